/*
 * jacobi_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously correct single-threaded CPU Jacobi over the GLOBAL grid.  It is
 * the parity oracle for the CUDA path in paper_conf_cluster_sagbilieinu25_b200/ and shares no
 * code with it (no headers, no helpers, no tables).  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load it.
 *
 * What it follows (PAPER.md = /root/reference/PAPER.md, "P:n" = line n):
 *   - P:410 (§VI-C "Jacobi 2D Solver"): a 5-point 2-D star stencil on an fp32 grid, split
 *     equally along y.  Domain decomposition with 1-row halos (Listings 1-3) reaches
 *     exactly the result of sequential Jacobi on the global grid, because each point reads
 *     only its 4 neighbours of the previous iterate -- so the oracle is that global Jacobi.
 *   - Reading G1: new = 0.25f * ((l + r) + (t + b)), IEEE fp32 round-to-nearest,
 *     no FMA contraction (built with -ffp-contract=off), no FTZ/DAZ (no -ffast-math).
 *   - Reading G2: columns 0 and NX-1 fixed; ring topology refreshes halo rows 0 and NY+1 from
 *     rows NY and 1 before every iteration; dirichlet topology keeps them fixed.
 *   - Reading G7 (north_star): at iterations k with k % norm_every == 0 it records
 *     sum over all updated points of (double)d*(double)d, d = new - old in fp32, summed
 *     sequentially in double (row-major order).  norm = sqrt(sum).
 *
 * Pins (tests/test_oracle.py): hand-worked 4x4 example (tests/golden/hand4x4.txt), periodic
 * 2-row example, exact-rational brute force, invariants, the discrete sin-sinh closed form,
 * dense-matrix Jacobi, subnormal front 4^-k.
 */
#include <stddef.h>
#include <stdlib.h>
#include <string.h>

#define IDX(j, i) ((size_t)(j) * (size_t)nx + (size_t)(i))

/* One Jacobi sweep A -> B over rows 1..ny, columns 1..nx-2 of a (ny+2) x nx array.
 * Returns the sequential double sum of squared updates when want_norm != 0, else 0. */
static double sweep(int nx, int ny, const float *A, float *B, int want_norm) {
    double s = 0.0;
    for (int j = 1; j <= ny; ++j) {
        for (int i = 1; i <= nx - 2; ++i) {
            float l = A[IDX(j, i - 1)];
            float r = A[IDX(j, i + 1)];
            float t = A[IDX(j - 1, i)];
            float b = A[IDX(j + 1, i)];
            float lr = l + r;
            float tb = t + b;
            float sum = lr + tb;
            float v = 0.25f * sum;
            if (want_norm) {
                float d = v - A[IDX(j, i)];
                s += (double)d * (double)d;
            }
            B[IDX(j, i)] = v;
        }
    }
    return s;
}

/* Ring topology: halo row 0 <- row ny, halo row ny+1 <- row 1 (every rank sends its
 * first computed row to top and its last to bottom each iteration; with one global grid that
 * is this wrap). */
static void refresh_ring(int nx, int ny, float *A) {
    memcpy(&A[IDX(0, 0)], &A[IDX(ny, 0)], (size_t)nx * sizeof(float));
    memcpy(&A[IDX(ny + 1, 0)], &A[IDX(1, 0)], (size_t)nx * sizeof(float));
}

/*
 * oracle_jacobi_run: run `iters` Jacobi iterations in place on g[(ny+2)*nx].
 *   ring        : 1 = ring (y periodic), 0 = dirichlet-y
 *   norm_every  : >0 -> sums[m] = sum of d^2 at iteration k = m*norm_every (k < iters);
 *                 <=0 -> no norms
 *   sums        : caller-allocated, ceil(iters/norm_every) doubles (may be NULL if norm_every<=0)
 * Returns 0 on success, -1 on bad arguments, -2 on allocation failure.
 */
int oracle_jacobi_run(int nx, int ny, int ring, float *g, int iters, int norm_every, double *sums) {
    if (nx < 3 || ny < 1 || iters < 0 || g == NULL) return -1;
    if (norm_every > 0 && sums == NULL) return -1;
    size_t n = (size_t)(ny + 2) * (size_t)nx;
    float *B = (float *)malloc(n * sizeof(float));
    if (!B) return -2;
    if (ring) refresh_ring(nx, ny, g);
    memcpy(B, g, n * sizeof(float)); /* fixed columns / dirichlet rows present in both buffers */
    float *A = g, *Bn = B;
    for (int k = 0; k < iters; ++k) {
        int want = (norm_every > 0) && (k % norm_every == 0);
        if (ring) refresh_ring(nx, ny, A);
        double s = sweep(nx, ny, A, Bn, want);
        if (want) sums[k / norm_every] = s;
        float *tmp = A; A = Bn; Bn = tmp;
    }
    if (ring) refresh_ring(nx, ny, A);
    if (A != g) memcpy(g, A, n * sizeof(float));
    free(B);
    return 0;
}

/* Number of norm records oracle_jacobi_run writes. */
int oracle_num_norms(int iters, int norm_every) {
    if (norm_every <= 0 || iters <= 0) return 0;
    return (iters + norm_every - 1) / norm_every;
}
