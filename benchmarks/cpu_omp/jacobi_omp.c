/*
 * jacobi_omp.c -- multi-core HOST baseline of the Jacobi hot path (bench.py "cpu_parallel").
 *
 * Not the product and not the oracle: the same global-grid Jacobi as oracle/jacobi_oracle.c
 * (PAPER.md P:410, 5-point star, fp32; reading G1 new = 0.25f*((l+r)+(t+b)), no FMA, no FTZ;
 * reading G2 ring / dirichlet halo rows), written for the host's cores: rows split over OpenMP
 * threads, the inner loop left to the compiler's vectoriser (IEEE single adds / multiplies in
 * the written order, -ffp-contract=off, no -ffast-math), the norm's squares summed in double
 * per thread and combined by the OpenMP reduction.  The grid is therefore bit-identical to the
 * oracle's; only the norm's summation order differs (tests/test_cpu_omp.py checks both).
 * It shares no code with the oracle or with the CUDA path.
 */
#include <omp.h>
#include <stddef.h>
#include <string.h>

#define AT(a, j, i) (a)[(size_t)(j) * (size_t)nx + (size_t)(i)]

int omp_threads(void) { return omp_get_max_threads(); }

/* `iters` iterations on the (ny+2) x nx array g (in place, ping-pong through `tmp` of the same
 * size).  ring != 0: rows 0 and ny+1 are refreshed from rows ny and 1 before every sweep.
 * sums[m] = sum of d^2 at iteration k = m * norm_every (norm_every <= 0: none). */
int omp_jacobi_run(int nx, int ny, int ring, float *g, float *tmp, int iters, int norm_every, double *sums) {
    if (nx < 3 || ny < 1 || iters < 0) return 1;
    float *a = g, *b = tmp;
    if (ring) {
        memcpy(&AT(a, 0, 0), &AT(a, ny, 0), (size_t)nx * sizeof(float));
        memcpy(&AT(a, ny + 1, 0), &AT(a, 1, 0), (size_t)nx * sizeof(float));
    }
    memcpy(b, a, (size_t)(ny + 2) * (size_t)nx * sizeof(float));
    int m = 0;
    for (int k = 0; k < iters; ++k) {
        if (ring) {
            memcpy(&AT(a, 0, 0), &AT(a, ny, 0), (size_t)nx * sizeof(float));
            memcpy(&AT(a, ny + 1, 0), &AT(a, 1, 0), (size_t)nx * sizeof(float));
        }
        const int want = norm_every > 0 && k % norm_every == 0;
        double s = 0.0;
#pragma omp parallel for schedule(static) reduction(+ : s)
        for (int j = 1; j <= ny; ++j) {
            const float *up = &AT(a, j - 1, 0), *row = &AT(a, j, 0), *dn = &AT(a, j + 1, 0);
            float *out = &AT(b, j, 0);
            for (int i = 1; i <= nx - 2; ++i) {
                const float lr = row[i - 1] + row[i + 1];
                const float tb = up[i] + dn[i];
                out[i] = 0.25f * (lr + tb);
            }
            if (want) {
                double t = 0.0;
                for (int i = 1; i <= nx - 2; ++i) {
                    const float d = out[i] - row[i];
                    t += (double)d * (double)d;
                }
                s += t;
            }
        }
        if (want && sums) sums[m++] = s;
        float *x = a;
        a = b;
        b = x;
    }
    if (ring) {  /* halo rows of the final iterate, as the oracle leaves them */
        memcpy(&AT(a, 0, 0), &AT(a, ny, 0), (size_t)nx * sizeof(float));
        memcpy(&AT(a, ny + 1, 0), &AT(a, 1, 0), (size_t)nx * sizeof(float));
    }
    if (a != g) memcpy(g, a, (size_t)(ny + 2) * (size_t)nx * sizeof(float));
    return 0;
}
