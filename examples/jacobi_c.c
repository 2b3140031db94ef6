/*
 * jacobi_c.c -- the Jacobi hot path driven from plain C through the C-ABI only
 * (include/uniconn.h), no Python, no torch: the paper's Listing 4 host loop.
 *
 *   jacobi_c NX NY ITERS NORM_EVERY MODE(0 host|1 device|2 partial) OUT.bin
 *
 * One rank (P = 1, ring topology, self-neighbour).  Writes the final (NY+2) x NX slab
 * (float32, row-major, halo rows included) followed by the norms (float64) to OUT.bin, so a
 * test can compare them with the oracle.  Exit code 0 on success.
 */
#include <stdio.h>
#include <stdlib.h>

#include "uniconn.h"

#define CHECK(call)                                                                    \
  do {                                                                                 \
    int rc_ = (call);                                                                  \
    if (rc_ != UC_OK) {                                                                \
      fprintf(stderr, "%s failed: %s\n", #call, uc_last_error());                      \
      return 1;                                                                        \
    }                                                                                  \
  } while (0)

int main(int argc, char** argv) {
  if (argc != 7) {
    fprintf(stderr, "usage: %s NX NY ITERS NORM_EVERY MODE OUT.bin\n", argv[0]);
    return 2;
  }
  const int nx = atoi(argv[1]), ny = atoi(argv[2]), iters = atoi(argv[3]), ne = atoi(argv[4]);
  const int mode = atoi(argv[5]);
  uc_env* env;
  uc_comm* comm;
  uc_coord* coord;
  uc_jacobi* J;
  /* Setup: Environment, Communicator, Coordinator (default stream), solver memory */
  CHECK(uc_env_init(0, 1, 0, NULL, NULL, &env));
  CHECK(uc_comm_create(env, 0, 0, &comm));
  CHECK(uc_coord_create(comm, (uc_mode)mode, NULL, &coord));
  CHECK(uc_jacobi_create(comm, nx, ny, 0x5EED, 0, &J));
  /* Progression: the time loop (one call runs all iterations; uc_jacobi_step is the per-
   * iteration form of Listing 4 lines 30-39) */
  const int nn = uc_jacobi_num_norms(J, iters, ne);
  double* norms = (double*)calloc(nn > 0 ? nn : 1, sizeof(double));
  CHECK(uc_jacobi_run(coord, J, iters, ne, norms, 0));
  CHECK(uc_coord_sync(coord));
  float* slab = (float*)malloc((size_t)(ny + 2) * nx * sizeof(float));
  CHECK(uc_jacobi_copy_out(coord, J, slab, 0));
  FILE* f = fopen(argv[6], "wb");
  if (!f) return 3;
  fwrite(slab, sizeof(float), (size_t)(ny + 2) * nx, f);
  fwrite(norms, sizeof(double), (size_t)nn, f);
  fclose(f);
  /* Termination */
  CHECK(uc_jacobi_destroy(J));
  CHECK(uc_coord_destroy(coord));
  CHECK(uc_comm_destroy(comm));
  CHECK(uc_env_finalize(env));
  free(slab);
  free(norms);
  printf("jacobi_c: %dx%d, %d iterations, %d norms, mode %d: OK\n", nx, ny, iters, nn, mode);
  return 0;
}
