/*
 * gen.c — host build of the synthetic-input generator (see gen_rng.h).
 * Used by tests/ (oracle inputs) and bench.py (host inputs); no method arithmetic.
 */
#include "gen_rng.h"
#ifdef _OPENMP
#include <omp.h>
#endif

/* Fill out[i*ld_out + j] for rows [r0, r0+nr), columns [c0, c0+nc) of a matrix with
 * `ncols_total` columns: element (i, c) uses index i*ncols_total + c. */
void gen_matrix_f32(uint64_t seed, uint64_t stream, int32_t kind, uint32_t zero_q24,
                    int64_t r0, int64_t nr, int64_t c0, int64_t nc, int64_t ncols_total,
                    float* out, int64_t ld_out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < nr; ++i) {
    for (int64_t j = 0; j < nc; ++j) {
      uint64_t idx = (uint64_t)((r0 + i) * ncols_total + (c0 + j));
      out[i * ld_out + j] = (kind == GEN_KIND_NORMAL) ? gen_normal_f32(seed, stream, idx)
                                                      : gen_pixel_f32(seed, stream, idx, zero_q24);
    }
  }
}

void gen_uniform_f64_array(uint64_t seed, uint64_t stream, int64_t i0, int64_t count, double* out) {
#pragma omp parallel for schedule(static)
  for (int64_t i = 0; i < count; ++i) out[i] = gen_uniform_f64(seed, stream, (uint64_t)(i0 + i));
}
