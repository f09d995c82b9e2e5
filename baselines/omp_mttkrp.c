/* omp_mttkrp.c -- the paper's own CPU method, COO-MTTKRP-OMP, as a second,
 * clearly labelled CPU baseline for bench.py (SURVEY 8(d) "optional"): fp32 arithmetic, the
 * nonzeros split across all OpenMP threads, every update of the output an `omp atomic`
 * ("data races ... handled by atomics").  Not the oracle (oracle/ is the single-thread
 * fp64 correctness reference) and not the target; no part of the GPU path uses it.
 *
 *   out(i_n(x), r) += val(x) * prod_{k != n} U^(k)(i_k(x), r)   (Eq. 3)
 */
#include <stdint.h>
#include <string.h>

int omp_mttkrp_coo(uint32_t order, const uint32_t *dims, uint64_t nnz, const uint32_t *const *inds,
                   const float *vals, uint32_t mode, const float *const *factors, uint32_t R, float *out)
{
    if (order < 1 || order > 8 || mode >= order || R < 1 || R > 256) return -1;
    memset(out, 0, (size_t)dims[mode] * R * sizeof(float));
#pragma omp parallel for schedule(static)
    for (int64_t x = 0; x < (int64_t)nnz; ++x) {
        float t[256];
        for (uint32_t r = 0; r < R; ++r) t[r] = vals[x];
        for (uint32_t k = 0; k < order; ++k) {
            if (k == mode) continue;
            const float *row = factors[k] + (uint64_t)inds[k][x] * R;
            for (uint32_t r = 0; r < R; ++r) t[r] *= row[r];
        }
        float *dst = out + (uint64_t)inds[mode][x] * R;
        for (uint32_t r = 0; r < R; ++r) {
#pragma omp atomic
            dst[r] += t[r];
        }
    }
    return 0;
}

#include <omp.h>
int omp_threads(void) { return omp_get_max_threads(); }
