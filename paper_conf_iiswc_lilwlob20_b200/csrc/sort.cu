// sort.cu -- device pre-processing primitives: stable lexicographic / Morton sorts
// (LSD passes of CUB radix sort, a library call used only in pre-processing),
// gathers, compaction, histograms.  Pre-processing trades for kernel time.
#include <cub/cub.cuh>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kThreads = 256;

inline unsigned grid_for(uint64_t n, int per_thread = 1) {
  uint64_t b = (n + uint64_t(kThreads) * per_thread - 1) / (uint64_t(kThreads) * per_thread);
  if (b < 1) b = 1;
  if (b > (1u << 30)) b = 1u << 30;
  return unsigned(b);
}

struct PackArgs {
  const uint32_t *comp[kMaxOrder];
  uint32_t shift[kMaxOrder];
  int nc;
};

__global__ void pack_keys_kernel(PackArgs a, const uint32_t *__restrict__ perm, uint64_t M,
                                 uint64_t *__restrict__ keys) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t p = perm[x];
    uint64_t k = 0;
    for (int c = 0; c < a.nc; ++c) k |= uint64_t(a.comp[c][p]) << a.shift[c];
    keys[x] = k;
  }
}

struct MortonArgs {
  const uint32_t *inds[kMaxOrder];
  uint32_t order;
  uint32_t pos_lo;  // first Morton bit position of this word
  uint32_t nbits;   // bits in this word
};

// Morton bit position of (level l, mode k) = l * N + (N - 1 - k)   (R#13)
__global__ void morton_word_kernel(MortonArgs a, const uint32_t *__restrict__ perm, uint64_t M,
                                   uint64_t *__restrict__ keys) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t p = perm[x];
    uint32_t c[kMaxOrder];
    for (uint32_t k = 0; k < a.order; ++k) c[k] = a.inds[k][p];
    uint64_t key = 0;
    for (uint32_t j = 0; j < a.nbits; ++j) {
      uint32_t pos = a.pos_lo + j;
      uint32_t l = pos / a.order;
      uint32_t k = a.order - 1 - pos % a.order;
      key |= uint64_t((c[k] >> l) & 1u) << j;
    }
    keys[x] = key;
  }
}

template <class T>
__global__ void gather_kernel(const T *__restrict__ in, const uint32_t *__restrict__ perm,
                              T *__restrict__ out, uint64_t M) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = in[perm[x]];
}

__global__ void iota_kernel(uint32_t *p, uint64_t M) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    p[x] = uint32_t(x);
}

__global__ void row_hist_kernel(const uint32_t *__restrict__ rows, uint64_t M,
                                unsigned long long *__restrict__ counts) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    atomicAdd(&counts[rows[x]], 1ull);
}

__global__ void lower_bound_kernel(const uint32_t *__restrict__ a, uint64_t M, uint32_t v,
                                   unsigned long long *out) {
  uint64_t lo = 0, hi = M;
  while (lo < hi) {
    uint64_t mid = lo + (hi - lo) / 2;
    if (a[mid] < v) lo = mid + 1; else hi = mid;
  }
  *out = lo;
}

struct LexArgs {
  const uint32_t *inds[kMaxOrder];
  uint32_t order;
};
__global__ void unsorted_flag_kernel(LexArgs a, uint64_t M, int *flag) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x + 1; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    int cmp = 0;
    for (uint32_t k = 0; k < a.order && cmp == 0; ++k) {
      uint32_t u = a.inds[k][x - 1], v = a.inds[k][x];
      cmp = (u < v) ? -1 : (u > v ? 1 : 0);
    }
    if (cmp > 0) *flag = 1;
  }
}

}  // namespace

void iota_u32(uint32_t *p, uint64_t M, cudaStream_t s) {
  if (!M) return;
  iota_kernel<<<grid_for(M, 4), kThreads, 0, s>>>(p, M);
  PASTA_LAUNCHED();
}

void gather_u32(const uint32_t *in, const uint32_t *perm, uint32_t *out, uint64_t M, cudaStream_t s) {
  if (!M) return;
  gather_kernel<uint32_t><<<grid_for(M, 4), kThreads, 0, s>>>(in, perm, out, M);
  PASTA_LAUNCHED();
}
void gather_f32(const float *in, const uint32_t *perm, float *out, uint64_t M, cudaStream_t s) {
  if (!M) return;
  gather_kernel<float><<<grid_for(M, 4), kThreads, 0, s>>>(in, perm, out, M);
  PASTA_LAUNCHED();
}
void gather_u8(const uint8_t *in, const uint32_t *perm, uint8_t *out, uint64_t M, cudaStream_t s) {
  if (!M) return;
  gather_kernel<uint8_t><<<grid_for(M, 4), kThreads, 0, s>>>(in, perm, out, M);
  PASTA_LAUNCHED();
}

static void radix_pass(DevArray<uint64_t> &keys, DevArray<uint64_t> &keys_alt, DevArray<uint32_t> &perm,
                       DevArray<uint32_t> &perm_alt, uint64_t M, int end_bit, cudaStream_t s) {
  cub::DoubleBuffer<uint64_t> kb(keys.p, keys_alt.p);
  cub::DoubleBuffer<uint32_t> vb(perm.p, perm_alt.p);
  size_t tmp_bytes = 0;
  PASTA_CUDA(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, kb, vb, M, 0, end_bit, s));
  DevArray<uint8_t> tmp(tmp_bytes, s);
  PASTA_CUDA(cub::DeviceRadixSort::SortPairs(tmp.p, tmp_bytes, kb, vb, M, 0, end_bit, s));
  count_launch();
  if (vb.Current() != perm.p) std::swap(perm, perm_alt);
  if (kb.Current() != keys.p) std::swap(keys, keys_alt);
  PASTA_CUDA(cudaStreamSynchronize(s));  // tmp is released at scope exit
}

void lexsort(const uint32_t *const *comps, const uint32_t *bits, int nc, DevArray<uint32_t> &perm,
             uint64_t M, cudaStream_t s) {
  if (M < 2) return;
  DevArray<uint64_t> keys(M, s), keys_alt(M, s);
  DevArray<uint32_t> perm_alt(M, s);
  int c = nc - 1;
  while (c >= 0) {
    // pack components (c0, c] into one 64-bit key, component c least significant
    uint32_t total = 0;
    int c0 = c;
    while (c0 >= 0 && total + bits[c0] <= 64) { total += bits[c0]; --c0; }
    if (total > 0) {
      PackArgs a{};
      uint32_t shift = 0;
      a.nc = 0;
      for (int j = c; j > c0; --j) {
        if (bits[j] == 0) continue;
        a.comp[a.nc] = comps[j];
        a.shift[a.nc] = shift;
        shift += bits[j];
        ++a.nc;
      }
      pack_keys_kernel<<<grid_for(M, 4), kThreads, 0, s>>>(a, perm.p, M, keys.p);
      PASTA_LAUNCHED();
      radix_pass(keys, keys_alt, perm, perm_alt, M, int(total), s);
    }
    c = c0;
  }
}

void morton_sort(const uint32_t *const *inds, uint32_t order, uint32_t Lm, DevArray<uint32_t> &perm,
                 uint64_t M, cudaStream_t s) {
  if (M < 2) return;
  uint32_t total = order * Lm;
  if (total == 0) return;
  DevArray<uint64_t> keys(M, s), keys_alt(M, s);
  DevArray<uint32_t> perm_alt(M, s);
  for (uint32_t lo = 0; lo < total; lo += 64) {  // least significant word first (LSD)
    MortonArgs a{};
    for (uint32_t k = 0; k < order; ++k) a.inds[k] = inds[k];
    a.order = order;
    a.pos_lo = lo;
    a.nbits = (total - lo) < 64 ? (total - lo) : 64;
    morton_word_kernel<<<grid_for(M, 4), kThreads, 0, s>>>(a, perm.p, M, keys.p);
    PASTA_LAUNCHED();
    radix_pass(keys, keys_alt, perm, perm_alt, M, int(a.nbits), s);
  }
}

uint64_t select_flagged(const uint8_t *flags, uint64_t M, DevArray<uint32_t> &idx_out, cudaStream_t s) {
  idx_out.alloc(M ? M : 1, s);
  if (!M) return 0;
  DevArray<int64_t> dcount(1, s);
  cub::CountingInputIterator<uint32_t> it(0);
  size_t tmp_bytes = 0;
  PASTA_CUDA(cub::DeviceSelect::Flagged(nullptr, tmp_bytes, it, flags, idx_out.p, dcount.p,
                                        int64_t(M), s));
  DevArray<uint8_t> tmp(tmp_bytes, s);
  PASTA_CUDA(cub::DeviceSelect::Flagged(tmp.p, tmp_bytes, it, flags, idx_out.p, dcount.p,
                                        int64_t(M), s));
  count_launch();
  int64_t h = 0;
  PASTA_CUDA(cudaMemcpyAsync(&h, dcount.p, sizeof(h), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  return uint64_t(h);
}

void row_counts_device(const uint32_t *rows, uint64_t nnz, uint32_t nrows, uint64_t *counts_host,
                       cudaStream_t s) {
  DevArray<unsigned long long> c(nrows ? nrows : 1, s);
  PASTA_CUDA(cudaMemsetAsync(c.p, 0, c.bytes(), s));
  if (nnz) {
    row_hist_kernel<<<grid_for(nnz, 8), kThreads, 0, s>>>(rows, nnz, c.p);
    PASTA_LAUNCHED();
  }
  PASTA_CUDA(cudaMemcpyAsync(counts_host, c.p, sizeof(uint64_t) * nrows, cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
}

uint64_t lower_bound_device(const uint32_t *a, uint64_t M, uint32_t v, cudaStream_t s) {
  DevArray<unsigned long long> d(1, s);
  lower_bound_kernel<<<1, 1, 0, s>>>(a, M, v, d.p);
  PASTA_LAUNCHED();
  unsigned long long h = 0;
  PASTA_CUDA(cudaMemcpyAsync(&h, d.p, sizeof(h), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  return h;
}

bool is_lex_sorted_device(const uint32_t *const *inds, uint32_t order, uint64_t M, cudaStream_t s) {
  if (M < 2) return true;
  DevArray<int> flag(1, s);
  PASTA_CUDA(cudaMemsetAsync(flag.p, 0, sizeof(int), s));
  LexArgs a{};
  for (uint32_t k = 0; k < order; ++k) a.inds[k] = inds[k];
  a.order = order;
  unsorted_flag_kernel<<<grid_for(M, 8), kThreads, 0, s>>>(a, M, flag.p);
  PASTA_LAUNCHED();
  int h = 0;
  PASTA_CUDA(cudaMemcpyAsync(&h, flag.p, sizeof(h), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  return h == 0;
}

}  // namespace pasta

// ------------------------------------------------------------------------------------------
// Frequency-aware L2 eviction priority for the COO factor gathers (see coo_mark_hot).
namespace pasta {
namespace {

__device__ __host__ inline uint32_t count_bucket(uint32_t c) {
  if (c == 0) return 0;
  uint32_t e = 31 - __builtin_clz(c);
  uint32_t m = e >= 3 ? (c >> (e - 3)) & 7u : (c << (3 - e)) & 7u;
  return 8 * e + m;
}

__device__ inline uint32_t count_bucket_dev(uint32_t c) {
  if (c == 0) return 0;
  uint32_t e = 31 - __clz(c);
  uint32_t m = e >= 3 ? (c >> (e - 3)) & 7u : (c << (3 - e)) & 7u;
  return 8 * e + m;
}

__global__ void count_rows_kernel(const uint32_t *__restrict__ rows, uint64_t M, uint32_t *__restrict__ cnt) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    atomicAdd(&cnt[rows[x]], 1u);
}

__global__ void bucket_hist_kernel(const uint32_t *__restrict__ cnt, uint64_t n,
                                   unsigned long long *__restrict__ hist) {
  __shared__ unsigned long long h[kCountBuckets];
  for (int b = threadIdx.x; b < kCountBuckets; b += blockDim.x) h[b] = 0;
  __syncthreads();
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n;
       i += uint64_t(gridDim.x) * blockDim.x)
    if (cnt[i]) atomicAdd(&h[count_bucket_dev(cnt[i])], 1ull);
  __syncthreads();
  for (int b = threadIdx.x; b < kCountBuckets; b += blockDim.x)
    if (h[b]) atomicAdd(&hist[b], h[b]);
}

// flag rows with lo <= bucket(count) < hi
__global__ void hot_flag_kernel(const uint32_t *__restrict__ cnt, uint64_t n, uint32_t lo, uint32_t hi,
                                uint8_t *__restrict__ flag) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n;
       i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t b = cnt[i] ? count_bucket_dev(cnt[i]) : 0u;
    flag[i] = cnt[i] && b >= lo && b < hi;
  }
}

__global__ void slot_map_kernel(const uint32_t *__restrict__ rows, uint64_t nh, uint64_t base,
                                uint32_t tag, uint32_t *__restrict__ slot_of, uint32_t *__restrict__ hot_rows) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s < nh;
       s += uint64_t(gridDim.x) * blockDim.x) {
    slot_of[rows[s]] = tag | uint32_t(base + s);
    hot_rows[base + s] = rows[s];
  }
}

__global__ void mark_hot_kernel(const uint32_t *__restrict__ src, const uint32_t *__restrict__ slot_of,
                                uint64_t M, uint32_t *__restrict__ dst) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t v = src[x];
    const uint32_t sl = __ldg(slot_of + v);
    dst[x] = sl != 0xFFFFFFFFu ? sl : v;  // sl carries its tier tag
  }
}

// hot_buf[s][:] = U[hot_rows[s]][:] for the slots [base, base + n) of one factor (float4)
__global__ void hot_fill_kernel(const float4 *__restrict__ U, const uint32_t *__restrict__ hot_rows,
                                uint64_t base, uint64_t n, uint32_t r4, float4 *__restrict__ buf) {
  for (uint64_t e = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; e < n * r4;
       e += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t s = e / r4, c = e % r4;
    buf[(base + s) * r4 + c] = __ldg(U + uint64_t(__ldg(hot_rows + base + s)) * r4 + c);
  }
}

void gather_any(const uint32_t *in, const uint32_t *perm, uint32_t *out, uint64_t n, cudaStream_t s) {
  if (n) gather_u32(in, perm, out, n, s);
}
void gather_any(const float *in, const uint32_t *perm, float *out, uint64_t n, cudaStream_t s) {
  if (n) gather_f32(in, perm, out, n, s);
}

// die-split segment of each nonzero (R#35); n01 counts the die-0 segments (half of ia == 0)
__global__ void split_seg_kernel(const uint32_t *__restrict__ ia, const uint32_t *__restrict__ ib, uint64_t M,
                                 uint32_t ka, uint32_t kb, uint32_t ta, uint32_t tb, uint32_t sh,
                                 uint32_t *__restrict__ seg, unsigned long long *__restrict__ n01) {
  unsigned long long c = 0;
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M; x += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t ha = die_half(ia[x] >> sh, ka, ta), hb = die_half(ib[x] >> sh, kb, tb);
    seg[x] = ha ? (hb ? 2u : 3u) : (hb ? 1u : 0u);
    c += ha == 0;
  }
  for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xFFFFFFFFu, c, o);
  if ((threadIdx.x & 31) == 0 && c) atomicAdd(n01, c);
}

unsigned grid8(uint64_t n) {
  uint64_t b = (n + 256 * 8 - 1) / (256 * 8);
  if (b < 1) b = 1;
  if (b > (1u << 30)) b = 1u << 30;
  return unsigned(b);
}

}  // namespace

static bool env_flag(const char *name) {
  const char *v = getenv(name);
  return v && *v && atoi(v) != 0;
}

// Hot-row cache for the COO factor gathers, two tiers.  The most frequent rows of the gathered
// factors (row nonzero counts, bucketed 8 per octave) are ranked jointly over the factors:
//  * shared-memory tier: as many as fit `smem_rows` rows (the kernel copies them into every
//    CTA's shared memory at launch, so their gathers never reach L2; on L2-resident factors
//    the kernel is bound by L2->SM bandwidth, and power-law-hot rows carry most gathers);
//  * L2 tier (`global_tier`, when the gathered factors exceed L2): the next rows, as many as fit
//    PASTA_HOT_MB (default 64 MB) at R*4 bytes per row, get contiguous slots of one buffer
//    refilled from the factors before every launch.  Packed hot rows fill whole L2 lines, and
//    their misses land on a 64-MB region instead of the whole factor: on H the DRAM bytes stay
//    about the same (8.10 vs 8.32 GB per launch) but the kernel runs 2.4x faster, because
//    scattered misses are bound by the rate of DRAM row activations (~37 G/s) and packed ones
//    are not (profiles/r02_coo_l2_tier_effect.txt; cache reuse is why MTTKRP beats its DRAM
//    roofline).
// The per-mode index copies hot_inds[k] encode 0xC0000000 | smem slot (slot numbered over all
// gathered factors, factor k at [hs_base[k], +hs_cnt[k])), 0x80000000 | L2-tier slot, or the
// plain row.  Needs dims < 2^30.
void coo_mark_hot(pasta_coo *x, uint32_t mode, uint32_t R, bool global_tier, uint32_t smem_rows,
                  cudaStream_t s, bool die_split) {
  CooModeCopy &mc = x->mc[mode];
  // the shared-memory tier filled to its budget from the next count bucket down: on
  // L2-resident factors (no L2 tier) every row it serves is an L1TEX wavefront saved (C2 0.757
  // -> 0.729 ms per mode); with DRAM-bound gathers it takes L1 from the in-flight misses (H 1.56
  // -> 1.71), so off there (profiles/r02_smem_fill_sweep.txt).  PASTA_HOT_SMEM_FILL overrides.
  const char *fenv = getenv("PASTA_HOT_SMEM_FILL");
  const bool smem_fill = (fenv && *fenv) ? atoi(fenv) != 0 : !global_tier;
  if (mc.hot_R == R && mc.hot_global == global_tier && mc.hot_smem_budget == smem_rows &&
      mc.split == die_split && mc.smem_fill == smem_fill)
    return;
  mc.smem_fill = smem_fill;
  // die split (R#35): two gathered factors, an L2 tier and a measured SM -> die map
  die_split = die_split && global_tier && x->order == 3;
  const DieMap *dmp = die_split ? &die_map() : nullptr;  // calibrates on first use only
  die_split = die_split && dmp->ok;
  mc.split = false;
  const char *env = getenv("PASTA_HOT_MB");
  // the die split holds half of each factor's tier per die, so the tier can be larger
  const double hot_mb = global_tier ? ((env && *env) ? atof(env) : (die_split ? 96.0 : 64.0)) : 0.0;
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  // die-0 shares: the first gathered factor in proportion to the dies' SM counts, the second
  // half and half, so both phases of both dies get work in proportion to their SMs
  uint32_t tsplit[kMaxOrder] = {};
  // the halves are made of 2-KB runs of factor rows (row >> split_sh): a die's L2 keeps whole
  // lines its SMs read, so rows of the two halves must not share lines (nor 2-KB chunks)
  uint32_t split_sh = 0;
  while (split_sh < 16 && (uint64_t(R) * 4u << split_sh) < 2048u) ++split_sh;
  if (die_split) {
    int j = 0;
    for (uint32_t k = 0; k < N; ++k) {
      if (k == mode) continue;
      tsplit[k] = j == 0 ? uint32_t(4294967296.0 * dmp->n[0] / double(dmp->n[0] + dmp->n[1])) : 0x80000000u;
      ++j;
    }
  }
  mc.hot_R = 0;
  for (uint32_t k = 0; k < N; ++k)
    if (x->dims[k] >= 0x40000000u) return;
  if ((hot_mb <= 0 && smem_rows == 0) || M == 0) return;
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode || x->counts_ready[k]) continue;
    x->row_count[k].alloc(x->dims[k], s);
    PASTA_CUDA(cudaMemsetAsync(x->row_count[k].p, 0, x->row_count[k].bytes(), s));
    count_rows_kernel<<<grid8(M), 256, 0, s>>>(x->inds[k].p, M, x->row_count[k].p);
    PASTA_LAUNCHED();
    DevArray<unsigned long long> h(kCountBuckets, s);
    PASTA_CUDA(cudaMemsetAsync(h.p, 0, h.bytes(), s));
    bucket_hist_kernel<<<grid8(x->dims[k]), 256, 0, s>>>(x->row_count[k].p, x->dims[k], h.p);
    PASTA_LAUNCHED();
    PASTA_CUDA(cudaMemcpyAsync(x->count_hist[k], h.p, h.bytes(), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    x->counts_ready[k] = true;
  }
  // smallest bucket such that the rows at or above it, over every gathered factor, fit a budget
  auto threshold = [&](double budget_rows) {
    uint32_t hb = kCountBuckets;
    double acc = 0.0;
    for (int b = kCountBuckets - 1; b >= 1; --b) {
      double add = 0.0;
      for (uint32_t k = 0; k < N; ++k)
        if (k != mode) add += double(x->count_hist[k][b]);
      if (acc + add > budget_rows) break;
      acc += add;
      hb = uint32_t(b);
    }
    return hb;
  };
  const uint32_t hsb = threshold(double(smem_rows));  // smem tier: bucket >= hsb
  const uint32_t hb =                                  // L2 tier: hb <= bucket < hsb
      hot_mb > 0 ? threshold(double(smem_rows) + hot_mb * 1048576.0 / (double(R) * 4.0)) : hsb;
  uint64_t smem_fill_extra[kMaxOrder] = {};
  if (smem_fill && hsb > 1 && hsb <= kCountBuckets && smem_rows > 0) {
    double in_tier = 0.0, next = 0.0;
    for (uint32_t k = 0; k < N; ++k) {
      if (k == mode) continue;
      for (uint32_t b = hsb; b < kCountBuckets; ++b) in_tier += double(x->count_hist[k][b]);
      next += double(x->count_hist[k][hsb - 1]);
    }
    const double left = double(smem_rows) - in_tier;
    if (left > 0 && next > 0)
      for (uint32_t k = 0; k < N; ++k)
        if (k != mode) smem_fill_extra[k] = uint64_t(double(x->count_hist[k][hsb - 1]) * std::min(1.0, left / next));
  }
  // both tiers -> contiguous slots (per tier, factor after factor, rows ascending)
  uint64_t total = 0, stotal = 0;
  std::vector<DevArray<uint32_t>> lists(N), slists(N);
  for (uint32_t k = 0; k < N; ++k) {
    mc.hot_base[k] = total;
    mc.hot_cnt[k] = 0;
    mc.hs_base[k] = stotal;
    mc.hs_cnt[k] = 0;
    if (k == mode) continue;
    DevArray<uint8_t> flag(x->dims[k], s);
    if (hsb < kCountBuckets) {
      hot_flag_kernel<<<grid8(x->dims[k]), 256, 0, s>>>(x->row_count[k].p, x->dims[k], hsb, kCountBuckets,
                                                        flag.p);
      PASTA_LAUNCHED();
      mc.hs_cnt[k] = select_flagged(flag.p, x->dims[k], slists[k], s);
      stotal += mc.hs_cnt[k];
    }
    // smem fill: the budget the whole buckets leave is filled with rows of the next bucket
    // down (each factor in proportion to its rows there; with an L2 tier they keep that slot too)
    if (hsb > 1 && hsb <= kCountBuckets && smem_fill_extra[k] > 0) {
      hot_flag_kernel<<<grid8(x->dims[k]), 256, 0, s>>>(x->row_count[k].p, x->dims[k], hsb - 1, hsb, flag.p);
      PASTA_LAUNCHED();
      DevArray<uint32_t> more;
      const uint64_t nm = std::min<uint64_t>(select_flagged(flag.p, x->dims[k], more, s), smem_fill_extra[k]);
      DevArray<uint32_t> cat(mc.hs_cnt[k] + nm, s);
      if (mc.hs_cnt[k])
        PASTA_CUDA(cudaMemcpyAsync(cat.p, slists[k].p, mc.hs_cnt[k] * 4, cudaMemcpyDeviceToDevice, s));
      PASTA_CUDA(cudaMemcpyAsync(cat.p + mc.hs_cnt[k], more.p, nm * 4, cudaMemcpyDeviceToDevice, s));
      PASTA_CUDA(cudaStreamSynchronize(s));
      slists[k] = std::move(cat);
      mc.hs_cnt[k] += nm;
      stotal += nm;
    }
    if (hb < hsb) {
      hot_flag_kernel<<<grid8(x->dims[k]), 256, 0, s>>>(x->row_count[k].p, x->dims[k], hb, hsb, flag.p);
      PASTA_LAUNCHED();
      mc.hot_cnt[k] = select_flagged(flag.p, x->dims[k], lists[k], s);
      total += mc.hot_cnt[k];
      if (die_split && mc.hot_cnt[k]) {  // L2-tier slots: this factor's half-0 rows first
        std::vector<uint32_t> hl(mc.hot_cnt[k]), part;
        part.reserve(hl.size());
        PASTA_CUDA(cudaMemcpyAsync(hl.data(), lists[k].p, hl.size() * 4, cudaMemcpyDeviceToHost, s));
        PASTA_CUDA(cudaStreamSynchronize(s));
        for (uint32_t r : hl) if (die_half(r >> split_sh, k, tsplit[k]) == 0) part.push_back(r);
        for (uint32_t r : hl) if (die_half(r >> split_sh, k, tsplit[k]) == 1) part.push_back(r);
        PASTA_CUDA(cudaMemcpyAsync(lists[k].p, part.data(), part.size() * 4, cudaMemcpyHostToDevice, s));
        PASTA_CUDA(cudaStreamSynchronize(s));
      }
    }
  }
  mc.hot_total = total;
  mc.hs_total = stotal;
  mc.hot_rows.alloc(total ? total : 1, s);
  mc.hot_buf.alloc((total ? total : 1) * R, s);
  mc.hs_rows.alloc(stotal ? stotal : 1, s);
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode) continue;
    DevArray<uint32_t> slot_of(x->dims[k], s);
    PASTA_CUDA(cudaMemsetAsync(slot_of.p, 0xFF, slot_of.bytes(), s));
    if (mc.hot_cnt[k]) {
      slot_map_kernel<<<grid8(mc.hot_cnt[k]), 256, 0, s>>>(lists[k].p, mc.hot_cnt[k], mc.hot_base[k],
                                                          0x80000000u, slot_of.p, mc.hot_rows.p);
      PASTA_LAUNCHED();
    }
    if (mc.hs_cnt[k]) {
      slot_map_kernel<<<grid8(mc.hs_cnt[k]), 256, 0, s>>>(slists[k].p, mc.hs_cnt[k], mc.hs_base[k],
                                                         0xC0000000u, slot_of.p, mc.hs_rows.p);
      PASTA_LAUNCHED();
    }
    if (mc.hot_inds[k].n != M) mc.hot_inds[k].alloc(M, s);
    mark_hot_kernel<<<grid8(M), 256, 0, s>>>(mc.inds[k], slot_of.p, M, mc.hot_inds[k].p);
    PASTA_LAUNCHED();
    PASTA_CUDA(cudaStreamSynchronize(s));  // slot_of is released at scope exit
  }
  if (die_split) {
    // nonzero segments (R#35): 0 = (0,0), 1 = (0,1) [die 0], 2 = (1,1), 3 = (1,0) [die 1]
    uint32_t ka = 0, kb = 0, j = 0;
    for (uint32_t k = 0; k < N; ++k) {
      if (k == mode) continue;
      (j++ == 0 ? ka : kb) = k;
    }
    DevArray<uint32_t> seg(M, s), perm(M, s);
    DevArray<unsigned long long> n01(1, s);
    PASTA_CUDA(cudaMemsetAsync(n01.p, 0, sizeof(unsigned long long), s));
    split_seg_kernel<<<grid8(M), 256, 0, s>>>(mc.inds[ka], mc.inds[kb], M, ka, kb, tsplit[ka], tsplit[kb], split_sh,
                                              seg.p, n01.p);
    PASTA_LAUNCHED();
    iota_u32(perm.p, M, s);
    const uint32_t *comps[1] = {seg.p};
    const uint32_t bits[1] = {2};
    lexsort(comps, bits, 1, perm, M, s);  // stable: rows stay sorted inside each segment
    seg.reset();
    unsigned long long h01 = 0;
    PASTA_CUDA(cudaMemcpyAsync(&h01, n01.p, sizeof(h01), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    // die 1's part starts 16-byte aligned (the kernel streams 4 nonzeros per cp.async); the
    // gap holds zero-valued nonzeros of row 0 (die 0 walks them; they add nothing)
    const uint64_t n0 = h01, x1 = (n0 + 3) & ~uint64_t(3), Mt = x1 + (M - n0);
    auto split_gather = [&](auto *in, auto *out) {
      gather_any(in, perm.p, out, n0, s);
      if (x1 > n0) PASTA_CUDA(cudaMemsetAsync(out + n0, 0, (x1 - n0) * 4, s));
      gather_any(in, perm.p + n0, out + x1, M - n0, s);
    };
    mc.split_irow.alloc(Mt, s);
    mc.split_val.alloc(Mt, s);
    split_gather(mc.inds[mode], mc.split_irow.p);
    split_gather(mc.val, mc.split_val.p);
    for (uint32_t k : {ka, kb}) {
      DevArray<uint32_t> tmp(Mt, s);
      split_gather(mc.hot_inds[k].p, tmp.p);
      std::swap(mc.hot_inds[k], tmp);
    }
    PASTA_CUDA(cudaStreamSynchronize(s));
    mc.split_x = x1;
    mc.split_n = Mt;
    mc.split_t[0] = tsplit[ka];
    mc.split_t[1] = tsplit[kb];
    mc.claim.alloc(2, s);
    mc.split = true;
  } else {
    mc.split_irow.reset();
    mc.split_val.reset();
  }
  mc.hot_bucket = hb;
  mc.hs_bucket = hsb;
  mc.hot_global = global_tier;
  mc.hot_smem_budget = smem_rows;
  mc.hot_R = R;
  if (getenv("PASTA_DEBUG")) {
    fprintf(stderr, "[pasta] hot cache mode %u R %u: smem budget %u rows (bucket >= %u, %llu rows), "
            "L2 tier %.0f MB (bucket >= %u, %llu rows) (", mode, R, smem_rows, hsb,
            (unsigned long long)stotal, hot_mb, hb, (unsigned long long)total);
    for (uint32_t k = 0; k < N; ++k)
      if (k != mode)
        fprintf(stderr, " k%u:%llu+%llu", k, (unsigned long long)mc.hs_cnt[k], (unsigned long long)mc.hot_cnt[k]);
    fprintf(stderr, " )\n");
  }
}

template <class MC>
static void hot_fill_t(const MC &mc, const float *const *factors, uint32_t order, uint32_t mode,
                       uint32_t R, cudaStream_t s) {
  for (uint32_t k = 0; k < order; ++k) {
    if (k == mode || mc.hot_cnt[k] == 0) continue;
    const uint64_t n = mc.hot_cnt[k] * (R / 4);
    uint64_t g = (n + 255) / 256;
    if (g > 148 * 32) g = 148 * 32;
    hot_fill_kernel<<<unsigned(g), 256, 0, s>>>(reinterpret_cast<const float4 *>(factors[k]), mc.hot_rows.p,
                                                mc.hot_base[k], mc.hot_cnt[k], R / 4,
                                                reinterpret_cast<float4 *>(mc.hot_buf.p));
    PASTA_LAUNCHED();
  }
}

}  // namespace pasta

namespace pasta {

void launch_hot_fill(const CooModeCopy &mc, const float *const *factors, uint32_t order, uint32_t mode,
                     uint32_t R, cudaStream_t s) {
  hot_fill_t(mc, factors, order, mode, R, s);
}
void launch_hot_fill(const HicooModeCopy &mc, const float *const *factors, uint32_t order, uint32_t mode,
                     uint32_t R, cudaStream_t s) {
  hot_fill_t(mc, factors, order, mode, R, s);
}

namespace {

// cnt[binds_k[b]] += entries of canonical block b: nonzeros per mode-k block row
__global__ void block_row_count_kernel(const uint64_t *__restrict__ bptr, const uint32_t *__restrict__ binds,
                                       uint64_t nb, unsigned long long *__restrict__ cnt) {
  for (uint64_t b = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; b < nb; b += uint64_t(gridDim.x) * blockDim.x)
    atomicAdd(&cnt[binds[b]], (unsigned long long)(bptr[b + 1] - bptr[b]));
}

// slice base (untagged: block << bb) -> tier tag | slot row, from the per-block-row map
__global__ void retag_base_kernel(uint32_t *__restrict__ base, uint64_t n, uint32_t bb,
                                  const uint32_t *__restrict__ map) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t v = base[i];
    if ((v >> 30) == 0u) {
      const uint32_t t = map[v >> bb];
      if (t != 0xFFFFFFFFu) base[i] = t;
    }
  }
}

// undo retag_base_kernel: tagged slot row -> original block << bb (tier_block: smem slot
// blocks of this factor, then its L2 slot blocks)
__global__ void untag_base_kernel(uint32_t *__restrict__ base, uint64_t n, uint32_t bb, uint32_t hs_base,
                                  uint32_t hot_base, uint32_t nsm, const uint32_t *__restrict__ tier_block) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t v = base[i], tag = v >> 30, slot = v & 0x3FFFFFFFu;
    if (tag == 3u) base[i] = tier_block[(slot - hs_base) >> bb] << bb;
    else if (tag == 2u) base[i] = tier_block[nsm + ((slot - hot_base) >> bb)] << bb;
  }
}

}  // namespace

// Hot-block tiers of the HiCOO row-slice copy (R#34): block rows of the gathered compressed
// factors ranked jointly by their nonzero count; the top ones fill the shared-memory tier
// (`smem_rows` rows = smem_rows / B blocks), the next ones the L2 tier (PASTA_HOT_MB, default
// 64 MB, when `global_tier`); the slices' bases of those blocks are retagged in place.
void hicoo_mark_hot(pasta_hicoo *h, uint32_t mode, uint32_t R, bool global_tier, uint32_t smem_rows,
                    cudaStream_t s) {
  HicooModeCopy &mc = h->mc[mode];
  if (mc.layout != 0) return;
  if (mc.hot_R == R && mc.hot_global == global_tier && mc.hot_smem_budget == smem_rows) return;
  const uint32_t N = h->order, bb = h->block_bits, B = 1u << bb;
  auto blocked = [&](uint32_t k) { return k != mode && ((h->cmask >> k) & 1u) != 0; };
  if (mc.tagged) {  // undo the previous tiers before re-ranking
    for (uint32_t k = 0; k < N; ++k) {
      if (!blocked(k) || (mc.hs_cnt[k] + mc.hot_cnt[k]) == 0) continue;
      untag_base_kernel<<<grid8(mc.nsb), 256, 0, s>>>(mc.sbbase[k].p, mc.nsb, bb, uint32_t(mc.hs_base[k]),
                                                       uint32_t(mc.hot_base[k]), uint32_t(mc.hs_cnt[k] >> bb),
                                                       mc.tier_block[k].p);
      PASTA_LAUNCHED();
    }
    mc.tagged = false;
  }
  // the ranking is cached per (R, budgets), also when it yields no tiers
  mc.hot_R = R;
  mc.hot_global = global_tier;
  mc.hot_smem_budget = smem_rows;
  mc.hs_total = mc.hot_total = 0;
  for (uint32_t k = 0; k < N; ++k) mc.hs_base[k] = mc.hs_cnt[k] = mc.hot_base[k] = mc.hot_cnt[k] = 0;
  for (uint32_t k = 0; k < N; ++k)
    if (h->dims[k] >= 0x40000000u) return;  // untagged bases must stay below 2^30
  const char *env = getenv("PASTA_HOT_MB");
  const double hot_mb = global_tier ? ((env && *env) ? atof(env) : 64.0) : 0.0;
  const uint64_t sm_blocks = smem_rows / B;
  const uint64_t l2_blocks = uint64_t(hot_mb * 1048576.0 / (double(B) * R * sizeof(float)));
  if ((sm_blocks == 0 && l2_blocks == 0) || h->nnz == 0 || mc.nsb == 0) return;
  struct Cand { unsigned long long cnt; uint32_t k, blk; };
  std::vector<Cand> cand;
  for (uint32_t k = 0; k < N; ++k) {
    if (!blocked(k)) continue;
    const uint64_t nbr = (uint64_t(h->dims[k]) + B - 1) >> bb;
    DevArray<unsigned long long> c(nbr, s);
    PASTA_CUDA(cudaMemsetAsync(c.p, 0, c.bytes(), s));
    block_row_count_kernel<<<grid8(h->nblocks), 256, 0, s>>>(h->bptr.p, h->binds[k].p, h->nblocks, c.p);
    PASTA_LAUNCHED();
    std::vector<unsigned long long> hc(nbr);
    PASTA_CUDA(cudaMemcpyAsync(hc.data(), c.p, c.bytes(), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    for (uint64_t b = 0; b < nbr; ++b)
      if (hc[b]) cand.push_back({hc[b], k, uint32_t(b)});
  }
  std::stable_sort(cand.begin(), cand.end(), [](const Cand &a, const Cand &b) { return a.cnt > b.cnt; });
  std::vector<std::vector<uint32_t>> smb(N), l2b(N);
  for (uint64_t i = 0; i < cand.size() && i < sm_blocks + l2_blocks; ++i)
    (i < sm_blocks ? smb : l2b)[cand[i].k].push_back(cand[i].blk);
  std::vector<uint32_t> hs_rows, hot_rows;
  for (uint32_t k = 0; k < N; ++k) {
    mc.hs_base[k] = hs_rows.size();
    for (uint32_t blk : smb[k])
      for (uint32_t e = 0; e < B; ++e) hs_rows.push_back(std::min<uint64_t>(uint64_t(blk) * B + e, h->dims[k] - 1));
    mc.hs_cnt[k] = hs_rows.size() - mc.hs_base[k];
    mc.hot_base[k] = hot_rows.size();
    for (uint32_t blk : l2b[k])
      for (uint32_t e = 0; e < B; ++e) hot_rows.push_back(std::min<uint64_t>(uint64_t(blk) * B + e, h->dims[k] - 1));
    mc.hot_cnt[k] = hot_rows.size() - mc.hot_base[k];
  }
  mc.hs_total = hs_rows.size();
  mc.hot_total = hot_rows.size();
  mc.hs_rows.alloc(std::max<size_t>(hs_rows.size(), 1), s);
  mc.hot_rows.alloc(std::max<size_t>(hot_rows.size(), 1), s);
  mc.hot_buf.alloc(std::max<uint64_t>(mc.hot_total, 1) * R, s);
  if (!hs_rows.empty())
    PASTA_CUDA(cudaMemcpyAsync(mc.hs_rows.p, hs_rows.data(), hs_rows.size() * 4, cudaMemcpyHostToDevice, s));
  if (!hot_rows.empty())
    PASTA_CUDA(cudaMemcpyAsync(mc.hot_rows.p, hot_rows.data(), hot_rows.size() * 4, cudaMemcpyHostToDevice, s));
  for (uint32_t k = 0; k < N; ++k) {
    if (!blocked(k) || (smb[k].empty() && l2b[k].empty())) continue;
    const uint64_t nbr = (uint64_t(h->dims[k]) + B - 1) >> bb;
    std::vector<uint32_t> map(nbr, 0xFFFFFFFFu), tb;
    for (size_t i = 0; i < smb[k].size(); ++i) {
      map[smb[k][i]] = 0xC0000000u | uint32_t(mc.hs_base[k] + i * B);
      tb.push_back(smb[k][i]);
    }
    for (size_t i = 0; i < l2b[k].size(); ++i) {
      map[l2b[k][i]] = 0x80000000u | uint32_t(mc.hot_base[k] + i * B);
      tb.push_back(l2b[k][i]);
    }
    DevArray<uint32_t> dmap(nbr, s);
    PASTA_CUDA(cudaMemcpyAsync(dmap.p, map.data(), nbr * 4, cudaMemcpyHostToDevice, s));
    mc.tier_block[k].alloc(tb.size(), s);
    PASTA_CUDA(cudaMemcpyAsync(mc.tier_block[k].p, tb.data(), tb.size() * 4, cudaMemcpyHostToDevice, s));
    retag_base_kernel<<<grid8(mc.nsb), 256, 0, s>>>(mc.sbbase[k].p, mc.nsb, bb, dmap.p);
    PASTA_LAUNCHED();
    PASTA_CUDA(cudaStreamSynchronize(s));  // dmap and the host vectors are released at scope exit
  }
  PASTA_CUDA(cudaStreamSynchronize(s));
  mc.tagged = mc.hs_total + mc.hot_total > 0;
  if (getenv("PASTA_DEBUG"))
    fprintf(stderr, "[pasta] hicoo hot blocks mode %u R %u: smem %llu rows, L2 %llu rows\n", mode, R,
            (unsigned long long)mc.hs_total, (unsigned long long)mc.hot_total);
}

namespace {
// cnt[i_k(x)] += 1 over the canonical HiCOO entries (i_k decoded from the block of entry x)
__global__ void hicoo_row_count_kernel(const uint64_t *__restrict__ bptr, uint64_t nb, const uint32_t *__restrict__ binds,
                                       const uint8_t *__restrict__ einds, const uint32_t *__restrict__ uinds,
                                       uint32_t bb, uint64_t M, uint32_t *__restrict__ cnt) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M; x += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t row;
    if (uinds) {
      row = uinds[x];
    } else {
      uint64_t lo = 0, hi = nb;
      while (hi - lo > 1) {
        const uint64_t mid = (lo + hi) / 2;
        if (bptr[mid] <= x) lo = mid; else hi = mid;
      }
      row = (binds[lo] << bb) | einds[x];
    }
    atomicAdd(&cnt[row], 1u);
  }
}
}  // namespace

void hicoo_mark_rows(pasta_hicoo *h, uint32_t mode, uint32_t R, uint32_t smem_rows, uint64_t max_words,
                     cudaStream_t s) {
  HicooModeCopy &mc = h->mc[mode];
  if (mc.rs_R == R && mc.rs_budget == smem_rows) return;
  const uint32_t N = h->order, bb = h->block_bits;
  mc.rs_R = R;
  mc.rs_budget = smem_rows;
  mc.rs_total = 0;
  uint64_t words = 0;
  for (uint32_t k = 0; k < N; ++k)
    if (k != mode) words += (uint64_t(h->dims[k]) + 31) / 32;
  if (smem_rows == 0 || h->nnz == 0 || words > max_words) return;
  struct Cand { uint32_t cnt, k, row; };
  std::vector<Cand> cand;
  std::vector<std::vector<uint32_t>> hc(N);
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode) continue;
    DevArray<uint32_t> c(h->dims[k], s);
    PASTA_CUDA(cudaMemsetAsync(c.p, 0, c.bytes(), s));
    const bool comp = (h->cmask >> k) & 1u;
    hicoo_row_count_kernel<<<grid8(h->nnz), 256, 0, s>>>(h->bptr.p, h->nblocks, comp ? h->binds[k].p : nullptr,
                                                         comp ? h->einds[k].p : nullptr, comp ? nullptr : h->uinds[k].p,
                                                         bb, h->nnz, c.p);
    PASTA_LAUNCHED();
    hc[k].resize(h->dims[k]);
    PASTA_CUDA(cudaMemcpyAsync(hc[k].data(), c.p, c.bytes(), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    for (uint32_t r = 0; r < h->dims[k]; ++r)
      if (hc[k][r]) cand.push_back({hc[k][r], k, r});
  }
  std::stable_sort(cand.begin(), cand.end(), [](const Cand &a, const Cand &b) { return a.cnt > b.cnt; });
  if (cand.size() > smem_rows) cand.resize(smem_rows);
  std::vector<std::vector<uint32_t>> rows(N);
  for (const Cand &c : cand) rows[c.k].push_back(c.row);
  std::vector<uint32_t> all;
  for (uint32_t k = 0; k < N; ++k) {
    mc.rs_base[k] = all.size();
    mc.rs_words[k] = 0;
    if (k == mode) continue;
    std::sort(rows[k].begin(), rows[k].end());  // slot order = row order (prefix counts)
    const uint64_t nw = (uint64_t(h->dims[k]) + 31) / 32;
    std::vector<uint32_t> bm(nw, 0), pre(nw, 0);
    for (uint32_t r : rows[k]) bm[r >> 5] |= 1u << (r & 31);
    uint32_t run = 0;
    for (uint64_t w = 0; w < nw; ++w) { pre[w] = run; run += uint32_t(__builtin_popcount(bm[w])); }
    mc.rs_words[k] = nw;
    mc.rs_bm[k].alloc(nw, s);
    mc.rs_pre[k].alloc(nw, s);
    PASTA_CUDA(cudaMemcpyAsync(mc.rs_bm[k].p, bm.data(), nw * 4, cudaMemcpyHostToDevice, s));
    PASTA_CUDA(cudaMemcpyAsync(mc.rs_pre[k].p, pre.data(), nw * 4, cudaMemcpyHostToDevice, s));
    all.insert(all.end(), rows[k].begin(), rows[k].end());
    PASTA_CUDA(cudaStreamSynchronize(s));
  }
  mc.rs_total = all.size();
  mc.rs_rows.alloc(std::max<size_t>(all.size(), 1), s);
  if (!all.empty())
    PASTA_CUDA(cudaMemcpyAsync(mc.rs_rows.p, all.data(), all.size() * 4, cudaMemcpyHostToDevice, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  if (getenv("PASTA_DEBUG"))
    fprintf(stderr, "[pasta] hicoo row tier mode %u R %u: %llu smem rows, %llu bitmap words\n", mode, R,
            (unsigned long long)mc.rs_total, (unsigned long long)words);
}

}  // namespace pasta
