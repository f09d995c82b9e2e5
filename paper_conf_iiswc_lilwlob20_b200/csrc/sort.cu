// sort.cu -- device pre-processing primitives: stable lexicographic / Morton sorts
// (LSD passes of CUB radix sort, a library call used only in pre-processing),
// gathers, compaction, histograms.  Pre-processing trades for kernel time.
#include <cub/cub.cuh>

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
