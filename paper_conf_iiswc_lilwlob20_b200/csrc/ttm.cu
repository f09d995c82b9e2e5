// ttm.cu -- mode-n fibers of a COO tensor for TTV / TTM (Eq. 1, Eq. 2).
// The paper pre-processes the fibers (f_ptr, M_F) and pre-allocates the semi-sparse
// output (sCOO) by the sparse-dense property: the output has one dense length-R
// vector per mode-n fiber.  Here the fibers become the rows of an order-2 COO matrix
// (fiber id, i_n), so TTM is the mode-0 MTTKRP of that matrix with the single factor U and runs
// on the same segmented-reduction kernel (TTV: R = 1).
#include <cub/cub.cuh>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kThreads = 256;

inline unsigned grid_for(uint64_t n) {
  uint64_t b = (n + kThreads * 4 - 1) / (kThreads * 4);
  if (b < 1) b = 1;
  if (b > (1u << 30)) b = 1u << 30;
  return unsigned(b);
}

struct Others {
  const uint32_t *c[kMaxOrder];
  uint32_t n;
};

// flag[x] = 1 iff sorted position x starts a new fiber (some i_k, k != mode, changes)
__global__ void fiber_flag_kernel(Others o, uint64_t M, uint32_t *__restrict__ flag) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t f = x == 0;
    if (x > 0)
      for (uint32_t j = 0; j < o.n; ++j) f |= o.c[j][x] != o.c[j][x - 1];
    flag[x] = f;
  }
}

__global__ void minus_one_kernel(uint32_t *__restrict__ v, uint64_t M) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    v[x] -= 1;
}

__global__ void u32_to_u8_kernel(const uint32_t *__restrict__ in, uint64_t M, uint8_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = uint8_t(in[x]);
}

}  // namespace

void coo_build_fibers(pasta_coo *x, uint32_t mode, cudaStream_t s) {
  if (x->fib[mode]) return;
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  auto fc = new FiberCopy();
  try {
    // sort by (i_k for k != mode, ascending k), then i_mode
    const uint32_t *comps[kMaxOrder];
    uint32_t bits[kMaxOrder];
    int nc = 0;
    for (uint32_t k = 0; k < N; ++k)
      if (k != mode) { comps[nc] = x->inds[k].p; bits[nc] = ceil_log2(x->dims[k]); ++nc; }
    comps[nc] = x->inds[mode].p;
    bits[nc] = ceil_log2(x->dims[mode]);
    ++nc;
    DevArray<uint32_t> perm(M, s);
    iota_u32(perm.p, M, s);
    lexsort(comps, bits, nc, perm, M, s);
    DevArray<uint32_t> sk[kMaxOrder];
    Others o{};
    for (uint32_t k = 0; k < N; ++k) {
      sk[k].alloc(M, s);
      gather_u32(x->inds[k].p, perm.p, sk[k].p, M, s);
      if (k != mode) o.c[o.n++] = sk[k].p;
    }
    pasta_coo &mat = fc->mat;
    mat.order = 2;
    mat.nnz = M;
    mat.device = x->device;
    mat.dims[1] = x->dims[mode];
    mat.val.alloc(M, s);
    gather_f32(x->val.p, perm.p, mat.val.p, M, s);
    mat.inds[1] = std::move(sk[mode]);
    // fiber ids: inclusive scan of the fiber-start flags, minus one
    DevArray<uint32_t> flag(M, s);
    mat.inds[0].alloc(M, s);
    uint64_t nf = 0;
    DevArray<uint32_t> starts;
    if (M) {
      fiber_flag_kernel<<<grid_for(M), kThreads, 0, s>>>(o, M, flag.p);
      PASTA_LAUNCHED();
      size_t tb = 0;
      PASTA_CUDA(cub::DeviceScan::InclusiveSum(nullptr, tb, flag.p, mat.inds[0].p, M, s));
      DevArray<uint8_t> tmp(tb, s);
      PASTA_CUDA(cub::DeviceScan::InclusiveSum(tmp.p, tb, flag.p, mat.inds[0].p, M, s));
      count_launch();
      minus_one_kernel<<<grid_for(M), kThreads, 0, s>>>(mat.inds[0].p, M);
      PASTA_LAUNCHED();
      DevArray<uint8_t> f8(M, s);
      u32_to_u8_kernel<<<grid_for(M), kThreads, 0, s>>>(flag.p, M, f8.p);
      PASTA_LAUNCHED();
      nf = select_flagged(f8.p, M, starts, s);
    }
    fc->nf = nf;
    mat.dims[0] = uint32_t(nf ? nf : 1);
    for (uint32_t k = 0; k < N; ++k) {
      if (k == mode) continue;
      fc->finds[k].alloc(nf, s);
      if (nf) gather_u32(sk[k].p, starts.p, fc->finds[k].p, nf, s);
    }
    mat.lex_sorted = true;  // sorted by (fiber id, i_mode)
    PASTA_CUDA(cudaStreamSynchronize(s));
  } catch (...) {
    delete fc;
    throw;
  }
  x->fib[mode] = fc;
}

}  // namespace pasta
