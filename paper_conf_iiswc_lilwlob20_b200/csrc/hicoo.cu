// hicoo.cu -- COO -> HiCOO conversion (R#10-R#14) and the per-mode
// HiCOO working copy used by the GPU MTTKRP (R#27).
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

struct Coords {
  const uint32_t *c[kMaxOrder];
  uint32_t order;
};

// flag[s] = 1 iff position s (Morton-sorted) starts a new block: (i_k >> b) differs for some k
__global__ void block_flag_kernel(Coords a, uint32_t bbits, uint64_t M, uint8_t *__restrict__ flag) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s < M;
       s += uint64_t(gridDim.x) * blockDim.x) {
    uint8_t f = (s == 0);
    if (s > 0)
      for (uint32_t k = 0; k < a.order; ++k) f |= ((a.c[k][s] >> bbits) != (a.c[k][s - 1] >> bbits));
    flag[s] = f;
  }
}

__global__ void emit_blocks_kernel(const uint32_t *__restrict__ starts, uint64_t nb, uint64_t M,
                                   const uint32_t *__restrict__ sc, uint32_t bbits,
                                   uint64_t *__restrict__ bptr, uint32_t *__restrict__ binds_k,
                                   int write_bptr) {
  for (uint64_t j = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; j <= nb;
       j += uint64_t(gridDim.x) * blockDim.x) {
    if (j == nb) {
      if (write_bptr) bptr[nb] = M;
      continue;
    }
    uint32_t s = starts[j];
    if (write_bptr) bptr[j] = s;
    binds_k[j] = sc[s] >> bbits;
  }
}

__global__ void emit_einds_kernel(const uint32_t *__restrict__ sc, uint64_t M, uint32_t mask,
                                  uint8_t *__restrict__ e) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s < M;
       s += uint64_t(gridDim.x) * blockDim.x)
    e[s] = uint8_t(sc[s] & mask);
}

// blk[x] = block containing entry x: last j with bptr[j] <= x
__global__ void entry_block_kernel(const uint64_t *__restrict__ bptr, uint64_t nb, uint64_t M,
                                   uint32_t *__restrict__ blk) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    uint64_t lo = 0, hi = nb;  // answer in [0, nb)
    while (hi - lo > 1) {
      uint64_t mid = (lo + hi) / 2;
      if (bptr[mid] <= x) lo = mid; else hi = mid;
    }
    blk[x] = uint32_t(lo);
  }
}

__global__ void gather_binds_kernel(const uint32_t *__restrict__ binds_n, const uint32_t *__restrict__ blk,
                                    uint64_t M, uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = binds_n[blk[x]];
}

__global__ void u8_to_u32_kernel(const uint8_t *__restrict__ in, uint64_t M, uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = in[x];
}

__global__ void sched_counts_kernel(const uint64_t *__restrict__ bptr, const uint32_t *__restrict__ sched,
                                    uint64_t nb, uint64_t *__restrict__ cnt) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s <= nb;
       s += uint64_t(gridDim.x) * blockDim.x) {
    if (s == nb) { cnt[s] = 0; continue; }
    uint32_t b = sched[s];
    cnt[s] = bptr[b + 1] - bptr[b];
  }
}

}  // namespace

void coo_to_hicoo_device(const pasta_coo *x, pasta_hicoo *h, cudaStream_t s) {
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  const uint32_t bb = h->block_bits;
  uint32_t Lm = 0;
  for (uint32_t k = 0; k < N; ++k) Lm = ceil_log2(x->dims[k]) > Lm ? ceil_log2(x->dims[k]) : Lm;
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  const uint32_t *canon[kMaxOrder];
  for (uint32_t k = 0; k < N; ++k) canon[k] = x->inds[k].p;
  morton_sort(canon, N, Lm, perm, M, s);

  DevArray<uint32_t> sc[kMaxOrder];
  Coords co{};
  co.order = N;
  for (uint32_t k = 0; k < N; ++k) {
    sc[k].alloc(M, s);
    gather_u32(canon[k], perm.p, sc[k].p, M, s);
    co.c[k] = sc[k].p;
  }
  uint64_t nb = 0;
  DevArray<uint32_t> starts;
  if (M) {
    DevArray<uint8_t> flag(M, s);
    block_flag_kernel<<<grid_for(M), kThreads, 0, s>>>(co, bb, M, flag.p);
    PASTA_LAUNCHED();
    nb = select_flagged(flag.p, M, starts, s);
  }
  h->nblocks = nb;
  h->nnz = M;
  h->bptr.alloc(nb + 1, s);
  if (!M) {
    uint64_t zero = 0;
    PASTA_CUDA(cudaMemcpyAsync(h->bptr.p, &zero, sizeof(zero), cudaMemcpyHostToDevice, s));
  }
  for (uint32_t k = 0; k < N; ++k) {
    h->binds[k].alloc(nb, s);
    h->einds[k].alloc(M, s);
    if (M) {
      emit_blocks_kernel<<<grid_for(nb + 1), kThreads, 0, s>>>(starts.p, nb, M, sc[k].p, bb, h->bptr.p,
                                                             h->binds[k].p, k == 0);
      PASTA_LAUNCHED();
      emit_einds_kernel<<<grid_for(M), kThreads, 0, s>>>(sc[k].p, M, (1u << bb) - 1u, h->einds[k].p);
      PASTA_LAUNCHED();
    }
  }
  h->val.alloc(M, s);
  gather_f32(x->val.p, perm.p, h->val.p, M, s);
  PASTA_CUDA(cudaStreamSynchronize(s));
}

// Per-mode copy (R#27): blocks stably sorted by binds_mode, entries inside a block stably
// sorted by einds_mode, so equal output rows are contiguous runs (segmented reduction).
void hicoo_prepare_mode(pasta_hicoo *h, uint32_t mode, cudaStream_t s) {
  HicooModeCopy &mc = h->mc[mode];
  if (mc.ready) return;
  const uint32_t N = h->order;
  const uint64_t M = h->nnz, nb = h->nblocks;
  const uint32_t bb = h->block_bits;
  mc.bptr.alloc(nb + 1, s);
  for (uint32_t k = 0; k < N; ++k) {
    mc.binds[k].alloc(nb, s);
    mc.einds[k].alloc(M, s);
  }
  mc.val.alloc(M, s);
  if (M == 0) {
    uint64_t zero = 0;
    PASTA_CUDA(cudaMemcpyAsync(mc.bptr.p, &zero, sizeof(zero), cudaMemcpyHostToDevice, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    mc.ready = true;
    return;
  }
  // entry permutation: (binds_mode[blk], blk, einds_mode)
  DevArray<uint32_t> blk(M, s), c0(M, s), c2(M, s);
  entry_block_kernel<<<grid_for(M), kThreads, 0, s>>>(h->bptr.p, nb, M, blk.p);
  PASTA_LAUNCHED();
  gather_binds_kernel<<<grid_for(M), kThreads, 0, s>>>(h->binds[mode].p, blk.p, M, c0.p);
  PASTA_LAUNCHED();
  u8_to_u32_kernel<<<grid_for(M), kThreads, 0, s>>>(h->einds[mode].p, M, c2.p);
  PASTA_LAUNCHED();
  uint64_t nbr = (uint64_t(h->dims[mode]) + (1ull << bb) - 1) >> bb;  // block rows of this mode
  const uint32_t *comps[3] = {c0.p, blk.p, c2.p};
  uint32_t bits[3] = {ceil_log2(nbr), ceil_log2(nb), bb};
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  lexsort(comps, bits, 3, perm, M, s);
  for (uint32_t k = 0; k < N; ++k) gather_u8(h->einds[k].p, perm.p, mc.einds[k].p, M, s);
  gather_f32(h->val.p, perm.p, mc.val.p, M, s);
  // block schedule: blocks stably sorted by binds_mode (same order the entries now follow)
  DevArray<uint32_t> sched(nb, s);
  iota_u32(sched.p, nb, s);
  const uint32_t *bc[1] = {h->binds[mode].p};
  uint32_t bbit[1] = {ceil_log2(nbr)};
  lexsort(bc, bbit, 1, sched, nb, s);
  DevArray<uint64_t> cnt(nb + 1, s);
  sched_counts_kernel<<<grid_for(nb + 1), kThreads, 0, s>>>(h->bptr.p, sched.p, nb, cnt.p);
  PASTA_LAUNCHED();
  size_t tmp_bytes = 0;
  PASTA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, cnt.p, mc.bptr.p, nb + 1, s));
  DevArray<uint8_t> tmp(tmp_bytes, s);
  PASTA_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tmp_bytes, cnt.p, mc.bptr.p, nb + 1, s));
  count_launch();
  for (uint32_t k = 0; k < N; ++k) gather_u32(h->binds[k].p, sched.p, mc.binds[k].p, nb, s);
  PASTA_CUDA(cudaStreamSynchronize(s));
  mc.ready = true;
}

}  // namespace pasta
