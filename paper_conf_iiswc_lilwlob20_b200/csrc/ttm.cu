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

// TTV (Eq. 1) on the fiberised matrix: y[f] = sum_{x in fiber f} val[x] * v[i_n[x]].
// Warp-level segmented reduction (the north_star's "warp-level segmented reduction
// (shuffles) over runs of equal output index, and atomics only at segment boundaries"): a warp
// takes a tile of 128 consecutive nonzeros, lane l the 4 at 4l (128-bit loads of fiber ids,
// i_n and values: fully coalesced); runs inside a lane are summed in registers; the lanes'
// trailing runs are combined by a 5-step segmented Kogge-Stone scan with shuffles; a run is
// written by the lane where it ends -- a plain store when it lies inside the tile (the fiber
// is exclusively this warp's), an atomicAdd when it touches the tile's first or last entry
// (it may continue in the neighbouring tile).  y must be zeroed.
__global__ void __launch_bounds__(256) ttv_segsum_kernel(const uint32_t *__restrict__ fid,
                                                         const uint32_t *__restrict__ in,
                                                         const float *__restrict__ val,
                                                         const float *__restrict__ v, uint64_t M,
                                                         float *__restrict__ y) {
  constexpr uint32_t kNone = 0xFFFFFFFFu;
  const unsigned full = 0xFFFFFFFFu;
  const int lane = threadIdx.x & 31;
  const uint64_t warp = (uint64_t(blockIdx.x) * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * blockDim.x) >> 5;
  for (uint64_t t0 = warp * 128; t0 < M; t0 += nwarps * 128) {
    const uint64_t x = t0 + 4 * uint64_t(lane);
    uint32_t f[4];
    float p[4];
    if (x + 3 < M) {
      const uint4 a = __ldg(reinterpret_cast<const uint4 *>(fid + x));
      const uint4 b = __ldg(reinterpret_cast<const uint4 *>(in + x));
      const float4 c = __ldg(reinterpret_cast<const float4 *>(val + x));
      f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w;
      p[0] = c.x * __ldg(v + b.x); p[1] = c.y * __ldg(v + b.y);
      p[2] = c.z * __ldg(v + b.z); p[3] = c.w * __ldg(v + b.w);
    } else {
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const bool ok = x + i < M;
        f[i] = ok ? fid[x + i] : kNone;
        p[i] = ok ? val[x + i] * __ldg(v + in[x + i]) : 0.f;
      }
    }
    const uint32_t tile_first = __shfl_sync(full, f[0], 0);
    // lane-local runs: first run, interior runs (complete, exclusive), trailing run
    const uint32_t ff = f[0];
    float first_sum = p[0];
    int i = 1;
    while (i < 4 && f[i] == ff) first_sum += p[i++];
    const bool single = i == 4;
    float last_sum = first_sum;
    uint32_t lf = ff;
    if (!single) {
      lf = f[i];
      last_sum = p[i];
      for (int j = i + 1; j < 4; ++j) {
        if (f[j] == lf) {
          last_sum += p[j];
        } else {
          y[lf] = last_sum;  // interior run: the whole fiber
          lf = f[j];
          last_sum = p[j];
        }
      }
    }
    const uint32_t tile_last = __shfl_sync(full, lf, 31);
    // segmented inclusive scan of the trailing runs across lanes
    const uint32_t plf = __shfl_up_sync(full, lf, 1);
    bool head = !single || lane == 0 || plf != ff;
    float sv = last_sum;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const float ov = __shfl_up_sync(full, sv, d);
      const bool oh = __shfl_up_sync(full, head, d);
      if (lane >= d) {
        if (!head) sv += ov;
        head = head || oh;
      }
    }
    const float carry_src = __shfl_up_sync(full, sv, 1);
    const uint32_t nff = __shfl_down_sync(full, ff, 1);
    auto emit = [&](uint32_t fb, float val_) {
      if (fb == kNone) return;
      if (fb == tile_first || fb == tile_last) atomicAdd(y + fb, val_);
      else y[fb] = val_;
    };
    if (!single) {
      const float carry = (lane > 0 && plf == ff) ? carry_src : 0.f;
      emit(ff, first_sum + carry);  // the first run ends inside this lane
    }
    if (lane == 31 || nff != lf) emit(lf, sv);  // the trailing run ends here
  }
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

void launch_ttv(const pasta_coo &mat, const float *v, float *y, cudaStream_t s) {
  const uint64_t M = mat.nnz;
  if (M == 0) return;
  const CooModeCopy &mc = mat.mc[0];
  const bool al = ((reinterpret_cast<uintptr_t>(mc.inds[0]) | reinterpret_cast<uintptr_t>(mc.inds[1]) |
                    reinterpret_cast<uintptr_t>(mc.val)) & 15u) == 0;
  if (!al) fail(PASTA_ECUDA, "ttv: fiber arrays not 16-byte aligned");
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  uint64_t want = (M + 128 * 8 - 1) / (128 * 8);
  uint64_t grid = uint64_t(sms) * 8;
  if (want < grid) grid = want;
  ttv_segsum_kernel<<<unsigned(grid), 256, 0, s>>>(mc.inds[0], mc.inds[1], mc.val, v, M, y);
  PASTA_LAUNCHED();
}

}  // namespace pasta
