// tew.cu -- tensor element-wise (TEW) and tensor-scalar (TS) operations
// (SURVEY NEXT-4): the streaming, trivially HBM-bound kernels of the suite (Table I: TEW 12M
// bytes / M flops, TS 8M bytes / M flops).
//
//   TS:  y = x op s on the values of X, same pattern (the output indices are set in
//        pre-processing).
//   TEW: z = x op y.  Same pattern (the benchmarked case): one pass over the values.
//        Different patterns (footnote 3): the output pattern is predicted first from
//        a merge of the two mode-0 lexicographic index lists (R#31: union for add/sub,
//        intersection for mul/div), then the values are computed per merged coordinate.
//
// Design for HBM: 128-bit loads with an L2 evict_first hint (each byte is used once),
// 128-bit stores (streaming .cs for TEW, plain for TS: measured), four vectors in flight per
// thread, a grid of 148 x 8 CTAs walking the arrays in grid-stride order.  IEEE fp32 operations (correctly rounded, incl. division).
#include <cub/cub.cuh>

#include <cstdlib>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kThreads = 256;

__device__ __forceinline__ float apply(uint32_t op, float a, float b) {
  switch (op) {
    case PASTA_OP_ADD: return __fadd_rn(a, b);
    case PASTA_OP_SUB: return __fsub_rn(a, b);
    case PASTA_OP_MUL: return __fmul_rn(a, b);
    default: return __fdiv_rn(a, b);
  }
}

__device__ __forceinline__ float4 ld_stream(const float4 *p, uint64_t pol) {
  float4 r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
      : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
      : "l"(p), "l"(pol));
  return r;
}

template <bool kCs>
__device__ __forceinline__ void st_stream(float4 *p, float4 v) {
  if (kCs)
    asm volatile("st.global.cs.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(p), "f"(v.x), "f"(v.y), "f"(v.z),
                 "f"(v.w)
                 : "memory");
  else
    *p = v;
}

// TS (b == nullptr: scalar s) and same-pattern TEW over n4 float4 + a scalar tail.
// kVec float4 in flight per thread; kCs: streaming (evict-first) stores.
template <uint32_t OP, bool kScalar, int kVec = 4, bool kCs = true>
__global__ void __launch_bounds__(kThreads) ew_kernel(const float *__restrict__ a, const float *__restrict__ b,
                                                      float s, float *__restrict__ out, uint64_t n) {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  const uint64_t n4 = n / 4;
  const float4 *a4 = reinterpret_cast<const float4 *>(a);
  const float4 *b4 = reinterpret_cast<const float4 *>(b);
  float4 *o4 = reinterpret_cast<float4 *>(out);
  const uint64_t stride = uint64_t(gridDim.x) * kThreads;
  uint64_t i = uint64_t(blockIdx.x) * kThreads + threadIdx.x;
  // main loop: kVec independent vectors in flight per thread
  for (; i + (kVec - 1) * stride < n4; i += kVec * stride) {
    float4 va[kVec], vb[kVec];
#pragma unroll
    for (int v = 0; v < kVec; ++v) va[v] = ld_stream(a4 + i + v * stride, pol);
    if (!kScalar) {
#pragma unroll
      for (int v = 0; v < kVec; ++v) vb[v] = ld_stream(b4 + i + v * stride, pol);
    }
#pragma unroll
    for (int v = 0; v < kVec; ++v) {
      const float4 y = kScalar ? make_float4(s, s, s, s) : vb[v];
      st_stream<kCs>(o4 + i + v * stride, make_float4(apply(OP, va[v].x, y.x), apply(OP, va[v].y, y.y),
                                                 apply(OP, va[v].z, y.z), apply(OP, va[v].w, y.w)));
    }
  }
  for (; i < n4; i += stride) {
    const float4 x = ld_stream(a4 + i, pol);
    const float4 y = kScalar ? make_float4(s, s, s, s) : ld_stream(b4 + i, pol);
    st_stream<kCs>(o4 + i, make_float4(apply(OP, x.x, y.x), apply(OP, x.y, y.y), apply(OP, x.z, y.z),
                                  apply(OP, x.w, y.w)));
  }
  // tail (n % 4 elements), and the whole array when the pointers are not 16-B aligned
  for (uint64_t e = n4 * 4 + uint64_t(blockIdx.x) * kThreads + threadIdx.x; e < n; e += stride)
    out[e] = apply(OP, a[e], kScalar ? s : b[e]);
}

template <uint32_t OP, bool kScalar>
__global__ void __launch_bounds__(kThreads) ew_scalar_kernel(const float *__restrict__ a, const float *__restrict__ b,
                                                             float s, float *__restrict__ out, uint64_t n) {
  for (uint64_t e = uint64_t(blockIdx.x) * kThreads + threadIdx.x; e < n; e += uint64_t(gridDim.x) * kThreads)
    out[e] = apply(OP, a[e], kScalar ? s : b[e]);
}

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

int sms() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

int ew_variant() {
  static int v = -1;
  if (v < 0) {
    const char *e = getenv("PASTA_EW_VARIANT");
    v = (e && *e) ? atoi(e) : 0;
  }
  return v;
}

template <uint32_t OP, bool kScalar>
void launch_ew_op(bool vec, const float *a, const float *b, float s, float *out, uint64_t n, cudaStream_t st) {
  // grid: 8 CTAs of 256 threads per SM (full occupancy), fewer for small arrays
  const int var = ew_variant();
  uint64_t want = (n / 4 + kThreads - 1) / kThreads;
  uint64_t grid = uint64_t(sms()) * (var == 4 ? 4 : 8);
  if (want < grid) grid = want ? want : 1;
  auto go = [&](auto k) {
    k<<<unsigned(grid), kThreads, 0, st>>>(a, b, s, out, n);
    PASTA_LAUNCHED();
  };
  if (!vec) return go(ew_scalar_kernel<OP, kScalar>);
  // PASTA_EW_VARIANT: tuning knob (1: 2 in flight, 2: 8 in flight, 3: plain stores, 5:
  // streaming stores).  Default (measured on B200, tools/ew_sweep.py): TS (1 read : 1 write)
  // with plain stores 6.0 TB/s vs 5.66 with .cs; TEW (2 : 1) with .cs stores 6.4 vs 6.2.
  switch (var) {
    case 1: go(ew_kernel<OP, kScalar, 2, true>); break;
    case 2: go(ew_kernel<OP, kScalar, 8, true>); break;
    case 3: go(ew_kernel<OP, kScalar, 4, false>); break;
    case 5: go(ew_kernel<OP, kScalar, 4, true>); break;
    default: go(ew_kernel<OP, kScalar, 4, !kScalar>); break;
  }
}

template <bool kScalar>
void launch_ew(uint32_t op, const float *a, const float *b, float s, float *out, uint64_t n, cudaStream_t st) {
  if (n == 0) return;
  const bool vec = aligned16(a) && aligned16(out) && (kScalar || aligned16(b));
  ProfScope prof(kProfEw, st);
  switch (op) {
    case PASTA_OP_ADD: launch_ew_op<PASTA_OP_ADD, kScalar>(vec, a, b, s, out, n, st); break;
    case PASTA_OP_SUB: launch_ew_op<PASTA_OP_SUB, kScalar>(vec, a, b, s, out, n, st); break;
    case PASTA_OP_MUL: launch_ew_op<PASTA_OP_MUL, kScalar>(vec, a, b, s, out, n, st); break;
    default: launch_ew_op<PASTA_OP_DIV, kScalar>(vec, a, b, s, out, n, st); break;
  }
}

inline unsigned grid_for(uint64_t n) {
  uint64_t b = (n + kThreads * 4 - 1) / (kThreads * 4);
  if (b < 1) b = 1;
  if (b > (1u << 30)) b = 1u << 30;
  return unsigned(b);
}

struct Idx {
  const uint32_t *c[kMaxOrder];
  uint32_t order;
};

// diff[0] = 1 iff the two index lists differ anywhere
__global__ void differ_kernel(Idx a, Idx b, uint64_t M, int *__restrict__ diff) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M; x += uint64_t(gridDim.x) * blockDim.x) {
    bool d = false;
    for (uint32_t k = 0; k < a.order; ++k) d |= a.c[k][x] != b.c[k][x];
    if (d) *diff = 1;
  }
}

// Merged list (x's sorted entries, then y's), permuted by a stable lexicographic sort:
// grp[s] = 1 iff sorted position s starts a new coordinate.
__global__ void group_flag_kernel(Idx cat, const uint32_t *__restrict__ perm, uint64_t T, uint8_t *__restrict__ grp) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s < T; s += uint64_t(gridDim.x) * blockDim.x) {
    uint8_t f = s == 0;
    if (s > 0)
      for (uint32_t k = 0; k < cat.order; ++k) f |= cat.c[k][perm[s]] != cat.c[k][perm[s - 1]];
    grp[s] = f;
  }
}

// For each group (start positions `starts`, count G): keep flag by op, duplicate detection.
__global__ void group_keep_kernel(const uint32_t *__restrict__ starts, uint64_t G, uint64_t T,
                                  const uint32_t *__restrict__ perm, uint64_t Mx, uint32_t op,
                                  uint32_t *__restrict__ keep, int *__restrict__ dup) {
  for (uint64_t g = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; g < G; g += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t s0 = starts[g], s1 = g + 1 < G ? starts[g + 1] : T;
    const uint64_t cnt = s1 - s0;
    if (cnt > 2 || (cnt == 2 && (perm[s0] < Mx) == (perm[s0 + 1] < Mx))) *dup = 1;
    const bool both = cnt == 2;
    keep[g] = (op == PASTA_OP_ADD || op == PASTA_OP_SUB) ? 1u : (both ? 1u : 0u);
  }
}

struct MergeOut {
  uint32_t *c[kMaxOrder];
  float *val;
};

__global__ void group_emit_kernel(Idx cat, const float *__restrict__ catv, const uint32_t *__restrict__ starts,
                                  uint64_t G, uint64_t T, const uint32_t *__restrict__ perm, uint64_t Mx,
                                  const uint32_t *__restrict__ keep, const uint64_t *__restrict__ pos, uint32_t op,
                                  MergeOut o) {
  for (uint64_t g = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; g < G; g += uint64_t(gridDim.x) * blockDim.x) {
    if (!keep[g]) continue;
    const uint64_t s0 = starts[g], s1 = g + 1 < G ? starts[g + 1] : T;
    const uint32_t p0 = perm[s0];
    float xv = 0.f, yv = 0.f;
    bool hx = false, hy = false;
    for (uint64_t s = s0; s < s1; ++s) {
      const uint32_t p = perm[s];
      if (p < Mx) { xv = catv[p]; hx = true; } else { yv = catv[p]; hy = true; }
    }
    float z;
    if (hx && hy) z = apply(op, xv, yv);
    else if (hx) z = xv;                                      // x op 0, op in {add, sub}
    else z = op == PASTA_OP_SUB ? __fsub_rn(0.f, yv) : yv;   // 0 op y
    const uint64_t w = pos[g];
    for (uint32_t k = 0; k < cat.order; ++k) o.c[k][w] = cat.c[k][p0];
    o.val[w] = z;
  }
}

__global__ void copy_u32_kernel(const uint32_t *__restrict__ a, uint32_t *__restrict__ b, uint64_t n) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    b[i] = a[i];
}

// All-gather by peer stores (a9): a contiguous float range copied into up to 8 replicas
// (local and CUDA-IPC-mapped peers); 128-bit loads once, one 128-bit store per replica.
struct Dst8 {
  float *d[8];
  uint32_t n;
};

__global__ void __launch_bounds__(kThreads) bcast_kernel(const float *__restrict__ src, uint64_t n, Dst8 dst) {
  uint64_t pol;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  const uint64_t n4 = n / 4, stride = uint64_t(gridDim.x) * kThreads;
  const float4 *s4 = reinterpret_cast<const float4 *>(src);
  for (uint64_t i = uint64_t(blockIdx.x) * kThreads + threadIdx.x; i < n4; i += stride) {
    const float4 v = ld_stream(s4 + i, pol);
    for (uint32_t k = 0; k < dst.n; ++k) reinterpret_cast<float4 *>(dst.d[k])[i] = v;
  }
  for (uint64_t e = n4 * 4 + uint64_t(blockIdx.x) * kThreads + threadIdx.x; e < n; e += stride)
    for (uint32_t k = 0; k < dst.n; ++k) dst.d[k][e] = src[e];
  __threadfence_system();
}

}  // namespace

void launch_ts(uint32_t op, const float *x, float s, float *y, uint64_t n, cudaStream_t st) {
  launch_ew<true>(op, x, nullptr, s, y, n, st);
}

void launch_tew(uint32_t op, const float *a, const float *b, float *z, uint64_t n, cudaStream_t st) {
  launch_ew<false>(op, a, b, 0.f, z, n, st);
}

void launch_bcast(const float *src, uint64_t n, float *const *dsts, uint32_t ndst, cudaStream_t st) {
  if (ndst < 1 || ndst > 8) fail(PASTA_EINVAL, "pasta_bcast_f32: 1..8 destinations");
  if (n == 0) return;
  Dst8 d{};
  d.n = ndst;
  bool al = aligned16(src);
  for (uint32_t k = 0; k < ndst; ++k) { d.d[k] = dsts[k]; al = al && aligned16(dsts[k]); }
  if (!al) fail(PASTA_EINVAL, "pasta_bcast_f32: pointers must be 16-byte aligned");
  uint64_t want = (n / 4 + kThreads - 1) / kThreads;
  uint64_t grid = uint64_t(sms()) * 8;
  if (want < grid) grid = want ? want : 1;
  bcast_kernel<<<unsigned(grid), kThreads, 0, st>>>(src, n, d);
  PASTA_LAUNCHED();
}

bool same_pattern_device(const pasta_coo *x, const pasta_coo *y, cudaStream_t s) {
  if (x->order != y->order || x->nnz != y->nnz) return false;
  for (uint32_t k = 0; k < x->order; ++k)
    if (x->dims[k] != y->dims[k]) return false;
  if (x->nnz == 0) return true;
  Idx a{}, b{};
  a.order = b.order = x->order;
  for (uint32_t k = 0; k < x->order; ++k) { a.c[k] = x->inds[k].p; b.c[k] = y->inds[k].p; }
  DevArray<int> d(1, s);
  PASTA_CUDA(cudaMemsetAsync(d.p, 0, sizeof(int), s));
  differ_kernel<<<grid_for(x->nnz), kThreads, 0, s>>>(a, b, x->nnz, d.p);
  PASTA_LAUNCHED();
  int h = 0;
  PASTA_CUDA(cudaMemcpyAsync(&h, d.p, sizeof(int), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  return h == 0;
}

void copy_pattern_device(const pasta_coo *x, pasta_coo *y, cudaStream_t s) {
  y->order = x->order;
  for (uint32_t k = 0; k < x->order; ++k) y->dims[k] = x->dims[k];
  y->nnz = x->nnz;
  y->device = x->device;
  y->lex_sorted = x->lex_sorted;
  for (uint32_t k = 0; k < x->order; ++k) {
    y->inds[k].alloc(x->nnz, s);
    if (x->nnz) {
      copy_u32_kernel<<<grid_for(x->nnz), kThreads, 0, s>>>(x->inds[k].p, y->inds[k].p, x->nnz);
      PASTA_LAUNCHED();
    }
  }
  y->val.alloc(x->nnz, s);
}

// General TEW (R#31): x, y have mode-0 lexicographic working copies (coo_prepare_mode(., 0)).
void tew_merge_device(const pasta_coo *x, const pasta_coo *y, uint32_t op, pasta_coo *z, cudaStream_t s) {
  const uint32_t N = x->order;
  const uint64_t Mx = x->nnz, My = y->nnz, T = Mx + My;
  if (T > 0xFFFFFFFEull) fail(PASTA_ERANGE, "tew: more than 2^32-2 merged nonzeros");
  const CooModeCopy &mx = x->mc[0], &my = y->mc[0];
  DevArray<uint32_t> cat[kMaxOrder];
  DevArray<float> catv(T, s);
  Idx ci{};
  ci.order = N;
  uint32_t bits[kMaxOrder];
  const uint32_t *comps[kMaxOrder];
  for (uint32_t k = 0; k < N; ++k) {
    cat[k].alloc(T, s);
    if (Mx) PASTA_CUDA(cudaMemcpyAsync(cat[k].p, mx.inds[k], Mx * 4, cudaMemcpyDeviceToDevice, s));
    if (My) PASTA_CUDA(cudaMemcpyAsync(cat[k].p + Mx, my.inds[k], My * 4, cudaMemcpyDeviceToDevice, s));
    ci.c[k] = cat[k].p;
    comps[k] = cat[k].p;
    bits[k] = ceil_log2(x->dims[k]);
  }
  if (Mx) PASTA_CUDA(cudaMemcpyAsync(catv.p, mx.val, Mx * 4, cudaMemcpyDeviceToDevice, s));
  if (My) PASTA_CUDA(cudaMemcpyAsync(catv.p + Mx, my.val, My * 4, cudaMemcpyDeviceToDevice, s));
  DevArray<uint32_t> perm(T, s);
  iota_u32(perm.p, T, s);
  lexsort(comps, bits, int(N), perm, T, s);  // stable: x's entry precedes y's on a tie
  uint64_t G = 0;
  DevArray<uint32_t> starts;
  if (T) {
    DevArray<uint8_t> grp(T, s);
    group_flag_kernel<<<grid_for(T), kThreads, 0, s>>>(ci, perm.p, T, grp.p);
    PASTA_LAUNCHED();
    G = select_flagged(grp.p, T, starts, s);
  }
  DevArray<uint32_t> keep(G + 1, s);
  DevArray<uint64_t> pos(G + 1, s);
  DevArray<int> dup(1, s);
  PASTA_CUDA(cudaMemsetAsync(dup.p, 0, sizeof(int), s));
  PASTA_CUDA(cudaMemsetAsync(keep.p, 0, (G + 1) * sizeof(uint32_t), s));
  if (G) {
    group_keep_kernel<<<grid_for(G), kThreads, 0, s>>>(starts.p, G, T, perm.p, Mx, op, keep.p, dup.p);
    PASTA_LAUNCHED();
  }
  size_t tb = 0;
  PASTA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, keep.p, pos.p, G + 1, s));
  DevArray<uint8_t> tmp(tb, s);
  PASTA_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tb, keep.p, pos.p, G + 1, s));
  count_launch();
  int hdup = 0;
  uint64_t nz = 0;
  PASTA_CUDA(cudaMemcpyAsync(&hdup, dup.p, sizeof(int), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaMemcpyAsync(&nz, pos.p + G, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  if (hdup) fail(PASTA_EINVAL, "tew: an input tensor repeats a coordinate");
  z->order = N;
  for (uint32_t k = 0; k < N; ++k) z->dims[k] = x->dims[k];
  z->nnz = nz;
  z->device = x->device;
  z->lex_sorted = true;
  MergeOut o{};
  for (uint32_t k = 0; k < N; ++k) {
    z->inds[k].alloc(nz, s);
    o.c[k] = z->inds[k].p;
  }
  z->val.alloc(nz, s);
  o.val = z->val.p;
  if (G) {
    group_emit_kernel<<<grid_for(G), kThreads, 0, s>>>(ci, catv.p, starts.p, G, T, perm.p, Mx, keep.p, pos.p, op, o);
    PASTA_LAUNCHED();
  }
  PASTA_CUDA(cudaStreamSynchronize(s));
}

}  // namespace pasta
