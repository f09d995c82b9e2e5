// cpals.cu -- CANDECOMP/PARAFAC by alternating least squares around the MTTKRP (SURVEY
// NEXT-1).  The paper names MTTKRP as CPD's most expensive kernel and lists CPD as
// future work; the ALS update itself is the textbook one of its ref. [1] (Kolda &
// Bader): for each mode n,
//     M   = X_(n) (KRP of U_k, k != n)                      (MTTKRP, mttkrp.cu)
//     V   = Hadamard_{k != n} (U_k^T U_k)                     (R x R)
//     U_n = M V^{-1};  lambda_r = ||U_n(:, r)||_2;  U_n(:, r) /= lambda_r
// and fit = 1 - ||X - [[lambda; U]]|| / ||X|| from ||X||^2, <X, Xhat> = sum_r lambda_r
// sum_i M(i, r) U_n(i, r) (last mode) and ||Xhat||^2 = lambda^T (Hadamard_k G_k) lambda.
// Building blocks are exported through the C ABI so the multi-GPU driver (parallel.py) can
// all-reduce the R x R partials and all-gather the owned rows in between.
#include <cmath>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kThreads = 256;
constexpr int kMaxR = 64;

unsigned grid_rows(uint64_t rows, int per_cta) {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  uint64_t b = (rows + per_cta - 1) / per_cta;
  uint64_t cap = uint64_t(sms) * 16;
  if (b > cap) b = cap;
  return unsigned(b < 1 ? 1 : b);
}

// G (R x R, fp64, row-major) += U^T U over rows [0, rows).  Row tiles of 64 are staged in
// shared memory; thread t accumulates the upper-triangle pairs t, t + 256, ... in fp64.
__global__ void __launch_bounds__(kThreads) gram_kernel(const float *__restrict__ U, uint64_t rows,
                                                        uint32_t R, double *__restrict__ G) {
  __shared__ float tile[64 * kMaxR];
  const uint32_t npairs = R * (R + 1) / 2;
  constexpr int kAcc = (kMaxR * (kMaxR + 1) / 2 + kThreads - 1) / kThreads;
  double acc[kAcc];
  uint32_t pa[kAcc], pb[kAcc];
  const int nacc = int((npairs + kThreads - 1) / kThreads);
  for (int q = 0; q < nacc; ++q) {
    acc[q] = 0.0;
    // pair index p -> (a, b) with a <= b, row-major over the upper triangle
    uint32_t a = 0, rem = threadIdx.x + q * kThreads;
    while (a < R && rem >= R - a) { rem -= R - a; ++a; }
    pa[q] = a;
    pb[q] = a + rem;
  }
  for (uint64_t r0 = uint64_t(blockIdx.x) * 64; r0 < rows; r0 += uint64_t(gridDim.x) * 64) {
    const uint32_t nr = uint32_t(rows - r0 < 64 ? rows - r0 : 64);
    __syncthreads();
    for (uint32_t e = threadIdx.x; e < nr * R; e += kThreads) tile[e] = U[r0 * R + e];
    __syncthreads();
    for (int q = 0; q < nacc; ++q) {
      const uint32_t p = threadIdx.x + q * kThreads;
      if (p >= npairs) break;
      const uint32_t a = pa[q], b = pb[q];
      float s = 0.f;  // <= 64 terms in fp32, tiles combined in fp64 (fp64 is a slow pipe here)
      for (uint32_t i = 0; i < nr; ++i) s = fmaf(tile[i * R + a], tile[i * R + b], s);
      acc[q] += double(s);
    }
  }
  for (int q = 0; q < nacc; ++q) {
    const uint32_t p = threadIdx.x + q * kThreads;
    if (p >= npairs) break;
    const uint32_t a = pa[q], b = pb[q];
    atomicAdd(&G[a * R + b], acc[q]);
    if (a != b) atomicAdd(&G[b * R + a], acc[q]);
  }
}

struct GramList {
  const double *g[kMaxOrder];
  uint32_t n;
};

// W = (Hadamard of the grams)^{-1}, fp64 Gauss-Jordan with partial pivoting in shared memory
// (R <= 64; run by one warp of every CTA that needs it).  A singular V gets a tiny ridge.
__device__ void hadamard_inverse(const GramList &gl, uint32_t R, double *V, double *W) {
  const int lane = threadIdx.x & 31;
  for (uint32_t e = lane; e < R * R; e += 32) {
    double v = 1.0;
    for (uint32_t k = 0; k < gl.n; ++k) v *= gl.g[k][e];
    V[e] = v;
    W[e] = (e / R == e % R) ? 1.0 : 0.0;
  }
  __syncwarp();
  double tr = 0.0;
  for (uint32_t j = 0; j < R; ++j) tr += V[j * R + j];
  const double ridge = 1e-14 * (tr > 0 ? tr : 1.0) / R;
  for (uint32_t c = 0; c < R; ++c) {
    // pivot: largest |V(r, c)| for r >= c (lane 0 decides, everyone reads)
    __syncwarp();
    uint32_t piv = c;
    double best = fabs(V[c * R + c]);
    for (uint32_t r = c + 1; r < R; ++r)
      if (fabs(V[r * R + c]) > best) { best = fabs(V[r * R + c]); piv = r; }
    __syncwarp();
    if (piv != c) {
      for (uint32_t e = lane; e < R; e += 32) {
        double t = V[c * R + e]; V[c * R + e] = V[piv * R + e]; V[piv * R + e] = t;
        t = W[c * R + e]; W[c * R + e] = W[piv * R + e]; W[piv * R + e] = t;
      }
    }
    __syncwarp();
    double d = V[c * R + c];
    if (fabs(d) < ridge) d = d < 0 ? -ridge : ridge;
    const double inv = 1.0 / d;
    __syncwarp();
    for (uint32_t e = lane; e < R; e += 32) {
      V[c * R + e] *= inv;
      W[c * R + e] *= inv;
    }
    __syncwarp();
    for (uint32_t r = 0; r < R; ++r) {
      if (r == c) continue;
      const double f = V[r * R + c];
      __syncwarp();
      for (uint32_t e = lane; e < R; e += 32) {
        V[r * R + e] -= f * V[c * R + e];
        W[r * R + e] -= f * W[c * R + e];
      }
      __syncwarp();
    }
  }
}

// U = M W (row by row, fp64 accumulation), colsq[r] += sum_i U(i, r)^2.  A sub-warp of
// `width` lanes (next power of two >= R, at most 32) handles one row; lane l owns columns
// l, l + width (R <= 64); M(i, a) is broadcast inside the sub-warp with shuffles and W is read
// from shared memory (consecutive lanes, consecutive columns: conflict-free).
__global__ void __launch_bounds__(kThreads) solve_kernel(const float *__restrict__ M, uint64_t rows,
                                                         uint32_t R, GramList gl, float *__restrict__ U,
                                                         double *__restrict__ colsq) {
  extern __shared__ double solve_smem[];  // V[R*R], W[R*R], csq[R], Wf[R*R] (fp32)
  double *V = solve_smem, *W = solve_smem + R * R, *csq = solve_smem + 2 * R * R;
  float *Wf = reinterpret_cast<float *>(solve_smem + 2 * R * R + R);
  if (threadIdx.x < 32) hadamard_inverse(gl, R, V, W);
  for (uint32_t r = threadIdx.x; r < R; r += kThreads) csq[r] = 0.0;
  __syncthreads();
  for (uint32_t e = threadIdx.x; e < R * R; e += kThreads) Wf[e] = float(W[e]);
  __syncthreads();
  uint32_t width = 1, lw = 0;
  while (width < R && width < 32) { width <<= 1; ++lw; }
  const uint32_t lane = threadIdx.x & 31, sub = lane / width, l = lane % width;
  const uint32_t rpw = 32 / width;
  const uint64_t warp = (uint64_t(blockIdx.x) * kThreads + threadIdx.x) >> 5;
  const uint64_t nwarps = (uint64_t(gridDim.x) * kThreads) >> 5;
  float mine[2] = {0.f, 0.f};
  constexpr int RB = 4;  // rows per sub-warp per step: independent loads and FMA chains
  for (uint64_t base = warp * rpw * RB; base < rows; base += nwarps * rpw * RB) {
    float mv[RB][2];
#pragma unroll
    for (int b = 0; b < RB; ++b) {
      const uint64_t i = base + uint64_t(b) * rpw + sub;
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const uint32_t c = l + width * q;
        mv[b][q] = (i < rows && c < R) ? M[i * R + c] : 0.f;
      }
    }
    float x[RB][2] = {};
    for (uint32_t a = 0; a < R; ++a) {
      const uint32_t q = a >> lw, src = sub * width + (a & (width - 1));
      float w[2];
#pragma unroll
      for (int q2 = 0; q2 < 2; ++q2) {
        const uint32_t c = l + width * q2;
        w[q2] = c < R ? Wf[a * R + c] : 0.f;
      }
#pragma unroll
      for (int b = 0; b < RB; ++b) {
        const float ma = __shfl_sync(0xffffffffu, q == 0 ? mv[b][0] : mv[b][1], src);
        x[b][0] = fmaf(ma, w[0], x[b][0]);
        x[b][1] = fmaf(ma, w[1], x[b][1]);
      }
    }
#pragma unroll
    for (int b = 0; b < RB; ++b) {
      const uint64_t i = base + uint64_t(b) * rpw + sub;
#pragma unroll
      for (int q2 = 0; q2 < 2; ++q2) {
        const uint32_t c = l + width * q2;
        if (i < rows && c < R) {
          U[i * R + c] = x[b][q2];
          mine[q2] = fmaf(x[b][q2], x[b][q2], mine[q2]);
        }
      }
    }
  }
  // reduce over the sub-warps (lanes with equal l hold the same columns)
#pragma unroll
  for (int q2 = 0; q2 < 2; ++q2) {
    double v = double(mine[q2]);
    for (uint32_t o = width; o < 32; o <<= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    const uint32_t c = l + width * q2;
    if (sub == 0 && c < R) atomicAdd(&csq[c], v);
  }
  __syncthreads();
  for (uint32_t r = threadIdx.x; r < R; r += kThreads) atomicAdd(&colsq[r], csq[r]);
}

// lambda_r = sqrt(colsq_r) (1 if zero); U(:, r) /= lambda_r.  VW = 4: float4 path (R % 4 == 0),
// 4 independent vectors per thread per step for memory-level parallelism.
template <int VW>
__global__ void normalize_kernel(float *__restrict__ U, uint64_t rows, uint32_t R,
                                 const double *__restrict__ colsq, double *__restrict__ lambda) {
  __shared__ float inv[kMaxR];
  for (uint32_t r = threadIdx.x; r < R; r += blockDim.x) {
    double l = sqrt(colsq[r]);
    l = l > 0 ? l : 1.0;
    inv[r] = float(1.0 / l);
    if (blockIdx.x == 0) lambda[r] = l;
  }
  __syncthreads();
  // blockDim is a multiple of R / VW, so the columns of a thread never change
  const uint32_t cv = R / VW;
  const uint32_t c0 = (threadIdx.x % cv) * VW;
  float f[VW];
#pragma unroll
  for (int i = 0; i < VW; ++i) f[i] = inv[c0 + i];
  const uint64_t n = rows * cv, stride = uint64_t(gridDim.x) * blockDim.x;
  uint64_t e = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x;
  for (; e + 3 * stride < n; e += 4 * stride) {
    if constexpr (VW == 4) {
      float4 *p = reinterpret_cast<float4 *>(U);
      float4 v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) v[j] = p[e + j * stride];
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        v[j].x *= f[0]; v[j].y *= f[1]; v[j].z *= f[2]; v[j].w *= f[3];
        p[e + j * stride] = v[j];
      }
    } else {
      float v[4];
#pragma unroll
      for (int j = 0; j < 4; ++j) v[j] = U[e + j * stride];
#pragma unroll
      for (int j = 0; j < 4; ++j) U[e + j * stride] = v[j] * f[0];
    }
  }
  for (; e < n; e += stride) {
    if constexpr (VW == 4) {
      float4 *p = reinterpret_cast<float4 *>(U);
      float4 v = p[e];
      v.x *= f[0]; v.y *= f[1]; v.z *= f[2]; v.w *= f[3];
      p[e] = v;
    } else {
      U[e] *= f[0];
    }
  }
}

// out += sum_{i, r} lambda_r A(i, r) B(i, r); fp32 products, fp64 partial sums every 64 terms
template <int VW>
__global__ void inner_kernel(const float *__restrict__ A, const float *__restrict__ B, uint64_t rows,
                             uint32_t R, const double *__restrict__ lambda, double *__restrict__ out) {
  const uint32_t cv = R / VW;
  const uint32_t c0 = (threadIdx.x % cv) * VW;  // blockDim is a multiple of R / VW
  float lc[VW];
#pragma unroll
  for (int i = 0; i < VW; ++i) lc[i] = float(lambda[c0 + i]);
  double s = 0.0;
  float part = 0.f;
  int cnt = 0;
  const uint64_t n = rows * cv, stride = uint64_t(gridDim.x) * blockDim.x;
  for (uint64_t e = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < n; e += stride) {
    if constexpr (VW == 4) {
      const float4 a = reinterpret_cast<const float4 *>(A)[e];
      const float4 b = reinterpret_cast<const float4 *>(B)[e];
      part = fmaf(lc[0] * a.x, b.x, part);
      part = fmaf(lc[1] * a.y, b.y, part);
      part = fmaf(lc[2] * a.z, b.z, part);
      part = fmaf(lc[3] * a.w, b.w, part);
    } else {
      part = fmaf(lc[0] * A[e], B[e], part);
    }
    if (++cnt == 16) { s += double(part); part = 0.f; cnt = 0; }
  }
  s += double(part);
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}

__global__ void sumsq_kernel(const float *__restrict__ v, uint64_t n, double *__restrict__ out) {
  double s = 0.0;
  for (uint64_t e = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < n;
       e += uint64_t(gridDim.x) * blockDim.x)
    s += double(v[e]) * double(v[e]);
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) atomicAdd(out, s);
}

}  // namespace

void launch_gram(const float *U, uint64_t rows, uint32_t R, double *G, cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  if (!rows) return;
  gram_kernel<<<grid_rows(rows, 64 * 8), kThreads, 0, s>>>(U, rows, R, G);
  PASTA_LAUNCHED();
}

void launch_solve(const float *M, uint64_t rows, uint32_t R, const double *const *grams, uint32_t ngrams,
                  float *U, double *colsq, cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  if (ngrams > kMaxOrder) fail(PASTA_EINVAL, "too many gram matrices");
  GramList gl{};
  gl.n = ngrams;
  for (uint32_t k = 0; k < ngrams; ++k) gl.g[k] = grams[k];
  const size_t smem = (2 * size_t(R) * R + R) * sizeof(double) + size_t(R) * R * sizeof(float);
  auto go = [&](auto kern) {
    if (smem > 48 * 1024)
      PASTA_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    kern<<<grid_rows(rows ? rows : 1, kThreads * 4), kThreads, smem, s>>>(M, rows, R, gl, U, colsq);
    PASTA_LAUNCHED();
  };
  go(solve_kernel);
}

void launch_normalize(float *U, uint64_t rows, uint32_t R, const double *colsq, double *lambda,
                      cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  const bool v4 = R % 4 == 0 && (reinterpret_cast<uintptr_t>(U) & 15) == 0;
  const uint32_t cv = v4 ? R / 4 : R;
  const int bd = int((kThreads / cv) * cv);  // a multiple of R / VW
  const uint64_t n = rows * cv;
  if (v4) normalize_kernel<4><<<grid_rows(n ? n : 1, bd * 4), bd, 0, s>>>(U, rows, R, colsq, lambda);
  else normalize_kernel<1><<<grid_rows(n ? n : 1, bd * 4), bd, 0, s>>>(U, rows, R, colsq, lambda);
  PASTA_LAUNCHED();
}

void launch_inner(const float *A, const float *B, uint64_t rows, uint32_t R, const double *lambda,
                  double *out, cudaStream_t s) {
  if (!rows) return;
  const bool v4 = R % 4 == 0 && ((reinterpret_cast<uintptr_t>(A) | reinterpret_cast<uintptr_t>(B)) & 15) == 0;
  const uint32_t cv = v4 ? R / 4 : R;
  const int bd = int((kThreads / cv) * cv);
  const uint64_t n = rows * cv;
  if (v4) inner_kernel<4><<<grid_rows(n, bd * 4), bd, 0, s>>>(A, B, rows, R, lambda, out);
  else inner_kernel<1><<<grid_rows(n, bd * 4), bd, 0, s>>>(A, B, rows, R, lambda, out);
  PASTA_LAUNCHED();
}

void launch_sumsq(const float *v, uint64_t n, double *out, cudaStream_t s) {
  if (!n) return;
  sumsq_kernel<<<grid_rows(n, kThreads * 8), kThreads, 0, s>>>(v, n, out);
  PASTA_LAUNCHED();
}

}  // namespace pasta
