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
  uint64_t cap = uint64_t(sms) * 4;
  if (b > cap) b = cap;
  return unsigned(b < 1 ? 1 : b);
}

// G (R x R, fp64, row-major) += U^T U over rows [0, rows).  Row tiles of 64 are staged in
// shared memory; thread t accumulates the upper-triangle pairs t, t + 256, ... in fp64.
__global__ void __launch_bounds__(kThreads) gram_kernel(const float *__restrict__ U, uint64_t rows,
                                                        uint32_t R, double *__restrict__ G) {
  __shared__ float tile[64 * kMaxR];
  const uint32_t npairs = R * (R + 1) / 2;
  double acc[(kMaxR * (kMaxR + 1) / 2 + kThreads - 1) / kThreads];
  const int nacc = int((npairs + kThreads - 1) / kThreads);
  for (int q = 0; q < nacc; ++q) acc[q] = 0.0;
  for (uint64_t r0 = uint64_t(blockIdx.x) * 64; r0 < rows; r0 += uint64_t(gridDim.x) * 64) {
    const uint32_t nr = uint32_t(rows - r0 < 64 ? rows - r0 : 64);
    __syncthreads();
    for (uint32_t e = threadIdx.x; e < nr * R; e += kThreads) tile[e] = U[r0 * R + e];
    __syncthreads();
    for (int q = 0; q < nacc; ++q) {
      const uint32_t p = threadIdx.x + q * kThreads;
      if (p >= npairs) break;
      // pair index p -> (a, b) with a <= b, row-major over the upper triangle
      uint32_t a = 0, rem = p;
      while (rem >= R - a) { rem -= R - a; ++a; }
      const uint32_t b = a + rem;
      double s = 0.0;
      for (uint32_t i = 0; i < nr; ++i) s += double(tile[i * R + a]) * double(tile[i * R + b]);
      acc[q] += s;
    }
  }
  for (int q = 0; q < nacc; ++q) {
    const uint32_t p = threadIdx.x + q * kThreads;
    if (p >= npairs) break;
    uint32_t a = 0, rem = p;
    while (rem >= R - a) { rem -= R - a; ++a; }
    const uint32_t b = a + rem;
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

// U = M W (row by row, fp64 accumulation), colsq[r] += sum_i U(i, r)^2.
__global__ void __launch_bounds__(kThreads) solve_kernel(const float *__restrict__ M, uint64_t rows,
                                                         uint32_t R, GramList gl, float *__restrict__ U,
                                                         double *__restrict__ colsq) {
  extern __shared__ double solve_smem[];  // V[R*R], W[R*R], csq[R]
  double *V = solve_smem, *W = solve_smem + R * R, *csq = solve_smem + 2 * R * R;
  if (threadIdx.x < 32) hadamard_inverse(gl, R, V, W);
  for (uint32_t r = threadIdx.x; r < R; r += kThreads) csq[r] = 0.0;
  __syncthreads();
  double mine[kMaxR];
  for (uint32_t r = 0; r < R; ++r) mine[r] = 0.0;
  for (uint64_t i = uint64_t(blockIdx.x) * kThreads + threadIdx.x; i < rows;
       i += uint64_t(gridDim.x) * kThreads) {
    double m[kMaxR];
    for (uint32_t a = 0; a < R; ++a) m[a] = M[i * R + a];
    for (uint32_t r = 0; r < R; ++r) {
      double x = 0.0;
      for (uint32_t a = 0; a < R; ++a) x += m[a] * W[a * R + r];
      U[i * R + r] = float(x);
      mine[r] += x * x;
    }
  }
  for (uint32_t r = 0; r < R; ++r) {
    double v = mine[r];
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if ((threadIdx.x & 31) == 0) atomicAdd(&csq[r], v);
  }
  __syncthreads();
  for (uint32_t r = threadIdx.x; r < R; r += kThreads) atomicAdd(&colsq[r], csq[r]);
}

// lambda_r = sqrt(colsq_r) (1 if zero); U(:, r) /= lambda_r
__global__ void normalize_kernel(float *__restrict__ U, uint64_t rows, uint32_t R,
                                 const double *__restrict__ colsq, double *__restrict__ lambda) {
  __shared__ double lam[kMaxR];
  for (uint32_t r = threadIdx.x; r < R; r += blockDim.x) {
    double l = sqrt(colsq[r]);
    lam[r] = l > 0 ? l : 1.0;
  }
  __syncthreads();
  if (blockIdx.x == 0)
    for (uint32_t r = threadIdx.x; r < R; r += blockDim.x) lambda[r] = lam[r];
  for (uint64_t e = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < rows * R;
       e += uint64_t(gridDim.x) * blockDim.x)
    U[e] = float(double(U[e]) / lam[e % R]);
}

// out += sum_{i, r} lambda_r A(i, r) B(i, r)
__global__ void inner_kernel(const float *__restrict__ A, const float *__restrict__ B, uint64_t rows,
                             uint32_t R, const double *__restrict__ lambda, double *__restrict__ out) {
  double s = 0.0;
  for (uint64_t e = uint64_t(blockIdx.x) * blockDim.x + threadIdx.x; e < rows * R;
       e += uint64_t(gridDim.x) * blockDim.x)
    s += lambda[e % R] * double(A[e]) * double(B[e]);
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
  const size_t smem = (2 * size_t(R) * R + R) * sizeof(double);
  if (smem > 48 * 1024)
    PASTA_CUDA(cudaFuncSetAttribute(solve_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  solve_kernel<<<grid_rows(rows ? rows : 1, kThreads * 4), kThreads, smem, s>>>(M, rows, R, gl, U, colsq);
  PASTA_LAUNCHED();
}

void launch_normalize(float *U, uint64_t rows, uint32_t R, const double *colsq, double *lambda,
                      cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  normalize_kernel<<<grid_rows(rows * R ? rows * R : 1, kThreads * 8), kThreads, 0, s>>>(U, rows, R, colsq,
                                                                                        lambda);
  PASTA_LAUNCHED();
}

void launch_inner(const float *A, const float *B, uint64_t rows, uint32_t R, const double *lambda,
                  double *out, cudaStream_t s) {
  if (!rows) return;
  inner_kernel<<<grid_rows(rows * R, kThreads * 8), kThreads, 0, s>>>(A, B, rows, R, lambda, out);
  PASTA_LAUNCHED();
}

void launch_sumsq(const float *v, uint64_t n, double *out, cudaStream_t s) {
  if (!n) return;
  sumsq_kernel<<<grid_rows(n, kThreads * 8), kThreads, 0, s>>>(v, n, out);
  PASTA_LAUNCHED();
}

}  // namespace pasta
