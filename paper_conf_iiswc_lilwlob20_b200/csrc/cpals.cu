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
#include <cstdlib>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kThreads = 256;
constexpr int kMaxR = 64;

int sm_count_cpals() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

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

// Tiled kernels for R in {4, 8, 16, 32, 64}: a CTA stages kTile rows of the I x R matrix in
// shared memory with coalesced 128-bit loads, then
//   gram_tile_kernel:  groups of (R/4)^2 threads own the 4 x 4 blocks of U^T U; group g sums
//                      rows g, g + G, ... of the tile (two LDS.128 broadcasts + 16 FMAs per
//                      row), fp32 over <= 64 rows, fp64 beyond; one fp64 atomic per entry per CTA.
//   apply_tile_kernel: thread t owns output column c = t % R with W(:, c) in registers and
//                      rows t / R + j * (256 / R) of the tile (LDS.128 broadcasts, R FMAs per
//                      row); stores are coalesced (consecutive threads, consecutive columns).
// Both are HBM-streaming passes over the factor-sized matrix (one read; apply also writes).
constexpr int kTile = 256;
// rows per staged tile: 256, fewer for R = 64 so that static shared memory stays <= 48 KB
template <int R>
constexpr int tile_rows() { return R <= 32 ? kTile : 64; }

// gram: 16 KB row tiles, double-buffered with cp.async so the next tile streams in while the
// current one is reduced (the single-buffered load -> sync -> compute loop ran at ~1.9 TB/s)
template <int R>
constexpr int gram_rows() { return R == 64 ? 32 : 4096 / R; }  // R = 64: + 32 KB of fp64 reduction

template <int R>
__global__ void __launch_bounds__(kThreads) gram_tile_kernel(const float *__restrict__ U, uint64_t rows,
                                                             double *__restrict__ G) {
  constexpr int RB = R / 4, GS = RB * RB, NG = kThreads / GS, T = gram_rows<R>();
  // a group reduces RPG rows of a full tile; the fp32 partials go to fp64 every FLUSH tiles
  // (<= 64 rows in fp32, as before), so the row loop of a full tile has no flush test
  constexpr int RPG = T / NG, FLUSH = 64 / RPG;
  static_assert(T % NG == 0 && RPG <= 64, "gram tile shape");
  __shared__ __align__(16) float tile[2][T * R];
  __shared__ double red[R * R];
  const int t = threadIdx.x, g = t / GS, blk = t % GS, ba = blk / RB, bb = blk % RB;
  float acc[4][4] = {};
  double acc64[4][4] = {};
  int tiles = 0;
  for (uint32_t e = t; e < R * R; e += kThreads) red[e] = 0.0;
  const uint64_t step = uint64_t(gridDim.x) * T;
  auto issue = [&](uint64_t r0, int b) {
    if (r0 < rows) {
      const int nr = int(rows - r0 < T ? rows - r0 : T);
      const float4 *src = reinterpret_cast<const float4 *>(U + r0 * R);
      for (int e = t; e < nr * RB; e += kThreads) {
        const uint32_t d = uint32_t(__cvta_generic_to_shared(reinterpret_cast<float4 *>(tile[b]) + e));
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src + e) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  auto row = [&](const float *tb, int i) {
    const float4 x = *reinterpret_cast<const float4 *>(tb + i * R + 4 * ba);
    const float4 y = *reinterpret_cast<const float4 *>(tb + i * R + 4 * bb);
    const float xa[4] = {x.x, x.y, x.z, x.w}, ya[4] = {y.x, y.y, y.z, y.w};
#pragma unroll
    for (int p = 0; p < 4; ++p)
#pragma unroll
      for (int q = 0; q < 4; ++q) acc[p][q] = fmaf(xa[p], ya[q], acc[p][q]);
  };
  int b = 0;
  issue(uint64_t(blockIdx.x) * T, 0);
  for (uint64_t r0 = uint64_t(blockIdx.x) * T; r0 < rows; r0 += step, b ^= 1) {
    const int nr = int(rows - r0 < T ? rows - r0 : T);
    issue(r0 + step, b ^ 1);
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    __syncthreads();
    const float *tb = tile[b];
    if (nr == T) {
#pragma unroll
      for (int j = 0; j < RPG; ++j) row(tb, g + j * NG);
    } else {
      for (int i = g; i < nr; i += NG) row(tb, i);
    }
    if (++tiles == FLUSH) {
#pragma unroll
      for (int p = 0; p < 4; ++p)
#pragma unroll
        for (int q = 0; q < 4; ++q) { acc64[p][q] += double(acc[p][q]); acc[p][q] = 0.f; }
      tiles = 0;
    }
    __syncthreads();  // tile[b] is refilled by the next iteration's issue
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
  __syncthreads();
#pragma unroll
  for (int p = 0; p < 4; ++p)
#pragma unroll
    for (int q = 0; q < 4; ++q) atomicAdd(&red[(4 * ba + p) * R + 4 * bb + q], acc64[p][q] + double(acc[p][q]));
  __syncthreads();
  for (uint32_t e = t; e < R * R; e += kThreads) atomicAdd(&G[e], red[e]);
}

template <int R>
__global__ void __launch_bounds__(kThreads) apply_tile_kernel(const float *__restrict__ M, uint64_t rows,
                                                              const float *__restrict__ W, float *__restrict__ U) {
  // row tiles double-buffered with cp.async (as in gram_tile_kernel): 16 KB per buffer
  constexpr int RB = R / 4, RPP = kThreads / R, T = gram_rows<R>();  // RPP: rows per pass
  __shared__ __align__(16) float tile[2][T * R];
  const int t = threadIdx.x, c = t % R, r = t / R;
  float w[R];
#pragma unroll
  for (int a = 0; a < R; ++a) w[a] = W[a * R + c];
  const uint64_t step = uint64_t(gridDim.x) * T;
  auto issue = [&](uint64_t r0, int b) {
    if (r0 < rows) {
      const int nr = int(rows - r0 < T ? rows - r0 : T);
      const float4 *src = reinterpret_cast<const float4 *>(M + r0 * R);
      for (int e = t; e < nr * RB; e += kThreads) {
        const uint32_t d = uint32_t(__cvta_generic_to_shared(reinterpret_cast<float4 *>(tile[b]) + e));
        asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(d), "l"(src + e) : "memory");
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  int b = 0;
  issue(uint64_t(blockIdx.x) * T, 0);
  for (uint64_t r0 = uint64_t(blockIdx.x) * T; r0 < rows; r0 += step, b ^= 1) {
    const int nr = int(rows - r0 < T ? rows - r0 : T);
    issue(r0 + step, b ^ 1);
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    __syncthreads();
    const float *tb = tile[b];
    auto row = [&](int i) {
      float acc = 0.f;
#pragma unroll
      for (int a = 0; a < R; a += 4) {
        const float4 m = *reinterpret_cast<const float4 *>(tb + i * R + a);
        acc = fmaf(m.x, w[a], acc);
        acc = fmaf(m.y, w[a + 1], acc);
        acc = fmaf(m.z, w[a + 2], acc);
        acc = fmaf(m.w, w[a + 3], acc);
      }
      U[(r0 + i) * R + c] = acc;
    };
    if (nr == T) {  // full tile: T / RPP rows per thread, unrolled (as in gram_tile_kernel)
#pragma unroll
      for (int j = 0; j < T / RPP; ++j) row(r + j * RPP);
    } else {
      for (int i = r; i < nr; i += RPP) row(i);
    }
    __syncthreads();  // tile[b] is refilled by the next iteration's issue
  }
  asm volatile("cp.async.wait_group 0;" ::: "memory");
}

// Fused factor update + all-gather over peer memory (a9 / NEXT-1, B200-native exchange):
// the rows [row_lo, row_hi) this rank owns are computed once (U = M Wn, as apply_tile_kernel)
// and stored into every replica of U_n -- the local one and each peer's, mapped through CUDA
// IPC (NVLink / NVSwitch P2P stores) -- so the all-gather overlaps the arithmetic tile by
// tile instead of following it as a separate collective.
struct DstList {
  float *d[kMaxOrder];
  uint32_t n;
};

template <int R>
__global__ void __launch_bounds__(kThreads) apply_bcast_kernel(const float *__restrict__ M, uint64_t row_lo,
                                                               uint64_t row_hi, const float *__restrict__ W,
                                                               DstList dst) {
  constexpr int RB = R / 4, RPP = kThreads / R, T = R <= 32 ? 256 : 64;
  __shared__ __align__(16) float tile[T * R];
  const int t = threadIdx.x, c = t % R, r = t / R;
  float w[R];
#pragma unroll
  for (int a = 0; a < R; ++a) w[a] = W[a * R + c];
  const uint64_t rows = row_hi - row_lo;
  for (uint64_t r0 = uint64_t(blockIdx.x) * T; r0 < rows; r0 += uint64_t(gridDim.x) * T) {
    const int nr = int(rows - r0 < T ? rows - r0 : T);
    __syncthreads();
    const float4 *src = reinterpret_cast<const float4 *>(M + (row_lo + r0) * R);
    float4 *sd = reinterpret_cast<float4 *>(tile);
    for (int e = t; e < nr * RB; e += kThreads) sd[e] = src[e];
    __syncthreads();
    for (int i = r; i < nr; i += RPP) {
      float acc = 0.f;
#pragma unroll
      for (int a = 0; a < R; a += 4) {
        const float4 m = *reinterpret_cast<const float4 *>(tile + i * R + a);
        acc = fmaf(m.x, w[a], acc);
        acc = fmaf(m.y, w[a + 1], acc);
        acc = fmaf(m.z, w[a + 2], acc);
        acc = fmaf(m.w, w[a + 3], acc);
      }
      const uint64_t off = (row_lo + r0 + i) * R + c;
      for (uint32_t k = 0; k < dst.n; ++k) dst.d[k][off] = acc;
    }
  }
  __threadfence_system();  // peer stores performed before the kernel is seen complete
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
// Wg != nullptr: the fp32 right-hand matrix is given (cpals_prep_kernel) and neither the
// inverse nor colsq is computed (colsq may be NULL).
__global__ void __launch_bounds__(kThreads) solve_kernel(const float *__restrict__ M, uint64_t rows,
                                                         uint32_t R, GramList gl, float *__restrict__ U,
                                                         double *__restrict__ colsq,
                                                         const float *__restrict__ Wg) {
  extern __shared__ double solve_smem[];  // V[R*R], W[R*R], csq[R], Wf[R*R] (fp32)
  double *V = solve_smem, *W = solve_smem + R * R, *csq = solve_smem + 2 * R * R;
  float *Wf = reinterpret_cast<float *>(solve_smem + 2 * R * R + R);
  if (Wg == nullptr && threadIdx.x < 32) hadamard_inverse(gl, R, V, W);
  for (uint32_t r = threadIdx.x; r < R; r += kThreads) csq[r] = 0.0;
  __syncthreads();
  for (uint32_t e = threadIdx.x; e < R * R; e += kThreads) Wf[e] = Wg ? Wg[e] : float(W[e]);
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
          if (colsq) mine[q2] = fmaf(x[b][q2], x[b][q2], mine[q2]);
        }
      }
    }
  }
  if (colsq == nullptr) return;  // uniform across the grid
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

// Fused CP-ALS epilogue algebra for mode n (one CTA), so that the factor update needs a
// single pass over M and none over U: with GM = M^T M (R x R, from gram_kernel on M),
//   W = V^{-1}, V = Hadamard_{k != n} G_k          (hadamard_inverse, one warp, fp64)
//   U = M W  =>  U^T U = W^T GM W =: GU,  lambda_r = sqrt(GU_rr)  (1 if GU_rr <= 0)
//   normalised U_n = M Wn,  Wn = W diag(1 / lambda),  G_n = GU ./ (lambda lambda^T).
// Same algebra as solve -> normalise -> gram (Kolda & Bader), without two of the
// three passes over the I_n x R factor.
__global__ void cpals_prep_kernel(const double *__restrict__ GM, GramList gl, uint32_t R,
                                  float *__restrict__ Wn, double *__restrict__ Gn,
                                  double *__restrict__ lambda) {
  extern __shared__ double prep_smem[];  // V[R*R], W[R*R], T[R*R], lam[R]
  double *V = prep_smem, *W = prep_smem + R * R, *T = prep_smem + 2 * R * R, *lam = prep_smem + 3 * R * R;
  if (threadIdx.x < 32) hadamard_inverse(gl, R, V, W);
  __syncthreads();
  for (uint32_t e = threadIdx.x; e < R * R; e += blockDim.x) {  // T = GM W
    const uint32_t a = e / R, c = e % R;
    double t = 0.0;
    for (uint32_t b = 0; b < R; ++b) t += GM[a * R + b] * W[b * R + c];
    T[e] = t;
  }
  __syncthreads();
  for (uint32_t e = threadIdx.x; e < R * R; e += blockDim.x) {  // GU = W^T T  (into V)
    const uint32_t a = e / R, c = e % R;
    double t = 0.0;
    for (uint32_t b = 0; b < R; ++b) t += W[b * R + a] * T[b * R + c];
    V[e] = t;
  }
  __syncthreads();
  for (uint32_t r = threadIdx.x; r < R; r += blockDim.x) {
    const double d = V[r * R + r];
    const double l = d > 0.0 ? sqrt(d) : 1.0;
    lam[r] = l;
    lambda[r] = l;
  }
  __syncthreads();
  for (uint32_t e = threadIdx.x; e < R * R; e += blockDim.x) {
    const uint32_t a = e / R, c = e % R;
    Gn[e] = V[e] / (lam[a] * lam[c]);
    Wn[e] = float(W[e] / lam[c]);
  }
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

bool tiled_ok(uint32_t R, const void *a, const void *b) {
  const bool al = ((reinterpret_cast<uintptr_t>(a) | reinterpret_cast<uintptr_t>(b)) & 15u) == 0;
  return al && (R == 4 || R == 8 || R == 16 || R == 32 || R == 64);
}

template <template <int> class K, class... Args>
void launch_tiled(uint32_t R, uint64_t rows, cudaStream_t s, Args... args) {
  // persistent-style grid: PASTA_TILE_CTAS_PER_SM (default 8) CTAs per SM walk the row tiles,
  // so the per-CTA prologue / epilogue (W load, smem and global reductions) is amortised
  static int per_sm = 0;
  if (!per_sm) {
    const char *e = getenv("PASTA_TILE_CTAS_PER_SM");
    per_sm = (e && *e) ? atoi(e) : 8;
    if (per_sm < 1) per_sm = 8;
  }
  unsigned grid = grid_rows(rows, kTile);
  const unsigned cap = unsigned(sm_count_cpals()) * unsigned(per_sm);
  if (grid > cap) grid = cap;
  switch (R) {
    case 4: K<4>::go(grid, s, args...); break;
    case 8: K<8>::go(grid, s, args...); break;
    case 16: K<16>::go(grid, s, args...); break;
    case 32: K<32>::go(grid, s, args...); break;
    default: K<64>::go(grid, s, args...); break;
  }
  PASTA_LAUNCHED();
}

template <int R>
struct GramTile {
  static void go(unsigned grid, cudaStream_t s, const float *U, uint64_t rows, double *G) {
    gram_tile_kernel<R><<<grid, kThreads, 0, s>>>(U, rows, G);
  }
};

template <int R>
struct ApplyTile {
  static void go(unsigned grid, cudaStream_t s, const float *M, uint64_t rows, const float *W, float *U) {
    apply_tile_kernel<R><<<grid, kThreads, 0, s>>>(M, rows, W, U);
  }
};

void launch_gram(const float *U, uint64_t rows, uint32_t R, double *G, cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  if (!rows) return;
  if (tiled_ok(R, U, U)) return launch_tiled<GramTile>(R, rows, s, U, rows, G);
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
    kern<<<grid_rows(rows ? rows : 1, kThreads * 4), kThreads, smem, s>>>(M, rows, R, gl, U, colsq, nullptr);
    PASTA_LAUNCHED();
  };
  go(solve_kernel);
}

void launch_cpals_prep(const double *GM, const double *const *grams, uint32_t ngrams, uint32_t R,
                       float *Wn, double *Gn, double *lambda, cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  if (ngrams > kMaxOrder) fail(PASTA_EINVAL, "too many gram matrices");
  GramList gl{};
  gl.n = ngrams;
  for (uint32_t k = 0; k < ngrams; ++k) gl.g[k] = grams[k];
  const size_t smem = (3 * size_t(R) * R + R) * sizeof(double);
  if (smem > 48 * 1024)
    PASTA_CUDA(cudaFuncSetAttribute(cpals_prep_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  cpals_prep_kernel<<<1, kThreads, smem, s>>>(GM, gl, R, Wn, Gn, lambda);
  PASTA_LAUNCHED();
}

void launch_apply(const float *M, uint64_t rows, uint32_t R, const float *Wn, float *U, cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  if (tiled_ok(R, M, U)) return launch_tiled<ApplyTile>(R, rows, s, M, rows, Wn, U);
  GramList gl{};
  const size_t smem = (2 * size_t(R) * R + R) * sizeof(double) + size_t(R) * R * sizeof(float);
  if (smem > 48 * 1024)
    PASTA_CUDA(cudaFuncSetAttribute(solve_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
  solve_kernel<<<grid_rows(rows ? rows : 1, kThreads * 4), kThreads, smem, s>>>(M, rows, R, gl, U, nullptr, Wn);
  PASTA_LAUNCHED();
}

template <int R>
struct ApplyBcast {
  static void go(unsigned grid, cudaStream_t s, const float *M, uint64_t lo, uint64_t hi, const float *W,
                 DstList d) {
    apply_bcast_kernel<R><<<grid, kThreads, 0, s>>>(M, lo, hi, W, d);
  }
};

void launch_apply_bcast(const float *M, uint64_t row_lo, uint64_t row_hi, uint32_t R, const float *Wn,
                        float *const *dsts, uint32_t ndst, cudaStream_t s) {
  if (!(R == 4 || R == 8 || R == 16 || R == 32 || R == 64))
    fail(PASTA_EUNSUPPORTED, "pasta_rows_times_bcast: R must be 4, 8, 16, 32 or 64");
  if (ndst < 1 || ndst > kMaxOrder) fail(PASTA_EINVAL, "pasta_rows_times_bcast: 1..8 destinations");
  if (row_hi <= row_lo) return;
  // the kernel reads M and writes the replicas with 128-bit accesses
  bool al = (reinterpret_cast<uintptr_t>(M) & 15) == 0;
  for (uint32_t k = 0; k < ndst; ++k) al = al && (reinterpret_cast<uintptr_t>(dsts[k]) & 15) == 0;
  if (!al) fail(PASTA_EINVAL, "pasta_rows_times_bcast: M and every destination must be 16-byte aligned");
  DstList d{};
  d.n = ndst;
  for (uint32_t k = 0; k < ndst; ++k) d.d[k] = dsts[k];
  launch_tiled<ApplyBcast>(R, row_hi - row_lo, s, M, row_lo, row_hi, Wn, d);
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

namespace {
// CP-ALS fit (one CTA, fp64): ||Xhat||^2 = lambda^T (Hadamard_k G_k) lambda, resid^2 =
// ||X||^2 + ||Xhat||^2 - 2 <X, Xhat>, fit = 1 - sqrt(max(resid^2, 0)) / ||X||.
__global__ void cpals_fit_kernel(GramList gl, uint32_t R, const double *__restrict__ lambda,
                                 const double *__restrict__ inner, double normx2, double *__restrict__ out) {
  __shared__ double red[kThreads / 32];
  double acc = 0.0;
  for (uint32_t e = threadIdx.x; e < R * R; e += blockDim.x) {
    const uint32_t a = e / R, b = e % R;
    double v = lambda[a] * lambda[b];
    for (uint32_t k = 0; k < gl.n; ++k) v *= gl.g[k][e];
    acc += v;
  }
  for (int o = 16; o; o >>= 1) acc += __shfl_xor_sync(0xFFFFFFFFu, acc, o);
  if ((threadIdx.x & 31) == 0) red[threadIdx.x >> 5] = acc;
  __syncthreads();
  if (threadIdx.x == 0) {
    double nx = 0.0;
    for (int w = 0; w < int(blockDim.x >> 5); ++w) nx += red[w];
    const double resid2 = normx2 + nx - 2.0 * inner[0];
    out[0] = normx2 > 0 ? 1.0 - sqrt(resid2 > 0 ? resid2 : 0.0) / sqrt(normx2) : 0.0;
    out[1] = nx;
  }
}
}  // namespace

void launch_cpals_fit(const double *const *grams, uint32_t ngrams, uint32_t R, const double *lambda,
                      const double *inner, double normx2, double *out, cudaStream_t s) {
  if (R > kMaxR) fail(PASTA_EUNSUPPORTED, "CP-ALS building blocks support R <= 64");
  if (ngrams > kMaxOrder) fail(PASTA_EINVAL, "at most 8 grams");
  GramList gl{};
  gl.n = ngrams;
  for (uint32_t k = 0; k < ngrams; ++k) gl.g[k] = grams[k];
  cpals_fit_kernel<<<1, kThreads, 0, s>>>(gl, R, lambda, inner, normx2, out);
  PASTA_LAUNCHED();
}

}  // namespace pasta
