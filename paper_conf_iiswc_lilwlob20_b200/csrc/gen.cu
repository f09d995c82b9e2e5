// gen.cu -- Stochastic Kronecker ("ball dropping") sparse tensor generator on the GPU
// (R#19-R#23).  Counter-based: draw d's randomness is a pure function of
// (seed, d, level), so the result is independent of launch geometry and identical to any
// other implementation of the same recipe (include/pasta.h documents it).
#include <cmath>
#include <vector>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kThreads = 256;
constexpr uint64_t kValueStream = 0xFFFF;

__constant__ double c_cum[1 << kMaxOrder];

struct GenArgs {
  uint32_t kind;  // 1: Kronecker ball dropping (also kind 0 = uniform table), 2: slice power law
  // kind 2 (R#30): per-mode cumulative weight tables (device) and their totals
  const double *cumk[kMaxOrder];
  uint32_t order;
  uint32_t ncell;
  uint32_t last_pos;  // last cell with positive weight (rounding fallback)
  double total;       // cum[ncell - 1]
  uint32_t L[kMaxOrder];
  uint32_t Lmax;
  uint32_t dims[kMaxOrder];
  uint64_t key;
};

__host__ __device__ inline uint64_t mix64(uint64_t z) {
  z ^= z >> 30;
  z *= 0xbf58476d1ce4e5b9ull;
  z ^= z >> 27;
  z *= 0x94d049bb133111ebull;
  z ^= z >> 31;
  return z;
}

__device__ inline double uniform01(uint64_t key, uint64_t d, uint64_t s) {
  uint64_t h = mix64(key ^ mix64((s << 40) | d));
  return __dmul_rn(__ull2double_rn(h >> 11), 1.0 / 9007199254740992.0);
}

__device__ inline bool draw_coords(const GenArgs &a, uint64_t d, uint32_t *c) {
  if (a.kind == 2) {
    // slice power law (R#30): i_k = first i with u(d, k) * cum_k[I_k - 1] < cum_k[i]
    for (uint32_t k = 0; k < a.order; ++k) {
      const double *cum = a.cumk[k];
      const uint32_t I = a.dims[k];
      const double u = __dmul_rn(uniform01(a.key, d, k), cum[I - 1]);
      uint32_t lo = 0, hi = I;
      while (lo < hi) {
        const uint32_t mid = lo + (hi - lo) / 2;
        if (u < cum[mid]) hi = mid; else lo = mid + 1;
      }
      c[k] = lo < I ? lo : I - 1;
    }
    return true;
  }
  for (uint32_t k = 0; k < a.order; ++k) c[k] = 0;
  for (uint32_t l = 0; l < a.Lmax; ++l) {
    double u = __dmul_rn(uniform01(a.key, d, l), a.total);
    uint32_t cell = a.last_pos;
    for (uint32_t j = 0; j < a.ncell; ++j)
      if (u < c_cum[j]) { cell = j; break; }
    for (uint32_t k = 0; k < a.order; ++k)
      if (l < a.L[k]) c[k] |= ((cell >> k) & 1u) << l;
  }
  bool ok = true;
  for (uint32_t k = 0; k < a.order; ++k) ok &= c[k] < a.dims[k];
  return ok;
}

__global__ void valid_flag_kernel(GenArgs a, uint64_t D, uint8_t *__restrict__ flag) {
  for (uint64_t d = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; d < D;
       d += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t c[kMaxOrder];
    flag[d] = draw_coords(a, d, c) ? 1 : 0;
  }
}

struct CoordOut {
  uint32_t *c[kMaxOrder];
};

__global__ void coords_kernel(GenArgs a, const uint32_t *__restrict__ did, uint64_t nv, CoordOut o) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < nv;
       x += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t c[kMaxOrder];
    draw_coords(a, did[x], c);
    for (uint32_t k = 0; k < a.order; ++k) o.c[k][x] = c[k];
  }
}

struct CoordIn {
  const uint32_t *c[kMaxOrder];
  uint32_t order;
};

// flag[s] = 1 iff sorted position s starts a new distinct coordinate
__global__ void first_flag_kernel(CoordIn a, const uint32_t *__restrict__ perm, uint64_t nv,
                                  uint8_t *__restrict__ flag) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s < nv;
       s += uint64_t(gridDim.x) * blockDim.x) {
    uint8_t f = 1;
    if (s > 0) {
      uint32_t p = perm[s], q = perm[s - 1];
      f = 0;
      for (uint32_t k = 0; k < a.order; ++k) f |= (a.c[k][p] != a.c[k][q]);
    }
    flag[s] = f;
  }
}

// firstd[u] = draw id of the first draw of unique coordinate u (sorted position uniq[u])
__global__ void firstd_kernel(const uint32_t *__restrict__ uniq, const uint32_t *__restrict__ perm,
                              const uint32_t *__restrict__ did, uint64_t nu, uint32_t *__restrict__ fd) {
  for (uint64_t u = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; u < nu;
       u += uint64_t(gridDim.x) * blockDim.x)
    fd[u] = did[perm[uniq[u]]];
}

__global__ void keep_flag_kernel(const uint32_t *__restrict__ fd, uint64_t nu, uint32_t thresh,
                                 uint8_t *__restrict__ flag) {
  for (uint64_t u = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; u < nu;
       u += uint64_t(gridDim.x) * blockDim.x)
    flag[u] = fd[u] <= thresh;
}

__global__ void emit_kernel(CoordIn a, const uint32_t *__restrict__ keep, const uint32_t *__restrict__ uniq,
                            const uint32_t *__restrict__ perm, const uint32_t *__restrict__ did, uint64_t M,
                            uint64_t key, double lo, double diff, CoordOut o, float *__restrict__ val) {
  for (uint64_t j = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; j < M;
       j += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t p = perm[uniq[keep[j]]];
    for (uint32_t k = 0; k < a.order; ++k) o.c[k][j] = a.c[k][p];
    double u = uniform01(key, did[p], kValueStream);
    val[j] = __double2float_rn(__dadd_rn(lo, __dmul_rn(diff, u)));
  }
}

inline unsigned grid_for(uint64_t n) {
  uint64_t b = (n + kThreads * 4 - 1) / (kThreads * 4);
  if (b < 1) b = 1;
  if (b > (1u << 30)) b = 1u << 30;
  return unsigned(b);
}

}  // namespace

// x->order, x->dims, x->nnz are set by the caller; fills x->inds / x->val.
void gen_powerlaw_device(pasta_coo *x, uint64_t seed, const double *table, uint32_t ncell,
                         float val_lo, float val_hi, cudaStream_t s, double alpha) {
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  GenArgs a{};
  a.order = N;
  a.kind = ncell == 0 ? 2 : 1;
  DevArray<double> cumk[kMaxOrder];
  if (a.kind == 2) {
    // weights w_i = (i + 1)^-alpha, running fp64 sums in ascending i, computed on the host so
    // that every implementation of the recipe reproduces the same table (include/pasta.h)
    std::vector<double> h;
    for (uint32_t k = 0; k < N; ++k) {
      h.resize(x->dims[k]);
      double run = 0.0;
      for (uint32_t i = 0; i < x->dims[k]; ++i) {
        run = run + std::pow(double(i) + 1.0, -alpha);
        h[i] = run;
      }
      cumk[k].alloc(x->dims[k], s);
      PASTA_CUDA(cudaMemcpyAsync(cumk[k].p, h.data(), sizeof(double) * x->dims[k], cudaMemcpyHostToDevice, s));
      PASTA_CUDA(cudaStreamSynchronize(s));
      a.cumk[k] = cumk[k].p;
    }
  }
  a.ncell = ncell;
  double cum[1 << kMaxOrder] = {};
  double run = 0.0;
  for (uint32_t c = 0; c < ncell; ++c) {
    run = run + table[c];
    cum[c] = run;
    if (table[c] > 0.0) a.last_pos = c;
  }
  a.total = run;
  if (ncell) PASTA_CUDA(cudaMemcpyToSymbolAsync(c_cum, cum, sizeof(double) * ncell, 0, cudaMemcpyHostToDevice, s));
  for (uint32_t k = 0; k < N; ++k) {
    a.dims[k] = x->dims[k];
    a.L[k] = ceil_log2(x->dims[k]);
    if (a.L[k] > a.Lmax) a.Lmax = a.L[k];
  }
  a.key = mix64(seed ^ 0x5851F42D4C957F2Dull);

  for (uint32_t k = 0; k < N; ++k) x->inds[k].alloc(M, s);
  x->val.alloc(M, s);
  if (M == 0) return;

  uint64_t D = M + M / 16 + 4096;
  const uint64_t cap = 64 * M + (1ull << 22);
  for (;;) {
    if (D >= 0xFFFFFFFFull) fail(PASTA_ERANGE, "gen_powerlaw: more than 2^32-2 draws needed");
    // 1. valid draws (stripping), compacted in draw order
    DevArray<uint8_t> flag(D, s);
    valid_flag_kernel<<<grid_for(D), kThreads, 0, s>>>(a, D, flag.p);
    PASTA_LAUNCHED();
    DevArray<uint32_t> did;
    uint64_t nv = select_flagged(flag.p, D, did, s);
    flag.reset();
    // 2. coordinates of valid draws, stable lexicographic sort (draw order inside ties)
    DevArray<uint32_t> coords[kMaxOrder];
    CoordOut co{};
    CoordIn ci{};
    ci.order = N;
    for (uint32_t k = 0; k < N; ++k) {
      coords[k].alloc(nv, s);
      co.c[k] = coords[k].p;
      ci.c[k] = coords[k].p;
    }
    if (nv) {
      coords_kernel<<<grid_for(nv), kThreads, 0, s>>>(a, did.p, nv, co);
      PASTA_LAUNCHED();
    }
    DevArray<uint32_t> perm(nv, s);
    iota_u32(perm.p, nv, s);
    const uint32_t *comps[kMaxOrder];
    uint32_t bits[kMaxOrder];
    for (uint32_t k = 0; k < N; ++k) { comps[k] = coords[k].p; bits[k] = a.L[k]; }
    lexsort(comps, bits, int(N), perm, nv, s);
    // 3. first occurrence of each distinct coordinate
    DevArray<uint8_t> f2(nv, s);
    if (nv) {
      first_flag_kernel<<<grid_for(nv), kThreads, 0, s>>>(ci, perm.p, nv, f2.p);
      PASTA_LAUNCHED();
    }
    DevArray<uint32_t> uniq;
    uint64_t nu = select_flagged(f2.p, nv, uniq, s);
    f2.reset();
    if (nu >= M) {
      // 4. keep the M earliest-first-drawn coordinates, in lexicographic order
      DevArray<uint32_t> fd(nu, s);
      firstd_kernel<<<grid_for(nu), kThreads, 0, s>>>(uniq.p, perm.p, did.p, nu, fd.p);
      PASTA_LAUNCHED();
      uint32_t thresh = 0xFFFFFFFFu;
      if (nu > M) {
        DevArray<uint32_t> fds(nu, s), ident(nu, s);
        iota_u32(ident.p, nu, s);
        const uint32_t *fc[1] = {fd.p};
        uint32_t fb[1] = {ceil_log2(D)};
        // sort a permutation by first-draw id; the M-th smallest is the threshold
        lexsort(fc, fb, 1, ident, nu, s);
        uint32_t pos = 0;
        PASTA_CUDA(cudaMemcpyAsync(&pos, ident.p + (M - 1), sizeof(pos), cudaMemcpyDeviceToHost, s));
        PASTA_CUDA(cudaStreamSynchronize(s));
        PASTA_CUDA(cudaMemcpyAsync(&thresh, fd.p + pos, sizeof(thresh), cudaMemcpyDeviceToHost, s));
        PASTA_CUDA(cudaStreamSynchronize(s));
      }
      DevArray<uint8_t> kf(nu, s);
      keep_flag_kernel<<<grid_for(nu), kThreads, 0, s>>>(fd.p, nu, thresh, kf.p);
      PASTA_LAUNCHED();
      DevArray<uint32_t> keep;
      uint64_t nk = select_flagged(kf.p, nu, keep, s);
      if (nk != M) fail(PASTA_ECUDA, "gen_powerlaw: internal selection mismatch");
      CoordOut out{};
      for (uint32_t k = 0; k < N; ++k) out.c[k] = x->inds[k].p;
      double lo = double(val_lo), diff = double(val_hi) - double(val_lo);
      emit_kernel<<<grid_for(M), kThreads, 0, s>>>(ci, keep.p, uniq.p, perm.p, did.p, M, a.key, lo,
                                                   diff, out, x->val.p);
      PASTA_LAUNCHED();
      PASTA_CUDA(cudaStreamSynchronize(s));
      return;
    }
    if (D >= cap) fail(PASTA_EINVAL, "gen_powerlaw: cannot reach nnz distinct coordinates");
    D = D + D / 2 + 2 * (M - nu) + 4096;
    if (D > cap) D = cap;
  }
}

namespace {

// Label permutation pi_k of [0, I_k) (R#22, include/pasta.h): cycle walking over a keyed
// bijection f of [0, 2^L) made of three rounds of (odd multiply, xor-shift, add) mod 2^L.
__host__ __device__ inline uint32_t relabel_index(uint32_t v, uint32_t dim, uint64_t key, uint32_t L) {
  const uint64_t m = (uint64_t(1) << L) - 1;
  uint64_t y = v;
  do {
    for (int r = 0; r < 3; ++r) {
      y = (y * (((key >> (16 * r)) & 0xFFFFull) | 1ull)) & m;
      if (L >= 2) y ^= y >> ((L + 1) / 2);
      y = (y + ((key >> (32 + 8 * r)) & 0xFFFFFFull)) & m;
    }
  } while (y >= dim);
  return uint32_t(y);
}

__global__ void relabel_kernel(uint32_t *inds, uint64_t M, uint32_t dim, uint64_t key, uint32_t L) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M; x += uint64_t(gridDim.x) * blockDim.x)
    inds[x] = relabel_index(inds[x], dim, key, L);
}

}  // namespace

// permute = 1 (R#22): relabel every mode by pi_k, then restore the lexicographic order
void relabel_device(pasta_coo *x, uint64_t seed, cudaStream_t s) {
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  if (M == 0) return;
  for (uint32_t k = 0; k < N; ++k) {
    relabel_kernel<<<grid_for(M), kThreads, 0, s>>>(x->inds[k].p, M, x->dims[k],
                                                    mix64(seed ^ 0xA0761D6478BD642Full ^ uint64_t(k)),
                                                    ceil_log2(x->dims[k]));
    PASTA_LAUNCHED();
  }
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  const uint32_t *comps[kMaxOrder];
  uint32_t bits[kMaxOrder];
  for (uint32_t k = 0; k < N; ++k) {
    comps[k] = x->inds[k].p;
    bits[k] = ceil_log2(x->dims[k]);
  }
  lexsort(comps, bits, int(N), perm, M, s);
  for (uint32_t k = 0; k < N; ++k) {
    DevArray<uint32_t> t(M, s);
    gather_u32(x->inds[k].p, perm.p, t.p, M, s);
    std::swap(x->inds[k], t);
  }
  DevArray<float> v(M, s);
  gather_f32(x->val.p, perm.p, v.p, M, s);
  std::swap(x->val, v);
  PASTA_CUDA(cudaStreamSynchronize(s));
}

}  // namespace pasta
