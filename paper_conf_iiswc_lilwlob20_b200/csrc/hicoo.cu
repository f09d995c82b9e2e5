// hicoo.cu -- COO -> HiCOO conversion (R#10-R#14) and the per-mode
// HiCOO working copy used by the GPU MTTKRP (R#27).
#include <cub/cub.cuh>

#include <cstdlib>
#include <vector>

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

__global__ void shift_u32_kernel(const uint32_t *__restrict__ in, uint64_t M, uint32_t sh,
                                 uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = in[x] >> sh;
}

__global__ void u8_to_u32_kernel(const uint8_t *__restrict__ in, uint64_t M, uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = in[x];
}

// light[x] = 1 iff the block of entry x holds fewer than heavy_min entries
__global__ void light_entry_kernel(const uint64_t *__restrict__ bptr, const uint32_t *__restrict__ blk,
                                   uint64_t M, uint32_t heavy_min, uint32_t *__restrict__ light) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    uint32_t b = blk[x];
    light[x] = (bptr[b + 1] - bptr[b]) < heavy_min ? 1u : 0u;
  }
}

__global__ void light_block_kernel(const uint64_t *__restrict__ bptr, uint64_t nb, uint32_t heavy_min,
                                   uint32_t *__restrict__ light) {
  for (uint64_t b = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; b < nb;
       b += uint64_t(gridDim.x) * blockDim.x)
    light[b] = (bptr[b + 1] - bptr[b]) < heavy_min ? 1u : 0u;
}

__global__ void piece_count_kernel(const uint64_t *__restrict__ bptr, uint64_t nh, uint32_t piece,
                                   uint64_t *__restrict__ cnt) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s <= nh;
       s += uint64_t(gridDim.x) * blockDim.x)
    cnt[s] = s == nh ? 0 : (bptr[s + 1] - bptr[s] + piece - 1) / piece;
}

__global__ void piece_emit_kernel(const uint64_t *__restrict__ off, uint64_t nh, uint32_t *__restrict__ out) {
  for (uint64_t s = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; s < nh;
       s += uint64_t(gridDim.x) * blockDim.x)
    for (uint64_t j = off[s]; j < off[s + 1]; ++j) {
      out[2 * j] = uint32_t(s);
      out[2 * j + 1] = uint32_t(j - off[s]);
    }
}

// rowslice: flag[x] = 1 iff position x starts a new (block, einds_mode) slice
__global__ void slice_flag_kernel(const uint32_t *__restrict__ blkp, const uint32_t *__restrict__ enp,
                                  uint64_t M, uint8_t *__restrict__ flag) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    flag[x] = (x == 0) || blkp[x] != blkp[x - 1] || enp[x] != enp[x - 1];
}

struct SliceOut {
  const uint32_t *binds[kMaxOrder];
  uint32_t *base[kMaxOrder];
  uint32_t order, mode, bbits;
  uint32_t cmask;  // gHiCOO: only compressed modes have block bases; an uncompressed mode's
                   // row comes in full (enp = i_mode)
};

__global__ void slice_emit_kernel(SliceOut o, const uint32_t *__restrict__ starts, uint64_t nsb, uint64_t M,
                                  const uint32_t *__restrict__ blkp, const uint32_t *__restrict__ enp,
                                  uint64_t *__restrict__ sbptr, uint32_t *__restrict__ sbrow) {
  for (uint64_t j = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; j <= nsb;
       j += uint64_t(gridDim.x) * blockDim.x) {
    if (j == nsb) { sbptr[nsb] = M; continue; }
    uint32_t x = starts[j];
    uint32_t b = blkp[x];
    sbptr[j] = x;
    sbrow[j] = ((o.cmask >> o.mode) & 1u) ? (o.binds[o.mode][b] << o.bbits) + enp[x] : enp[x];
    for (uint32_t k = 0; k < o.order; ++k)
      if (k != o.mode && ((o.cmask >> k) & 1u)) o.base[k][j] = o.binds[k][b] << o.bbits;
  }
}

// ---- R#36 tier blocks (row-granular hot-row tiers of the row-slice copy) ----
struct TierArgs {
  const uint32_t *binds[kMaxOrder];
  const uint8_t *einds[kMaxOrder];
  const uint32_t *rank[kMaxOrder];  // null: not ranked (no tiers)
  uint32_t ntier[kMaxOrder];        // tier blocks of mode k (smem ones first)
  uint32_t nbr[kMaxOrder];          // block rows of mode k: keys >= nbr are tier blocks
  uint32_t *key[kMaxOrder];
  uint8_t *e[kMaxOrder];
  uint32_t order, bbits;
};

// per entry x of the canonical copy and tiered mode k: the row's heat rank rho; a row of tier
// block m = rho >> b (m < ntier) gets key nbr + m and element index rho & (B - 1), any other row
// keeps its canonical block (key binds_k) and element index
__global__ void tier_entry_kernel(TierArgs t, const uint32_t *__restrict__ blk, uint64_t M) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t b = blk[x];
    for (uint32_t k = 0; k < t.order; ++k) {
      if (!t.key[k]) continue;  // the target mode, uncompressed modes
      const uint32_t bk = t.binds[k][b], ek = t.einds[k][x];
      if (t.rank[k] && t.ntier[k]) {
        const uint32_t rho = t.rank[k][(bk << t.bbits) | ek];
        const uint32_t m = rho >> t.bbits;
        if (m < t.ntier[k]) {
          t.key[k][x] = t.nbr[k] + m;
          t.e[k][x] = uint8_t(rho & ((1u << t.bbits) - 1u));
          continue;
        }
      }
      t.key[k][x] = bk;
      t.e[k][x] = uint8_t(ek);
    }
  }
}

struct TierEmit {
  const uint32_t *key[kMaxOrder];  // sorted keys (tiered or plain compressed other modes)
  uint32_t *base[kMaxOrder];
  uint32_t nbr[kMaxOrder], sblk[kMaxOrder], hs_base[kMaxOrder], hot_base[kMaxOrder];
  uint32_t order, mode, bbits;
};

// slice j (first entry starts[j]): row, and per compressed other mode the block base -- plain
// (binds_k << b) or the tier tag | first slot of the tier block
__global__ void slice_emit_tier_kernel(TierEmit o, const uint32_t *__restrict__ starts, uint64_t nsb, uint64_t M,
                                       const uint32_t *__restrict__ rowp, uint64_t *__restrict__ sbptr,
                                       uint32_t *__restrict__ sbrow) {
  for (uint64_t j = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; j <= nsb;
       j += uint64_t(gridDim.x) * blockDim.x) {
    if (j == nsb) { sbptr[nsb] = M; continue; }
    const uint32_t x = starts[j];
    sbptr[j] = x;
    sbrow[j] = rowp[x];
    for (uint32_t k = 0; k < o.order; ++k) {
      if (!o.base[k]) continue;
      const uint32_t key = o.key[k][x];
      uint32_t v;
      if (key < o.nbr[k]) {
        v = key << o.bbits;
      } else {
        const uint32_t m = key - o.nbr[k];
        v = m < o.sblk[k] ? (0xC0000000u | (o.hs_base[k] + (m << o.bbits)))
                          : (0x80000000u | (o.hot_base[k] + ((m - o.sblk[k]) << o.bbits)));
      }
      o.base[k][j] = v;
    }
  }
}

__global__ void full_row_kernel(const uint32_t *__restrict__ binds_n, const uint32_t *__restrict__ blk,
                                const uint8_t *__restrict__ einds_n, uint32_t bb, uint64_t M,
                                uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = (binds_n[blk[x]] << bb) | einds_n[x];
}

__global__ void entry_row_count_kernel(const uint32_t *__restrict__ binds_k, const uint32_t *__restrict__ blk,
                                       const uint8_t *__restrict__ einds_k, uint32_t bb, uint64_t M,
                                       uint32_t *__restrict__ cnt) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    atomicAdd(&cnt[(binds_k[blk[x]] << bb) | einds_k[x]], 1u);
}

__global__ void coord_count_kernel(const uint32_t *__restrict__ c, uint64_t M, uint32_t *__restrict__ cnt) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x)
    atomicAdd(&cnt[c[x]], 1u);
}

// gHiCOO uncompressed mode (R#36): the entry's full coordinate, or the tag | slot of its tier row
__global__ void tier_coord_kernel(const uint32_t *__restrict__ c, const uint32_t *__restrict__ perm, uint64_t M,
                                  const uint32_t *__restrict__ rank, uint32_t nrank_tier, uint32_t nrank_smem,
                                  uint32_t hs_base, uint32_t hot_base, uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M;
       x += uint64_t(gridDim.x) * blockDim.x) {
    const uint32_t v = c[perm[x]], rho = rank[v];
    out[x] = rho >= nrank_tier ? v
             : rho < nrank_smem ? (0xC0000000u | (hs_base + rho))
                                : (0x80000000u | (hot_base + rho - nrank_smem));
  }
}

__global__ void scatter_rank_kernel(const uint32_t *__restrict__ order, uint32_t n, uint32_t *__restrict__ rank) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    rank[order[i]] = uint32_t(i);
}

// heat[m] = sum of the sorted counts of ranks [m B, m B + B)
__global__ void block_heat_kernel(const uint32_t *__restrict__ sorted, uint32_t n, uint32_t bb,
                                  unsigned long long *__restrict__ heat) {
  const uint64_t nb = (uint64_t(n) + (1u << bb) - 1) >> bb;
  for (uint64_t m = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; m < nb; m += uint64_t(gridDim.x) * blockDim.x) {
    unsigned long long h = 0;
    const uint64_t e = std::min<uint64_t>(n, (m + 1) << bb);
    for (uint64_t i = m << bb; i < e; ++i) h += sorted[i];
    heat[m] = h;
  }
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

// COO -> HiCOO / gHiCOO.  HiCOO (cmask = all modes): Morton order of the full coordinates.
// gHiCOO (R#29): stable lexicographic sort by the uncompressed modes first, then a
// stable Morton sort by the compressed modes, which gives Morton order of the compressed
// coordinates with ties in lexicographic order of the uncompressed ones; blocks split where
// (i_k >> b) changes for a compressed k; uncompressed modes keep their u32 coordinates.
void coo_to_hicoo_device(const pasta_coo *x, pasta_hicoo *h, cudaStream_t s) {
  const uint32_t N = x->order;
  const uint64_t M = x->nnz;
  const uint32_t bb = h->block_bits;
  const uint32_t cmask = h->cmask;
  uint32_t Lm = 0, nc = 0, nu = 0;
  const uint32_t *comp[kMaxOrder], *unc[kMaxOrder];
  uint32_t ubits[kMaxOrder];
  for (uint32_t k = 0; k < N; ++k) {
    if ((cmask >> k) & 1u) {
      comp[nc++] = x->inds[k].p;
      if (ceil_log2(x->dims[k]) > Lm) Lm = ceil_log2(x->dims[k]);
    } else {
      ubits[nu] = ceil_log2(x->dims[k]);
      unc[nu++] = x->inds[k].p;
    }
  }
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  if (nu) lexsort(unc, ubits, int(nu), perm, M, s);
  morton_sort(comp, nc, Lm, perm, M, s);

  DevArray<uint32_t> sc[kMaxOrder];
  Coords co{};
  co.order = 0;
  for (uint32_t k = 0; k < N; ++k) {
    sc[k].alloc(M, s);
    gather_u32(x->inds[k].p, perm.p, sc[k].p, M, s);
    if ((cmask >> k) & 1u) co.c[co.order++] = sc[k].p;
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
  bool bptr_written = false;
  for (uint32_t k = 0; k < N; ++k) {
    if (!((cmask >> k) & 1u)) {
      h->uinds[k] = std::move(sc[k]);  // full coordinates, already in gHiCOO order
      continue;
    }
    h->binds[k].alloc(nb, s);
    h->einds[k].alloc(M, s);
    if (M) {
      emit_blocks_kernel<<<grid_for(nb + 1), kThreads, 0, s>>>(starts.p, nb, M, sc[k].p, bb, h->bptr.p,
                                                             h->binds[k].p, !bptr_written);
      PASTA_LAUNCHED();
      bptr_written = true;
      emit_einds_kernel<<<grid_for(M), kThreads, 0, s>>>(sc[k].p, M, (1u << bb) - 1u, h->einds[k].p);
      PASTA_LAUNCHED();
    }
  }
  h->val.alloc(M, s);
  gather_f32(x->val.p, perm.p, h->val.p, M, s);
  PASTA_CUDA(cudaStreamSynchronize(s));
}

uint64_t count_blocks_device(const pasta_coo *x, uint32_t block_bits, uint32_t cmask, cudaStream_t s) {
  const uint64_t M = x->nnz;
  if (M == 0) return 0;
  const uint32_t N = x->order;
  DevArray<uint32_t> keys[kMaxOrder];
  const uint32_t *comps[kMaxOrder];
  uint32_t bits[kMaxOrder];
  int nc = 0;
  Coords co{};
  for (uint32_t k = 0; k < N; ++k) {
    if (!((cmask >> k) & 1u)) continue;
    keys[nc].alloc(M, s);
    shift_u32_kernel<<<grid_for(M), kThreads, 0, s>>>(x->inds[k].p, M, block_bits, keys[nc].p);
    PASTA_LAUNCHED();
    comps[nc] = keys[nc].p;
    uint32_t l = ceil_log2(x->dims[k]);
    bits[nc] = l > block_bits ? l - block_bits : 0;
    ++nc;
  }
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  lexsort(comps, bits, nc, perm, M, s);
  DevArray<uint32_t> sk[kMaxOrder];
  for (int c = 0; c < nc; ++c) {
    sk[c].alloc(M, s);
    gather_u32(keys[c].p, perm.p, sk[c].p, M, s);
    co.c[c] = sk[c].p;
  }
  co.order = uint32_t(nc);
  DevArray<uint8_t> flag(M, s);
  block_flag_kernel<<<grid_for(M), kThreads, 0, s>>>(co, 0, M, flag.p);
  PASTA_LAUNCHED();
  DevArray<uint32_t> starts;
  return select_flagged(flag.p, M, starts, s);
}

// Per-mode copy (R#27): blocks stably sorted by (light, binds_mode), entries inside a block
// stably sorted by einds_mode, so equal output rows are contiguous runs (segmented
// reduction); heavy blocks come first and get CTA work items (pieces) for the tile-staged
// kernel.
// R#36: the tier blocks of each compressed other mode (see hicoo_tier_rows)
struct TierPlan {
  uint32_t ntier[kMaxOrder] = {}, sblk[kMaxOrder] = {};
  uint32_t hs_base[kMaxOrder] = {}, hot_base[kMaxOrder] = {};
};

static void hicoo_prepare_rowslice_tiered(pasta_hicoo *h, uint32_t mode, const TierPlan &tp, cudaStream_t s);

static void hicoo_prepare_rowslice(pasta_hicoo *h, uint32_t mode, cudaStream_t s, const TierPlan *tp = nullptr) {
  HicooModeCopy &mc = h->mc[mode];
  const uint32_t N = h->order;
  const uint64_t M = h->nnz, nb = h->nblocks;
  const uint32_t bb = h->block_bits;
  auto comp = [&](uint32_t k) { return ((h->cmask >> k) & 1u) != 0; };
  mc.layout = 0;
  // derived per-copy caches of the launcher are rebuilt for the new slices
  mc.run_sb_run = 0;
  mc.run_sb.reset();
  mc.sbend32.reset();
  mc.win_sb.reset();
  mc.tagged = false;
  mc.hot_R = 0;
  if (tp && M > 0) return hicoo_prepare_rowslice_tiered(h, mode, *tp, s);
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode) continue;
    if (comp(k)) mc.einds[k].alloc(M, s); else mc.uinds[k].alloc(M, s);
  }
  mc.val.alloc(M, s);
  if (M == 0) {
    mc.nsb = 0;
    mc.sbptr.alloc(1, s);
    uint64_t zero = 0;
    PASTA_CUDA(cudaMemcpyAsync(mc.sbptr.p, &zero, sizeof(zero), cudaMemcpyHostToDevice, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    mc.ready = true;
    return;
  }
  // entry order: (output row, blk), the row as (binds_mode[blk], einds_mode) when the mode is
  // compressed, else the full i_mode (gHiCOO); ties keep the canonical order (stable)
  DevArray<uint32_t> blk(M, s), c0, en;
  entry_block_kernel<<<grid_for(M), kThreads, 0, s>>>(h->bptr.p, nb, M, blk.p);
  PASTA_LAUNCHED();
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  const uint32_t *en_src;
  if (comp(mode)) {
    c0.alloc(M, s);
    en.alloc(M, s);
    gather_binds_kernel<<<grid_for(M), kThreads, 0, s>>>(h->binds[mode].p, blk.p, M, c0.p);
    PASTA_LAUNCHED();
    u8_to_u32_kernel<<<grid_for(M), kThreads, 0, s>>>(h->einds[mode].p, M, en.p);
    PASTA_LAUNCHED();
    uint64_t nbr = (uint64_t(h->dims[mode]) + (1ull << bb) - 1) >> bb;
    const uint32_t *comps[3] = {c0.p, en.p, blk.p};
    uint32_t bits[3] = {ceil_log2(nbr), bb, ceil_log2(nb)};
    lexsort(comps, bits, 3, perm, M, s);
    c0.reset();
    en_src = en.p;
  } else {
    const uint32_t *comps[2] = {h->uinds[mode].p, blk.p};
    uint32_t bits[2] = {ceil_log2(h->dims[mode]), ceil_log2(nb)};
    lexsort(comps, bits, 2, perm, M, s);
    en_src = h->uinds[mode].p;
  }
  DevArray<uint32_t> blkp(M, s), enp(M, s);
  gather_u32(blk.p, perm.p, blkp.p, M, s);
  gather_u32(en_src, perm.p, enp.p, M, s);
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode) continue;
    if (comp(k)) gather_u8(h->einds[k].p, perm.p, mc.einds[k].p, M, s);
    else gather_u32(h->uinds[k].p, perm.p, mc.uinds[k].p, M, s);
  }
  gather_f32(h->val.p, perm.p, mc.val.p, M, s);
  DevArray<uint8_t> flag(M, s);
  slice_flag_kernel<<<grid_for(M), kThreads, 0, s>>>(blkp.p, enp.p, M, flag.p);
  PASTA_LAUNCHED();
  DevArray<uint32_t> starts;
  mc.nsb = select_flagged(flag.p, M, starts, s);
  mc.sbptr.alloc(mc.nsb + 1, s);
  // slice rows / bases carry kSlicePad zero slots past nsb: the raw-staged decode copies 36
  // aligned slots from any window's first slice without bounds checks
  mc.sbrow.alloc(mc.nsb + kSlicePad, s);
  PASTA_CUDA(cudaMemsetAsync(mc.sbrow.p + mc.nsb, 0, kSlicePad * 4, s));
  SliceOut o{};
  o.order = N;
  o.mode = mode;
  o.bbits = bb;
  o.cmask = h->cmask;
  for (uint32_t k = 0; k < N; ++k) {
    o.binds[k] = h->binds[k].p;
    if (k != mode && comp(k)) {
      mc.sbbase[k].alloc(mc.nsb + kSlicePad, s);
      PASTA_CUDA(cudaMemsetAsync(mc.sbbase[k].p + mc.nsb, 0, kSlicePad * 4, s));
      o.base[k] = mc.sbbase[k].p;
    }
  }
  slice_emit_kernel<<<grid_for(mc.nsb + 1), kThreads, 0, s>>>(o, starts.p, mc.nsb, M, blkp.p, enp.p,
                                                              mc.sbptr.p, mc.sbrow.p);
  PASTA_LAUNCHED();
  PASTA_CUDA(cudaStreamSynchronize(s));
  mc.ready = true;
  if (getenv("PASTA_DEBUG"))
    fprintf(stderr, "[pasta] hicoo row slices mode %u: %llu slices\n", mode, (unsigned long long)mc.nsb);
}

// Row-slice copy over tier blocks (R#36).  Every compressed other mode k has its rows ranked by
// nonzero count (h->rt_rank[k]); the rows of ranks [0, ntier_k B) form ntier_k synthetic "tier
// blocks" of B consecutive ranks -- the first sblk_k in the shared-memory tier, the rest in the
// packed L2-tier buffer -- and an entry on such a row is re-blocked: block key nbr_k + m,
// element index rho & (B - 1).  Entries are ordered by (output row, block key of every
// compressed other mode); a slice = equal row and keys; a slice base of a tier block is the
// tier tag | its first slot, so the decode's base + e lands on the row's slot directly and the
// kernel gathers through the same tiers as the COO hot-row cache (WA 10).  Every row of a tier
// block is hot (ranks, not row numbers), so a tier line holds only hot rows.
static void hicoo_prepare_rowslice_tiered(pasta_hicoo *h, uint32_t mode, const TierPlan &tp, cudaStream_t s) {
  HicooModeCopy &mc = h->mc[mode];
  const uint32_t N = h->order;
  const uint64_t M = h->nnz, nb = h->nblocks;
  const uint32_t bb = h->block_bits, B = 1u << bb;
  auto comp = [&](uint32_t k) { return ((h->cmask >> k) & 1u) != 0; };
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode) continue;
    if (comp(k)) mc.einds[k].alloc(M, s); else mc.uinds[k].alloc(M, s);
  }
  mc.val.alloc(M, s);
  DevArray<uint32_t> blk(M, s), rowfull;
  entry_block_kernel<<<grid_for(M), kThreads, 0, s>>>(h->bptr.p, nb, M, blk.p);
  PASTA_LAUNCHED();
  const uint32_t *row_src;
  if (comp(mode)) {
    rowfull.alloc(M, s);
    full_row_kernel<<<grid_for(M), kThreads, 0, s>>>(h->binds[mode].p, blk.p, h->einds[mode].p, bb, M, rowfull.p);
    PASTA_LAUNCHED();
    row_src = rowfull.p;
  } else {
    row_src = h->uinds[mode].p;
  }
  TierArgs ta{};
  ta.order = N;
  ta.bbits = bb;
  DevArray<uint32_t> key[kMaxOrder];
  DevArray<uint8_t> e[kMaxOrder];
  const uint32_t *comps[kMaxOrder + 1];
  uint32_t bits[kMaxOrder + 1];
  int nc = 0;
  comps[nc] = row_src;
  bits[nc++] = ceil_log2(h->dims[mode]);
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode || !comp(k)) continue;
    key[k].alloc(M, s);
    e[k].alloc(M, s);
    ta.binds[k] = h->binds[k].p;
    ta.einds[k] = h->einds[k].p;
    ta.rank[k] = h->rt_rank[k].p;
    ta.ntier[k] = tp.ntier[k];
    ta.nbr[k] = uint32_t((uint64_t(h->dims[k]) + B - 1) >> bb);
    ta.key[k] = key[k].p;
    ta.e[k] = e[k].p;
    comps[nc] = key[k].p;
    bits[nc++] = ceil_log2(uint64_t(ta.nbr[k]) + tp.ntier[k]);
  }
  tier_entry_kernel<<<grid_for(M), kThreads, 0, s>>>(ta, blk.p, M);
  PASTA_LAUNCHED();
  blk.reset();
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  lexsort(comps, bits, nc, perm, M, s);
  DevArray<uint32_t> rowp(M, s), keyp[kMaxOrder];
  gather_u32(row_src, perm.p, rowp.p, M, s);
  rowfull.reset();
  Coords co{};
  co.order = 0;
  co.c[co.order++] = rowp.p;
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode) continue;
    if (comp(k)) {
      keyp[k].alloc(M, s);
      gather_u32(key[k].p, perm.p, keyp[k].p, M, s);
      gather_u8(e[k].p, perm.p, mc.einds[k].p, M, s);
      co.c[co.order++] = keyp[k].p;
      key[k].reset();
      e[k].reset();
    } else if (tp.ntier[k]) {
      tier_coord_kernel<<<grid_for(M), kThreads, 0, s>>>(h->uinds[k].p, perm.p, M, h->rt_rank[k].p, tp.ntier[k] << bb,
                                                         tp.sblk[k] << bb, tp.hs_base[k], tp.hot_base[k],
                                                         mc.uinds[k].p);
      PASTA_LAUNCHED();
    } else {
      gather_u32(h->uinds[k].p, perm.p, mc.uinds[k].p, M, s);
    }
  }
  gather_f32(h->val.p, perm.p, mc.val.p, M, s);
  perm.reset();
  DevArray<uint8_t> flag(M, s);
  block_flag_kernel<<<grid_for(M), kThreads, 0, s>>>(co, 0, M, flag.p);
  PASTA_LAUNCHED();
  DevArray<uint32_t> starts;
  mc.nsb = select_flagged(flag.p, M, starts, s);
  flag.reset();
  mc.sbptr.alloc(mc.nsb + 1, s);
  mc.sbrow.alloc(mc.nsb + kSlicePad, s);
  PASTA_CUDA(cudaMemsetAsync(mc.sbrow.p + mc.nsb, 0, kSlicePad * 4, s));
  TierEmit o{};
  o.order = N;
  o.mode = mode;
  o.bbits = bb;
  for (uint32_t k = 0; k < N; ++k) {
    if (k == mode || !comp(k)) continue;
    mc.sbbase[k].alloc(mc.nsb + kSlicePad, s);
    PASTA_CUDA(cudaMemsetAsync(mc.sbbase[k].p + mc.nsb, 0, kSlicePad * 4, s));
    o.key[k] = keyp[k].p;
    o.base[k] = mc.sbbase[k].p;
    o.nbr[k] = ta.nbr[k];
    o.sblk[k] = tp.sblk[k];
    o.hs_base[k] = tp.hs_base[k];
    o.hot_base[k] = tp.hot_base[k];
  }
  slice_emit_tier_kernel<<<grid_for(mc.nsb + 1), kThreads, 0, s>>>(o, starts.p, mc.nsb, M, rowp.p, mc.sbptr.p,
                                                                   mc.sbrow.p);
  PASTA_LAUNCHED();
  PASTA_CUDA(cudaStreamSynchronize(s));
  mc.ready = true;
}

// heat ranking of mode k's rows (R#36), cached on the handle: counts over the canonical entries,
// rows sorted by count descending (ties by row, ascending: the radix sort is stable), rank =
// inverse permutation, and the heat of every block of B consecutive ranks
static void hicoo_rank_mode(pasta_hicoo *h, uint32_t k, const uint32_t *blk, cudaStream_t s) {
  if (h->rt_ready[k]) return;
  const uint32_t n = h->dims[k], bb = h->block_bits;
  const uint64_t M = h->nnz;
  DevArray<uint32_t> cnt(n, s), cnt_sorted(n, s), rows(n, s);
  PASTA_CUDA(cudaMemsetAsync(cnt.p, 0, cnt.bytes(), s));
  if ((h->cmask >> k) & 1u)
    entry_row_count_kernel<<<grid_for(M), kThreads, 0, s>>>(h->binds[k].p, blk, h->einds[k].p, bb, M, cnt.p);
  else  // gHiCOO uncompressed mode: full coordinates
    coord_count_kernel<<<grid_for(M), kThreads, 0, s>>>(h->uinds[k].p, M, cnt.p);
  PASTA_LAUNCHED();
  iota_u32(rows.p, n, s);
  h->rt_order[k].alloc(n, s);
  size_t tb = 0;
  PASTA_CUDA(cub::DeviceRadixSort::SortPairsDescending(nullptr, tb, cnt.p, cnt_sorted.p, rows.p, h->rt_order[k].p,
                                                        int64_t(n), 0, 32, s));
  DevArray<uint8_t> tmp(tb, s);
  PASTA_CUDA(cub::DeviceRadixSort::SortPairsDescending(tmp.p, tb, cnt.p, cnt_sorted.p, rows.p, h->rt_order[k].p,
                                                        int64_t(n), 0, 32, s));
  count_launch();
  h->rt_rank[k].alloc(n, s);
  scatter_rank_kernel<<<grid_for(n), kThreads, 0, s>>>(h->rt_order[k].p, n, h->rt_rank[k].p);
  PASTA_LAUNCHED();
  const uint64_t nbk = (uint64_t(n) + (1u << bb) - 1) >> bb;
  DevArray<unsigned long long> heat(nbk, s);
  block_heat_kernel<<<grid_for(nbk), kThreads, 0, s>>>(cnt_sorted.p, n, bb, heat.p);
  PASTA_LAUNCHED();
  h->rt_heat[k].resize(nbk);
  PASTA_CUDA(cudaMemcpyAsync(h->rt_heat[k].data(), heat.p, heat.bytes(), cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  h->rt_ready[k] = true;
}

// R#36: tier blocks for the row-slice copy of `mode`, budgets as the COO hot-row cache
// (`smem_rows` shared-memory rows; PASTA_HOT_MB, default 64 MB, of L2 tier when `global_tier`).
// Tier blocks of all compressed other modes are taken greedily by heat (each mode's block
// heats are non-increasing, so every mode's tier is a prefix of its ranking: smem blocks
// first, then L2 blocks).  Rebuilds the copy when the plan changes; on = false restores the
// plain copy.
void hicoo_tier_rows(pasta_hicoo *h, uint32_t mode, uint32_t R, bool on, bool global_tier, uint32_t smem_rows,
                     cudaStream_t s) {
  HicooModeCopy &mc = h->mc[mode];
  if (!mc.ready || mc.layout != 0) return;
  const bool want = on && h->nnz > 0;
  if (!want) {
    if (mc.rt_on) {
      hicoo_prepare_rowslice(h, mode, s);
      mc.rt_on = false;
      mc.rt_R = 0;
    }
    return;
  }
  if (mc.rt_on && mc.rt_R == R && mc.rt_global == global_tier && mc.rt_budget == smem_rows) return;
  const uint32_t N = h->order, bb = h->block_bits, B = 1u << bb;
  // every gathered mode: compressed ones through re-blocked slices, uncompressed (gHiCOO) ones
  // through tagged per-entry coordinates
  auto tiered = [&](uint32_t k) { return k != mode; };
  bool ok = true;
  for (uint32_t k = 0; k < N; ++k)
    if (h->dims[k] >= 0x40000000u) ok = false;  // tagged bases need slots below 2^30
  const char *env = getenv("PASTA_HOT_MB");
  const double hot_mb = global_tier ? ((env && *env) ? atof(env) : 64.0) : 0.0;
  const uint64_t sm_blocks = smem_rows >> bb;
  const uint64_t l2_blocks = uint64_t(hot_mb * 1048576.0 / (double(B) * R * sizeof(float)));
  TierPlan tp{};
  uint64_t hs_total = 0, hot_total = 0;
  if (ok && sm_blocks + l2_blocks > 0) {
    {
      DevArray<uint32_t> blk(h->nnz, s);
      entry_block_kernel<<<grid_for(h->nnz), kThreads, 0, s>>>(h->bptr.p, h->nblocks, h->nnz, blk.p);
      PASTA_LAUNCHED();
      for (uint32_t k = 0; k < N; ++k)
        if (tiered(k)) hicoo_rank_mode(h, k, blk.p, s);
    }
    uint64_t p[kMaxOrder] = {};
    for (uint64_t i = 0; i < sm_blocks + l2_blocks; ++i) {
      int best = -1;
      unsigned long long bh = 0;
      for (uint32_t k = 0; k < N; ++k)
        if (tiered(k) && p[k] < h->rt_heat[k].size() && h->rt_heat[k][p[k]] > bh) {
          bh = h->rt_heat[k][p[k]];
          best = int(k);
        }
      if (best < 0) break;
      if (i < sm_blocks) ++tp.sblk[best];
      ++tp.ntier[best];
      ++p[best];
    }
    for (uint32_t k = 0; k < N; ++k) {
      tp.hs_base[k] = uint32_t(hs_total);
      hs_total += uint64_t(tp.sblk[k]) << bb;
    }
    for (uint32_t k = 0; k < N; ++k) {
      tp.hot_base[k] = uint32_t(hot_total);
      hot_total += uint64_t(tp.ntier[k] - tp.sblk[k]) << bb;
    }
  }
  // slot -> factor row lists: the ranking's prefixes (slots past a mode's last row hold row 0)
  mc.hs_total = hs_total;
  mc.hot_total = hot_total;
  mc.hs_rows.alloc(std::max<uint64_t>(hs_total, 1), s);
  mc.hot_rows.alloc(std::max<uint64_t>(hot_total, 1), s);
  PASTA_CUDA(cudaMemsetAsync(mc.hs_rows.p, 0, mc.hs_rows.bytes(), s));
  PASTA_CUDA(cudaMemsetAsync(mc.hot_rows.p, 0, mc.hot_rows.bytes(), s));
  mc.hot_buf.alloc(std::max<uint64_t>(hot_total, 1) * R, s);
  for (uint32_t k = 0; k < N; ++k) {
    mc.hs_base[k] = tp.hs_base[k];
    mc.hs_cnt[k] = uint64_t(tp.sblk[k]) << bb;
    mc.hot_base[k] = tp.hot_base[k];
    mc.hot_cnt[k] = uint64_t(tp.ntier[k] - tp.sblk[k]) << bb;
    if (!tp.ntier[k]) continue;
    const uint64_t n = h->dims[k];
    const uint64_t ns = std::min<uint64_t>(mc.hs_cnt[k], n);
    if (ns)
      PASTA_CUDA(cudaMemcpyAsync(mc.hs_rows.p + mc.hs_base[k], h->rt_order[k].p, ns * 4, cudaMemcpyDeviceToDevice, s));
    const uint64_t h0 = mc.hs_cnt[k];
    const uint64_t nh = h0 < n ? std::min<uint64_t>(mc.hot_cnt[k], n - h0) : 0;
    if (nh)
      PASTA_CUDA(cudaMemcpyAsync(mc.hot_rows.p + mc.hot_base[k], h->rt_order[k].p + h0, nh * 4,
                                 cudaMemcpyDeviceToDevice, s));
  }
  hicoo_prepare_rowslice(h, mode, s, &tp);
  // hicoo_prepare_rowslice cleared the R#34 state; these describe the R#36 tiers
  mc.hs_total = hs_total;
  mc.hot_total = hot_total;
  for (uint32_t k = 0; k < N; ++k) {
    mc.hs_base[k] = tp.hs_base[k];
    mc.hs_cnt[k] = uint64_t(tp.sblk[k]) << bb;
    mc.hot_base[k] = tp.hot_base[k];
    mc.hot_cnt[k] = uint64_t(tp.ntier[k] - tp.sblk[k]) << bb;
  }
  mc.rt_on = true;
  mc.rt_R = R;
  mc.rt_global = global_tier;
  mc.rt_budget = smem_rows;
  if (getenv("PASTA_DEBUG")) {
    double tot = 0.0, cov = 0.0;
    for (uint32_t k = 0; k < N; ++k)
      if (tiered(k) && h->rt_ready[k])
        for (size_t m = 0; m < h->rt_heat[k].size(); ++m) {
          tot += double(h->rt_heat[k][m]);
          if (m < tp.ntier[k]) cov += double(h->rt_heat[k][m]);
        }
    fprintf(stderr, "[pasta] hicoo tier blocks mode %u R %u: smem %llu rows, L2 %llu rows, %llu slices, "
            "%.3f of the gathers (", mode, R, (unsigned long long)hs_total, (unsigned long long)hot_total,
            (unsigned long long)mc.nsb, tot > 0 ? cov / tot : 0.0);
    for (uint32_t k = 0; k < N; ++k)
      if (tiered(k)) fprintf(stderr, " k%u:%u+%u", k, tp.sblk[k], tp.ntier[k] - tp.sblk[k]);
    fprintf(stderr, " )\n");
  }
}

void hicoo_prepare_mode(pasta_hicoo *h, uint32_t mode, cudaStream_t s) {
  HicooModeCopy &mc = h->mc[mode];
  if (mc.ready) return;
  const char *lay = getenv("PASTA_HICOO_LAYOUT");
  const bool full = h->cmask == (1u << h->order) - 1u;  // the block layout needs every mode blocked
  if (!full || !(lay && std::string(lay) == "block")) return hicoo_prepare_rowslice(h, mode, s);
  mc.layout = 1;
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
  // Heavy blocks (>= heavy_min entries: staging their factor tiles pays, Table I's
  // min{n_b B, M} term) go first, light ones after; each part by binds_mode.
  const char *env = getenv("PASTA_HICOO_HEAVY");
  mc.heavy_min = (env && *env) ? uint32_t(atoi(env)) : 256u;
  if (mc.heavy_min == 0) mc.heavy_min = 0xFFFFFFFFu;  // 0 disables the heavy path
  // entry permutation: (light[blk], binds_mode[blk], blk, einds_mode)
  DevArray<uint32_t> blk(M, s), c0(M, s), c2(M, s), lt(M, s);
  entry_block_kernel<<<grid_for(M), kThreads, 0, s>>>(h->bptr.p, nb, M, blk.p);
  PASTA_LAUNCHED();
  gather_binds_kernel<<<grid_for(M), kThreads, 0, s>>>(h->binds[mode].p, blk.p, M, c0.p);
  PASTA_LAUNCHED();
  u8_to_u32_kernel<<<grid_for(M), kThreads, 0, s>>>(h->einds[mode].p, M, c2.p);
  PASTA_LAUNCHED();
  light_entry_kernel<<<grid_for(M), kThreads, 0, s>>>(h->bptr.p, blk.p, M, mc.heavy_min, lt.p);
  PASTA_LAUNCHED();
  uint64_t nbr = (uint64_t(h->dims[mode]) + (1ull << bb) - 1) >> bb;  // block rows of this mode
  const uint32_t *comps[4] = {lt.p, c0.p, blk.p, c2.p};
  uint32_t bits[4] = {1, ceil_log2(nbr), ceil_log2(nb), bb};
  DevArray<uint32_t> perm(M, s);
  iota_u32(perm.p, M, s);
  lexsort(comps, bits, 4, perm, M, s);
  for (uint32_t k = 0; k < N; ++k) gather_u8(h->einds[k].p, perm.p, mc.einds[k].p, M, s);
  gather_f32(h->val.p, perm.p, mc.val.p, M, s);
  // block schedule: blocks stably sorted by (light, binds_mode), the order entries now follow
  DevArray<uint32_t> sched(nb, s), blt(nb, s);
  iota_u32(sched.p, nb, s);
  light_block_kernel<<<grid_for(nb), kThreads, 0, s>>>(h->bptr.p, nb, mc.heavy_min, blt.p);
  PASTA_LAUNCHED();
  const uint32_t *bc[2] = {blt.p, h->binds[mode].p};
  uint32_t bbit[2] = {1, ceil_log2(nbr)};
  lexsort(bc, bbit, 2, sched, nb, s);
  DevArray<uint64_t> cnt(nb + 1, s);
  sched_counts_kernel<<<grid_for(nb + 1), kThreads, 0, s>>>(h->bptr.p, sched.p, nb, cnt.p);
  PASTA_LAUNCHED();
  size_t tmp_bytes = 0;
  PASTA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tmp_bytes, cnt.p, mc.bptr.p, nb + 1, s));
  DevArray<uint8_t> tmp(tmp_bytes, s);
  PASTA_CUDA(cub::DeviceScan::ExclusiveSum(tmp.p, tmp_bytes, cnt.p, mc.bptr.p, nb + 1, s));
  count_launch();
  // number of heavy blocks = blocks whose light flag is 0
  {
    std::vector<uint32_t> hl(nb);
    PASTA_CUDA(cudaMemcpyAsync(hl.data(), blt.p, nb * sizeof(uint32_t), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    uint64_t nh = 0;
    for (uint64_t b = 0; b < nb; ++b) nh += hl[b] == 0;
    mc.n_heavy = nh;
  }
  PASTA_CUDA(cudaMemcpyAsync(&mc.heavy_nnz, mc.bptr.p + mc.n_heavy, sizeof(uint64_t),
                             cudaMemcpyDeviceToHost, s));
  PASTA_CUDA(cudaStreamSynchronize(s));
  // CTA work items of the heavy part: (block, piece) with at most `piece` entries each
  if (mc.n_heavy) {
    DevArray<uint64_t> pc(mc.n_heavy + 1, s), off(mc.n_heavy + 1, s);
    piece_count_kernel<<<grid_for(mc.n_heavy + 1), kThreads, 0, s>>>(mc.bptr.p, mc.n_heavy, mc.piece, pc.p);
    PASTA_LAUNCHED();
    size_t tb = 0;
    PASTA_CUDA(cub::DeviceScan::ExclusiveSum(nullptr, tb, pc.p, off.p, mc.n_heavy + 1, s));
    DevArray<uint8_t> t2(tb, s);
    PASTA_CUDA(cub::DeviceScan::ExclusiveSum(t2.p, tb, pc.p, off.p, mc.n_heavy + 1, s));
    count_launch();
    PASTA_CUDA(cudaMemcpyAsync(&mc.n_pieces, off.p + mc.n_heavy, sizeof(uint64_t), cudaMemcpyDeviceToHost, s));
    PASTA_CUDA(cudaStreamSynchronize(s));
    mc.pieces.alloc(2 * mc.n_pieces, s);
    piece_emit_kernel<<<grid_for(mc.n_heavy), kThreads, 0, s>>>(off.p, mc.n_heavy, mc.pieces.p);
    PASTA_LAUNCHED();
  }
  for (uint32_t k = 0; k < N; ++k) gather_u32(h->binds[k].p, sched.p, mc.binds[k].p, nb, s);
  PASTA_CUDA(cudaStreamSynchronize(s));
  mc.ready = true;
}

namespace {
// full coordinate of every entry (canonical gHiCOO order): binds_k[blk] << b | einds_k, or uinds_k
__global__ void decode_coord_kernel(const uint32_t *__restrict__ blk, const uint32_t *__restrict__ binds,
                                    const uint8_t *__restrict__ einds, const uint32_t *__restrict__ uinds,
                                    uint32_t bb, uint64_t M, uint32_t *__restrict__ out) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M; x += uint64_t(gridDim.x) * blockDim.x)
    out[x] = uinds ? uinds[x] : ((binds[blk[x]] << bb) | einds[x]);
}
__global__ void range_flag_kernel(const uint32_t *__restrict__ c, uint64_t M, uint32_t lo, uint32_t hi,
                                  uint8_t *__restrict__ flag) {
  for (uint64_t x = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; x < M; x += uint64_t(gridDim.x) * blockDim.x)
    flag[x] = c[x] >= lo && c[x] < hi;
}
}  // namespace

// The entries of `h` with row_lo <= i_mode < row_hi, as a HiCOO handle of the same shape,
// block size and mask: the canonical order restricted to the
// subset (a Morton / gHiCOO order restricted to a subset is that subset's order), blocks
// re-cut where a compressed mode's block index changes -- the conversion of the sub-tensor.
void hicoo_shard_device(const pasta_hicoo *h, uint32_t mode, uint32_t row_lo, uint32_t row_hi, pasta_hicoo *y,
                        cudaStream_t s) {
  const uint32_t N = h->order, bb = h->block_bits, cmask = h->cmask;
  const uint64_t M = h->nnz;
  y->order = N;
  for (uint32_t k = 0; k < N; ++k) y->dims[k] = h->dims[k];
  y->block_bits = bb;
  y->cmask = cmask;
  y->device = h->device;
  DevArray<uint32_t> blk(M, s);
  if (M) {
    entry_block_kernel<<<grid_for(M), kThreads, 0, s>>>(h->bptr.p, h->nblocks, M, blk.p);
    PASTA_LAUNCHED();
  }
  auto decode = [&](uint32_t k, uint32_t *out) {
    const bool comp = (cmask >> k) & 1u;
    decode_coord_kernel<<<grid_for(M), kThreads, 0, s>>>(blk.p, comp ? h->binds[k].p : nullptr,
                                                         comp ? h->einds[k].p : nullptr,
                                                         comp ? nullptr : h->uinds[k].p, bb, M, out);
    PASTA_LAUNCHED();
  };
  DevArray<uint32_t> idx;
  uint64_t Ms = 0;
  if (M) {
    DevArray<uint32_t> rows(M, s);
    decode(mode, rows.p);
    DevArray<uint8_t> flag(M, s);
    range_flag_kernel<<<grid_for(M), kThreads, 0, s>>>(rows.p, M, row_lo, row_hi, flag.p);
    PASTA_LAUNCHED();
    Ms = select_flagged(flag.p, M, idx, s);
  }
  DevArray<uint32_t> sc[kMaxOrder];
  Coords co{};
  co.order = 0;
  for (uint32_t k = 0; k < N; ++k) {
    sc[k].alloc(Ms, s);
    if (Ms) {
      DevArray<uint32_t> full(M, s);
      decode(k, full.p);
      gather_u32(full.p, idx.p, sc[k].p, Ms, s);
    }
    if ((cmask >> k) & 1u) co.c[co.order++] = sc[k].p;
  }
  uint64_t nb = 0;
  DevArray<uint32_t> starts;
  if (Ms) {
    DevArray<uint8_t> flag(Ms, s);
    block_flag_kernel<<<grid_for(Ms), kThreads, 0, s>>>(co, bb, Ms, flag.p);
    PASTA_LAUNCHED();
    nb = select_flagged(flag.p, Ms, starts, s);
  }
  y->nblocks = nb;
  y->nnz = Ms;
  y->bptr.alloc(nb + 1, s);
  if (!Ms) {
    uint64_t zero = 0;
    PASTA_CUDA(cudaMemcpyAsync(y->bptr.p, &zero, sizeof(zero), cudaMemcpyHostToDevice, s));
  }
  bool bptr_written = false;
  for (uint32_t k = 0; k < N; ++k) {
    if (!((cmask >> k) & 1u)) {
      y->uinds[k] = std::move(sc[k]);
      continue;
    }
    y->binds[k].alloc(nb, s);
    y->einds[k].alloc(Ms, s);
    if (Ms) {
      emit_blocks_kernel<<<grid_for(nb + 1), kThreads, 0, s>>>(starts.p, nb, Ms, sc[k].p, bb, y->bptr.p,
                                                             y->binds[k].p, !bptr_written);
      PASTA_LAUNCHED();
      bptr_written = true;
      emit_einds_kernel<<<grid_for(Ms), kThreads, 0, s>>>(sc[k].p, Ms, (1u << bb) - 1u, y->einds[k].p);
      PASTA_LAUNCHED();
    }
  }
  y->val.alloc(Ms, s);
  if (Ms) gather_f32(h->val.p, idx.p, y->val.p, Ms, s);
  y->shard_mode = int(mode);
  y->row_lo = row_lo;
  y->row_hi = row_hi;
  PASTA_CUDA(cudaStreamSynchronize(s));
}

}  // namespace pasta
