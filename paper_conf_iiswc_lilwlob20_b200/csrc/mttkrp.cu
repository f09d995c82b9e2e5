// mttkrp.cu -- sm_100a MTTKRP kernels on COO (a6) and HiCOO (a7), and the output zero-fill (a5).
//
// What is computed (Eq. 3; Eq. 4; folded into the nonzero loop):
//     out(i_n(x), r) += val(x) * prod_{k != n} U^(k)(i_k(x), r)
//
// Design (B200-first, not the paper's P100/V100 kernels):
//   * Input is the mode-n working copy: nonzeros sorted so equal output rows are contiguous
//     (COO: lexicographic from mode n; HiCOO: blocks by binds_n, entries by einds_n, R#27).
//   * A warp owns a contiguous chunk of nonzeros; its 32 lanes form G = 32/LPN groups of LPN
//     lanes.  Group g walks a contiguous run of S = chunk/G nonzeros; within the group each
//     lane owns VW (=4 -> one 128-bit LDG) consecutive columns r of every factor row, so one
//     group-load fetches a whole 4R-byte row (64 B at R = 16) -- the coalescing direction the
//     paper's 2-D blocks use (x = R).
//   * Index/value streams: 128-bit vector loads (4 nonzeros per load per array, COO) or
//     32-bit loads of 4 packed 8-bit element indices (HiCOO).
//   * All U gathers of an unrolled step are issued before any is consumed (memory-level
//     parallelism is the whole game for this gather-bound kernel).
//   * Rank-R partial sums stay in registers while the output row does not change
//     (segmented reduction over runs of equal i_n).  A finished segment that began and
//     ended inside the run is owned by this group alone -> plain 128-bit store; the first
//     and last segment of a run may be shared with neighbours -> red.global.add.v4.f32
//     (one vector atomic per boundary, not per nonzero, cf. P:157/P:282 atomics).
//   * No tensor cores: the path is a gather/scatter, not a dense contraction.
#include <algorithm>
#include <cstdlib>
#include <type_traits>

#include "internal.cuh"

namespace pasta {

namespace {

constexpr int kWarpsPerCta = 8;
constexpr int kThreads = kWarpsPerCta * 32;

struct KArgs {
  uint64_t nnz;      // absolute end of the processed range
  uint64_t x_begin;  // absolute start (multiple of 4)
  uint64_t x_skip;   // entries below this absolute position are not processed
  uint64_t b_begin;  // HiCOO: first block of the range
  uint64_t chunk;  // nonzeros per warp; chunk % (4 * G) == 0
  uint32_t order, R;
  // COO streams (mode-n copy)
  const uint32_t *irow;                 // i_n
  const uint32_t *io[kMaxOrder - 1];    // i_k, k != n, ascending k
  const float *val;
  // HiCOO streams (mode-n copy)
  const uint64_t *bptr;
  uint64_t nblocks;
  const uint32_t *brow;
  const uint32_t *bo[kMaxOrder - 1];
  const uint8_t *erow;
  const uint8_t *eo[kMaxOrder - 1];
  uint32_t bbits;
  // HiCOO row-slice copy (layout 0)
  const uint64_t *sbptr;
  uint64_t nsb;
  const uint32_t *sbrow;
  const uint32_t *sbbase[kMaxOrder - 1];
  // gHiCOO (R#29): bit j set <=> other-mode slot j is uncompressed: its u32 coordinates come
  // from io[j] (no slice base); clear -> 8-bit element index eo[j] + slice base
  uint32_t wide;
  // factors of the other modes (ascending k), output
  const float *Uo[kMaxOrder - 1];
  float *out;
  // L2 eviction-priority hints (bit 0: streams evict_first, bit 1: gathers evict_last,
  // bit 2: output stores / atomics evict_first); see Policies
  uint32_t cache_mode;
  // io[] carry hot tags (coo_mark_hot): 0x80000000 | slot of hot_buf (L2 tier),
  // 0xC0000000 | slot of the shared-memory tier (coo_staged_kernel<..., HS = true>)
  uint32_t hot_marked;
  const float *hot_buf;
  // shared-memory tier: slot -> factor row; other-mode slot j owns slots [hs_lo[j], hs_lo[j+1])
  const uint32_t *hs_rows;
  uint32_t hs_lo[kMaxOrder];
  // HiCOO row slices decoded into the staged kernel (WA 9): run_sb[r] = slice holding entry
  // r * (chunk / G), the first entry of group run r
  const uint64_t *run_sb;
  // die split (R#35, HS kernels): die 0's CTAs take the chunks of [0, split_x), die 1's those
  // of [split_x, nnz), claimed dynamically (claim[die], zeroed per launch); every segment
  // flush is an atomic (a row appears in up to four segments)
  uint32_t split;
  uint64_t split_x;
  unsigned long long *claim;
  const int8_t *die_of;
  // HiCOO raw-staged decode (WA 11): win_sb[w] = slice holding entry 32 w; u32 slice ends;
  // words per group window of the raw buffer (layout: see coo_staged_kernel)
  const uint32_t *win_sb;
  const uint32_t *sbend32;
  uint32_t raw_words;
  // fused MTTKRP + all-gather (WA 15): every flush also goes to the peers' replicas of the
  // output (CUDA-IPC mapped, NVLink / NVSwitch P2P stores and atomics); outs[0] = out
  float *outs[kMaxOrder];
  uint32_t nout;
  // HiCOO row tier (WA 16): per other-mode slot j a bitmap of the factor rows held in the
  // shared-memory tier (bit i of word w = row 32 w + i) and, per word, the number of tier rows
  // before it; both copied into shared memory after the tier rows, rs_off[j] words apart
  const uint32_t *rs_bm[kMaxOrder - 1];
  const uint32_t *rs_pre[kMaxOrder - 1];
  uint32_t rs_words[kMaxOrder - 1];
};

// Per-thread L2 cache policies (createpolicy, sm_80+): the nonzero stream is touched once
// and must not displace the power-law-hot factor rows, which is what L2 is for here.
struct Policies {
  uint64_t stream, gather, cold, out;
  __device__ __forceinline__ explicit Policies(uint32_t mode) {
    uint64_t first, normal, last;
    asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(first));
    asm("createpolicy.fractional.L2::evict_normal.b64 %0, 1.0;" : "=l"(normal));
    asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(last));
    stream = (mode & 1) ? first : normal;
    gather = (mode & 2) ? last : normal;
    // bit 3: gathers of COLD rows (not in a hot tier) evict_first, so that the rows that are
    // used once or twice per launch do not push the hot tier out of L2
    cold = (mode & 8) ? first : gather;
    out = (mode & 4) ? first : normal;
  }
};

__device__ __forceinline__ uint4 ld_stream_u4(const void *p, uint64_t pol) {
  uint4 r;
  asm("ld.global.nc.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ uint32_t ld_stream_u32(const void *p, uint64_t pol) {
  uint32_t r;
  asm("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(r) : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ float4 ld_gather_f4(const float *p, uint64_t pol) {
  float4 r;
  asm("ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%4], %5;"
      : "=f"(r.x), "=f"(r.y), "=f"(r.z), "=f"(r.w)
      : "l"(p), "l"(pol));
  return r;
}

template <int VW>
struct Vec {
  float v[VW];
};

template <int VW>
__device__ __forceinline__ Vec<VW> ldg_vec(const float *p, uint64_t pol) {
  Vec<VW> r;
  if constexpr (VW == 4) {
    float4 t = ld_gather_f4(p, pol);
    r.v[0] = t.x; r.v[1] = t.y; r.v[2] = t.z; r.v[3] = t.w;
  } else {
#pragma unroll
    for (int i = 0; i < VW; ++i) r.v[i] = __ldg(p + i);
  }
  return r;
}

// One predicated 128-bit load from either shared memory (ps) or global memory (pg), without a
// branch: divergent per-group branches would serialise the batch of independent gathers.
template <bool L1NA = false>
__device__ __forceinline__ Vec<4> ld_tiered(uint32_t saddr, const float *gp, uint64_t pol, int ps, int pg) {
  Vec<4> r;
  if constexpr (L1NA) {  // the global gather does not allocate in L1
    asm volatile(
        "{\n\t.reg .pred ps, pg;\n\t"
        "setp.ne.s32 ps, %5, 0;\n\t"
        "setp.ne.s32 pg, %6, 0;\n\t"
        "@ps ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];\n\t"
        "@pg ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%7], %8;\n\t}"
        : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3])
        : "r"(saddr), "r"(ps), "r"(pg), "l"(gp), "l"(pol));
  } else {
    asm volatile(
        "{\n\t.reg .pred ps, pg;\n\t"
        "setp.ne.s32 ps, %5, 0;\n\t"
        "setp.ne.s32 pg, %6, 0;\n\t"
        "@ps ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];\n\t"
        "@pg ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%7], %8;\n\t}"
        : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3])
        : "r"(saddr), "r"(ps), "r"(pg), "l"(gp), "l"(pol));
  }
  return r;
}

// Three-way predicated 128-bit load: shared-memory tier (ps), L2-tier buffer (ph, policy ph_pol)
// or a cold factor row (pc, policy pc_pol); gp is the global address of whichever of the two.
__device__ __forceinline__ Vec<4> ld_tiered3(uint32_t saddr, const float *gp, uint64_t ph_pol, uint64_t pc_pol,
                                             int ps, int ph, int pc) {
  Vec<4> r;
  asm volatile(
      "{\n\t.reg .pred ps, ph, pc;\n\t"
      "setp.ne.s32 ps, %5, 0;\n\t"
      "setp.ne.s32 ph, %6, 0;\n\t"
      "setp.ne.s32 pc, %7, 0;\n\t"
      "@ps ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];\n\t"
      "@ph ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%8], %9;\n\t"
      "@pc ld.global.nc.L2::cache_hint.v4.f32 {%0, %1, %2, %3}, [%8], %10;\n\t}"
      : "=f"(r.v[0]), "=f"(r.v[1]), "=f"(r.v[2]), "=f"(r.v[3])
      : "r"(saddr), "r"(ps), "r"(ph), "r"(pc), "l"(gp), "l"(ph_pol), "l"(pc_pol));
  return r;
}

template <int VW>
__device__ __forceinline__ void red_vec(float *p, const Vec<VW> &a, uint64_t pol) {
  if constexpr (VW == 4) {
    asm volatile("red.global.add.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p),
                 "f"(a.v[0]), "f"(a.v[1]), "f"(a.v[2]), "f"(a.v[3]), "l"(pol)
                 : "memory");
  } else {
#pragma unroll
    for (int i = 0; i < VW; ++i) atomicAdd(p + i, a.v[i]);
  }
}

template <int VW>
__device__ __forceinline__ void st_vec(float *p, const Vec<VW> &a, uint64_t pol) {
  if constexpr (VW == 4) {
    asm volatile("st.global.L2::cache_hint.v4.f32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(p), "f"(a.v[0]),
                 "f"(a.v[1]), "f"(a.v[2]), "f"(a.v[3]), "l"(pol)
                 : "memory");
  } else {
#pragma unroll
    for (int i = 0; i < VW; ++i) p[i] = a.v[i];
  }
}

// Index source policies --------------------------------------------------------------------
// load(x, cnt, row[], idx[][], v[]) fills U entries starting at x (cnt valid, x % 4 == 0).

template <int NO, int U>
struct CooSrc {
  // rows are globally sorted: a segment strictly inside a run is owned by that run
  static constexpr bool kSortedRows = true;
  static constexpr int kMinBlocks = 1;
  uint64_t pol;
  __device__ __forceinline__ void init(const KArgs &, uint64_t, uint64_t p) { pol = p; }
  __device__ __forceinline__ void load(const KArgs &a, uint64_t x, int cnt, uint32_t (&row)[U],
                                       uint32_t (&idx)[NO > 0 ? NO : kMaxOrder - 1][U], float (&v)[U], int no) {
    if (cnt == U && (x & 3) == 0) {
#pragma unroll
      for (int q = 0; q < U; q += 4) {
        uint4 r4 = ld_stream_u4(a.irow + x + q, pol);
        row[q] = r4.x; row[q + 1] = r4.y; row[q + 2] = r4.z; row[q + 3] = r4.w;
        uint4 v4 = ld_stream_u4(a.val + x + q, pol);
        v[q] = __uint_as_float(v4.x); v[q + 1] = __uint_as_float(v4.y);
        v[q + 2] = __uint_as_float(v4.z); v[q + 3] = __uint_as_float(v4.w);
#pragma unroll
        for (int j = 0; j < (NO > 0 ? NO : kMaxOrder - 1); ++j) {
          if (j < no) {
            uint4 i4 = ld_stream_u4(a.io[j] + x + q, pol);
            idx[j][q] = i4.x; idx[j][q + 1] = i4.y; idx[j][q + 2] = i4.z; idx[j][q + 3] = i4.w;
          }
        }
      }
    } else {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (u < cnt) {
          row[u] = __ldg(a.irow + x + u);
          v[u] = __ldg(a.val + x + u);
#pragma unroll
          for (int j = 0; j < (NO > 0 ? NO : kMaxOrder - 1); ++j)
            if (j < no) idx[j][u] = __ldg(a.io[j] + x + u);
        }
      }
    }
  }
};

template <int NO, int U>
struct HicooSrc {
  // rows repeat across blocks of one block row (R#27): every flush is an atomic
  static constexpr bool kSortedRows = false;
  static constexpr int kMinBlocks = 2;
  uint64_t b, bend;
  uint32_t base_row;
  uint32_t base[NO > 0 ? NO : kMaxOrder - 1];
  int no;
  uint64_t pol;
  __device__ __forceinline__ void set_block(const KArgs &a) {
    bend = __ldg(a.bptr + b + 1);
    base_row = __ldg(a.brow + b) << a.bbits;
#pragma unroll
    for (int j = 0; j < (NO > 0 ? NO : kMaxOrder - 1); ++j)
      if (j < no) base[j] = __ldg(a.bo[j] + b) << a.bbits;
  }
  __device__ __forceinline__ void init(const KArgs &a, uint64_t x0, uint64_t p) {
    pol = p;
    no = int(a.order) - 1;
    uint64_t lo = a.b_begin, hi = a.nblocks;  // last block with bptr[b] <= x0
    while (hi - lo > 1) {
      uint64_t mid = (lo + hi) / 2;
      if (__ldg(a.bptr + mid) <= x0) lo = mid; else hi = mid;
    }
    b = lo;
    set_block(a);
  }
  __device__ __forceinline__ void load(const KArgs &a, uint64_t x, int cnt, uint32_t (&row)[U],
                                       uint32_t (&idx)[NO > 0 ? NO : kMaxOrder - 1][U], float (&v)[U], int) {
    uint32_t er[U], ej[NO > 0 ? NO : kMaxOrder - 1][U];
    if (cnt == U && (x & 3) == 0) {
#pragma unroll
      for (int q = 0; q < U; q += 4) {
        uint32_t w = ld_stream_u32(a.erow + x + q, pol);
        er[q] = w & 0xff; er[q + 1] = (w >> 8) & 0xff; er[q + 2] = (w >> 16) & 0xff; er[q + 3] = w >> 24;
        uint4 v4 = ld_stream_u4(a.val + x + q, pol);
        v[q] = __uint_as_float(v4.x); v[q + 1] = __uint_as_float(v4.y);
        v[q + 2] = __uint_as_float(v4.z); v[q + 3] = __uint_as_float(v4.w);
#pragma unroll
        for (int j = 0; j < (NO > 0 ? NO : kMaxOrder - 1); ++j) {
          if (j < no) {
            uint32_t e = ld_stream_u32(a.eo[j] + x + q, pol);
            ej[j][q] = e & 0xff; ej[j][q + 1] = (e >> 8) & 0xff; ej[j][q + 2] = (e >> 16) & 0xff;
            ej[j][q + 3] = e >> 24;
          }
        }
      }
    } else {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (u < cnt) {
          er[u] = __ldg(a.erow + x + u);
          v[u] = __ldg(a.val + x + u);
#pragma unroll
          for (int j = 0; j < (NO > 0 ? NO : kMaxOrder - 1); ++j)
            if (j < no) ej[j][u] = __ldg(a.eo[j] + x + u);
        }
      }
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (u < cnt) {
        while (x + u >= bend) { ++b; set_block(a); }  // walk to the entry's block
        row[u] = base_row + er[u];
#pragma unroll
        for (int j = 0; j < (NO > 0 ? NO : kMaxOrder - 1); ++j)
          if (j < no) idx[j][u] = base[j] + ej[j][u];
      }
    }
  }
};

// HiCOO row-slice policy (layout 0, R#27): a slice = the entries of one block that share
// einds_n; slices are ordered by output row, so rows are globally sorted as in COO.  Per
// entry only the 8-bit element indices of the other modes and the value are streamed; the
// row and the other-mode block bases (Alg. 3's rebased pointers) come per slice.
// gHiCOO (R#29): an uncompressed other mode streams its u32 coordinate instead
// (KArgs::wide), an uncompressed target mode makes a slice = the entries of a block sharing
// i_n.  The wide test is warp-uniform.
template <int NO, int U>
struct HicooRowSrc {
  static constexpr bool kSortedRows = true;
  static constexpr int kMinBlocks = 2;  // cap registers at 128: >= 16 resident warps per SM
  static constexpr int NOA = NO > 0 ? NO : kMaxOrder - 1;
  // current slice (the one holding the next entry).  A step of U entries spans at most U
  // slices, so each step loads the metadata of slices sb+1 .. sb+U-1 at once (independent
  // loads, one latency per step) instead of walking slice after slice with a dependent load
  // each -- at ~1 entry per slice (hypersparse tensors) the walk was the kernel's critical path.
  uint64_t sb, sbend;
  uint32_t srow;
  uint32_t base[NOA];
  int no;
  uint32_t wide;
  uint64_t pol;
  __device__ __forceinline__ void init(const KArgs &a, uint64_t x0, uint64_t p) {
    pol = p;
    no = int(a.order) - 1;
    wide = a.wide;
    uint64_t lo = 0, hi = a.nsb;  // last slice with sbptr[sb] <= x0
    while (hi - lo > 1) {
      uint64_t mid = (lo + hi) / 2;
      if (__ldg(a.sbptr + mid) <= x0) lo = mid; else hi = mid;
    }
    sb = lo;
    sbend = __ldg(a.sbptr + sb + 1);
    srow = __ldg(a.sbrow + sb);
#pragma unroll
    for (int j = 0; j < NOA; ++j)
      if (j < no) base[j] = ((wide >> j) & 1u) ? 0u : __ldg(a.sbbase[j] + sb);
  }
  __device__ __forceinline__ void load(const KArgs &a, uint64_t x, int cnt, uint32_t (&row)[U],
                                       uint32_t (&idx)[NOA][U], float (&v)[U], int) {
    // slice window: slot 0 = current slice, slots 1 .. U-1 = the next ones (clamped)
    uint64_t wend[U];
    uint32_t wrow[U], wbase[NOA][U];
    wend[0] = sbend;
    wrow[0] = srow;
#pragma unroll
    for (int j = 0; j < NOA; ++j) wbase[j][0] = base[j];
#pragma unroll
    for (int t = 1; t < U; ++t) {
      const uint64_t st = sb + t < a.nsb ? sb + t : a.nsb - 1;
      wend[t] = __ldg(a.sbptr + st + 1);
      wrow[t] = __ldg(a.sbrow + st);
#pragma unroll
      for (int j = 0; j < NOA; ++j)
        if (j < no) wbase[j][t] = ((wide >> j) & 1u) ? 0u : __ldg(a.sbbase[j] + st);
    }
    uint32_t ej[NOA][U];
    if (cnt == U && (x & 3) == 0) {
#pragma unroll
      for (int q = 0; q < U; q += 4) {
        uint4 v4 = ld_stream_u4(a.val + x + q, pol);
        v[q] = __uint_as_float(v4.x); v[q + 1] = __uint_as_float(v4.y);
        v[q + 2] = __uint_as_float(v4.z); v[q + 3] = __uint_as_float(v4.w);
#pragma unroll
        for (int j = 0; j < NOA; ++j) {
          if (j < no) {
            if ((wide >> j) & 1u) {
              uint4 i4 = ld_stream_u4(a.io[j] + x + q, pol);
              ej[j][q] = i4.x; ej[j][q + 1] = i4.y; ej[j][q + 2] = i4.z; ej[j][q + 3] = i4.w;
            } else {
              uint32_t e = ld_stream_u32(a.eo[j] + x + q, pol);
              ej[j][q] = e & 0xff; ej[j][q + 1] = (e >> 8) & 0xff; ej[j][q + 2] = (e >> 16) & 0xff;
              ej[j][q + 3] = e >> 24;
            }
          }
        }
      }
    } else {
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (u < cnt) {
          v[u] = __ldg(a.val + x + u);
#pragma unroll
          for (int j = 0; j < NOA; ++j)
            if (j < no) ej[j][u] = ((wide >> j) & 1u) ? __ldg(a.io[j] + x + u) : uint32_t(__ldg(a.eo[j] + x + u));
        }
      }
    }
    // entry u lies in window slot c_u = #{t : wend[t] <= x + u} (ends ascend); selects are
    // unrolled compares so the window stays in registers
    int clast = 0;
#pragma unroll
    for (int u = 0; u < U; ++u) {
      if (u < cnt) {
        int c = 0;
#pragma unroll
        for (int t = 0; t < U - 1; ++t) c += (x + u >= wend[t]) ? 1 : 0;
        uint32_t r = wrow[0];
        uint32_t bsel[NOA];
#pragma unroll
        for (int j = 0; j < NOA; ++j) bsel[j] = wbase[j][0];
#pragma unroll
        for (int t = 1; t < U; ++t) {
          if (c == t) {
            r = wrow[t];
#pragma unroll
            for (int j = 0; j < NOA; ++j) bsel[j] = wbase[j][t];
          }
        }
        row[u] = r;
#pragma unroll
        for (int j = 0; j < NOA; ++j)
          if (j < no) idx[j][u] = bsel[j] + ej[j][u];
        clast = c;
      }
    }
    // the slice of the last entry becomes the current one
#pragma unroll
    for (int t = 1; t < U; ++t) {
      if (clast == t) {
        sbend = wend[t];
        srow = wrow[t];
#pragma unroll
        for (int j = 0; j < NOA; ++j) base[j] = wbase[j][t];
      }
    }
    sb += uint64_t(clast);
    // the next entry may start the following slice: advance once more if so (slot clast + 1
    // is loaded when clast + 1 < U; otherwise the next step's window starts from here)
    if (x + cnt >= sbend) {
      const uint64_t st = sb + 1 < a.nsb ? sb + 1 : a.nsb - 1;
      sb = st;
      sbend = __ldg(a.sbptr + st + 1);
      srow = __ldg(a.sbrow + st);
#pragma unroll
      for (int j = 0; j < NOA; ++j)
        if (j < no) base[j] = ((wide >> j) & 1u) ? 0u : __ldg(a.sbbase[j] + st);
    }
  }
};

// NO = number of other modes (order - 1) when specialised, 0 = generic (<= kMaxOrder - 1).
// Kernel variant knobs: U nonzeros per unrolled step, PF = software-pipelined prefetch of
// the next step's index/value stream (so the stream latency hides behind the gathers),
// MINB = minimum resident CTAs per SM requested from ptxas (register cap).
template <int U_, bool PF_, int MINB_>
struct Tune {
  static constexpr int U = U_;
  static constexpr bool PF = PF_;
  static constexpr int MINB = MINB_;
};

// NO = number of other modes (order - 1) when specialised, 0 = generic (<= kMaxOrder - 1).
template <class Src, int NO, int LPN, int VW, class T>
__global__ void __launch_bounds__(kThreads, T::MINB) mttkrp_kernel(const KArgs a) {
  constexpr int U = T::U;
  constexpr int G = 32 / LPN;
  constexpr int NOA = NO > 0 ? NO : kMaxOrder - 1;  // register array extent
  const int lane = threadIdx.x & 31;
  const int g = lane / LPN, lig = lane % LPN;
  const uint64_t w = uint64_t(blockIdx.x) * kWarpsPerCta + (threadIdx.x >> 5);
  const uint64_t c0 = a.x_begin + w * a.chunk;
  if (c0 >= a.nnz) return;
  const uint64_t S = a.chunk / G;
  uint64_t x0 = c0 + uint64_t(g) * S;
  uint64_t x1 = x0 + S;
  if (x1 > a.nnz) x1 = a.nnz;
  if (x0 < a.x_skip) x0 = a.x_skip;
  if (x0 >= x1) return;
  const int no = NO > 0 ? NO : int(a.order) - 1;
  const uint32_t R = a.R;
  const Policies pol(a.cache_mode);

  for (uint32_t col = uint32_t(lig) * VW; col < R; col += LPN * VW) {
    Src src;
    src.init(a, x0, pol.stream);
    Vec<VW> acc;
#pragma unroll
    for (int i = 0; i < VW; ++i) acc.v[i] = 0.f;
    uint32_t cur = 0xFFFFFFFFu;
    bool first = true;
    uint32_t row[U];
    uint32_t idx[NOA][U];
    float v[U];
    int cnt = (x1 - x0) >= uint64_t(U) ? U : int(x1 - x0);
    if (T::PF) src.load(a, x0, cnt, row, idx, v, no);
    for (uint64_t x = x0; x < x1; x += U) {
      uint32_t rown[U];
      uint32_t idxn[NOA][U];
      float vn[U];
      const uint64_t xn = x + U;
      const int cntn = xn >= x1 ? 0 : ((x1 - xn) >= uint64_t(U) ? U : int(x1 - xn));
      if (T::PF) {
        if (cntn > 0) src.load(a, xn, cntn, rown, idxn, vn, no);  // next step's stream
      } else {
        src.load(a, x, cnt, row, idx, v, no);
      }
      // issue every gather of this step before consuming any
      Vec<VW> f[NOA][U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
#pragma unroll
        for (int j = 0; j < NOA; ++j) {
          if (j < no && u < cnt) f[j][u] = ldg_vec<VW>(a.Uo[j] + uint64_t(idx[j][u]) * R + col, pol.gather);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (u < cnt) {
          Vec<VW> t;
#pragma unroll
          for (int i = 0; i < VW; ++i) t.v[i] = v[u];
#pragma unroll
          for (int j = 0; j < NOA; ++j) {
            if (j < no) {
#pragma unroll
              for (int i = 0; i < VW; ++i) t.v[i] *= f[j][u].v[i];
            }
          }
          if (row[u] == cur) {
#pragma unroll
            for (int i = 0; i < VW; ++i) acc.v[i] += t.v[i];
          } else {
            if (cur != 0xFFFFFFFFu) {
              float *dst = a.out + uint64_t(cur) * R + col;
              if (first || !Src::kSortedRows) red_vec<VW>(dst, acc, pol.out); else st_vec<VW>(dst, acc, pol.out);
              first = false;
            }
            cur = row[u];
            acc = t;
          }
        }
      }
      if (T::PF) {
#pragma unroll
        for (int u = 0; u < U; ++u) {
          row[u] = rown[u];
          v[u] = vn[u];
#pragma unroll
          for (int j = 0; j < NOA; ++j) idx[j][u] = idxn[j][u];
        }
      }
      cnt = cntn;
    }
    if (cur != 0xFFFFFFFFu) red_vec<VW>(a.out + uint64_t(cur) * R + col, acc, pol.out);
  }
}

// ---------------------------------------------------------------------------------------
// HiCOO heavy-block kernel (a7, dense part).  One CTA per work item = one tensor block (or a
// <= `piece`-entry slice of a huge one), the paper's HiCOO-GPU mapping, made B200-
// native: thread 0 stages the block's (N-1) factor-row tiles U_k[bk*B .. bk*B+B) -- contiguous
// B*R*4-byte ranges, Alg. 3's rebased pointers C_b, B_b -- into shared memory with
// 1-D TMA bulk copies (cp.async.bulk, completion on an mbarrier); the CTA's 64 lane groups
// then walk contiguous runs of the block's entries (sorted by einds_n), gather rows from the
// staged tiles (LDS.128), keep rank-R partial sums in registers while einds_n repeats, and
// flush each finished segment with one red.global.add.v4.f32.
struct HArgs {
  const uint32_t *pieces;
  uint32_t piece;
  const uint64_t *bptr;
  const uint32_t *brow;
  const uint32_t *bo[kMaxOrder - 1];
  const uint8_t *erow;
  const uint8_t *eo[kMaxOrder - 1];
  const float *val;
  const float *Uo[kMaxOrder - 1];
  uint32_t dims_o[kMaxOrder - 1];
  float *out;
  uint32_t order, R, bbits;
  uint32_t cache_mode;
};

__device__ __forceinline__ uint32_t smem_addr(const void *p) {
  return uint32_t(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_wait(uint32_t addr, uint32_t parity) {
  uint32_t done = 0;
  do {
    asm volatile(
        "{\n\t.reg .pred p;\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
        "selp.u32 %0, 1, 0, p;\n\t}"
        : "=r"(done)
        : "r"(addr), "r"(parity)
        : "memory");
  } while (!done);
}

template <int NO, int LPN>
__global__ void __launch_bounds__(kThreads) hicoo_heavy_kernel(const HArgs a) {
  extern __shared__ __align__(128) float tiles[];  // [no][B][R]
  __shared__ __align__(8) uint64_t mbar;
  constexpr int G = 32 / LPN;
  constexpr int NOA = NO > 0 ? NO : kMaxOrder - 1;
  constexpr int U = 4;
  const int no = NO > 0 ? NO : int(a.order) - 1;
  const uint32_t R = a.R;
  const uint32_t B = 1u << a.bbits;
  const uint32_t s = __ldg(a.pieces + 2 * blockIdx.x);
  const uint32_t pj = __ldg(a.pieces + 2 * blockIdx.x + 1);
  const uint64_t eb = __ldg(a.bptr + s), ee = __ldg(a.bptr + s + 1);
  const uint64_t lo = eb + uint64_t(pj) * a.piece;
  const uint64_t hi = (lo + a.piece < ee) ? lo + a.piece : ee;
  const uint32_t mb = smem_addr(&mbar);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mb) : "memory");
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t total = 0;
    uint32_t bytes[NOA];
    uint64_t base[NOA];
#pragma unroll
    for (int j = 0; j < NOA; ++j) {
      if (j < no) {
        base[j] = uint64_t(__ldg(a.bo[j] + s)) << a.bbits;
        uint64_t rows = a.dims_o[j] - base[j];
        if (rows > B) rows = B;
        bytes[j] = uint32_t(rows * R * 4u);
        total += bytes[j];
      }
    }
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mb), "r"(total) : "memory");
#pragma unroll
    for (int j = 0; j < NOA; ++j) {
      if (j < no)
        asm volatile(
            "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                smem_addr(tiles + size_t(j) * B * R)),
            "l"(a.Uo[j] + base[j] * R), "r"(bytes[j]), "r"(mb)
            : "memory");
    }
  }
  const uint32_t base_row = __ldg(a.brow + s) << a.bbits;
  const int lane = threadIdx.x & 31, g = lane / LPN, lig = lane % LPN;
  const int gid = int(threadIdx.x >> 5) * G + g;
  const uint64_t ngroups = uint64_t(kWarpsPerCta) * G;
  const uint64_t run = (hi - lo + ngroups - 1) / ngroups;
  const uint64_t x0 = lo + uint64_t(gid) * run;
  const uint64_t x1 = (x0 + run < hi) ? x0 + run : hi;
  const Policies pol(a.cache_mode);
  mbar_wait(mb, 0);  // every thread waits: the tiles have landed
  if (x0 >= x1) return;

  for (uint32_t col = uint32_t(lig) * 4; col < R; col += LPN * 4) {
    Vec<4> acc;
#pragma unroll
    for (int i = 0; i < 4; ++i) acc.v[i] = 0.f;
    uint32_t cur = 0xFFFFFFFFu;
    for (uint64_t x = x0; x < x1; x += U) {
      const int cnt = (x1 - x) >= uint64_t(U) ? U : int(x1 - x);
      uint32_t er[U], ej[NOA][U];
      float v[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (u < cnt) {
          er[u] = __ldg(a.erow + x + u);
          v[u] = __ldg(a.val + x + u);
#pragma unroll
          for (int j = 0; j < NOA; ++j)
            if (j < no) ej[j][u] = __ldg(a.eo[j] + x + u);
        }
      }
#pragma unroll
      for (int u = 0; u < U; ++u) {
        if (u < cnt) {
          Vec<4> t;
#pragma unroll
          for (int i = 0; i < 4; ++i) t.v[i] = v[u];
#pragma unroll
          for (int j = 0; j < NOA; ++j) {
            if (j < no) {
              const float4 f =
                  *reinterpret_cast<const float4 *>(tiles + (size_t(j) * B + ej[j][u]) * R + col);
              t.v[0] *= f.x; t.v[1] *= f.y; t.v[2] *= f.z; t.v[3] *= f.w;
            }
          }
          if (er[u] == cur) {
#pragma unroll
            for (int i = 0; i < 4; ++i) acc.v[i] += t.v[i];
          } else {
            if (cur != 0xFFFFFFFFu) red_vec<4>(a.out + uint64_t(base_row + cur) * R + col, acc, pol.out);
            cur = er[u];
            acc = t;
          }
        }
      }
    }
    if (cur != 0xFFFFFFFFu) red_vec<4>(a.out + uint64_t(base_row + cur) * R + col, acc, pol.out);
  }
}

// ---------------------------------------------------------------------------------------
// COO MTTKRP with a shared-memory-staged nonzero stream (a6, default vector path).
// Same work decomposition as mttkrp_kernel (warp chunk = G groups x `run` contiguous
// nonzeros, 4-lane groups own 16-B column slices of every factor row), but the index/value
// stream is copied global->shared by the whole warp with cp.async (LDGSTS, L1-bypassing
// .cg, L2 evict_first policy: every 128-B line is consumed by one copy, so the stream never
// needs to linger in L2 and does not displace power-law-hot factor rows), double-buffered
// one stage (32 nonzeros per group) ahead of the gathers.
// WA: 0/1/2 buffer-address forms (see the launcher); 3, 4, 5 are measurement probes that
// decompose the kernel time (3: no output writes, 4: no factor gathers, 5: stream only).
// HS (persistent, 16 warps, one CTA per SM): the shared-memory tier of the hot-row cache --
// the most frequent factor rows are copied into shared memory once per CTA, and gathers of
// entries tagged 0xC0000000 | slot read them there instead of from L2.
template <int NO, int LPN, int WA, bool HS, int WPC_ = 16, int SG_ = 32, int U_ = 4>
__global__ void __launch_bounds__(HS ? WPC_ * 32 : kThreads, HS ? 1 : (WA == 6 ? 3 : 2))
    coo_staged_kernel(const KArgs a) {
  constexpr int WPC = HS ? WPC_ : kWarpsPerCta;
  // 7: HS kernel without the L2 tier (no hot_buf rows) whose gathered factors are < 4 GB each:
  // no base-pointer select, 32-bit byte offsets.  9: HiCOO row slices decoded warp-wide into
  // the stage buffer (no hot tiers, 64-bit offsets).  10: the same decode with the hot-block
  // tiers (R#34): decoded coordinates carry the tier tags of their retagged slice bases
  // 11: HiCOO row slices whose raw arrays (values, 8-bit element indices, slice ends, rows,
  // block bases) are copied into shared memory with cp.async one stage ahead and decoded from
  // there -- the decode of WA 9 waits on dependent global loads every stage
  constexpr bool kHicRaw = WA == 11;
  // 16: WA 9's decode with a ROW-granular shared-memory tier: the decoded coordinate of a hot
  // row (bitmap + per-word prefix count, in shared memory) is retagged 0xC0000000 | smem slot,
  // and the gathers use the WA 7 path (shared memory or a plain row, 32-bit byte offsets)
  constexpr bool kHicRows = WA == 16;
  // 17: WA 9's decode with tagged slice bases of the shared-memory tier only (R#36 tier blocks
  // without an L2 tier): the gathers take the WA 7 path (shared memory or a plain row, 32-bit
  // byte offsets)
  constexpr bool kHic = WA == 9 || WA == 10 || kHicRaw || kHicRows || WA == 17;
  constexpr bool kL2T = WA != 7 && WA != 9 && WA != 11 && WA != 16 && WA != 17;
  constexpr bool kGather = WA != 4 && WA != 5;
  constexpr bool kWrite = WA != 3 && WA != 5;
  constexpr int kBuf = (WA == 0 || WA == 2) ? WA : 1;  // 6: form 1 with 3 CTAs per SM
  constexpr int G = 32 / LPN;
  constexpr int SG = SG_;         // nonzeros per group per stage (32 or 16)
  constexpr int CG = SG / 4;      // 16-B chunks per group and array
  constexpr int GL = 8 / CG;      // groups per 128-B line
  constexpr int SW = G * SG;      // nonzeros per warp per stage
  constexpr int NA = NO + 2;      // arrays: i_n, i_k (k != n), val
  constexpr int U = U_;           // nonzeros per group per step (4 or 8; divides SG)
  extern __shared__ __align__(16) uint32_t stage_buf[];  // [warp][2][NA][SW]
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int g = lane / LPN, lig = lane % LPN;
  uint32_t *wbuf = stage_buf + size_t(warp) * 2 * NA * SW;
  constexpr uint32_t R = 4 * LPN;  // the launcher picks LPN = R / 4 (R = 16 or 32)
  float *hs_tile = reinterpret_cast<float *>(stage_buf + size_t(WPC) * 2 * NA * SW);
  const uint32_t hs_saddr = smem_addr(hs_tile);
  if constexpr (HS) {  // fill the shared-memory tier: hs_tile[slot][:] = U_j[hs_rows[slot]][:]
    const uint32_t r4 = R / 4, n4 = a.hs_lo[NO] * r4;
    for (uint32_t e = threadIdx.x; e < n4; e += blockDim.x) {
      const uint32_t slot = e / r4, c = e % r4;
      int j = 0;
#pragma unroll
      for (int jj = 1; jj < NO; ++jj) j += slot >= a.hs_lo[jj];
      const float4 *Uj = reinterpret_cast<const float4 *>(a.Uo[j]);
      reinterpret_cast<float4 *>(hs_tile)[e] = __ldg(Uj + uint64_t(__ldg(a.hs_rows + slot)) * r4 + c);
    }
    if constexpr (kHicRows) {  // the tier's row bitmaps and per-word prefixes, after the rows
      uint32_t *rs = reinterpret_cast<uint32_t *>(hs_tile + size_t(a.hs_lo[NO]) * R);
#pragma unroll
      for (int j = 0; j < NO; ++j) {
        for (uint32_t w = threadIdx.x; w < a.rs_words[j]; w += blockDim.x) {
          rs[w] = __ldg(a.rs_bm[j] + w);
          rs[a.rs_words[j] + w] = __ldg(a.rs_pre[j] + w);
        }
        rs += 2 * a.rs_words[j];
      }
    }
    __syncthreads();
  }
  // the nonzero range this CTA works on: all of them, or its die's half (die split)
  // die split (dyn): die 0's range is [0, split_x), die 1's [split_x, nnz); a CTA claims the
  // chunks of its own die's range first, then (work stealing) the other die's, so every chunk is
  // processed whatever the CTA placement (a CTA may not exist on some die at all)
  const bool dyn = HS && !kHic && a.split;
  int die = 0;
  if (dyn) {
    uint32_t sm;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(sm));
    die = a.die_of[sm];
  }
  auto range_end = [&](uint64_t c) { return (dyn && c < a.split_x) ? a.split_x : a.nnz; };
  const uint64_t nchunks = (a.nnz + a.chunk - 1) / a.chunk;  // static schedule
  const uint64_t wstep = HS ? uint64_t(gridDim.x) * WPC : nchunks;
  const uint64_t run = a.chunk / G;  // multiple of SG
  const int nstages = int(run / SG);
  const uint32_t col = uint32_t(lig) * 4;
  const Policies pol(a.cache_mode | 1u);  // the staged stream is always evict_first
  // one L2 policy for every gather: a per-lane choice forces a predicated R2UR of the policy
  // descriptor per load, and separate predicated loads per policy (hot rows evict_last, cold
  // ones evict_first) measured 2x slower on H (profiles/r01_hs_sweep.txt)
  const uint32_t *src[NA];
  src[0] = a.irow;
#pragma unroll
  for (int j = 0; j < NO; ++j) src[1 + j] = a.io[j];
  src[NA - 1] = reinterpret_cast<const uint32_t *>(a.val);

  // issue the cp.async copies of stage s of the chunk starting at cc into dst (one commit
  // group; an empty group when cc is past the end, so that wait_group counts stay uniform)
  auto issue_to = [&](uint64_t cc, int s, uint32_t *dst) {
    const uint64_t xend = range_end(cc);
    if (cc < xend) {
      for (int i = lane; i < SW / 4; i += 32) {  // 16-B chunks of one array
        const int gi = i / (SG / 4), k = i % (SG / 4);
        const uint64_t pos = cc + uint64_t(gi) * run + uint64_t(s) * SG + uint64_t(k) * 4;
        const int valid = pos >= xend ? 0 : (xend - pos >= 4 ? 16 : int(xend - pos) * 4);
#pragma unroll
        for (int arr = 0; arr < NA; ++arr) {
          // 16-B chunk k of group gi lands at chunk k ^ ((gi / GL) % CG) of the group's region:
          // the groups of a warp then read different bank quads at every step
          const uint32_t d = smem_addr(dst + arr * SW + gi * SG + ((k ^ (gi / GL)) & (CG - 1)) * 4);
          const uint32_t *sp = src[arr] + (valid ? pos : 0);
          if (kBuf == 2) {
            asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(d), "l"(sp), "r"(valid)
                         : "memory");
          } else {
            asm volatile("cp.async.cg.shared.global.L2::cache_hint [%0], [%1], 16, %2, %3;" ::"r"(d),
                         "l"(sp), "r"(valid), "l"(pol.stream)
                         : "memory");
          }
        }
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  // HiCOO decode (WA 9, SG == 32): for each group window of 32 entries, lane l takes entry
  // p + l and slice slot sb + l (the window's entries lie in at most 32 consecutive slices);
  // an entry's slot = #{slots whose end <= entry} by a 5-step shuffle search over the sorted
  // slot ends; row and block bases come from the owning lane by shuffle; i_k = base + e_k
  // (Alg. 3's rebased pointers).  gsb[g] = current slice of group g (warp-uniform).
  uint32_t gsb[G];  // slice indices < nnz < 2^32 (API)
  uint32_t rs_j[NO > 0 ? NO : 1];  // WA 16: shared addresses of each mode's bitmap (prefixes follow)
  if constexpr (kHicRows) {
    uint32_t rs = hs_saddr + a.hs_lo[NO] * R * 4u;
#pragma unroll
    for (int j = 0; j < NO; ++j) {
      rs_j[j] = rs;
      rs += 8u * a.rs_words[j];
    }
  }
  auto lds32 = [](uint32_t addr) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(addr));
    return v;
  };
  // The loads of GB groups' windows are issued together (branch-free, so the compiler can
  // hoist them past the previous group's shuffles) before any is consumed: one memory latency
  // per batch of groups instead of one per group.
  auto decode_to = [&](uint64_t cc, int s, uint32_t *dst) {
    if (cc >= a.nnz) return;
    const uint64_t r0 = cc / run;
    if (s == 0) {
      const uint64_t nruns = (a.nnz + run - 1) / run;
#pragma unroll
      for (int gi = 0; gi < G; ++gi) gsb[gi] = uint32_t(__ldg(a.run_sb + (r0 + gi < nruns ? r0 + gi : nruns - 1)));
    }
#ifdef PASTA_DECODE_GB
    constexpr int GB = G < PASTA_DECODE_GB ? G : PASTA_DECODE_GB;
#else
    constexpr int GB = G < 4 ? G : ((NO >= 3 || kHicRows) ? 2 : 4);
#endif
    constexpr int NOA = NO > 0 ? NO : 1;
#pragma unroll
    for (int gb = 0; gb < G; gb += GB) {
      uint32_t eabs[GB];
      uint32_t srow[GB], sbase[GB][NOA], e[GB][NOA];
      float v[GB];
#pragma unroll
      for (int q = 0; q < GB; ++q) {  // loads only
        const uint64_t p = cc + uint64_t(gb + q) * run + uint64_t(s) * SG;
        const uint64_t sb0 = gsb[gb + q];
        const uint64_t st = sb0 + lane < a.nsb ? sb0 + lane : a.nsb - 1;
        // the slice and entry arrays are read once per launch: cache-streaming loads (ld.cs,
        // evict-first in L2), like the COO stream, so they do not push the tiers and hot factor
        // rows out of L2.  (The same loads with an L2::cache_hint policy operand faulted for
        // order-2 instantiations at R >= 32 under ptxas 12.9.)
        eabs[q] = __ldcs(a.sbend32 + st);  // = sbptr[st + 1]
        srow[q] = __ldcs(a.sbrow + st);
#pragma unroll
        for (int j = 0; j < NO; ++j) sbase[q][j] = ((a.wide >> j) & 1u) ? 0u : __ldcs(a.sbbase[j] + st);
        const uint64_t x = p + lane;
        const bool ok = x < a.nnz;
        v[q] = ok ? __ldcs(a.val + x) : 0.f;
#pragma unroll
        for (int j = 0; j < NO; ++j)
          e[q][j] = !ok ? 0u : ((a.wide >> j) & 1u) ? __ldcs(a.io[j] + x) : uint32_t(__ldcs(a.eo[j] + x));
      }
#pragma unroll
      for (int q = 0; q < GB; ++q) {
        const int gi = gb + q;
        const uint64_t p = cc + uint64_t(gi) * run + uint64_t(s) * SG;
        if (p >= a.nnz) continue;  // warp-uniform
        const uint64_t sb0 = gsb[gi];
        const uint32_t erel = eabs[q] - uint32_t(p) > 64u ? 64u : eabs[q] - uint32_t(p);
        int c = 0;  // <= 31: slot 0 holds entry p, so 32 entries span at most 32 slots
#pragma unroll
        for (int k = 16; k >= 1; k >>= 1) {
          const uint32_t et = __shfl_sync(0xFFFFFFFFu, erel, c + k - 1);
          if (et <= uint32_t(lane)) c += k;
        }
        const uint32_t row = __shfl_sync(0xFFFFFFFFu, srow[q], c);
        const int d = gi * SG + (((lane / 4) ^ (gi / GL)) & (CG - 1)) * 4 + (lane & 3);
        dst[d] = row;
#pragma unroll
        for (int j = 0; j < NO; ++j) {
          uint32_t id = __shfl_sync(0xFFFFFFFFu, sbase[q][j], c) + e[q][j];
          if constexpr (kHicRows) {  // hot row -> its shared-memory slot
            const uint32_t w = id >> 5;
            const uint32_t bits = lds32(rs_j[j] + 4u * w);
            if ((bits >> (id & 31)) & 1u)
              id = 0xC0000000u | (a.hs_lo[j] + lds32(rs_j[j] + 4u * (a.rs_words[j] + w)) +
                                  __popc(bits & ((1u << (id & 31)) - 1u)));
          }
          dst[(1 + j) * SW + d] = id;
        }
        dst[(NA - 1) * SW + d] = __float_as_uint(v[q]);
        // the next window starts at the slice holding entry p + SG: the last entry's slice, or
        // the one after it when that slice ends inside this window
        const uint64_t nleft = a.nnz - p;
        const int last = nleft >= uint64_t(SG) ? SG - 1 : int(nleft) - 1;
        const int clast = __shfl_sync(0xFFFFFFFFu, c, last);
        const uint32_t elast = __shfl_sync(0xFFFFFFFFu, erel, clast);
        gsb[gi] = uint32_t(sb0) + uint32_t(clast) + (elast <= uint32_t(SG) ? 1u : 0u);
      }
    }
  };
  // ---- WA 11: raw windows.  Per group window (32 entries from p, slices from sb0), at word
  // offsets: [0] sb0 & 3 | [4, 36) values | per other mode j: 8 words of 8-bit einds, or 32 of
  // u32 coordinates (gHiCOO wide) | 36 slice ends (u32, slots (sb0 & ~3) + t) | 36 slice rows |
  // per compressed mode j: 36 block bases.  The slice arrays are padded (ends with nnz) so the
  // aligned 36-slot copies never leave them.
  uint32_t *raw = reinterpret_cast<uint32_t *>(hs_tile + size_t(a.hs_lo[NO]) * R) + size_t(warp) * G * a.raw_words;
  int off_e[NO > 0 ? NO : 1], off_b[NO > 0 ? NO : 1], off_end = 36, off_row = 72;
  if constexpr (kHicRaw) {
    int o = 36;
#pragma unroll
    for (int j = 0; j < NO; ++j) { off_e[j] = o; o += ((a.wide >> j) & 1u) ? 32 : 8; }
    off_end = o;
    off_row = o + 36;
    o += 72;
#pragma unroll
    for (int j = 0; j < NO; ++j) { off_b[j] = o; o += ((a.wide >> j) & 1u) ? 0 : 36; }
  }
  const uint64_t nst_total = (uint64_t(a.chunk) / G) / SG;  // stages per chunk
  // the position after (cc, s) in this warp's static schedule (cc = a.nnz: none)
  auto next_pos = [&](uint64_t &cc, int &s) {
    if (cc >= a.nnz) return;
    if (uint64_t(s) + 1 < nst_total) { ++s; return; }
    s = 0;
    cc += wstep * a.chunk;
    if (cc >= a.nnz) cc = a.nnz;
  };
  auto win_of = [&](uint64_t cc, int s) -> uint32_t {  // lane gi < G: win_sb of its group
    const uint64_t p = cc + uint64_t(lane) * (a.chunk / G) + uint64_t(s) * SG;
    return (lane < G && p < a.nnz) ? __ldg(a.win_sb + p / 32) : 0u;
  };
  auto raw_issue = [&](uint64_t cc, int s, uint32_t wsb) {
    if (cc < a.nnz) {
#pragma unroll 1
      for (int gi = 0; gi < G; ++gi) {
        const uint64_t p = cc + uint64_t(gi) * (a.chunk / G) + uint64_t(s) * SG;
        if (p >= a.nnz) break;  // warp-uniform; later groups start later
        const uint32_t sb0 = __shfl_sync(0xFFFFFFFFu, wsb, gi);
        uint32_t *rw = raw + gi * a.raw_words;
        if (lane == 0) rw[0] = sb0 & 3u;
        const uint32_t sa = sb0 & ~3u;
        auto cp16 = [&](uint32_t *dst, const void *src, int valid) {
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_addr(dst)), "l"(src),
                       "r"(valid) : "memory");
        };
        const uint64_t left = a.nnz - p;  // entries of this window that exist (>= 1)
        if (lane < 8) {  // values
          const uint64_t q = uint64_t(lane) * 4;
          cp16(rw + 4 + lane * 4, a.val + (q < left ? p + q : 0), q < left ? int(left - q >= 4 ? 16 : (left - q) * 4) : 0);
        }
#pragma unroll
        for (int j = 0; j < NO; ++j) {
          if ((a.wide >> j) & 1u) {
            if (lane < 8) {
              const uint64_t q = uint64_t(lane) * 4;
              cp16(rw + off_e[j] + lane * 4, a.io[j] + (q < left ? p + q : 0),
                   q < left ? int(left - q >= 4 ? 16 : (left - q) * 4) : 0);
            }
          } else if (lane < 2) {
            const uint64_t q = uint64_t(lane) * 16;
            cp16(rw + off_e[j] + lane * 4, a.eo[j] + (q < left ? p + q : 0),
                 q < left ? int(left - q >= 16 ? 16 : left - q) : 0);
          }
        }
        if (lane < 9) {  // 36 slots of ends, rows and bases from the aligned slot sa
          cp16(rw + off_end + lane * 4, a.sbend32 + sa + lane * 4, 16);
          cp16(rw + off_row + lane * 4, a.sbrow + sa + lane * 4, 16);
#pragma unroll
          for (int j = 0; j < NO; ++j)
            if (!((a.wide >> j) & 1u)) cp16(rw + off_b[j] + lane * 4, a.sbbase[j] + sa + lane * 4, 16);
        }
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };
  // decode a landed raw stage into a stage buffer (same output as decode_to)
  auto raw_decode = [&](uint64_t cc, int s, uint32_t *dst) {
    if (cc >= a.nnz) return;
#pragma unroll 1
    for (int gi = 0; gi < G; ++gi) {
      const uint64_t p = cc + uint64_t(gi) * (a.chunk / G) + uint64_t(s) * SG;
      if (p >= a.nnz) break;
      const uint32_t *rw = raw + gi * a.raw_words;
      const uint32_t bi = rw[0] + uint32_t(lane);
      const uint32_t p32 = uint32_t(p);
      const uint32_t eabs = rw[off_end + bi];
      const uint32_t erel = eabs - p32 > 64u ? 64u : eabs - p32;
      const uint32_t srow = rw[off_row + bi];
      const bool ok = p + lane < a.nnz;
      const float v = ok ? __uint_as_float(rw[4 + lane]) : 0.f;
      uint32_t sbase[NO > 0 ? NO : 1], e[NO > 0 ? NO : 1];
#pragma unroll
      for (int j = 0; j < NO; ++j) {
        const bool wj = (a.wide >> j) & 1u;
        sbase[j] = wj ? 0u : rw[off_b[j] + bi];
        e[j] = !ok ? 0u : wj ? rw[off_e[j] + lane] : ((rw[off_e[j] + (lane >> 2)] >> (8 * (lane & 3))) & 0xFFu);
      }
      int c = 0;
#pragma unroll
      for (int k = 16; k >= 1; k >>= 1) {
        const uint32_t et = __shfl_sync(0xFFFFFFFFu, erel, c + k - 1);
        if (et <= uint32_t(lane)) c += k;
      }
      const uint32_t row = __shfl_sync(0xFFFFFFFFu, srow, c);
      const int d = gi * SG + (((lane / 4) ^ (gi / GL)) & (CG - 1)) * 4 + (lane & 3);
      dst[d] = row;
#pragma unroll
      for (int j = 0; j < NO; ++j) dst[(1 + j) * SW + d] = __shfl_sync(0xFFFFFFFFu, sbase[j], c) + e[j];
      dst[(NA - 1) * SW + d] = __float_as_uint(v);
    }
  };
  uint32_t wsb_next = 0;
  bool raw_primed = false;
  auto issue = [&](uint64_t cc, int s, int b) {
    if constexpr (kHicRaw) {
      uint64_t c2 = cc;
      int s2 = s;
      next_pos(c2, s2);
      if (!raw_primed) {  // first position of this warp: raw-issue it synchronously
        raw_issue(cc, s, win_of(cc, s));
        wsb_next = win_of(c2, s2);
        raw_primed = true;
      }
      asm volatile("cp.async.wait_group 0;" ::: "memory");
      __syncwarp();
      raw_decode(cc, s, wbuf + b * NA * SW);
      __syncwarp();  // every lane has read the raw buffer before it is refilled
      raw_issue(c2, s2, wsb_next);
      uint64_t c3 = c2;
      int s3 = s2;
      next_pos(c3, s3);
      wsb_next = win_of(c3, s3);
      return;
    }
    if constexpr (kHic) {
      decode_to(cc, s, wbuf + b * NA * SW);
      return;
    }
    if (kBuf == 1) {
      if (b) issue_to(cc, s, wbuf + NA * SW); else issue_to(cc, s, wbuf);
    } else {
      issue_to(cc, s, wbuf + b * NA * SW);
    }
  };

  // The stream is pipelined across the warp's chunks: the last stage of a chunk prefetches
  // stage 0 of the next one, so a persistent warp never waits on a cold pipeline.
  // Chunk schedule: static round robin, or (die split) chunks of the die's range claimed with
  // one atomic per chunk -- the CTA -> SM placement is not known in advance, so a static
  // split by die rank could skip or repeat chunks.  The claim of the chunk after next is
  // issued at the start of a chunk and consumed at its end (its latency hides behind it).
  auto claim_issue = [&](int d) -> unsigned long long {
    unsigned long long v = 0;
    if (lane == 0) v = atomicAdd(a.claim + d, 1ull);
    return v;
  };
  auto claim_get = [&](unsigned long long v) { return uint64_t(__shfl_sync(0xFFFFFFFFu, v, 0)); };
  const uint64_t kDone = a.nnz;
  int dcl = die;            // die range currently claimed from
  bool stolen = false;      // switched to the other die's range
  // chunk index v of range d -> first entry, or (range exhausted) steal once from the other
  auto resolve = [&](uint64_t v, int d) -> uint64_t {
    for (;;) {
      const uint64_t base = d ? a.split_x : 0, end = d ? a.nnz : a.split_x;
      if (v < (end - base + a.chunk - 1) / a.chunk) return base + v * a.chunk;
      if (stolen) return kDone;
      stolen = true;
      dcl = d = 1 - d;
      v = claim_get(claim_issue(d));
    }
  };
  int bsel = 0;
  uint64_t c0, cn;  // first entry of the current / next chunk (kDone: none)
  if (dyn) {
    c0 = resolve(claim_get(claim_issue(dcl)), dcl);
    cn = c0 < kDone ? resolve(claim_get(claim_issue(dcl)), dcl) : kDone;
  } else {
    const uint64_t w0 = uint64_t(blockIdx.x) * WPC + warp;
    c0 = w0 < nchunks ? w0 * a.chunk : kDone;
    cn = w0 + wstep < nchunks ? (w0 + wstep) * a.chunk : kDone;
  }
  if (c0 < kDone) issue(c0, 0, 0);
  while (c0 < kDone) {
  const int dpend = dcl;  // claim of the chunk after next, in flight during this chunk
  const unsigned long long pend = (dyn && cn < kDone) ? claim_issue(dpend) : 0ull;
  const uint64_t x0 = c0 + uint64_t(g) * run;
  const uint64_t xend = range_end(c0);
  const uint64_t x1 = (x0 + run < xend) ? x0 + run : xend;
  Vec<4> acc;
#pragma unroll
  for (int i = 0; i < 4; ++i) acc.v[i] = 0.f;
  uint32_t cur = 0xFFFFFFFFu;
  bool first = true;
  const bool active = x0 < x1 && col < R;
  for (int s = 0; s < nstages; ++s) {
    if (s + 1 < nstages) issue(c0, s + 1, bsel ^ 1);
    else issue(cn, 0, bsel ^ 1);
    asm volatile("cp.async.wait_group 1;" ::: "memory");
    __syncwarp();
    const uint32_t *buf = wbuf + bsel * NA * SW + g * SG;
    const uint64_t sx = x0 + uint64_t(s) * SG;  // first nonzero of this stage for the group
    if (active && sx < x1) {
      const int scnt = (x1 - sx) >= uint64_t(SG) ? SG : int(x1 - sx);
#pragma unroll 1
      for (int q = 0; q < scnt; q += U) {
        const int cnt = (scnt - q) >= U ? U : scnt - q;
        uint32_t row[U];
        float v[U];
        uint32_t idx[NO][U];
#pragma unroll
        for (int p = 0; p < U / 4; ++p) {
          const int qs = ((((q / 4) + p) ^ (g / GL)) & (CG - 1)) * 4;  // swizzled chunk (see issue_to)
          const uint4 r4 = *reinterpret_cast<const uint4 *>(buf + qs);
          const uint4 v4 = *reinterpret_cast<const uint4 *>(buf + (NA - 1) * SW + qs);
          row[4 * p] = r4.x; row[4 * p + 1] = r4.y; row[4 * p + 2] = r4.z; row[4 * p + 3] = r4.w;
          v[4 * p] = __uint_as_float(v4.x); v[4 * p + 1] = __uint_as_float(v4.y);
          v[4 * p + 2] = __uint_as_float(v4.z); v[4 * p + 3] = __uint_as_float(v4.w);
#pragma unroll
          for (int j = 0; j < NO; ++j) {
            const uint4 i4 = *reinterpret_cast<const uint4 *>(buf + (1 + j) * SW + qs);
            idx[j][4 * p] = i4.x; idx[j][4 * p + 1] = i4.y; idx[j][4 * p + 2] = i4.z; idx[j][4 * p + 3] = i4.w;
          }
        }
        Vec<4> f[NO][U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
#pragma unroll
          for (int j = 0; j < NO; ++j) {
            if (kGather) {
              const uint32_t id = idx[j][u];
              if constexpr (WA == 9 || WA == 11) {  // decoded HiCOO coordinate: plain factor row
                if (u < cnt) f[j][u] = ldg_vec<4>(a.Uo[j] + uint64_t(id) * R + col, pol.gather);
              } else if constexpr (HS) {  // shared-memory tier, L2-tier buffer or plain factor row
                const bool in_s = (id >> 30) == 3u;
                if constexpr (kL2T) {
                  const bool in_h = (id >> 30) == 2u;
                  const uint64_t off = uint64_t(id & 0x3FFFFFFFu) * R + col;
                  const float *gptr = (in_h ? a.hot_buf : a.Uo[j]) + off;
                  if constexpr (WA == 12)  // cold rows with their own L2 policy (Policies::cold)
                    f[j][u] = ld_tiered3(hs_saddr + uint32_t(off) * 4u, gptr, pol.gather, pol.cold, u < cnt && in_s,
                                         u < cnt && in_h, u < cnt && !in_s && !in_h);
                  else
                    f[j][u] = ld_tiered<WA == 13>(hs_saddr + uint32_t(off) * 4u, gptr, pol.gather, u < cnt && in_s,
                                                  u < cnt && !in_s);
                } else {
                  const uint32_t boff = ((id & 0x3FFFFFFFu) * R + col) * 4u;  // < 4 GB
                  const float *gptr = reinterpret_cast<const float *>(
                      reinterpret_cast<const char *>(a.Uo[j]) + boff);
                  f[j][u] = ld_tiered(hs_saddr + boff, gptr, pol.gather, u < cnt && in_s, u < cnt && !in_s);
                }
              } else {
                const float *base = a.Uo[j];
                uint32_t row = id;
                if (a.hot_marked && (id >> 31)) {  // a row of the packed L2-tier buffer
                  base = a.hot_buf;
                  row = id & 0x3FFFFFFFu;
                }
                if (u < cnt) f[j][u] = ldg_vec<4>(base + uint64_t(row) * R + col, pol.gather);
              }
            } else {
#pragma unroll
              for (int i = 0; i < 4; ++i) f[j][u].v[i] = __uint_as_float(idx[j][u] | 0x3f800000u);
            }
          }
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          if (u < cnt) {
            Vec<4> t;
#pragma unroll
            for (int i = 0; i < 4; ++i) t.v[i] = v[u];
#pragma unroll
            for (int j = 0; j < NO; ++j) {
#pragma unroll
              for (int i = 0; i < 4; ++i) t.v[i] *= f[j][u].v[i];
            }
            if (row[u] == cur) {
#pragma unroll
              for (int i = 0; i < 4; ++i) acc.v[i] += t.v[i];
            } else {
              if (cur != 0xFFFFFFFFu) {
                float *dst = a.out + uint64_t(cur) * R + col;
                if constexpr (WA == 15) {  // the same flush into every replica
                  for (uint32_t d = 0; d < a.nout; ++d) {
                    float *dd = a.outs[d] + uint64_t(cur) * R + col;
                    if (first || dyn) red_vec<4>(dd, acc, pol.out); else st_vec<4>(dd, acc, pol.out);
                  }
                } else if (kWrite) {
                  if (first || dyn) red_vec<4>(dst, acc, pol.out); else st_vec<4>(dst, acc, pol.out);
                } else if (acc.v[0] == 1.2345e-30f) {
                  st_vec<4>(dst, acc, pol.out);  // keeps the arithmetic live in probes
                }
                first = false;
              }
              cur = row[u];
              acc = t;
            }
          }
        }
      }
    }
    __syncwarp();  // the buffer of this stage is refilled at the start of the next one
    bsel ^= 1;
  }
  if (active && cur != 0xFFFFFFFFu && (kWrite || acc.v[0] == 1.2345e-30f)) {
    if constexpr (WA == 15) {
      for (uint32_t d = 0; d < a.nout; ++d) red_vec<4>(a.outs[d] + uint64_t(cur) * R + col, acc, pol.out);
    } else {
      red_vec<4>(a.out + uint64_t(cur) * R + col, acc, pol.out);
    }
  }
  const uint64_t cprev = c0;
  c0 = cn;
  if (dyn) cn = c0 < kDone ? resolve(claim_get(pend), dpend) : kDone;
  else cn = (c0 < kDone && cprev / a.chunk + 2 * wstep < nchunks) ? (cprev / a.chunk + 2 * wstep) * a.chunk : kDone;
  }  // chunk loop
  if constexpr (WA == 15) __threadfence_system();  // the peer stores, before the kernel ends
}

template <int VW>
__global__ void zero_rows_kernel(float *__restrict__ out, uint64_t n) {
  for (uint64_t e = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; e < n;
       e += uint64_t(gridDim.x) * blockDim.x) {
    if constexpr (VW == 4) reinterpret_cast<float4 *>(out)[e] = make_float4(0.f, 0.f, 0.f, 0.f);
    else out[e] = 0.f;
  }
}

int sm_count() {
  static int n = 0;
  if (!n) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
    if (n <= 0) n = 148;
  }
  return n;
}

template <class Src, int NO, int LPN, int VW, class T>
void launch_t(const KArgs &a, cudaStream_t s) {
  uint64_t nwarps = (a.nnz - a.x_begin + a.chunk - 1) / a.chunk;
  uint64_t nblk = (nwarps + kWarpsPerCta - 1) / kWarpsPerCta;
  if (nblk == 0) return;
  if (nblk > 0x7FFFFFFFull) fail(PASTA_ERANGE, "mttkrp: grid too large");
  mttkrp_kernel<Src, NO, LPN, VW, T><<<unsigned(nblk), kThreads, 0, s>>>(a);
  PASTA_LAUNCHED();
}

template <class Src>
using TuneDefault = Tune<4, false, Src::kMinBlocks>;

// Variants selectable with PASTA_MTTKRP_VARIANT for tuning sweeps (vector path, N = 3, 4,
// R = 16 / 32).
template <template <int, int> class SrcT, int NO, int LPN>
void launch_variant(const KArgs &a, int variant, cudaStream_t s) {
  switch (variant) {
    case 1: launch_t<SrcT<NO, 4>, NO, LPN, 4, Tune<4, true, 1>>(a, s); break;
    case 2: launch_t<SrcT<NO, 8>, NO, LPN, 4, Tune<8, false, 1>>(a, s); break;
    case 3: launch_t<SrcT<NO, 4>, NO, LPN, 4, Tune<4, true, 3>>(a, s); break;
    case 4: launch_t<SrcT<NO, 8>, NO, LPN, 4, Tune<8, true, 2>>(a, s); break;
    case 5: launch_t<SrcT<NO, 4>, NO, LPN, 4, Tune<4, false, 4>>(a, s); break;
    case 6: launch_t<SrcT<NO, 4>, NO, LPN, 4, Tune<4, false, 3>>(a, s); break;
    case 7: launch_t<SrcT<NO, 8>, NO, LPN, 4, Tune<8, false, 2>>(a, s); break;
    default: launch_t<SrcT<NO, 4>, NO, LPN, 4, TuneDefault<SrcT<NO, 4>>>(a, s); break;
  }
}

template <template <int, int> class SrcT, int NO, int VW>
void launch_lpn(const KArgs &a, int lpn, int variant, cudaStream_t s) {
  if constexpr (VW == 4 && (NO == 2 || NO == 3)) {
    if (lpn == 4) return launch_variant<SrcT, NO, 4>(a, variant, s);
    if (lpn == 8) return launch_variant<SrcT, NO, 8>(a, variant, s);
  }
  switch (lpn) {
    case 1: launch_t<SrcT<NO, 4>, NO, 1, VW, TuneDefault<SrcT<NO, 4>>>(a, s); break;
    case 2: launch_t<SrcT<NO, 4>, NO, 2, VW, TuneDefault<SrcT<NO, 4>>>(a, s); break;
    case 4: launch_t<SrcT<NO, 4>, NO, 4, VW, TuneDefault<SrcT<NO, 4>>>(a, s); break;
    case 8: launch_t<SrcT<NO, 4>, NO, 8, VW, TuneDefault<SrcT<NO, 4>>>(a, s); break;
    case 16: launch_t<SrcT<NO, 4>, NO, 16, VW, TuneDefault<SrcT<NO, 4>>>(a, s); break;
    default: launch_t<SrcT<NO, 4>, NO, 32, VW, TuneDefault<SrcT<NO, 4>>>(a, s); break;
  }
}

int env_int(const char *name, int dflt) {
  const char *v = getenv(name);
  return (v && *v) ? atoi(v) : dflt;
}

template <template <int, int> class SrcT>
void dispatch(KArgs &a, bool vec4, cudaStream_t s) {
  // lanes per nonzero: smallest power of two covering R / VW columns, at most 32
  const uint32_t VWv = vec4 ? 4 : 1;
  uint32_t need = (a.R + VWv - 1) / VWv;
  int lpn = 1;
  while (lpn < 32 && uint32_t(lpn) < need) lpn <<= 1;
  const int G = 32 / lpn;
  // run length per group (multiple of 8), chunk = G * run
  uint64_t run = uint64_t(env_int("PASTA_MTTKRP_RUN", 128));
  run = run < 8 ? 8 : (run / 8) * 8;
  a.chunk = uint64_t(G) * run;
  const int variant = env_int("PASTA_MTTKRP_VARIANT", 0);
  a.cache_mode = uint32_t(env_int("PASTA_MTTKRP_CACHE", 0));
  const int no = int(a.order) - 1;
  if (vec4) {
    if (no == 2) launch_lpn<SrcT, 2, 4>(a, lpn, variant, s);
    else if (no == 3) launch_lpn<SrcT, 3, 4>(a, lpn, variant, s);
    else launch_lpn<SrcT, 0, 4>(a, lpn, variant, s);
  } else {
    if (no == 2) launch_lpn<SrcT, 2, 1>(a, lpn, variant, s);
    else if (no == 3) launch_lpn<SrcT, 3, 1>(a, lpn, variant, s);
    else launch_lpn<SrcT, 0, 1>(a, lpn, variant, s);
  }
}

bool aligned16(const void *p) { return (reinterpret_cast<uintptr_t>(p) & 15u) == 0; }

}  // namespace

void launch_zero_rows(float *out, uint64_t row_lo, uint64_t row_hi, uint32_t R, cudaStream_t s) {
  if (row_hi <= row_lo) return;
  ProfScope prof(kProfZero, s);
  float *p = out + row_lo * R;
  uint64_t n = (row_hi - row_lo) * uint64_t(R);
  uint64_t grid = uint64_t(sm_count()) * 8;
  if (aligned16(p) && n % 4 == 0) {
    zero_rows_kernel<4><<<unsigned(grid), 256, 0, s>>>(p, n / 4);
  } else {
    zero_rows_kernel<1><<<unsigned(grid), 256, 0, s>>>(p, n);
  }
  PASTA_LAUNCHED();
}

// Runtime (order - 1, lanes per nonzero) -> compile-time tags for the staged kernels
// (R = 4 * LPN in {8, 16, 32, 64}).
template <class F>
static void with_lpn(int lpn, F &&f) {
  switch (lpn) {
    case 2: f(std::integral_constant<int, 2>()); break;
    case 4: f(std::integral_constant<int, 4>()); break;
    case 8: f(std::integral_constant<int, 8>()); break;
    default: f(std::integral_constant<int, 16>()); break;
  }
}
template <int MAXNO, class F>
static void with_no_lpn(int no, int lpn, F &&f) {
  with_lpn(lpn, [&](auto L) {
    if (no == 1) f(std::integral_constant<int, 1>(), L);
    else if (no == 2 || MAXNO == 2) f(std::integral_constant<int, 2>(), L);
    else f(std::integral_constant<int, 3>(), L);
  });
}
static bool staged_rank(uint32_t R) { return R == 8 || R == 16 || R == 32 || R == 64; }

static bool vec4_ok(uint32_t order, uint32_t mode, const float *const *factors, uint32_t R,
                    const float *out) {
  if (R % 4 != 0 || !aligned16(out)) return false;
  for (uint32_t k = 0; k < order; ++k)
    if (k != mode && !aligned16(factors[k])) return false;
  return true;
}

void launch_coo_mttkrp(const pasta_coo *x, uint32_t mode, const float *const *factors, uint32_t R,
                       float *out, cudaStream_t s) {
  launch_coo_mttkrp_bcast(x, mode, factors, R, &out, 1, s);
}

// the rows this handle owns, copied from outs[0] into the peers' replicas outs[1..]
static void bcast_owned_rows(const pasta_coo *x, uint32_t mode, uint32_t R, float *const *outs, uint32_t nout,
                             cudaStream_t s) {
  uint64_t lo = 0, hi = x->dims[mode];
  if (x->shard_mode == int(mode)) { lo = x->row_lo; hi = x->row_hi; }
  if (hi <= lo) return;
  float *dsts[kMaxOrder];
  for (uint32_t d = 1; d < nout; ++d) dsts[d - 1] = outs[d] + lo * R;
  launch_bcast(outs[0] + lo * R, (hi - lo) * R, dsts, nout - 1, s);
}

// nout > 1: the fused MTTKRP + all-gather -- every flush is written into outs[0] (local) and
// into the peers' replicas outs[1..]; the staged persistent kernel (WA 15) when it applies,
// else the local kernel followed by a peer copy of the owned rows
void launch_coo_mttkrp_bcast(const pasta_coo *x, uint32_t mode, const float *const *factors, uint32_t R,
                             float *const *outs, uint32_t nout, cudaStream_t s) {
  float *out = outs[0];
  const CooModeCopy &mc = x->mc[mode];
  KArgs a{};
  a.nnz = x->nnz;
  a.order = x->order;
  a.R = R;
  a.irow = mc.inds[mode];
  a.val = mc.val;
  int j = 0;
  for (uint32_t k = 0; k < x->order; ++k) {
    if (k == mode) continue;
    a.io[j] = mc.inds[k];
    a.Uo[j] = factors[k];
    ++j;
  }
  a.out = out;
  if (a.nnz == 0) return;
  ProfScope prof(kProfCoo, s);
  const bool vec4 = vec4_ok(x->order, mode, factors, R, out);
  const int staged = env_int("PASTA_COO_STAGED", 1);
  const int no = int(x->order) - 1;
  // no == 1: order-2 matrices, e.g. the fiberised (fiber, i_n) matrix of TTM (ttm.cu)
  if (staged && vec4 && staged_rank(R) && (no >= 1 && no <= 3)) {
    // the hot-row cache pays only when the gathered factors do not fit in L2 already
    static int l2 = 0;
    if (!l2) {
      int dev = 0;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
      if (l2 <= 0) l2 = 126 << 20;
    }
    uint64_t gathered = 0;
    for (uint32_t k = 0; k < x->order; ++k)
      if (k != mode) gathered += uint64_t(x->dims[k]) * R * sizeof(float);
    // effective L2 for random row gathers is ~half the nominal size
    // (profiles/r01_l2_capacity_microbench.txt)
    const bool want_hot = env_int("PASTA_HOT_FORCE", 0) || gathered > uint64_t(l2) / 2;
    const int lpn = int(R / 4);  // 2, 4, 8 or 16 lanes per nonzero, 16 B of each factor row per lane
    const int G = 32 / lpn;
    // Persistent HS kernel (one 16-warp CTA per SM) with the shared-memory tier of the hot-row
    // cache.  Tier size: on L2-resident factors (no L2 tier) the kernel is bound by L2->SM
    // bandwidth and every smem row helps, so the tier takes what the staging buffers leave of
    // the 227 KB; on DRAM-bound gathers (L2 tier on) the L1 that the shared-memory carve-out
    // leaves holds the in-flight misses, so the tier stays at 512 rows (measured cliff between
    // 512 and 1024 rows on H and C3: 1.89 -> 2.17 ms, 1.84 -> 3.2 ms; profiles/r01_hs_sweep.txt).
    // PASTA_HOT_SMEM=0 selects the non-persistent kernel; PASTA_HOT_SMEM_ROWS caps the tier.
    // HS shape (warps per CTA, nonzeros per group per stage, nonzeros per group step):
    // PASTA_HS_CFG = 0 (16, 32, 4), 1 (24, 16, 4), 2 (16, 32, 8; orders 2 and 3).  More gathers
    // in flight is the lever: 24 warps fit 80 registers for order 3 (H 1.81 -> 1.64 ms, C2
    // 0.83 -> 0.77, C3 1.78 -> 1.58) but spill for order 4 (C4 0.74 -> 0.80); 8-deep steps
    // (126 registers, 16 warps) gain another 5-7 % where the gathers go to DRAM (H 1.69 ->
    // 1.57, C5 27.2 -> 26.6) but lose on L2-resident factors, whose shared-memory tier shrinks
    // (C2 0.80 -> 0.88).  32 warps spill for every order; 8 warps x 16-deep steps (220
    // registers) and 12 warps x 8-deep steps are slower everywhere (H 1.80 / 1.73 ms).
    // (R = 8 with DRAM-bound gathers: the 32-deep shape does not fit -> non-persistent kernel,
    // which measured faster there than forcing the 16-deep shape: H 1.80 vs 2.01 ms)
    // L2-resident factors: 20 warps x 16-deep (order <= 3) / 16 x 16-deep (order 4) -- the
    // shallower stage leaves the shared-memory tier 256-640 more rows (C2 0.728 -> 0.699, C4
    // 0.687 -> 0.676 ms per mode, profiles/r02_smem_fill_sweep.txt)
    const int hs_cfg = env_int("PASTA_HS_CFG", no <= 2 ? (want_hot ? 2 : 6) : (want_hot ? 0 : 5));
    const int hs_wpc = hs_cfg == 1 ? 24 : hs_cfg == 6 ? 20 : 16;
    const int hs_sg = (hs_cfg == 1 || hs_cfg == 5 || hs_cfg == 6) ? 16 : 32;  // 5: 16 x 16 x 4, 6: 20 x 16 x 4
    const size_t stage_hs = size_t(hs_wpc) * 2 * (no + 2) * (G * hs_sg) * sizeof(uint32_t);
    const size_t smem_cap = 227 * 1024;
    uint32_t hs_rows_budget =
        stage_hs < smem_cap ? uint32_t((smem_cap - stage_hs) / (size_t(R) * sizeof(float))) : 0u;
    if (want_hot) hs_rows_budget = std::min(hs_rows_budget, uint32_t(env_int("PASTA_HOT_SMEM_DRAM", 512)));
    if (const int cap = env_int("PASTA_HOT_SMEM_ROWS", 0)) hs_rows_budget = std::min(hs_rows_budget, uint32_t(cap));
    bool hs = env_int("PASTA_HOT_SMEM", 1) != 0 && hs_rows_budget >= 64;
    // die split (R#35): order 3 with DRAM-bound gathers (an L2 tier), persistent kernel only
    const bool split_want = env_int("PASTA_DIE_SPLIT", 0) != 0 && no == 2 && want_hot;
    if (hs) {
      // the nonzero order changes with the die split: wait for launches still reading the copy
      const_cast<CooModeCopy &>(mc).fence.wait(s);
      coo_mark_hot(const_cast<pasta_coo *>(x), mode, R, want_hot, hs_rows_budget, s, split_want);
      if (mc.hot_R != R || mc.hs_total == 0) hs = false;
    }
    if (!hs && want_hot) coo_mark_hot(const_cast<pasta_coo *>(x), mode, R, true, 0, s);
    if ((hs || want_hot) && mc.hot_R == R) {
      a.hot_marked = 1;
      a.hot_buf = mc.hot_buf.p;
      a.hs_rows = mc.hs_rows.p;
      int jj = 0;
      for (uint32_t k = 0; k < x->order; ++k)
        if (k != mode) {
          a.hs_lo[jj] = uint32_t(mc.hs_base[k]);
          a.io[jj++] = mc.hot_inds[k].p;
        }
      a.hs_lo[jj] = uint32_t(mc.hs_total);
      // hot_buf is shared by every launch on this handle and mode: wait for the previous one
      const_cast<CooModeCopy &>(mc).fence.wait(s);
      if (mc.hot_total) launch_hot_fill(mc, factors, x->order, mode, R, s);
      if (hs && mc.split) {
        a.nnz = mc.split_n;
        a.irow = mc.split_irow.p;
        a.val = mc.split_val.p;
        a.split = 1;
        a.split_x = mc.split_x;
        a.claim = mc.claim.p;
        a.die_of = die_map().d_die;
        PASTA_CUDA(cudaMemsetAsync(mc.claim.p, 0, 2 * sizeof(unsigned long long), s));
      }
    }
    // run per group: short runs on DRAM-bound gathers, longer ones on L2-resident factors
    // (fewer boundary atomics); measured on H (64: 1.82, 128: 1.87 ms per mode), C2 (128 and
    // 256: 0.83 ms) and C4 (128: 0.74, 256: 0.76 ms); profiles/r01_hs_sweep.txt
    uint64_t run = uint64_t(env_int("PASTA_MTTKRP_RUN", want_hot ? 64 : 128));
    run = run < 32 ? 32 : (run / 32) * 32;
    a.chunk = uint64_t(G) * run;
    a.cache_mode = uint32_t(env_int("PASTA_MTTKRP_CACHE", 0));
    const size_t smem = hs ? stage_hs + size_t(mc.hs_total) * R * sizeof(float)
                           : size_t(kWarpsPerCta) * 2 * (no + 2) * (G * 32) * sizeof(uint32_t);
    uint64_t nwarps = (a.nnz + a.chunk - 1) / a.chunk;
    uint64_t nblk = hs ? std::min<uint64_t>((nwarps + hs_wpc - 1) / hs_wpc, uint64_t(sm_count()))
                       : (nwarps + kWarpsPerCta - 1) / kWarpsPerCta;
    // PASTA_HOT_PERSIST=1: launch with an L2 access-policy window marking the hot-row buffer
    // persisting (within the device's persisting carve-out)
    const bool persist = a.hot_marked && env_int("PASTA_HOT_PERSIST", 0);
    auto go = [&](auto kern) {
      PASTA_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
      if (!persist) {
        kern<<<unsigned(nblk), hs ? hs_wpc * 32 : kThreads, smem, s>>>(a);
      } else {
        // the device-wide persisting carve-out is set for this launch only and restored
        // right after it (it would otherwise shrink the normal L2 of every later kernel)
        size_t prev_carve = 0, carve = 0;
        const size_t want = mc.hot_buf.bytes();
        {
          int dev = 0, maxp = 0;
          cudaGetDevice(&dev);
          cudaDeviceGetAttribute(&maxp, cudaDevAttrMaxPersistingL2CacheSize, dev);
          carve = size_t(maxp);
          PASTA_CUDA(cudaDeviceGetLimit(&prev_carve, cudaLimitPersistingL2CacheSize));
          PASTA_CUDA(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, carve));
        }
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(unsigned(nblk));
        cfg.blockDim = dim3(hs ? hs_wpc * 32 : kThreads);
        cfg.dynamicSmemBytes = smem;
        cfg.stream = s;
        cudaLaunchAttribute attr[1];
        attr[0].id = cudaLaunchAttributeAccessPolicyWindow;
        attr[0].val.accessPolicyWindow.base_ptr = mc.hot_buf.p;
        attr[0].val.accessPolicyWindow.num_bytes = want;
        attr[0].val.accessPolicyWindow.hitRatio = want <= carve ? 1.0f : float(double(carve) / double(want));
        attr[0].val.accessPolicyWindow.hitProp = cudaAccessPropertyPersisting;
        attr[0].val.accessPolicyWindow.missProp = cudaAccessPropertyStreaming;
        cfg.attrs = attr;
        cfg.numAttrs = 1;
        PASTA_CUDA(cudaLaunchKernelEx(&cfg, kern, a));
        PASTA_CUDA(cudaDeviceSetLimit(cudaLimitPersistingL2CacheSize, prev_carve));
      }
      PASTA_LAUNCHED();
      if (a.hot_marked) const_cast<CooModeCopy &>(mc).fence.record(s);
    };
    // WA 1 (default): one code path per buffer.  ptxas 12.9 turns the computed buffer
    // offset into an [R+UR] LDGSTS operand that, combined with the L2 cache-policy
    // descriptor, raises "illegal instruction" on sm_100a for some instantiations (observed
    // with compute-sanitizer); WA 2 drops the L2 hint instead; WA 0 is the plain form.
    const int wa = env_int("PASTA_STAGED_WA", 1);
    auto pick = [&](auto tag) {
      constexpr int W = decltype(tag)::value;
      if (lpn != 4 && lpn != 8) {  // R = 8 / 64: the default code path only
        with_no_lpn<3>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 1, false>); });
      } else if (no == 1 && lpn == 4) go(coo_staged_kernel<1, 4, 1, false>);  // one code path for order 2
      else if (no == 1) go(coo_staged_kernel<1, 8, 1, false>);
      else if (no == 2 && lpn == 4) go(coo_staged_kernel<2, 4, W, false>);
      else if (no == 2) go(coo_staged_kernel<2, 8, W, false>);
      else if (lpn == 4) go(coo_staged_kernel<3, 4, W, false>);
      else go(coo_staged_kernel<3, 8, W, false>);
    };
    // WA 7 = the HS kernel without the L2 tier (no tag-2 entries): no base-pointer select
    uint64_t max_factor = 0;
    for (uint32_t k = 0; k < x->order; ++k)
      if (k != mode) max_factor = std::max<uint64_t>(max_factor, uint64_t(x->dims[k]) * R * sizeof(float));
    const bool l2t = mc.hot_total > 0 || max_factor >= (uint64_t(1) << 32);
    auto pick_hs = [&](auto wtag, auto stag) {
      constexpr int W = decltype(wtag)::value, S = decltype(stag)::value;
      with_no_lpn<3>(no, lpn, [&](auto NOt, auto Lt) {
        if (l2t) go(coo_staged_kernel<NOt.value, Lt.value, 1, true, W, S>);
        else go(coo_staged_kernel<NOt.value, Lt.value, 7, true, W, S>);
      });
    };
    using I16 = std::integral_constant<int, 16>;
    a.nout = nout;
    for (uint32_t d = 0; d < nout && d < uint32_t(kMaxOrder); ++d) a.outs[d] = outs[d];
    if (hs && nout > 1) {  // fused MTTKRP + all-gather over peer memory, same shape as below
      if (hs_cfg == 1)
        with_no_lpn<3>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 15, true, 24, 16, 4>); });
      else if (hs_cfg == 5)
        with_no_lpn<3>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 15, true, 16, 16, 4>); });
      else if (hs_cfg == 6)
        with_no_lpn<3>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 15, true, 20, 16, 4>); });
      else if (hs_cfg == 2 && no <= 2)
        with_no_lpn<2>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 15, true, 16, 32, 8>); });
      else
        with_no_lpn<3>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 15, true, 16, 32, 4>); });
      return;
    }
    if (hs) {
      if (hs_cfg == 1) pick_hs(std::integral_constant<int, 24>(), I16());
      else if (hs_cfg == 5) pick_hs(I16(), I16());
      else if (hs_cfg == 6) pick_hs(std::integral_constant<int, 20>(), I16());
      else if (hs_cfg == 2 && no <= 2 && l2t && (a.cache_mode & 8u))  // cold gathers evict_first
        with_no_lpn<2>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 12, true, 16, 32, 8>); });
      else if (hs_cfg == 2 && no <= 2 && l2t && env_int("PASTA_GATHER_L1NA", 0))  // gathers skip L1
        with_no_lpn<2>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 13, true, 16, 32, 8>); });
      else if (hs_cfg == 2 && no <= 2)
        with_no_lpn<2>(no, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 1, true, 16, 32, 8>); });
      else pick_hs(I16(), std::integral_constant<int, 32>());
    } else if (wa == 1) pick(std::integral_constant<int, 1>());
    else if (wa == 2) pick(std::integral_constant<int, 2>());
    else if (wa == 3) pick(std::integral_constant<int, 3>());
    else if (wa == 4) pick(std::integral_constant<int, 4>());
    else if (wa == 5) pick(std::integral_constant<int, 5>());
    else if (wa == 6) pick(std::integral_constant<int, 6>());
    else pick(std::integral_constant<int, 0>());
    if (nout > 1) bcast_owned_rows(x, mode, R, outs, nout, s);
    return;
  }
  dispatch<CooSrc>(a, vec4, s);
  if (nout > 1) bcast_owned_rows(x, mode, R, outs, nout, s);
}

template <int NO>
void launch_heavy_lpn(const HArgs &h, int lpn, uint64_t n_pieces, size_t smem, cudaStream_t s) {
  auto go = [&](auto kern) {
    if (smem > 48 * 1024)
      PASTA_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
    kern<<<unsigned(n_pieces), kThreads, smem, s>>>(h);
    PASTA_LAUNCHED();
  };
  switch (lpn) {
    case 1: go(hicoo_heavy_kernel<NO, 1>); break;
    case 2: go(hicoo_heavy_kernel<NO, 2>); break;
    case 4: go(hicoo_heavy_kernel<NO, 4>); break;
    case 8: go(hicoo_heavy_kernel<NO, 8>); break;
    case 16: go(hicoo_heavy_kernel<NO, 16>); break;
    default: go(hicoo_heavy_kernel<NO, 32>); break;
  }
}

namespace {
// win_sb[w] = last slice s with sbptr[s] <= 32 w; end32[s] = sbptr[s + 1] (u32), nnz past nsb
__global__ void win_slice_kernel(const uint64_t *__restrict__ sbptr, uint64_t nsb, uint64_t nwin,
                                 uint32_t *__restrict__ win_sb) {
  for (uint64_t w = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; w < nwin; w += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t x = w * 32;
    uint64_t lo = 0, hi = nsb;
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) / 2;
      if (sbptr[mid] <= x) lo = mid; else hi = mid;
    }
    win_sb[w] = uint32_t(lo);
  }
}
__global__ void end32_kernel(const uint64_t *__restrict__ sbptr, uint64_t nsb, uint64_t nnz, uint64_t n,
                             uint32_t *__restrict__ end32) {
  for (uint64_t i = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; i < n; i += uint64_t(gridDim.x) * blockDim.x)
    end32[i] = uint32_t(i < nsb ? sbptr[i + 1] : nnz);
}
// run_sb[r] = last slice s with sbptr[s] <= r * run (the slice holding entry r * run)
__global__ void run_slice_kernel(const uint64_t *__restrict__ sbptr, uint64_t nsb, uint64_t run,
                                 uint64_t nruns, uint64_t *__restrict__ run_sb) {
  for (uint64_t r = blockIdx.x * uint64_t(blockDim.x) + threadIdx.x; r < nruns;
       r += uint64_t(gridDim.x) * blockDim.x) {
    const uint64_t x = r * run;
    uint64_t lo = 0, hi = nsb;
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) / 2;
      if (sbptr[mid] <= x) lo = mid; else hi = mid;
    }
    run_sb[r] = lo;
  }
}
}  // namespace

void launch_hicoo_mttkrp(const pasta_hicoo *h, uint32_t mode, const float *const *factors,
                         uint32_t R, float *out, cudaStream_t s) {
  const HicooModeCopy &mc = h->mc[mode];
  const int hno = int(h->order) - 1;
  // staging of 16 warps x 2 buffers x (N+1) arrays x 32 entries per group (R = 8: 16 groups
  // per warp -> 256 KB at N = 3, too large: the slice walk below takes it)
  const size_t hic_smem = size_t(16) * 2 * (hno + 2) * (size_t(32) / std::max<uint32_t>(R / 4, 1u) * 32) * 4;
  if (mc.layout == 0 && env_int("PASTA_HICOO_STAGED", 1) && staged_rank(R) && hno >= 1 &&
      hno <= 3 && h->nnz > 0 && hic_smem <= 227 * 1024 && vec4_ok(h->order, mode, factors, R, out)) {
    // Row slices decoded warp-wide into the persistent staged COO kernel (WA 9)
    HicooModeCopy &mcw = const_cast<HicooModeCopy &>(mc);
    const int lpn = int(R / 4);
    const int G = 32 / lpn;
    const size_t stage = size_t(16) * 2 * (hno + 2) * (G * 32) * sizeof(uint32_t);
    // hot-row tiers: 2 (default) = tier blocks (R#36, the copy rebuilt over heat-ranked blocks
    // of the gathered modes), 1 = hot-block tiers (R#34, slice bases of whole canonical blocks
    // retagged), 0 = none.  Budgets as the COO hot-row cache: an L2 tier when the gathered
    // factors exceed half the L2, a shared-memory tier of what the stage buffers leave (512
    // rows when the gathers go to DRAM)
    // Default (PASTA_HICOO_HOT unset): tier blocks when every gathered factor exceeds twice
    // the L2 -- measured: H (two 512-MB factors) 3.04 -> 2.60 ms per mode; C3 (a 20- or 102-MB
    // factor next to the 1.8-GB one) 2.41 -> 2.63 and the L2-resident C2 / C4 1.08 -> 1.20 / 1.15
    // -> 1.29, where the tiered gathers' extra instructions outweigh the misses they save
    // (profiles/r02_hicoo_tier_sweep.txt)
    static int l2 = 0;
    if (!l2) {
      int dev = 0;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&l2, cudaDevAttrL2CacheSize, dev);
      if (l2 <= 0) l2 = 126 << 20;
    }
    uint64_t gathered = 0, min_gathered = ~uint64_t(0);
    for (uint32_t k = 0; k < h->order; ++k)
      if (k != mode) {
        const uint64_t b = uint64_t(h->dims[k]) * R * sizeof(float);
        gathered += b;
        min_gathered = std::min(min_gathered, b);
      }
    const int hot_env = env_int("PASTA_HICOO_HOT", -1);
    const int hot_mode = !env_int("PASTA_HOT_SMEM", 1) ? 0
                         : hot_env >= 0                 ? hot_env
                         : (min_gathered > 2 * uint64_t(l2) ? 2 : 0);
    bool want_hot = false;
    uint32_t budget = 0;
    {
      want_hot = env_int("PASTA_HOT_FORCE", 0) || gathered > uint64_t(l2) / 2;
      budget = stage < 227 * 1024 ? uint32_t((227 * 1024 - stage) / (size_t(R) * sizeof(float))) : 0u;
      if (want_hot) budget = std::min(budget, uint32_t(env_int("PASTA_HOT_SMEM_DRAM", 512)));
      if (const int cap = env_int("PASTA_HOT_SMEM_ROWS", 0)) budget = std::min(budget, uint32_t(cap));
    }
    // every launch on this copy reads its slices: a rebuild or retag waits for the previous one
    mcw.fence.wait(s);
    hicoo_tier_rows(const_cast<pasta_hicoo *>(h), mode, R, hot_mode == 2, want_hot, budget, s);
    KArgs a{};
    a.nnz = h->nnz;
    a.order = h->order;
    a.R = R;
    a.sbptr = mc.sbptr.p;
    a.nsb = mc.nsb;
    a.sbrow = mc.sbrow.p;
    a.val = mc.val.p;
    int j = 0;
    for (uint32_t k = 0; k < h->order; ++k) {
      if (k == mode) continue;
      if ((h->cmask >> k) & 1u) {
        a.sbbase[j] = mc.sbbase[k].p;
        a.eo[j] = mc.einds[k].p;
      } else {
        a.io[j] = mc.uinds[k].p;
        a.wide |= 1u << j;
      }
      a.Uo[j] = factors[k];
      ++j;
    }
    a.out = out;
    uint64_t run = uint64_t(env_int("PASTA_MTTKRP_RUN", 128));
    run = run < 32 ? 32 : (run / 32) * 32;
    a.chunk = uint64_t(G) * run;
    const uint64_t nruns = (a.nnz + run - 1) / run;
    if (mcw.run_sb_run != run || mcw.run_sb.n != nruns) {
      mcw.run_sb.alloc(nruns, s);
      uint64_t g = (nruns + 255) / 256;
      if (g > 148 * 32) g = 148 * 32;
      run_slice_kernel<<<unsigned(g), 256, 0, s>>>(mc.sbptr.p, mc.nsb, run, nruns, mcw.run_sb.p);
      PASTA_LAUNCHED();
      mcw.run_sb_run = run;
    }
    a.run_sb = mcw.run_sb.p;
    bool tiers = false;
    if (hot_mode == 2) {
      tiers = mc.rt_on && mc.rt_R == R && (mc.hs_total + mc.hot_total) > 0;
    } else if (hot_mode != 1) {
      if (mc.tagged) hicoo_mark_hot(const_cast<pasta_hicoo *>(h), mode, R, false, 0, s);  // untag
    } else {
      hicoo_mark_hot(const_cast<pasta_hicoo *>(h), mode, R, want_hot, budget, s);
      tiers = mc.hot_R == R && (mc.hs_total + mc.hot_total) > 0;
    }
    if (tiers) {
      a.hot_marked = 1;
      a.hot_buf = mc.hot_buf.p;
      a.hs_rows = mc.hs_rows.p;
      int jj = 0;
      for (uint32_t k = 0; k < h->order; ++k)
        if (k != mode) a.hs_lo[jj++] = uint32_t(mc.hs_base[k]);
      a.hs_lo[jj] = uint32_t(mc.hs_total);
      if (mc.hot_total) launch_hot_fill(mc, factors, h->order, mode, R, s);
    }
    // raw-staged decode (WA 11): orders 2 and 3 (R >= 16: a warp's raw windows and stage
    // buffers fit the 227 KB), no tiers; PASTA_HICOO_RAW=0 keeps the WA 9 decode
    uint32_t raw_words = 36 + 72;
    for (int j = 0; j < hno; ++j) raw_words += ((a.wide >> j) & 1u) ? 32 : 8 + 36;
    const size_t raw_bytes = size_t(16) * G * raw_words * 4;
    const bool use_raw = !tiers && hno <= 2 && env_int("PASTA_HICOO_RAW", 0) && stage + raw_bytes <= 227 * 1024 &&
                         h->nnz < 0xFFFFFFFFull;
    // u32 slice ends (nnz < 2^32 by the API): half the bytes and registers of sbptr in the decode
    if (mcw.sbend32.n != mc.nsb + kSlicePad) {
      mcw.sbend32.alloc(mc.nsb + kSlicePad, s);
      uint64_t g = (mc.nsb + kSlicePad + 255) / 256;
      if (g > 148 * 32) g = 148 * 32;
      end32_kernel<<<unsigned(g), 256, 0, s>>>(mc.sbptr.p, mc.nsb, h->nnz, mc.nsb + kSlicePad, mcw.sbend32.p);
      PASTA_LAUNCHED();
    }
    a.sbend32 = mcw.sbend32.p;
    if (use_raw) {
      const uint64_t nwin = (h->nnz + 31) / 32;
      if (mcw.win_sb.n != nwin) {
        mcw.win_sb.alloc(nwin, s);
        uint64_t g = (nwin + 255) / 256;
        if (g > 148 * 32) g = 148 * 32;
        win_slice_kernel<<<unsigned(g), 256, 0, s>>>(mc.sbptr.p, mc.nsb, nwin, mcw.win_sb.p);
        PASTA_LAUNCHED();
      }
      a.win_sb = mcw.win_sb.p;
      a.raw_words = raw_words;
    }
    // row-granular shared-memory tier (WA 16) when the factors are L2-resident and every
    // gathered mode's row bitmap fits next to the stage buffers (C2- / C4-like tensors)
    uint64_t max_factor16 = 0, words = 0;
    uint64_t gathered16 = 0;
    for (uint32_t k = 0; k < h->order; ++k)
      if (k != mode) {
        max_factor16 = std::max<uint64_t>(max_factor16, uint64_t(h->dims[k]) * R * sizeof(float));
        gathered16 += uint64_t(h->dims[k]) * R * sizeof(float);
        words += (uint64_t(h->dims[k]) + 31) / 32;
      }
    static int l2b = 0;
    if (!l2b) {
      int dev = 0;
      cudaGetDevice(&dev);
      cudaDeviceGetAttribute(&l2b, cudaDevAttrL2CacheSize, dev);
      if (l2b <= 0) l2b = 126 << 20;
    }
    bool rowtier = false;
    if (!tiers && !use_raw && env_int("PASTA_HICOO_ROWTIER", 0) && max_factor16 < (uint64_t(1) << 32) &&
        gathered16 <= uint64_t(l2b) / 2 && stage + 8 * words + 64 * R * 4 <= 227 * 1024) {
      uint32_t budget = uint32_t((227 * 1024 - stage - 8 * words) / (size_t(R) * 4));
      if (const int cap = env_int("PASTA_HOT_SMEM_ROWS", 0)) budget = std::min(budget, uint32_t(cap));
      hicoo_mark_rows(const_cast<pasta_hicoo *>(h), mode, R, budget, (227 * 1024 - stage) / 8, s);
      rowtier = mc.rs_R == R && mc.rs_total > 0;
    }
    if (rowtier) {
      a.hs_rows = mc.rs_rows.p;
      int jj = 0;
      for (uint32_t k = 0; k < h->order; ++k)
        if (k != mode) {
          a.hs_lo[jj] = uint32_t(mc.rs_base[k]);
          a.rs_bm[jj] = mc.rs_bm[k].p;
          a.rs_pre[jj] = mc.rs_pre[k].p;
          a.rs_words[jj] = uint32_t(mc.rs_words[k]);
          ++jj;
        }
      a.hs_lo[jj] = uint32_t(mc.rs_total);
    }
    ProfScope prof(kProfHicoo, s);
    // shape: 0 = 16 warps x 4-nonzero steps; 2 = 16 x 8 (spills here: H 3.59 ms); 3 = 12 warps x
    // 8-nonzero steps (168 registers), the default with an L2 tier at order 3 (H 2.61 -> 2.53 ms,
    // profiles/r02_hicoo_tier_sweep.txt)
    const int cfg = env_int("PASTA_HS_CFG", (tiers && mc.hot_total > 0 && hno <= 2) ? 3 : 0);
    uint64_t max_gf = 0;
    for (uint32_t k = 0; k < h->order; ++k)
      if (k != mode) max_gf = std::max<uint64_t>(max_gf, uint64_t(h->dims[k]) * R * sizeof(float));
    // kernel choice (below) and its warps per CTA
    const bool wa17 = tiers && mc.hot_total == 0 && max_gf < (uint64_t(1) << 32);
    const int wpc = wa17 || rowtier || use_raw ? 16
                    : tiers                    ? ((cfg == 3 && hno <= 2) ? 12 : 16)
                                               : 16;
    const size_t smem = stage * wpc / 16 + (tiers ? size_t(mc.hs_total) * R * sizeof(float) : 0) + (use_raw ? raw_bytes : 0) +
                        (rowtier ? size_t(mc.rs_total) * R * sizeof(float) + 8 * words : 0);
    const uint64_t nwarps = (a.nnz + a.chunk - 1) / a.chunk;
    const uint64_t nblk = std::min<uint64_t>((nwarps + wpc - 1) / wpc, uint64_t(sm_count()));
    auto go = [&](auto kern) {
      PASTA_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, int(smem)));
      kern<<<unsigned(nblk), wpc * 32, smem, s>>>(a);
      PASTA_LAUNCHED();
      mcw.fence.record(s);
    };
    if (wa17)  // smem tier only: WA 17
      with_no_lpn<3>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 17, true, 16, 32, 4>); });
    else if (rowtier)
      with_no_lpn<3>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 16, true, 16, 32, 4>); });
    else if (use_raw)
      with_no_lpn<2>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 11, true, 16, 32, 4>); });
    else if (tiers) {
      if (cfg == 2 && hno <= 2)  // 8-nonzero steps (the COO shape on DRAM-bound gathers)
        with_no_lpn<2>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 10, true, 16, 32, 8>); });
      else if (cfg == 3 && hno <= 2)  // 12 warps x 8-nonzero steps: 168 registers, no spills
        with_no_lpn<2>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 10, true, 12, 32, 8>); });
      else
        with_no_lpn<3>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 10, true, 16, 32, 4>); });
    } else if (cfg == 2 && hno <= 2)
      with_no_lpn<2>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 9, true, 16, 32, 8>); });
    else
      with_no_lpn<3>(hno, lpn, [&](auto NOt, auto Lt) { go(coo_staged_kernel<NOt.value, Lt.value, 9, true, 16, 32, 4>); });
    return;
  }
  if (mc.layout == 0) {
    // the generic row-slice kernel reads plain block bases: undo any hot-block tagging
    HicooModeCopy &mcw = const_cast<HicooModeCopy &>(mc);
    if (mc.tagged || mc.rt_on) {
      mcw.fence.wait(s);
      if (mc.tagged) hicoo_mark_hot(const_cast<pasta_hicoo *>(h), mode, R, false, 0, s);
      hicoo_tier_rows(const_cast<pasta_hicoo *>(h), mode, R, false, false, 0, s);
    }
    KArgs a{};
    a.nnz = h->nnz;
    a.order = h->order;
    a.R = R;
    a.sbptr = mc.sbptr.p;
    a.nsb = mc.nsb;
    a.sbrow = mc.sbrow.p;
    a.val = mc.val.p;
    int j = 0;
    for (uint32_t k = 0; k < h->order; ++k) {
      if (k == mode) continue;
      if ((h->cmask >> k) & 1u) {
        a.sbbase[j] = mc.sbbase[k].p;
        a.eo[j] = mc.einds[k].p;
      } else {
        a.io[j] = mc.uinds[k].p;
        a.wide |= 1u << j;
      }
      a.Uo[j] = factors[k];
      ++j;
    }
    a.out = out;
    if (a.nnz == 0) return;
    ProfScope prof(kProfHicoo, s);
    dispatch<HicooRowSrc>(a, vec4_ok(h->order, mode, factors, R, out), s);
    return;
  }
  KArgs a{};
  a.nnz = h->nnz;
  a.order = h->order;
  a.R = R;
  a.bptr = mc.bptr.p;
  a.nblocks = h->nblocks;
  a.brow = mc.binds[mode].p;
  a.erow = mc.einds[mode].p;
  a.val = mc.val.p;
  a.bbits = h->block_bits;
  HArgs ha{};
  int j = 0;
  for (uint32_t k = 0; k < h->order; ++k) {
    if (k == mode) continue;
    a.bo[j] = mc.binds[k].p;
    a.eo[j] = mc.einds[k].p;
    a.Uo[j] = factors[k];
    ha.bo[j] = mc.binds[k].p;
    ha.eo[j] = mc.einds[k].p;
    ha.Uo[j] = factors[k];
    ha.dims_o[j] = h->dims[k];
    ++j;
  }
  a.out = out;
  if (a.nnz == 0) return;
  ProfScope prof(kProfHicoo, s);
  const bool vec4 = vec4_ok(h->order, mode, factors, R, out);
  const size_t smem = size_t(h->order - 1) * (size_t(1) << h->block_bits) * R * sizeof(float);
  const bool heavy = vec4 && mc.n_pieces > 0 && smem <= 160 * 1024;
  if (heavy) {
    ha.pieces = mc.pieces.p;
    ha.piece = mc.piece;
    ha.bptr = mc.bptr.p;
    ha.brow = mc.binds[mode].p;
    ha.erow = mc.einds[mode].p;
    ha.val = mc.val.p;
    ha.out = out;
    ha.order = h->order;
    ha.R = R;
    ha.bbits = h->block_bits;
    ha.cache_mode = uint32_t(env_int("PASTA_MTTKRP_CACHE", 0));
    uint32_t need = (R + 3) / 4;
    int lpn = 1;
    while (lpn < 32 && uint32_t(lpn) < need) lpn <<= 1;
    const int no = int(h->order) - 1;
    if (no == 2) launch_heavy_lpn<2>(ha, lpn, mc.n_pieces, smem, s);
    else if (no == 3) launch_heavy_lpn<3>(ha, lpn, mc.n_pieces, smem, s);
    else launch_heavy_lpn<0>(ha, lpn, mc.n_pieces, smem, s);
    // the light blocks: warp runs over the rest of the per-mode copy (the run grid starts
    // 16-byte aligned; entries before heavy_nnz are skipped)
    a.x_begin = mc.heavy_nnz & ~uint64_t(3);
    a.x_skip = mc.heavy_nnz;
    a.b_begin = mc.n_heavy;
    if (mc.heavy_nnz == h->nnz) return;
  }
  dispatch<HicooSrc>(a, vec4, s);
}

}  // namespace pasta
