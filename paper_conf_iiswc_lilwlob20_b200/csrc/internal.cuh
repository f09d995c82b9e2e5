// internal.cuh -- shared internals of libpasta (never installed; not part of the ABI).
// Citations: P:N = line N of the paper text; R#k = DESIGN.md reading k.
#pragma once

#include <cuda_runtime.h>

#include <atomic>
#include <cstdint>
#include <cstring>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "../../include/pasta.h"

namespace pasta {

constexpr int kMaxOrder = PASTA_MAX_ORDER;

// ----------------------------------------------------------------------------- errors
struct Error {
  pasta_status code;
  std::string msg;
};
[[noreturn]] inline void fail(pasta_status code, const std::string &msg) { throw Error{code, msg}; }
void set_last_error(pasta_status code, const std::string &msg);

#define PASTA_CUDA(expr)                                                                  \
  do {                                                                                    \
    cudaError_t _e = (expr);                                                              \
    if (_e != cudaSuccess)                                                                \
      ::pasta::fail(PASTA_ECUDA, std::string(#expr) + ": " + cudaGetErrorString(_e));     \
  } while (0)

#define PASTA_LAUNCHED()                                                                  \
  do {                                                                                    \
    ::pasta::count_launch();                                                              \
    cudaError_t _e = cudaGetLastError();                                                  \
    if (_e != cudaSuccess)                                                                \
      ::pasta::fail(PASTA_ECUDA, std::string("kernel launch: ") + cudaGetErrorString(_e)); \
  } while (0)

void count_launch();

// ----------------------------------------------------------------------------- memory
void *dev_alloc(size_t bytes, cudaStream_t s);
void dev_free(void *p, cudaStream_t s);

// Owning device array (allocated through the allocator hook, else cudaMalloc).
template <class T>
struct DevArray {
  T *p = nullptr;
  size_t n = 0;
  DevArray() = default;
  explicit DevArray(size_t count, cudaStream_t s = nullptr) { alloc(count, s); }
  DevArray(const DevArray &) = delete;
  DevArray &operator=(const DevArray &) = delete;
  DevArray(DevArray &&o) noexcept : p(o.p), n(o.n) { o.p = nullptr; o.n = 0; }
  DevArray &operator=(DevArray &&o) noexcept {
    if (this != &o) { reset(); p = o.p; n = o.n; o.p = nullptr; o.n = 0; }
    return *this;
  }
  ~DevArray() { reset(); }
  void alloc(size_t count, cudaStream_t s = nullptr) {
    reset();
    n = count;
    // rounded up to 64 bytes: the kernels' 16-byte vector and cp.async reads of a ragged tail
    // (with a partial src-size) stay inside the allocation
    p = static_cast<T *>(dev_alloc(((count ? count : 1) * sizeof(T) + 63) & ~size_t(63), s));
  }
  void reset() {
    if (p) dev_free(p, nullptr);
    p = nullptr;
    n = 0;
  }
  T *get() const { return p; }
  size_t bytes() const { return n * sizeof(T); }
};

// SM -> die map of the current device (die.cu): measured once per device; ok = two
// plausible groups found (else no die split is used).  d_die: device copy, die of %smid.
constexpr int kMaxSms = 1024;
struct DieMap {
  bool ok = false;
  int sms = 0;
  int n[2] = {0, 0};
  int8_t die[kMaxSms] = {};
  int8_t *d_die = nullptr;
};
const DieMap &die_map();

// Which half of factor k's rows a row belongs to in the die split (R#35): a fixed hash of
// (row, k) compared with the die-0 share t (of 2^32).  Host (slot order of the L2 tier) and
// device (nonzero classes) use the same function.
__host__ __device__ inline uint32_t die_half(uint32_t row, uint32_t k, uint32_t t) {
  uint32_t x = row * 0x9E3779B1u ^ (k * 0x85EBCA77u + 0x165667B1u);
  x ^= x >> 16;
  x *= 0x7FEB352Du;
  x ^= x >> 15;
  x *= 0x846CA68Bu;
  x ^= x >> 16;
  return x < t ? 0u : 1u;
}

// Completion of the last launch that used a handle's per-mode mutable state (the hot-row
// buffer, refilled from the factors before every launch): a launch on another stream waits
// for it, so same-handle MTTKRPs on two streams are ordered instead of racing on the buffer.
struct LaunchFence {
  cudaEvent_t e = nullptr;
  LaunchFence() = default;
  LaunchFence(const LaunchFence &) = delete;
  LaunchFence &operator=(const LaunchFence &) = delete;
  ~LaunchFence() { if (e) cudaEventDestroy(e); }
  void wait(cudaStream_t s) { if (e) cudaStreamWaitEvent(s, e, 0); }
  void record(cudaStream_t s) {
    if (!e) cudaEventCreateWithFlags(&e, cudaEventDisableTiming);
    cudaEventRecord(e, s);
  }
};

// Copy streams and events of the end-to-end host path (created on first use).
// Two staging slots: step i of a batch uses slot i & 1, so that step i+1's uploads overlap
// step i's downloads.  f: factor k of a slot landed; o: output m of a slot computed; od:
// output m of a slot downloaded (slot reusable); kd: every kernel of a slot done.
struct E2EStreams {
  cudaStream_t h2d = nullptr, d2h = nullptr;
  cudaEvent_t f[2][kMaxOrder] = {}, o[2][kMaxOrder] = {}, od[2][kMaxOrder] = {}, kd[2] = {};
  cudaEvent_t start = nullptr;
  bool ready = false;
  void init() {
    if (ready) return;
    cudaStreamCreateWithFlags(&h2d, cudaStreamNonBlocking);
    cudaStreamCreateWithFlags(&d2h, cudaStreamNonBlocking);
    for (int b = 0; b < 2; ++b) {
      for (int k = 0; k < kMaxOrder; ++k) {
        cudaEventCreateWithFlags(&f[b][k], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&o[b][k], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&od[b][k], cudaEventDisableTiming);
      }
      cudaEventCreateWithFlags(&kd[b], cudaEventDisableTiming);
    }
    cudaEventCreateWithFlags(&start, cudaEventDisableTiming);
    ready = true;
  }
  ~E2EStreams() {
    if (!ready) return;
    for (int b = 0; b < 2; ++b) {
      for (int k = 0; k < kMaxOrder; ++k) {
        cudaEventDestroy(f[b][k]);
        cudaEventDestroy(o[b][k]);
        cudaEventDestroy(od[b][k]);
      }
      cudaEventDestroy(kd[b]);
    }
    cudaEventDestroy(start);
    cudaStreamDestroy(h2d);
    cudaStreamDestroy(d2h);
  }
};

// ----------------------------------------------------------------------------- handles
struct CooModeCopy {
  bool ready = false;
  const uint32_t *inds[kMaxOrder] = {};  // sorted by (i_mode, i_mode+1, ...), may alias canon
  const float *val = nullptr;
  DevArray<uint32_t> own_inds[kMaxOrder];
  DevArray<float> own_val;
  // Hot-row cache (coo_mark_hot), two tiers for rank hot_R: the most frequent rows of the
  // gathered factors in every CTA's shared memory (hs_*), the next ones packed into one
  // contiguous buffer that fits the L2 budget (hot_*).  hot_inds[k] (k != mode) = inds[k] for
  // cold entries, 0xC0000000 | smem slot, 0x80000000 | slot into hot_buf.
  uint32_t hot_R = 0;       // 0: not marked
  bool hot_global = false;  // L2 tier requested
  uint32_t hot_smem_budget = 0;
  uint32_t hot_bucket = 0;  // rows with hot_bucket <= count bucket < hs_bucket: L2 tier
  uint32_t hs_bucket = 0;   // rows with count bucket >= hs_bucket: smem tier
  DevArray<uint32_t> hs_rows;           // smem slot -> factor row, factor k at [hs_base[k], +hs_cnt[k])
  uint64_t hs_base[kMaxOrder] = {}, hs_cnt[kMaxOrder] = {}, hs_total = 0;
  DevArray<uint32_t> hot_inds[kMaxOrder];
  DevArray<uint32_t> hot_rows;          // slot -> factor row, factor k at [hot_base[k], +hot_cnt[k])
  uint64_t hot_base[kMaxOrder] = {}, hot_cnt[kMaxOrder] = {}, hot_total = 0;
  DevArray<float> hot_buf;              // hot_total x R, refilled from the factors every launch
  LaunchFence fence;                    // last launch that read hot_buf
  // Die split (R#35, order 3 with an L2 tier): each gathered factor's rows are split into two
  // halves (die_half); nonzeros are reordered into 4 row-sorted segments by (half of the first
  // gathered row, half of the second): die 0 walks [0, split_x) = (0,0) then (0,1), die 1 walks
  // [split_x, split_n) = (1,1) then (1,0), so at any time the two dies gather disjoint halves of
  // both factors and each die's L2 holds only its half of the hot rows.  The L2-tier slots of
  // each factor are ordered half 0 first.  split_irow / split_val / hot_inds hold that order.
  bool split = false;
  uint64_t split_x = 0;                 // die 1's first position (16-byte aligned)
  uint64_t split_n = 0;                 // length of the split arrays (nnz + alignment gap)
  uint32_t split_t[2] = {};             // die-0 shares of the two gathered factors (of 2^32)
  DevArray<uint32_t> split_irow;
  DevArray<float> split_val;
  DevArray<unsigned long long> claim;   // per-die chunk counters, zeroed before each launch
  bool smem_fill = false;               // PASTA_HOT_SMEM_FILL: smem tier filled from the next bucket
};

constexpr int kCountBuckets = 256;  // 8 sub-buckets per octave of a row's nonzero count
constexpr uint64_t kSlicePad = 40;  // padding slots after the row-slice arrays (raw decode)

struct HicooModeCopy {
  bool ready = false;
  // blocks ordered (heavy first, then light; each part by binds_mode), entries inside a block
  // by einds_mode (R#27)
  DevArray<uint64_t> bptr;               // nblocks + 1
  DevArray<uint32_t> binds[kMaxOrder];   // nblocks each
  DevArray<uint8_t> einds[kMaxOrder];    // nnz each
  DevArray<float> val;                   // nnz
  uint64_t n_heavy = 0;                  // blocks [0, n_heavy) hold >= heavy_min entries
  uint64_t heavy_nnz = 0;                // = bptr[n_heavy]
  uint32_t heavy_min = 0;
  uint32_t piece = 4096;                 // max entries per CTA work item
  DevArray<uint32_t> pieces;             // 2 per item: (block, piece index within block)
  uint64_t n_pieces = 0;
  // layout 0 ("row slices", default): entries sorted by output row across the blocks of a
  // block row; a slice = the entries of one block sharing einds_mode, with its own row and
  // other-mode block bases.  Uses einds[k] (k != mode) and val; not bptr/binds/pieces.
  // layout 1 ("blocks"): the block-major copy above (heavy blocks TMA-staged).
  int layout = 0;
  uint64_t nsb = 0;
  DevArray<uint64_t> sbptr;              // nsb + 1
  DevArray<uint32_t> sbrow;              // nsb: output row of the slice
  DevArray<uint32_t> sbbase[kMaxOrder];  // nsb each (k != mode, k compressed): binds_k << block_bits
  DevArray<uint32_t> uinds[kMaxOrder];   // gHiCOO: nnz each (k != mode, k uncompressed): i_k
  // staged decode (launch_hicoo_mttkrp): slice holding the first entry of every group run
  DevArray<uint64_t> run_sb;
  uint64_t run_sb_run = 0;
  // raw-staged decode (WA 11): slice holding entry 32 w of every 32-entry window w, and the
  // slice ends as u32 padded with nnz (kSlicePad slots)
  DevArray<uint32_t> win_sb;
  DevArray<uint32_t> sbend32;
  // Hot-BLOCK tiers (hicoo_mark_hot, R#34): the row-slice copy has no per-entry coordinate
  // to retag (entries carry 8-bit offsets from a per-slice block base), so the tiers of the
  // COO hot-row cache are built at block granularity: the most frequent block rows [b B,
  // b B + B) of each gathered (compressed) factor go whole into the shared-memory tier or
  // the packed L2-tier buffer, and the slice bases sbbase[k] of those blocks are retagged in
  // place to 0xC0000000 | smem row slot / 0x80000000 | L2 row slot (slot = tier block x B,
  // so base + einds stays inside the block's slots).  Same slot lists and fill kernel as the
  // COO tiers; tier_block[k] lists the original block of every (smem, then L2) slot block so
  // the retagging can be undone when R or the budgets change.
  uint32_t hot_R = 0;
  bool hot_global = false;
  uint32_t hot_smem_budget = 0;
  DevArray<uint32_t> hs_rows;
  uint64_t hs_base[kMaxOrder] = {}, hs_cnt[kMaxOrder] = {}, hs_total = 0;
  DevArray<uint32_t> hot_rows;
  uint64_t hot_base[kMaxOrder] = {}, hot_cnt[kMaxOrder] = {}, hot_total = 0;
  DevArray<float> hot_buf;
  DevArray<uint32_t> tier_block[kMaxOrder];
  bool tagged = false;
  LaunchFence fence;
  // row-granular shared-memory tier of the staged decode (WA 16, hicoo_mark_rows): hot rows of
  // each gathered mode (ascending) in rs_rows, per mode k a bitmap rs_bm[k] over its rows and
  // the per-word prefix counts rs_pre[k]; cached for (rs_R, rs_budget)
  uint32_t rs_R = 0, rs_budget = 0;
  uint64_t rs_total = 0, rs_base[kMaxOrder] = {}, rs_words[kMaxOrder] = {};
  DevArray<uint32_t> rs_rows;
  DevArray<uint32_t> rs_bm[kMaxOrder], rs_pre[kMaxOrder];
  // tier blocks (R#36, hicoo_tier_rows): the copy itself was built over the heat-ranked tier
  // blocks of the gathered modes for (rt_R, rt_global, rt_budget); hs_* / hot_* describe them
  bool rt_on = false;
  uint32_t rt_R = 0, rt_budget = 0;
  bool rt_global = false;
};

}  // namespace pasta

namespace pasta {
// Mode-n fibers of a COO tensor (TTV/TTM): nonzeros sorted by the other modes
// then i_n; `mat` is the order-2 COO (fiber id, i_n) with the same values, so that
// TTM = mode-0 MTTKRP of `mat` with the single factor U (Eq. 2 = Eq. 3 on the fiberised matrix).
struct FiberCopy;
}  // namespace pasta

struct pasta_coo {
  uint32_t order = 0;
  uint32_t dims[pasta::kMaxOrder] = {};
  uint64_t nnz = 0;
  int device = 0;
  bool lex_sorted = false;  // canonical order == mode-0 lexicographic order
  pasta::DevArray<uint32_t> inds[pasta::kMaxOrder];
  pasta::DevArray<float> val;
  pasta::CooModeCopy mc[pasta::kMaxOrder];
  int shard_mode = -1;  // >= 0: this handle is the [row_lo, row_hi) shard of that mode
  uint32_t row_lo = 0, row_hi = 0;
  // e2e staging (pasta_mttkrp_coo_allmodes_host)
  uint32_t stage_R[2] = {};
  pasta::DevArray<float> stage_f[2][pasta::kMaxOrder];
  pasta::DevArray<float> stage_o[2][pasta::kMaxOrder];
  pasta::E2EStreams e2e;
  // per-mode row nonzero counts (device u32) and their bucket histogram (host)
  bool counts_ready[pasta::kMaxOrder] = {};
  pasta::DevArray<uint32_t> row_count[pasta::kMaxOrder];
  uint64_t count_hist[pasta::kMaxOrder][pasta::kCountBuckets] = {};
  pasta::FiberCopy *fib[pasta::kMaxOrder] = {};
  ~pasta_coo();
  std::mutex mu;
};

struct pasta_hicoo {
  uint32_t order = 0;
  uint32_t dims[pasta::kMaxOrder] = {};
  uint32_t block_bits = 7;
  // gHiCOO (R#29): bit k set <=> mode k is blocked (binds_k, einds_k); the
  // other modes keep full u32 coordinates (uinds_k).  HiCOO = all bits set.
  uint32_t cmask = 0;
  uint64_t nblocks = 0;
  uint64_t nnz = 0;
  int device = 0;
  pasta::DevArray<uint64_t> bptr;
  pasta::DevArray<uint32_t> binds[pasta::kMaxOrder];
  pasta::DevArray<uint8_t> einds[pasta::kMaxOrder];
  pasta::DevArray<uint32_t> uinds[pasta::kMaxOrder];
  pasta::DevArray<float> val;
  pasta::HicooModeCopy mc[pasta::kMaxOrder];
  // R#36 heat ranking per mode (rows by nonzero count, descending): order, its inverse, and
  // the heat of every block of 2^block_bits consecutive ranks (host)
  bool rt_ready[pasta::kMaxOrder] = {};
  pasta::DevArray<uint32_t> rt_order[pasta::kMaxOrder], rt_rank[pasta::kMaxOrder];
  std::vector<unsigned long long> rt_heat[pasta::kMaxOrder];
  int shard_mode = -1;  // >= 0: the [row_lo, row_hi) shard of that mode (pasta_hicoo_shard)
  uint32_t row_lo = 0, row_hi = 0;
  std::mutex mu;
};

namespace pasta {

struct FiberCopy {
  uint64_t nf = 0;
  pasta::DevArray<uint32_t> finds[kMaxOrder];  // fiber coordinates (k != mode), nf each
  pasta_coo mat;                               // order 2: (fiber id, i_mode), lex sorted
};

inline uint32_t ceil_log2(uint64_t v) {
  uint32_t l = 0;
  while (l < 64 && (uint64_t(1) << l) < v) ++l;
  return l;
}

// ------------------------------------------------------------------------- sort helpers
// Stable lexicographic sort of the permutation `perm` (length M, initialised by the
// caller) by device u32 component arrays comps[0] (most significant) .. comps[nc-1],
// where comps[c] has bits[c] significant bits.  Indexing: key of position x is
// comps[c][perm[x]].  Implemented as LSD passes of CUB radix sort over 64-bit packed keys.
void lexsort(const uint32_t *const *comps, const uint32_t *bits, int nc, DevArray<uint32_t> &perm,
             uint64_t M, cudaStream_t s);
// Morton-order sort (R#13) of the coordinate arrays `inds` (order N): stable, by the
// level-major interleave of Lm-bit coordinates.  perm initialised by the caller.
void morton_sort(const uint32_t *const *inds, uint32_t order, uint32_t Lm, DevArray<uint32_t> &perm,
                 uint64_t M, cudaStream_t s);
// out[x] = in[perm[x]]
void gather_u32(const uint32_t *in, const uint32_t *perm, uint32_t *out, uint64_t M, cudaStream_t s);
void gather_f32(const float *in, const uint32_t *perm, float *out, uint64_t M, cudaStream_t s);
void gather_u8(const uint8_t *in, const uint32_t *perm, uint8_t *out, uint64_t M, cudaStream_t s);
void iota_u32(uint32_t *p, uint64_t M, cudaStream_t s);
// idx_out[0..count) = positions x < M with flags[x] != 0, ascending.  Returns count.
uint64_t select_flagged(const uint8_t *flags, uint64_t M, DevArray<uint32_t> &idx_out, cudaStream_t s);

// ------------------------------------------------------------------------- operations
void coo_prepare_mode(pasta_coo *x, uint32_t mode, cudaStream_t s);
void hicoo_prepare_mode(pasta_hicoo *h, uint32_t mode, cudaStream_t s);
// ncell = 0 selects the slice power-law generator (kind 2, exponent alpha; R#30)
void gen_powerlaw_device(pasta_coo *x, uint64_t seed, const double *table, uint32_t ncell,
                         float val_lo, float val_hi, cudaStream_t s, double alpha = 1.0);
void coo_to_hicoo_device(const pasta_coo *x, pasta_hicoo *h, cudaStream_t s);  // honours h->cmask
void hicoo_shard_device(const pasta_hicoo *h, uint32_t mode, uint32_t row_lo, uint32_t row_hi, pasta_hicoo *y,
                        cudaStream_t s);
// generator label permutation (permute = 1, R#22): relabel every mode, re-sort lexicographically
void relabel_device(pasta_coo *x, uint64_t seed, cudaStream_t s);
// number of distinct block keys (i_k >> block_bits, k in cmask) of a COO tensor
uint64_t count_blocks_device(const pasta_coo *x, uint32_t block_bits, uint32_t cmask, cudaStream_t s);

void launch_zero_rows(float *out, uint64_t row_lo, uint64_t row_hi, uint32_t R, cudaStream_t s);
void launch_coo_mttkrp(const pasta_coo *x, uint32_t mode, const float *const *factors, uint32_t R,
                       float *out, cudaStream_t s);
// fused MTTKRP + all-gather: outs[0] local output, outs[1..nout) peers' replicas (nout <= 8)
void launch_coo_mttkrp_bcast(const pasta_coo *x, uint32_t mode, const float *const *factors, uint32_t R,
                             float *const *outs, uint32_t nout, cudaStream_t s);
void launch_hicoo_mttkrp(const pasta_hicoo *h, uint32_t mode, const float *const *factors,
                         uint32_t R, float *out, cudaStream_t s);
void launch_gram(const float *U, uint64_t rows, uint32_t R, double *G, cudaStream_t s);
void launch_solve(const float *M, uint64_t rows, uint32_t R, const double *const *grams, uint32_t ngrams,
                  float *U, double *colsq, cudaStream_t s);
void launch_normalize(float *U, uint64_t rows, uint32_t R, const double *colsq, double *lambda,
                      cudaStream_t s);
// fused CP-ALS epilogue: from GM = M^T M and the other grams -> Wn (fp32), G_n, lambda
void launch_cpals_prep(const double *GM, const double *const *grams, uint32_t ngrams, uint32_t R,
                       float *Wn, double *Gn, double *lambda, cudaStream_t s);
// U = M Wn (rows x R times R x R)
void launch_apply(const float *M, uint64_t rows, uint32_t R, const float *Wn, float *U, cudaStream_t s);
// rows [row_lo, row_hi) of M Wn stored into each of `ndst` full-size replicas (local / peer)
void launch_apply_bcast(const float *M, uint64_t row_lo, uint64_t row_hi, uint32_t R, const float *Wn,
                        float *const *dsts, uint32_t ndst, cudaStream_t s);
void launch_inner(const float *A, const float *B, uint64_t rows, uint32_t R, const double *lambda,
                  double *out, cudaStream_t s);
void launch_sumsq(const float *v, uint64_t n, double *out, cudaStream_t s);
// out[0] = CP-ALS fit, out[1] = ||Xhat||^2 (device), from the grams, lambda and <X, Xhat>
void launch_cpals_fit(const double *const *grams, uint32_t ngrams, uint32_t R, const double *lambda,
                      const double *inner, double normx2, double *out, cudaStream_t s);
void coo_mark_hot(pasta_coo *x, uint32_t mode, uint32_t R, bool global_tier, uint32_t smem_rows,
                  cudaStream_t s, bool die_split = false);
void coo_build_fibers(pasta_coo *x, uint32_t mode, cudaStream_t s);
// TTV on the fiberised matrix (warp-level segmented reduction); y zeroed by the caller
void launch_ttv(const pasta_coo &mat, const float *v, float *y, cudaStream_t s);
void launch_hot_fill(const CooModeCopy &mc, const float *const *factors, uint32_t order, uint32_t mode,
                     uint32_t R, cudaStream_t s);
void launch_hot_fill(const HicooModeCopy &mc, const float *const *factors, uint32_t order, uint32_t mode,
                     uint32_t R, cudaStream_t s);
// hot-block tiers of the HiCOO row-slice copy of `mode` (R#34); no-op when already marked for
// (R, global_tier, smem_rows) or when the copy is not the row-slice layout
void hicoo_mark_hot(pasta_hicoo *h, uint32_t mode, uint32_t R, bool global_tier, uint32_t smem_rows,
                    cudaStream_t s);
// row-granular shared-memory tier of the HiCOO staged decode (WA 16): the `smem_rows` most
// frequent rows of the gathered modes, with per-mode bitmaps of at most max_words words
void hicoo_mark_rows(pasta_hicoo *h, uint32_t mode, uint32_t R, uint32_t smem_rows, uint64_t max_words,
                     cudaStream_t s);
// tier blocks of the HiCOO row-slice copy of `mode` (R#36): rebuilds the copy over heat-ranked
// tier blocks of the gathered modes (on), or back to the plain copy (!on); cached per plan
void hicoo_tier_rows(pasta_hicoo *h, uint32_t mode, uint32_t R, bool on, bool global_tier, uint32_t smem_rows,
                     cudaStream_t s);
void row_counts_device(const uint32_t *rows, uint64_t nnz, uint32_t nrows, uint64_t *counts_host,
                       cudaStream_t s);
// first position x in the sorted array a[0..M) with a[x] >= v (device binary search).
uint64_t lower_bound_device(const uint32_t *a, uint64_t M, uint32_t v, cudaStream_t s);
bool is_lex_sorted_device(const uint32_t *const *inds, uint32_t order, uint64_t M, cudaStream_t s);

// TEW / TS (tew.cu)
void launch_ts(uint32_t op, const float *x, float s, float *y, uint64_t n, cudaStream_t st);
void launch_tew(uint32_t op, const float *a, const float *b, float *z, uint64_t n, cudaStream_t st);
bool same_pattern_device(const pasta_coo *x, const pasta_coo *y, cudaStream_t s);
void launch_bcast(const float *src, uint64_t n, float *const *dsts, uint32_t ndst, cudaStream_t st);
void copy_pattern_device(const pasta_coo *x, pasta_coo *y, cudaStream_t s);
void tew_merge_device(const pasta_coo *x, const pasta_coo *y, uint32_t op, pasta_coo *z, cudaStream_t s);

// ------------------------------------------------------------------------- profiling
enum ProfKind { kProfCoo = 0, kProfHicoo = 1, kProfZero = 2, kProfEw = 3, kProfKinds = 4 };
struct ProfScope {
  cudaEvent_t a = nullptr, b = nullptr;
  int kind;
  cudaStream_t s;
  ProfScope(int kind, cudaStream_t s);
  ~ProfScope();
};

}  // namespace pasta
