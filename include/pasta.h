/*
 * pasta.h -- C ABI of libpasta, a B200-native (sm_100a) sparse MTTKRP library on COO and
 * HiCOO tensors, after Li et al., "A Sparse Tensor Benchmark Suite for CPUs and GPUs"
 * (IISWC'20).  "P:N" cites line N of that paper's text; "R#k" cites reading k
 * of DESIGN.md ("Readings of the paper").
 *
 * Conventions for every entry point
 *   - Returns pasta_status; nothing throws or aborts across the ABI.  On a non-OK status
 *     pasta_last_error() returns a thread-local, human-readable message.
 *   - Arguments are validated before any side effect (EINVAL / ERANGE).  A CUDA launch or
 *     runtime failure maps to PASTA_ECUDA.  Faults of asynchronous kernels surface at the
 *     next synchronising call.
 *   - Tensor handles (pasta_coo, pasta_hicoo) are opaque and library-owned; free them with
 *     pasta_*_free (NULL-safe).  Their arrays live in device memory of the device that was
 *     current at creation.  Handles are immutable after creation except for lazily built,
 *     cached per-mode copies (pasta_*_prepare); calls on one handle must be serialised by
 *     the caller until every mode it uses is prepared, after which they are thread-safe.
 *   - Factor and output matrices are caller-owned DEVICE memory (e.g. torch tensors),
 *     row-major [I_k][R] with leading dimension R (footnote 2; Alg. 3's bi*B*R
 *     rebasing; R#4).  The library never frees them.
 *   - Indices are 0-based uint32 ("32 bits"), values fp32.  Modes are
 *     0-based (R#6).  Maximum order PASTA_MAX_ORDER.
 *   - `stream` is a cudaStream_t (NULL = legacy default stream).  MTTKRP calls are
 *     asynchronous on it; creation / conversion / export calls synchronise.
 */
#ifndef PASTA_H
#define PASTA_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PASTA_MAX_ORDER 8

typedef enum {
    PASTA_OK = 0,
    PASTA_EINVAL = -1,       /* invalid argument (NULL pointer, mode >= order, R == 0, ...) */
    PASTA_EIO = -2,          /* file could not be opened / read / written                  */
    PASTA_EFORMAT = -3,      /* malformed input file                                        */
    PASTA_ERANGE = -4,       /* an index >= its dimension, a size beyond 32-bit limits      */
    PASTA_ENOMEM = -5,       /* host or device allocation failed                             */
    PASTA_ECUDA = -6,        /* CUDA runtime / launch error                                  */
    PASTA_EUNSUPPORTED = -7  /* valid request this build does not implement                  */
} pasta_status;

typedef struct pasta_coo pasta_coo;     /* COO tensor, device-resident          */
typedef struct pasta_hicoo pasta_hicoo; /* HiCOO tensor, device-resident        */

/* Optional device allocator hook (e.g. torch's caching allocator).  alloc returns device
 * memory of `bytes` usable on `stream` or NULL; free releases it.  NULL hook -> cudaMalloc. */
typedef struct {
    void *(*alloc)(size_t bytes, void *stream, void *ctx);
    void (*free)(void *ptr, void *stream, void *ctx);
    void *ctx;
} pasta_allocator;

/* Thread-local text describing the last non-OK status of this thread ("" if none). */
const char *pasta_last_error(void);
/* Library version string, e.g. "pasta-b200 0.1 sm_100a". */
const char *pasta_version(void);
/* Install (or with NULL, remove) the device allocator hook.  Affects later allocations. */
pasta_status pasta_set_allocator(const pasta_allocator *alloc);

/* ---------------------------------------------------------------- ingest (a1) --------- */

/* Load a COO tensor from a FROSTT-style text file (R#17): one nonzero per line,
 * whitespace-separated 1-based indices followed by the value; '#' lines are comments.
 * The order is the token count of the first data line minus one; dims are the per-mode
 * maximum index.  Repeated coordinates are kept as separate nonzeros (MTTKRP is linear in
 * them, R#15).  A file that starts with the 8 bytes "PASTAB01" is read as the binary cache
 * instead (.pbin, written by pasta_save_coo): little-endian u32 order, u32 0, u64 nnz,
 * u32 dims[order], then the 0-based u32 indices of mode 0, 1, ..., order-1 (nnz each) and
 * the nnz f32 values; its dims are the stored ones, and its size must match the header.
 * Errors: EIO (open/read), EFORMAT (ragged line, index 0, bad number; bad .pbin header or
 * size), ERANGE (index > 2^32-1, index >= a stored dim, or > 2^32-2 nonzeros). */
pasta_status pasta_load_coo(const char *path, pasta_coo **out);

/* Write `x` (canonical order): as the binary cache when `path` ends in ".pbin" (format
 * above; bit-exact round trip including dims), else as a 1-based text file readable by
 * pasta_load_coo (values with 9 significant digits: exact fp32 round trip).  EIO on failure. */
pasta_status pasta_save_coo(const pasta_coo *x, const char *path);

/* Create a COO tensor from HOST arrays (copied; the caller keeps ownership).
 * inds: `order` pointers to nnz uint32 each; vals: nnz floats.  Every index must be
 * < dims[k] (ERANGE otherwise).  The input order is kept as the canonical order. */
pasta_status pasta_coo_from_arrays(uint32_t order, const uint32_t *dims, uint64_t nnz,
                                   const uint32_t *const *inds, const float *vals,
                                   pasta_coo **out);

/* Synthetic tensor generator parameters (R#19-R#23). */
typedef struct {
    uint32_t kind;            /* 0 uniform (q = 0.5), 1 Stochastic Kronecker (default),
                                 2 FireHose-style slice power law (R#30)                     */
    const double *initiator;  /* 2^order non-negative cell weights, cell c sets bit k of mode
                                 k's index to (c >> k) & 1; NULL -> product form from q     */
    double q;                 /* product-form P(bit = 0) per mode per level; 0 -> 0.75      */
    uint32_t permute;         /* 1: relabel every mode by pi_k after the draws (R#22), see  */
                              /* below; 0 keeps the generator's fractal locality (default)  */
    float val_lo, val_hi;     /* values uniform in [val_lo, val_hi); both 0 -> [-1, 1)       */
    double alpha;             /* kind 2: power-law exponent in (0, 8]; 0 -> 1.0              */
} pasta_gen_params;

/* Stochastic Kronecker tensor by ball dropping (R#20-R#21): draw d chooses, at each
 * level l < L_k = ceil(log2 I_k), an initiator cell with the counter-based uniform
 * u(d, l) = (mix64(K ^ mix64((l << 40) | d)) >> 11) * 2^-53,  K = mix64(seed ^
 * 0x5851F42D4C957F2D), mix64 = SplitMix64 finaliser; mode k takes the cell's bit k as bit l
 * of i_k; draws with any i_k >= I_k are stripped.  The tensor is the first `nnz` distinct
 * coordinates in draw order, each with value lo + (hi - lo) * u(d_first, 0xFFFF) (fp64,
 * rounded to fp32), stored in lexicographic (i_0, ..., i_{N-1}) order.  Runs on the GPU.
 *
 * kind 2 -- slice power law, the FireHose-style generator of the irregular tensors (P:225,
 * P:229, Table II s4-s6/s10-s15; R#30): "combines graphs together to form
 * slices ... repeated on an (N-1)th-order tensor"; every mode index is drawn independently
 * from P(i) ~ (i+1)^-alpha, i < I_k, so each slice is a power-law graph without clustering
 * (P:229).  Table: w_i = pow(i + 1, -alpha), cum_i = running fp64 sum over ascending i
 * (computed on the host).  Draw d, mode k: u = u(d, k) * cum_{I_k - 1} (fp64 product);
 * i_k = the first i with u < cum_i, else I_k - 1.  No draw is stripped; the tensor is the
 * first `nnz` distinct coordinates in draw order with the values of kind 1, lexicographic.
 * dims <= 2^27 per mode (ERANGE otherwise).
 * permute = 1 (R#22): afterwards mode k's indices are relabelled by the bijection pi_k of
 * [0, I_k): with L = ceil(log2 I_k), m = 2^L - 1, K = mix64(seed ^ 0xA0761D6478BD642F ^ k),
 * f(v) = three rounds r = 0, 1, 2 of { v = v * (((K >> 16r) & 0xFFFF) | 1) & m;
 * v ^= v >> ceil(L/2) (L >= 2); v = (v + ((K >> (32 + 8r)) & 0xFFFFFF)) & m } and
 * pi_k(v) = the first f^j(v), j >= 1, below I_k (cycle walking); the nonzeros are then
 * re-sorted lexicographically (values travel with their coordinates).
 * Errors: EINVAL (order, dims, nnz > prod dims, bad initiator, alpha, permute > 1), ERANGE
 * (more than 2^32-2 draws would be needed). */
pasta_status pasta_gen_powerlaw(uint32_t order, const uint32_t *dims, uint64_t nnz,
                                uint64_t seed, const pasta_gen_params *params,
                                pasta_coo **out);

/* ------------------------------------------------------------- formats (a2, a3) ------ */

/* HiCOO conversion (R#10-R#14): Morton (Z) order of the full
 * coordinates (level-major interleave, MSB level first, mode 0 first within a level; ties
 * by canonical position), blocks of B = 2^block_bits per mode (block_bits 1..8; 7 -> the
 * paper's B = 128), bptr u64, binds u32 = i >> b, einds u8 = i & (B-1).  Bit-exact
 * with the oracle's conversion.  Runs on the GPU. */
pasta_status pasta_coo_to_hicoo(const pasta_coo *x, uint32_t block_bits, pasta_hicoo **out);

/* gHiCOO conversion (Fig. 2(b); R#29): "pick which modes to be
 * compressed in units of blocks for HiCOO and which stay in COO format", for hypersparse
 * tensors whose HiCOO blocks hold one or few nonzeros.  Bit k of `cmask`
 * set <=> mode k is blocked (binds_k u32 per block, einds_k u8 per nonzero); the other modes
 * keep their u32 coordinates per nonzero (uinds_k).  Order: Morton order (R#13) of the
 * compressed modes' coordinates, ties lexicographic over the uncompressed modes in ascending
 * mode order, then canonical position; a block starts where i_k >> b changes for a
 * compressed k.  cmask = all modes is exactly pasta_coo_to_hicoo; cmask = 0 picks the mask
 * with pasta_ghicoo_auto_mask.  Bit-exact with the oracle's conversion.  The result is a
 * pasta_hicoo handle: pasta_mttkrp_hicoo / pasta_hicoo_prepare / pasta_hicoo_info accept it
 * (row-slice layout; an uncompressed target mode makes a slice = the entries of one block
 * that share i_mode).  Errors: EINVAL (NULL, block_bits outside 1..8, cmask bits >= order). */
pasta_status pasta_coo_to_ghicoo(const pasta_coo *x, uint32_t block_bits, uint32_t cmask,
                                 pasta_hicoo **out);
/* Hypersparse-aware mode choice for gHiCOO: the mask minimising the gHiCOO storage
 *   bytes(mask) = (N_c + 4 N_u + 4) M + (8 + 4 N_c) n_b(mask)
 * (Table I's HiCOO storage, generalised; N_c / N_u compressed / uncompressed modes,
 * n_b(mask) = number of distinct (i_k >> b, k in mask) keys, counted on the GPU).  Exhaustive
 * over all non-empty masks for order <= 4 (ties -> smallest mask value), greedy forward
 * selection from the best single mode above.  `bytes` (may be NULL) receives the minimum. */
pasta_status pasta_ghicoo_auto_mask(const pasta_coo *x, uint32_t block_bits, uint32_t *cmask,
                                    uint64_t *bytes);

/* Build (once; cached in the handle) the mode-`mode` working copy: for COO the nonzeros
 * stably sorted lexicographically by (i_mode, i_mode+1, ..., i_mode-1) (a2);
 * for HiCOO (R#27) by default "row slices" (the entries of a block that share einds_mode,
 * slices ordered by output row), or with PASTA_HICOO_LAYOUT=block the blocks stably sorted by
 * binds_mode with entries by einds_mode (dense blocks then run one per CTA with TMA-staged
 * factor tiles).  Optional: MTTKRP prepares on first use. */
pasta_status pasta_coo_prepare(pasta_coo *x, uint32_t mode, void *stream);
/* Free the mode-`mode` working copy of `x` and its caches (hot-row tiers, die split), after
 * the launches that read them; the next use prepares it again.  Lets a caller keep only one
 * sorted copy alive at a time (e.g. while cutting per-mode shards). */
pasta_status pasta_coo_release_mode(pasta_coo *x, uint32_t mode);
pasta_status pasta_hicoo_prepare(pasta_hicoo *h, uint32_t mode, void *stream);

/* --------------------------------------------------------------- MTTKRP (a5-a8) ------ */

/* out = X_(mode) (U^(N-1) (.) ... (.) U^(mode+1) (.) U^(mode-1) (.) ... (.) U^(0))
 * (Eq. 3; Eq. 4) computed directly over the nonzeros:
 *   out(i_mode(x), r) += val(x) * prod_{k != mode} U^(k)(i_k(x), r).
 * factors: `order` DEVICE pointers, U^(k) row-major [dims[k]][R]; factors[mode] is not
 * read and may be NULL.  out: DEVICE [dims[mode]][R] row-major, OVERWRITTEN (zeroed, then
 * accumulated, R#1) on the rows this handle owns: all rows, or [row_lo, row_hi) of a shard
 * made for this mode.  fp32 arithmetic; partial sums combined with fp32 atomics at segment
 * boundaries (R#24).  Asynchronous on `stream`.  Prepares the mode on first use
 * (synchronising once).  R >= 1 (any value; R % 4 == 0 and 16-byte aligned pointers take
 * the 128-bit vector path).  For R in {8, 16, 32, 64} the first call per (mode, R) also
 * ranks the gathered factors' rows by nonzero count (hot-row cache, synchronising once; one
 * cached ranking per mode: alternating R on one handle re-ranks at every change).  The
 * L2-tier buffer is per handle and refilled from `factors` at every launch; the library
 * orders same-handle launches that use it (a launch on another stream waits for the previous
 * one through an event), so concurrent calls are safe but do not overlap.  Thread-safe: the
 * handle's caches are built and the launches enqueued under the handle's lock.  The cache tags
 * use the top two bits of the indices, so it is off for tensors with a dimension >= 2^30 (the
 * kernels then gather every row from the factors). */
pasta_status pasta_mttkrp_coo(pasta_coo *x, uint32_t mode, const float *const *factors,
                              uint32_t R, float *out, void *stream);
/* As pasta_mttkrp_coo over the HiCOO handle's per-mode working copy (Alg. 3; R#27).
 * When every gathered factor exceeds twice the L2 (or PASTA_HICOO_HOT=2), the first call per
 * (mode, R) rebuilds that copy over heat-ranked "tier blocks" of the gathered modes (R#36:
 * hot rows served from the shared-memory / L2-tier buffers, synchronising once); the canonical
 * HiCOO arrays (pasta_hicoo_export) never change.  Same concurrency and thread-safety as
 * pasta_mttkrp_coo. */
pasta_status pasta_mttkrp_hicoo(pasta_hicoo *h, uint32_t mode, const float *const *factors,
                                uint32_t R, float *out, void *stream);
/* Fused MTTKRP + all-gather over peer memory (a9; SURVEY 8(e) "fused variant"): as
 * pasta_mttkrp_coo with out = outs[0], and every flush of a finished row segment is also stored
 * (or atomically added) into outs[1 .. nout) -- the other ranks' replicas of the output,
 * mapped with pasta_ipc_open -- so the rows this handle owns (all, or its shard's
 * [row_lo, row_hi)) reach every replica while the kernel runs, tile by tile, over NVLink /
 * NVSwitch P2P stores instead of a separate collective.  The owned rows are zeroed in every
 * replica first.  nout in 1..8, all 16-byte aligned.  Ordering: the caller makes sure no rank
 * still reads its replicas' rows before the call (a collective before it) and that peers read
 * them only after it (a collective after it on the stream); the kernel ends with a
 * system-scope fence. */
pasta_status pasta_mttkrp_coo_bcast(pasta_coo *x, uint32_t mode, const float *const *factors,
                                    uint32_t R, float *const *outs, uint32_t nout, void *stream);

/* End-to-end variant over ALL modes with HOST buffers (the e2e path): copies the `order`
 * factor matrices host->device (pinned host memory gives full PCIe/C2C bandwidth), computes
 * MTTKRP for every mode into library-owned device buffers, copies the `order` results back
 * to host_out[k] ([dims[k]][R] row-major; for a shard handle only its rows [row_lo, row_hi)
 * of the shard mode are written, the other host rows are left as they were) and synchronises
 * `stream`.  Device staging buffers (2 slots x order x (factor + output)) are cached in the
 * handle until pasta_coo_release_staging or pasta_coo_free. */
pasta_status pasta_mttkrp_coo_allmodes_host(pasta_coo *x, const float *const *host_factors,
                                            uint32_t R, float *const *host_out, void *stream);
/* `nsteps` independent all-modes steps in one call (a stream of factor sets, e.g. serving):
 * step i reads host_factors[i*order + k] and writes host_out[i*order + m] (same shapes as
 * above; the arrays hold nsteps*order pointers).  Two device staging slots: step i+1's
 * uploads overlap step i's downloads, so the per-step cost approaches the larger of the two
 * transfer totals instead of their sum.  Every step's copies still happen.  Returns after the
 * last result is in host memory; nsteps = 0 is a no-op. */
pasta_status pasta_mttkrp_coo_allmodes_host_batch(pasta_coo *x, uint32_t nsteps,
                                                  const float *const *host_factors, uint32_t R,
                                                  float *const *host_out, void *stream);

/* Free the e2e staging buffers of `x` (after the copies in flight have finished); the next
 * host-buffer call allocates them again. */
pasta_status pasta_coo_release_staging(pasta_coo *x);

/* --------------------------------------------------------------- multi-GPU (a9) ------ */

/* counts[r] = number of nonzeros with i_mode == r, r < dims[mode] (HOST uint64 buffer). */
pasta_status pasta_coo_row_counts(const pasta_coo *x, uint32_t mode, uint64_t *counts);
/* Host-only: nnz-balanced contiguous row ranges.  bounds[p] = min{ r : S(r) >= p*T/nparts }
 * with S(r) = sum_{i<r} counts[i], T = S(nrows); bounds[0] = 0, bounds[nparts] = nrows.
 * bounds has nparts + 1 entries.  Needs no GPU. */
pasta_status pasta_row_partition(uint32_t nrows, const uint64_t *counts, uint32_t nparts,
                                 uint32_t *bounds);
/* pasta_coo_row_counts + pasta_row_partition. */
pasta_status pasta_coo_partition(const pasta_coo *x, uint32_t mode, uint32_t nparts,
                                 uint32_t *bounds);
/* New handle holding the nonzeros with row_lo <= i_mode < row_hi (global indices and dims
 * kept; the mode-`mode` copy comes prepared).  MTTKRP of that mode on the shard writes only
 * rows [row_lo, row_hi) of `out`. */
pasta_status pasta_coo_shard(pasta_coo *x, uint32_t mode, uint32_t row_lo, uint32_t row_hi,
                             pasta_coo **out);
/* HiCOO (or gHiCOO) shard: a new handle of the same shape,
 * block size and mask holding the entries with row_lo <= i_mode < row_hi, in the canonical
 * order restricted to them, with blocks re-cut where a compressed mode's block index changes:
 * bit-exact with the conversion of that sub-tensor.  MTTKRP of that mode on the shard writes
 * only rows [row_lo, row_hi) of `out`.  Row bounds: pasta_row_partition / pasta_coo_partition. */
pasta_status pasta_hicoo_shard(const pasta_hicoo *h, uint32_t mode, uint32_t row_lo, uint32_t row_hi,
                               pasta_hicoo **out);

/* ------------------------------------------------------- CP-ALS -------- */
/* CANDECOMP/PARAFAC by alternating least squares around the MTTKRP: the paper's motivation
 * for MTTKRP ("most computationally expensive kernel in CPD"; CPD listed as future work
 * P:380).  The update is the textbook one of the paper's ref. [1] (Kolda & Bader).  All
 * matrices are DEVICE memory; R <= 64 (EUNSUPPORTED otherwise).  Building blocks accumulate
 * (+=) into fp64 outputs so that row-partitioned callers can all-reduce partial results. */

/* G (R x R, fp64, row-major) += U^T U for U row-major [rows][R] fp32. */
pasta_status pasta_gram(const float *U, uint64_t rows, uint32_t R, double *G, void *stream);
/* U = M V^{-1} with V = Hadamard product of the `ngrams` R x R matrices grams[] (HOST array of
 * DEVICE pointers; the grams of every mode but the updated one), inverted in fp64 (partial-
 * pivot Gauss-Jordan, tiny ridge if singular); colsq[r] += sum_i U(i, r)^2 (fp64). */
pasta_status pasta_cpals_solve(const float *M, uint64_t rows, uint32_t R, const double *const *grams,
                               uint32_t ngrams, float *U, double *colsq, void *stream);
/* Fused CP-ALS update algebra (one CTA, fp64): from GM = M^T M (R x R, e.g. pasta_gram of the
 * MTTKRP output, all-reduced across row shards) and the other modes' grams G_k:
 *   W = (Hadamard_k G_k)^{-1};  GU = W^T GM W (= U^T U for U = M W);
 *   lambda_r = sqrt(GU_rr) (1 if GU_rr <= 0);  Wn = W diag(1/lambda) (fp32, row-major R x R);
 *   Gn = GU ./ (lambda lambda^T)  (the gram of the normalised factor).
 * The normalised factor is then U_n = M Wn (pasta_rows_times): the solve, the column
 * normalisation and the gram of the factor without the two extra passes over U_n.  DEVICE
 * pointers; R <= 64 (EUNSUPPORTED otherwise). */
/* CP-ALS fit (P:93 via Kolda-Bader, one CTA, fp64): ||Xhat||^2 = lambda^T (Hadamard of the
 * `ngrams` R x R grams, every mode's) lambda, resid^2 = normx2 + ||Xhat||^2 - 2 inner[0],
 * *fit (HOST) = 1 - sqrt(max(resid^2, 0)) / sqrt(normx2) (0 when normx2 = 0).  grams, lambda
 * (R doubles) and inner (<X, Xhat>, 1 double, e.g. all-reduced pasta_weighted_inner) are
 * DEVICE pointers; synchronises `stream`.  R <= 64. */
pasta_status pasta_cpals_fit(const double *const *grams, uint32_t ngrams, uint32_t R, const double *lambda,
                             const double *inner, double normx2, double *fit, void *stream);
pasta_status pasta_cpals_prepare(const double *GM, const double *const *grams, uint32_t ngrams,
                                 uint32_t R, float *Wn, double *Gn, double *lambda, void *stream);
/* U = M Wn: rows x R (row-major, fp32) times R x R (fp32).  DEVICE pointers; R <= 64. */
pasta_status pasta_rows_times(const float *M, uint64_t rows, uint32_t R, const float *Wn, float *U,
                              void *stream);
/* The factor update fused with its all-gather (a9): rows [row_lo, row_hi) of
 * M Wn (M: DEVICE [rows][R], the rank's MTTKRP output rows at their global positions) are
 * computed once and stored into each of the `ndst` (1..8) full-size replicas dsts[k]
 * ([rows][R], row-major): the local factor and the peers' factors mapped with
 * pasta_ipc_open (P2P stores over NVLink / NVSwitch).  The kernel ends with a system-scope
 * fence; the caller orders the peers' next reads after it (a collective on the stream).
 * R in {4, 8, 16, 32, 64} (EUNSUPPORTED otherwise). */
pasta_status pasta_rows_times_bcast(const float *M, uint64_t row_lo, uint64_t row_hi, uint32_t R,
                                    const float *Wn, float *const *dsts, uint32_t ndst, void *stream);

/* Peer memory (CUDA IPC) for the fused exchange.  pasta_dev_alloc returns an exportable
 * device allocation (cudaMalloc base pointer; free with pasta_dev_free);
 * pasta_ipc_get_handle writes its PASTA_IPC_HANDLE_BYTES-byte handle; another process maps
 * it with pasta_ipc_open (peer access enabled lazily) and unmaps with pasta_ipc_close. */
#define PASTA_IPC_HANDLE_BYTES 64
/* The all-gather of owned rows by peer stores (a9): dsts[k][i] = src[i] for i < n and each of
 * the `ndst` (1..8) destinations (local or pasta_ipc_open-mapped peer buffers, all 16-byte
 * aligned; EINVAL otherwise).  Ends with a system-scope fence; the caller orders the peers'
 * reads after it. */
pasta_status pasta_bcast_f32(const float *src, uint64_t n, float *const *dsts, uint32_t ndst,
                             void *stream);
pasta_status pasta_dev_alloc(uint64_t bytes, void **ptr);
pasta_status pasta_dev_free(void *ptr);
pasta_status pasta_ipc_get_handle(void *base, void *handle);
pasta_status pasta_ipc_open(const void *handle, void **ptr);
pasta_status pasta_ipc_close(void *ptr);
/* lambda[r] = sqrt(colsq[r]) (1 where zero); U(:, r) /= lambda[r].  lambda: DEVICE fp64 [R]. */
pasta_status pasta_normalize_columns(float *U, uint64_t rows, uint32_t R, const double *colsq,
                                     double *lambda, void *stream);
/* out += sum_{i, r} lambda[r] A(i, r) B(i, r)   (out: DEVICE fp64 scalar). */
pasta_status pasta_weighted_inner(const float *A, const float *B, uint64_t rows, uint32_t R,
                                  const double *lambda, double *out, void *stream);
/* ||X||_F^2 = sum of squared values (HOST result). */
pasta_status pasta_coo_norm2(const pasta_coo *x, double *out);
/* Single-GPU CP-ALS: factors[k] (DEVICE [dims[k]][R], the initial guess on entry, the result
 * on exit, columns normalised), lambda (HOST fp64 [R], out), fit_history (HOST fp64
 * [max_iters], out: fit = 1 - ||X - [[lambda; U]]|| / ||X|| after each sweep over the modes),
 * iters (out).  Stops when |fit - previous fit| < tol. */
pasta_status pasta_cpals_coo(pasta_coo *x, uint32_t R, uint32_t max_iters, double tol,
                             float *const *factors, double *lambda, double *fit_history,
                             uint32_t *iters, void *stream);

/* ------------------------------------------------- TTV / TTM --------- */
/* Tensor-times-vector (Eq. 1) and tensor-times-matrix (Eq. 2) in mode `mode`.
 * The result is semi-sparse (sCOO): one dense vector of length R per mode-n fiber of X
 * (sparse-dense property), fibers in lexicographic order of their coordinates over the
 * modes k != mode.  The fibers are pre-processed once per mode and cached. */

/* Build (cached) the mode-`mode` fibers; *nfibers = M_F. */
pasta_status pasta_coo_fibers(pasta_coo *x, uint32_t mode, uint64_t *nfibers, void *stream);
/* Copy the fiber coordinates to HOST buffers: inds[k] (k != mode) gets M_F uint32; inds[mode]
 * is not touched (may be NULL). */
pasta_status pasta_coo_fiber_export(pasta_coo *x, uint32_t mode, uint32_t *const *inds);
/* out (DEVICE [M_F][R], OVERWRITTEN) = X x_mode U with U DEVICE row-major [dims[mode]][R]. */
pasta_status pasta_ttm_coo(pasta_coo *x, uint32_t mode, const float *U, uint32_t R, float *out,
                           void *stream);
/* out (DEVICE [M_F]) = X x_mode v with v DEVICE [dims[mode]] (TTM with R = 1). */
pasta_status pasta_ttv_coo(pasta_coo *x, uint32_t mode, const float *v, float *out, void *stream);

/* ------------------------------------------------------- TEW / TS ---- */

/* Element-wise operators: z = x op y. */
enum { PASTA_OP_ADD = 0, PASTA_OP_SUB = 1, PASTA_OP_MUL = 2, PASTA_OP_DIV = 3 };

/* Tensor-scalar (TS) on a value array: out[i] = vals[i] op s, i < n, IEEE fp32
 * (correctly rounded, division included).  DEVICE arrays (out may equal vals).  Async on
 * `stream`.  Table I: M flops, 8M bytes. */
pasta_status pasta_ts(const float *vals, uint64_t n, uint32_t op, float s, float *out, void *stream);
/* Tensor element-wise (TEW) of two tensors with the same non-zero pattern, on their
 * value arrays: out[i] = a[i] op b[i].  DEVICE arrays.  Table I: M flops, 12M bytes. */
pasta_status pasta_tew(const float *a, const float *b, uint64_t n, uint32_t op, float *out,
                       void *stream);
/* Device pointer to the canonical value array of `x` (library-owned, valid until free). */
pasta_status pasta_coo_values(const pasta_coo *x, float **vals);
/* Y = X op s (TS) as a new tensor: the output indices are copied in pre-processing (the
 * output pattern is the input's), then the values come from pasta_ts. */
pasta_status pasta_coo_ts(const pasta_coo *x, uint32_t op, float s, pasta_coo **out);
/* Z = X op Y (TEW) for tensors of the same order and shape.  Same pattern (same
 * canonical index arrays, checked on the GPU): Z has X's pattern and z_i = x_i op y_i.
 * Different patterns (R#31): the output pattern is predicted from a merge of both mode-0
 * lexicographic index lists -- the union for add/sub (a missing operand contributes
 * nothing: z = x, or z = 0 - y), the intersection for mul/div -- and Z is stored in
 * lexicographic order.  Errors: EINVAL (order/shape mismatch, a repeated coordinate inside
 * one input in the merge case), ERANGE (more than 2^32-2 merged entries). */
pasta_status pasta_coo_tew(pasta_coo *x, pasta_coo *y, uint32_t op, pasta_coo **out);

/* ------------------------------------------------------------ introspection ---------- */

pasta_status pasta_coo_info(const pasta_coo *x, uint32_t *order, uint32_t *dims,
                            uint64_t *nnz);
/* Copy the canonical arrays to HOST buffers (inds: `order` pointers to nnz uint32). */
pasta_status pasta_coo_export(const pasta_coo *x, uint32_t *const *inds, float *vals);
/* Copy the mode-`mode` sorted copy to HOST buffers (prepares it if needed). */
pasta_status pasta_coo_export_mode(pasta_coo *x, uint32_t mode, uint32_t *const *inds,
                                   float *vals);
pasta_status pasta_hicoo_info(const pasta_hicoo *h, uint32_t *order, uint32_t *dims,
                              uint32_t *block_bits, uint64_t *nblocks, uint64_t *nnz);
/* Copy the canonical (Morton-ordered) HiCOO arrays to HOST buffers: bptr[nblocks+1],
 * binds: `order` pointers to nblocks uint32, einds: `order` pointers to nnz uint8, vals. */
pasta_status pasta_hicoo_export(const pasta_hicoo *h, uint64_t *bptr, uint32_t *const *binds,
                                uint8_t *const *einds, float *vals);
/* gHiCOO: the compression mask of a handle (all bits for a HiCOO handle). */
pasta_status pasta_ghicoo_info(const pasta_hicoo *h, uint32_t *cmask);
/* Copy the canonical gHiCOO arrays to HOST buffers: bptr[nblocks+1]; for compressed modes
 * binds[k] (nblocks u32) and einds[k] (nnz u8); for uncompressed modes uinds[k] (nnz u32).
 * NULL array pointers (or NULL entries) are skipped.  pasta_hicoo_export rejects (EINVAL) a
 * handle that is not fully compressed. */
pasta_status pasta_ghicoo_export(const pasta_hicoo *h, uint64_t *bptr, uint32_t *const *binds,
                                 uint8_t *const *einds, uint32_t *const *uinds, float *vals);
void pasta_coo_free(pasta_coo *x);
void pasta_hicoo_free(pasta_hicoo *h);

/* -------------------------------------------------------------- measurement ---------- */

/* Number of kernels this library has launched in this process (all kinds). */
uint64_t pasta_launch_count(void);
/* The current device's SM -> die map used by the die-split COO MTTKRP (R#35; measured once
 * per device and process, see csrc/die.cu): *nsms = number of SMs (0 when no plausible two-die
 * map was found or PASTA_DIE_SPLIT=0), die_of_sm[s] (HOST buffer of >= *nsms entries, may be
 * NULL) = 0 or 1 for SM id s, n_die[2] (may be NULL) = SMs per die.  Launches a calibration
 * kernel on first use (synchronises the device). */
pasta_status pasta_die_map(uint32_t *nsms, int8_t *die_of_sm, uint32_t *n_die);
/* When enabled, every MTTKRP main-kernel launch is bracketed by CUDA events recorded on
 * its own stream.  pasta_profile_read synchronises those events and returns the summed
 * device time (ms) and the launch count of kernel family `which` (0 = COO MTTKRP,
 * 1 = HiCOO MTTKRP, 2 = output zero-fill, 3 = TEW/TS), then clears the record if `reset`. */
pasta_status pasta_profile_enable(int on);
pasta_status pasta_profile_read(uint32_t which, double *total_ms, uint64_t *launches,
                                int reset);

#ifdef __cplusplus
}
#endif
#endif /* PASTA_H */
