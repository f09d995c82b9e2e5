/*
 * oracle.c -- plain, slow, single-threaded fp64 CPU oracle for the PASTA MTTKRP hot path.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or call this library.  The product
 * path (libpasta.so, paper_conf_iiswc_lilwlob20_b200/) never does, and it shares no
 * source, header, table or helper with this file.
 *
 * Citations: "P:N" = line N of the paper text (/root/reference/PAPER.md,
 * Li et al., "A Sparse Tensor Benchmark Suite for CPUs and GPUs", IISWC'20).
 * "R#k" = reading k in DESIGN.md section "Readings of the paper".
 *
 * Every routine below follows the definition or algorithm it cites in the order the
 * paper states it; the only library primitive used is qsort.  Compile with
 * -ffp-contract=off so that no multiply-add is fused (the generator's fp64 cell
 * decision must be reproducible bit for bit, R#20).
 *
 * Pins (tests/test_oracle_*.py): brute force X_(n)(KRP) on dense tiny tensors,
 * rank-1 closed form, all-ones slice sums, N=2 SpMM (scipy), R=1 chained TTV,
 * linearity/order/mode-permutation invariants, an independent Python Morton
 * conversion, HiCOO storage formula, binomial popcount marginal of the
 * generator.  No routine here is "parity unpinned".
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define ORACLE_MAX_ORDER 8

/* ------------------------------------------------------------------------- */
/* O-MTTKRP: Eq. 3 with the Khatri-Rao product of Eq. 4 folded  */
/* into the nonzero loop, as the paper describes (Alg. 3). */
/*   Mref(i_n(x), r) += val(x) * prod_{k != n} U^(k)(i_k(x), r)               */
/*   Aref(i_n(x), r) += |val(x) * prod_{k != n} U^(k)(i_k(x), r)|             */
/* Factors are row-major [I_k][R] (footnote 2; R#4).                   */
/* Returns 0, or -1 on invalid arguments.                                     */
/* ------------------------------------------------------------------------- */
int oracle_mttkrp(uint32_t order, const uint32_t *dims, uint64_t nnz,
                  const uint32_t *const *inds, const float *vals, uint32_t mode,
                  const float *const *factors, uint32_t R, double *Mref, double *Aref)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || mode >= order || R < 1) return -1;
    uint64_t rows = dims[mode];
    for (uint64_t e = 0; e < rows * R; ++e) { Mref[e] = 0.0; Aref[e] = 0.0; }
    for (uint64_t x = 0; x < nnz; ++x) {
        uint64_t i = inds[mode][x];
        for (uint32_t r = 0; r < R; ++r) {
            double t = (double)vals[x];
            for (uint32_t k = 0; k < order; ++k) {
                if (k == mode) continue;
                t *= (double)factors[k][(uint64_t)inds[k][x] * R + r];
            }
            Mref[i * R + r] += t;
            Aref[i * R + r] += fabs(t);
        }
    }
    return 0;
}

/* Same definition restricted to a set of output rows (for full-size sampled
 * parity).  rows[] must be strictly increasing; Mref/Aref are [nsel][R]. */
int oracle_mttkrp_rows(uint32_t order, const uint32_t *dims, uint64_t nnz,
                       const uint32_t *const *inds, const float *vals, uint32_t mode,
                       const float *const *factors, uint32_t R, uint32_t nsel,
                       const uint32_t *rows, double *Mref, double *Aref)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || mode >= order || R < 1) return -1;
    (void)dims;
    for (uint64_t e = 0; e < (uint64_t)nsel * R; ++e) { Mref[e] = 0.0; Aref[e] = 0.0; }
    for (uint64_t x = 0; x < nnz; ++x) {
        uint32_t i = inds[mode][x];
        /* binary search i in rows[0..nsel) */
        uint32_t lo = 0, hi = nsel;
        while (lo < hi) {
            uint32_t mid = lo + (hi - lo) / 2;
            if (rows[mid] < i) lo = mid + 1; else hi = mid;
        }
        if (lo == nsel || rows[lo] != i) continue;
        for (uint32_t r = 0; r < R; ++r) {
            double t = (double)vals[x];
            for (uint32_t k = 0; k < order; ++k) {
                if (k == mode) continue;
                t *= (double)factors[k][(uint64_t)inds[k][x] * R + r];
            }
            Mref[(uint64_t)lo * R + r] += t;
            Aref[(uint64_t)lo * R + r] += fabs(t);
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O-HiCOO-MTTKRP (Alg. 3): for block b, the pointers are rebased   */
/* by binds(b)*B*R, i.e. i_k = binds_k(b)*B + einds_k(x) (R#5: A_b means the  */
/* output).  Then the same accumulation as O-MTTKRP.                          */
/* ------------------------------------------------------------------------- */
int oracle_mttkrp_hicoo(uint32_t order, const uint32_t *dims, uint32_t block_bits,
                        uint64_t nblocks, const uint64_t *bptr,
                        const uint32_t *const *binds, const uint8_t *const *einds,
                        const float *vals, uint32_t mode, const float *const *factors,
                        uint32_t R, double *Mref, double *Aref)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || mode >= order || R < 1) return -1;
    uint64_t B = 1ull << block_bits;
    uint64_t rows = dims[mode];
    for (uint64_t e = 0; e < rows * R; ++e) { Mref[e] = 0.0; Aref[e] = 0.0; }
    for (uint64_t b = 0; b < nblocks; ++b) {
        for (uint64_t x = bptr[b]; x < bptr[b + 1]; ++x) {
            uint64_t i = (uint64_t)binds[mode][b] * B + einds[mode][x];
            for (uint32_t r = 0; r < R; ++r) {
                double t = (double)vals[x];
                for (uint32_t k = 0; k < order; ++k) {
                    if (k == mode) continue;
                    uint64_t ik = (uint64_t)binds[k][b] * B + einds[k][x];
                    t *= (double)factors[k][ik * R + r];
                }
                Mref[i * R + r] += t;
                Aref[i * R + r] += fabs(t);
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* Sorting helpers (qsort over an index permutation; ties broken by original  */
/* position so that the result is a stable sort, R#15).                       */
/* ------------------------------------------------------------------------- */
static uint32_t g_order;
static const uint32_t *const *g_inds;
static uint32_t g_first_mode;

/* O-mode-sort comparator: lexicographic on (i_n, i_{n+1 mod N}, ..., i_{n-1}),
 * which makes equal output rows contiguous (a2; "pre-processing to trade
 * for less kernel computation time", "naturally sorted in a mode order"). */
static int cmp_mode_lex(const void *pa, const void *pb)
{
    uint64_t a = *(const uint64_t *)pa, b = *(const uint64_t *)pb;
    for (uint32_t j = 0; j < g_order; ++j) {
        uint32_t k = (g_first_mode + j) % g_order;
        uint32_t va = g_inds[k][a], vb = g_inds[k][b];
        if (va != vb) return va < vb ? -1 : 1;
    }
    return a < b ? -1 : (a > b ? 1 : 0);
}

/* Morton (Z) order comparator for HiCOO ("Morton order sorting implied by
 * the HiCOO format"; R#13): the first differing bit of the level-major
 * interleave (MSB level first, mode 0 first within a level) decides.  That bit
 * lives in mode k* = argmax_k msb(a_k XOR b_k), ties to the smallest k. */
static int msb_less(uint32_t x, uint32_t y) { return x < y && x < (x ^ y); }
static int cmp_morton(const void *pa, const void *pb)
{
    uint64_t a = *(const uint64_t *)pa, b = *(const uint64_t *)pb;
    int best = -1;
    uint32_t best_x = 0;
    for (uint32_t k = 0; k < g_order; ++k) {
        uint32_t x = g_inds[k][a] ^ g_inds[k][b];
        if (msb_less(best_x, x)) { best = (int)k; best_x = x; }
    }
    if (best >= 0) {
        uint32_t va = g_inds[best][a], vb = g_inds[best][b];
        return va < vb ? -1 : 1;
    }
    return a < b ? -1 : (a > b ? 1 : 0);
}

/* Mode-n sort of a COO tensor.  Writes the permuted copy into out_inds/out_vals. */
int oracle_mode_sort(uint32_t order, uint64_t nnz, const uint32_t *const *inds,
                     const float *vals, uint32_t mode, uint32_t *const *out_inds,
                     float *out_vals)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || mode >= order) return -1;
    uint64_t *perm = (uint64_t *)malloc((nnz ? nnz : 1) * sizeof(uint64_t));
    if (!perm) return -2;
    for (uint64_t x = 0; x < nnz; ++x) perm[x] = x;
    g_order = order; g_inds = inds; g_first_mode = mode;
    qsort(perm, nnz, sizeof(uint64_t), cmp_mode_lex);
    for (uint64_t x = 0; x < nnz; ++x) {
        for (uint32_t k = 0; k < order; ++k) out_inds[k][x] = inds[k][perm[x]];
        out_vals[x] = vals[perm[x]];
    }
    free(perm);
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O-HiCOO conversion (R#10, R#12-R#14):             */
/*  1. sort nonzeros into Morton order of their full coordinates;             */
/*  2. scan: a new block starts where (i_k >> b) differs for any k;           */
/*  3. emit bptr (u64, bptr[n_b] = M), binds_k(blk) = i_k >> b (u32),          */
/*     einds_k(x) = i_k & (B-1) (u8), val (bitwise copy).                     */
/* Output arrays are caller-allocated with capacity M (bptr: M+1).            */
/* Returns n_b (>= 0) or -1 on invalid arguments.                             */
/* ------------------------------------------------------------------------- */
int64_t oracle_coo_to_hicoo(uint32_t order, uint64_t nnz, const uint32_t *const *inds,
                            const float *vals, uint32_t block_bits, uint64_t *bptr,
                            uint32_t *const *binds, uint8_t *const *einds, float *out_vals)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || block_bits < 1 || block_bits > 8) return -1;
    uint64_t *perm = (uint64_t *)malloc((nnz ? nnz : 1) * sizeof(uint64_t));
    if (!perm) return -2;
    for (uint64_t x = 0; x < nnz; ++x) perm[x] = x;
    g_order = order; g_inds = inds;
    qsort(perm, nnz, sizeof(uint64_t), cmp_morton);
    uint32_t emask = (1u << block_bits) - 1u;
    int64_t nb = 0;
    for (uint64_t x = 0; x < nnz; ++x) {
        uint64_t p = perm[x];
        int new_block = (x == 0);
        if (!new_block) {
            uint64_t q = perm[x - 1];
            for (uint32_t k = 0; k < order; ++k)
                if ((inds[k][p] >> block_bits) != (inds[k][q] >> block_bits)) new_block = 1;
        }
        if (new_block) {
            bptr[nb] = x;
            for (uint32_t k = 0; k < order; ++k) binds[k][nb] = inds[k][p] >> block_bits;
            ++nb;
        }
        for (uint32_t k = 0; k < order; ++k) einds[k][x] = (uint8_t)(inds[k][p] & emask);
        out_vals[x] = vals[p];
    }
    bptr[nb] = nnz;
    free(perm);
    return nb;
}

/* ------------------------------------------------------------------------- */
/* Stochastic Kronecker ("ball-dropping") tensor generator, P:223-227 (R#19-  */
/* R#23).  Counter-based randomness so the product generator can implement    */
/* the very same draw sequence independently:                                 */
/*   mix64 = SplitMix64 finaliser;  K = mix64(seed ^ 0x5851F42D4C957F2D);     */
/*   h(d, s) = mix64(K ^ mix64((s << 40) | d));  u = (h >> 11) * 2^-53.       */
/* Draw d, level l (s = l): choose initiator cell c = first c with            */
/*   u * cum[last] < cum[c]   (cum = running fp64 sum of the 2^N table);      */
/* mode k takes bit ((c >> k) & 1) at bit position l while l < L_k =          */
/* ceil(log2 I_k).  A draw with any i_k >= I_k is stripped.           */
/* Value of draw d: (float)(lo + (hi - lo) * u(d, 0xFFFF)).                   */
/* Result: the first M distinct coordinates in draw order (each keeps the     */
/* value of its first draw), emitted in lexicographic (i_0, ..., i_{N-1})     */
/* order.  Returns 0, -1 invalid, -2 no memory, -3 could not reach M.         */
/* ------------------------------------------------------------------------- */
static uint64_t mix64(uint64_t z)
{
    z ^= z >> 30; z *= 0xbf58476d1ce4e5b9ull;
    z ^= z >> 27; z *= 0x94d049bb133111ebull;
    z ^= z >> 31;
    return z;
}
static double gen_uniform(uint64_t key, uint64_t d, uint64_t s)
{
    uint64_t h = mix64(key ^ mix64((s << 40) | d));
    return (double)(h >> 11) * (1.0 / 9007199254740992.0);
}

typedef struct { uint32_t c[ORACLE_MAX_ORDER]; uint64_t d; } draw_rec;
static uint32_t g_gen_order;
static int cmp_draw_coords_then_d(const void *pa, const void *pb)
{
    const draw_rec *a = (const draw_rec *)pa, *b = (const draw_rec *)pb;
    for (uint32_t k = 0; k < g_gen_order; ++k)
        if (a->c[k] != b->c[k]) return a->c[k] < b->c[k] ? -1 : 1;
    return a->d < b->d ? -1 : (a->d > b->d ? 1 : 0);
}
static int cmp_draw_d(const void *pa, const void *pb)
{
    const draw_rec *a = (const draw_rec *)pa, *b = (const draw_rec *)pb;
    return a->d < b->d ? -1 : (a->d > b->d ? 1 : 0);
}

/* Common tail of both generators: D draws produced by draw(), invalid ones    */
/* stripped, the first nnz distinct coordinates in draw order kept, emitted in */
/* lexicographic order with value lo + (hi - lo) * u(d_first, 0xFFFF).        */
typedef int (*draw_fn)(const void *ctx, uint64_t d, uint32_t *c);
static int gen_common(uint32_t order, uint64_t nnz, uint64_t key, draw_fn draw, const void *ctx,
                      float val_lo, float val_hi, uint32_t *const *out_inds, float *out_vals)
{
    uint64_t D = nnz + nnz / 16 + 4096;
    uint64_t cap = 64 * nnz + (1ull << 22);
    for (;;) {
        draw_rec *rec = (draw_rec *)malloc(D * sizeof(draw_rec));
        if (!rec) return -2;
        uint64_t nvalid = 0;
        for (uint64_t d = 0; d < D; ++d) {
            draw_rec r;
            memset(&r, 0, sizeof(r));
            r.d = d;
            if (draw(ctx, d, r.c)) rec[nvalid++] = r;
        }
        g_gen_order = order;
        qsort(rec, nvalid, sizeof(draw_rec), cmp_draw_coords_then_d);
        uint64_t nuniq = 0;
        for (uint64_t x = 0; x < nvalid; ++x) {
            int dup = 0;
            if (nuniq > 0) {
                dup = 1;
                for (uint32_t k = 0; k < order; ++k)
                    if (rec[x].c[k] != rec[nuniq - 1].c[k]) dup = 0;
            }
            if (!dup) rec[nuniq++] = rec[x];
        }
        if (nuniq >= nnz) {
            qsort(rec, nuniq, sizeof(draw_rec), cmp_draw_d);           /* first-drawn order */
            qsort(rec, nnz, sizeof(draw_rec), cmp_draw_coords_then_d); /* keep M, lex order */
            double lo = (double)val_lo, diff = (double)val_hi - (double)val_lo;
            for (uint64_t x = 0; x < nnz; ++x) {
                for (uint32_t k = 0; k < order; ++k) out_inds[k][x] = rec[x].c[k];
                double u = gen_uniform(key, rec[x].d, 0xFFFF);
                double v = lo + diff * u;
                out_vals[x] = (float)v;
            }
            free(rec);
            return 0;
        }
        free(rec);
        if (D >= cap) return -3;
        D = D + D / 2 + 2 * (nnz - nuniq) + 4096; /* geometric growth */
        if (D > cap) D = cap;
    }
}

typedef struct {
    uint32_t order, ncell, last_pos, Lmax;
    uint32_t L[ORACLE_MAX_ORDER];
    const uint32_t *dims;
    const double *cum;
    double run;
    uint64_t key;
} kron_ctx;

static int kron_draw(const void *vctx, uint64_t d, uint32_t *c)
{
    const kron_ctx *x = (const kron_ctx *)vctx;
    for (uint32_t l = 0; l < x->Lmax; ++l) {
        double u = gen_uniform(x->key, d, l) * x->run;
        uint32_t cell = x->last_pos;
        for (uint32_t j = 0; j < x->ncell; ++j)
            if (u < x->cum[j]) { cell = j; break; }
        for (uint32_t k = 0; k < x->order; ++k)
            if (l < x->L[k]) c[k] |= ((cell >> k) & 1u) << l;
    }
    for (uint32_t k = 0; k < x->order; ++k) if (c[k] >= x->dims[k]) return 0;
    return 1;
}

int oracle_gen_powerlaw(uint32_t order, const uint32_t *dims, uint64_t nnz, uint64_t seed,
                        const double *initiator, double q, float val_lo, float val_hi,
                        uint32_t *const *out_inds, float *out_vals)
{
    if (order < 1 || order > ORACLE_MAX_ORDER) return -1;
    uint32_t ncell = 1u << order;
    double table[1u << ORACLE_MAX_ORDER], cum[1u << ORACLE_MAX_ORDER];
    if (initiator) {
        for (uint32_t c = 0; c < ncell; ++c) table[c] = initiator[c];
    } else {
        if (!(q > 0.0 && q < 1.0)) q = 0.75;
        for (uint32_t c = 0; c < ncell; ++c) {
            double p = 1.0;
            for (uint32_t k = 0; k < order; ++k) p = p * (((c >> k) & 1u) ? (1.0 - q) : q);
            table[c] = p;
        }
    }
    double run = 0.0;
    uint32_t last_pos = 0;
    for (uint32_t c = 0; c < ncell; ++c) {
        if (table[c] < 0.0) return -1;
        run = run + table[c];
        cum[c] = run;
        if (table[c] > 0.0) last_pos = c;
    }
    if (!(run > 0.0)) return -1;
    kron_ctx ctx;
    memset(&ctx, 0, sizeof(ctx));
    double cells = 1.0;
    for (uint32_t k = 0; k < order; ++k) {
        if (dims[k] < 1) return -1;
        uint32_t l = 0;
        while (l < 32 && ((uint64_t)1 << l) < dims[k]) ++l;
        ctx.L[k] = l;
        if (l > ctx.Lmax) ctx.Lmax = l;
        cells *= (double)dims[k];
    }
    if ((double)nnz > cells) return -1;
    ctx.order = order; ctx.ncell = ncell; ctx.last_pos = last_pos;
    ctx.dims = dims; ctx.cum = cum; ctx.run = run;
    ctx.key = mix64(seed ^ 0x5851F42D4C957F2Dull);
    return gen_common(order, nnz, ctx.key, kron_draw, &ctx, val_lo, val_hi, out_inds, out_vals);
}

/* ------------------------------------------------------------------------- */
/* Slice power-law generator (FireHose-style;    */
/* R#30).  "combines graphs together to form slices of a hypergraph ... when  */
/* repeated on an (N-1)th-order tensor, will generate a sparse tensor with N  */
/* modes": every mode index is drawn independently from the discrete power   */
/* law P(i) ~ (i+1)^(-alpha), i < I_k, so each slice is a power-law graph     */
/* (no clustering) and slices are combined the same way.               */
/* Table: w_i = pow(i+1, -alpha), cum_i = running fp64 sum (i ascending).     */
/* Draw d, mode k: u = u(d, k) * cum_{I_k-1}; i_k = the first i with         */
/* u < cum_i (binary search), else I_k - 1.  Then gen_common.                 */
/* ------------------------------------------------------------------------- */
typedef struct {
    uint32_t order;
    const uint32_t *dims;
    double *cum[ORACLE_MAX_ORDER];
    uint64_t key;
} slice_ctx;

static int slice_draw(const void *vctx, uint64_t d, uint32_t *c)
{
    const slice_ctx *x = (const slice_ctx *)vctx;
    for (uint32_t k = 0; k < x->order; ++k) {
        const double *cum = x->cum[k];
        uint32_t I = x->dims[k];
        double u = gen_uniform(x->key, d, k) * cum[I - 1];
        uint32_t lo = 0, hi = I; /* first i in [lo, hi) with u < cum[i]; hi = none */
        while (lo < hi) {
            uint32_t mid = lo + (hi - lo) / 2;
            if (u < cum[mid]) hi = mid; else lo = mid + 1;
        }
        c[k] = lo < I ? lo : I - 1;
    }
    return 1;
}

int oracle_gen_slice_powerlaw(uint32_t order, const uint32_t *dims, uint64_t nnz, uint64_t seed,
                              double alpha, float val_lo, float val_hi,
                              uint32_t *const *out_inds, float *out_vals)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || !(alpha >= 0.0 && alpha <= 8.0)) return -1;
    slice_ctx ctx;
    memset(&ctx, 0, sizeof(ctx));
    double cells = 1.0;
    for (uint32_t k = 0; k < order; ++k) {
        if (dims[k] < 1) return -1;
        cells *= (double)dims[k];
    }
    if ((double)nnz > cells) return -1;
    int rc = 0;
    for (uint32_t k = 0; k < order && rc == 0; ++k) {
        ctx.cum[k] = (double *)malloc((size_t)dims[k] * sizeof(double));
        if (!ctx.cum[k]) { rc = -2; break; }
        double run = 0.0;
        for (uint32_t i = 0; i < dims[k]; ++i) {
            run = run + pow((double)i + 1.0, -alpha);
            ctx.cum[k][i] = run;
        }
    }
    if (rc == 0) {
        ctx.order = order; ctx.dims = dims;
        ctx.key = mix64(seed ^ 0x5851F42D4C957F2Dull);
        rc = gen_common(order, nnz, ctx.key, slice_draw, &ctx, val_lo, val_hi, out_inds, out_vals);
    }
    for (uint32_t k = 0; k < order; ++k) free(ctx.cum[k]);
    return rc;
}

/* ------------------------------------------------------------------------- */
/* O-TTM / O-TTV: Eq. 2 and Eq. 1 over nonzeros: */
/*   y(i_1..i_{n-1}, r, i_{n+1}..i_N) = sum_{i_n} x(..., i_n, ...) u(i_n, r)  */
/* The output is semi-sparse (sCOO): one dense length-R vector per      */
/* mode-n fiber of X (the sparse-dense property).  Fibers are emitted   */
/* in lexicographic order of their coordinates (modes k != n, ascending k);   */
/* TTV is the R = 1 case with u = v.  fiber_inds: order arrays (capacity nnz, */
/* the mode-n array is left untouched); y, yabs: capacity nnz * R (fp64).      */
/* Returns the number of fibers, or -1 on invalid arguments.                  */
/* ------------------------------------------------------------------------- */
static uint32_t g_fib_mode;
static int cmp_fiber_then_n(const void *pa, const void *pb)
{
    uint64_t a = *(const uint64_t *)pa, b = *(const uint64_t *)pb;
    for (uint32_t k = 0; k < g_order; ++k) {
        if (k == g_fib_mode) continue;
        uint32_t va = g_inds[k][a], vb = g_inds[k][b];
        if (va != vb) return va < vb ? -1 : 1;
    }
    uint32_t va = g_inds[g_fib_mode][a], vb = g_inds[g_fib_mode][b];
    if (va != vb) return va < vb ? -1 : 1;
    return a < b ? -1 : (a > b ? 1 : 0);
}

int64_t oracle_ttm(uint32_t order, const uint32_t *dims, uint64_t nnz, const uint32_t *const *inds,
                   const float *vals, uint32_t mode, const float *U, uint32_t R,
                   uint32_t *const *fiber_inds, double *y, double *yabs)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || mode >= order || R < 1) return -1;
    (void)dims;
    uint64_t *perm = (uint64_t *)malloc((nnz ? nnz : 1) * sizeof(uint64_t));
    if (!perm) return -2;
    for (uint64_t x = 0; x < nnz; ++x) perm[x] = x;
    g_order = order; g_inds = inds; g_fib_mode = mode;
    qsort(perm, nnz, sizeof(uint64_t), cmp_fiber_then_n);
    int64_t nf = 0;
    for (uint64_t q = 0; q < nnz; ++q) {
        uint64_t x = perm[q];
        int new_fiber = (q == 0);
        if (!new_fiber) {
            uint64_t p = perm[q - 1];
            for (uint32_t k = 0; k < order; ++k)
                if (k != mode && inds[k][x] != inds[k][p]) new_fiber = 1;
        }
        if (new_fiber) {
            for (uint32_t k = 0; k < order; ++k)
                if (k != mode) fiber_inds[k][nf] = inds[k][x];
            for (uint32_t r = 0; r < R; ++r) { y[nf * R + r] = 0.0; yabs[nf * R + r] = 0.0; }
            ++nf;
        }
        for (uint32_t r = 0; r < R; ++r) {
            double t = (double)vals[x] * (double)U[(uint64_t)inds[mode][x] * R + r];
            y[(nf - 1) * R + r] += t;
            yabs[(nf - 1) * R + r] += fabs(t);
        }
    }
    free(perm);
    return nf;
}

/* ------------------------------------------------------------------------- */
/* O-gHiCOO conversion (Fig. 2(b); R#29):           */
/* "pick which modes to be compressed in units of blocks for HiCOO and which  */
/* stay in COO format".  cmask bit k set <=> mode k is compressed (blocked).  */
/*  1. sort nonzeros by the Morton order of the COMPRESSED modes' coordinates */
/*     (same level-major convention as HiCOO, R#13, restricted to those       */
/*     modes), ties by the uncompressed coordinates in ascending mode order   */
/*     (lexicographic), then by input position (stable);                      */
/*  2. scan: a new block starts where (i_k >> b) differs for a compressed k;  */
/*  3. emit bptr (u64), binds_k (u32) and einds_k (u8) for compressed k, the  */
/*     full coordinate inds_k (u32, as in COO) for uncompressed k, and val.   */
/* cmask = all modes is HiCOO; cmask = {0} is the mode-0 lexicographic order. */
/* Arrays of the other kind are left untouched.  Returns n_b or -1.           */
/* ------------------------------------------------------------------------- */
static uint32_t g_cmask;
static int cmp_ghicoo(const void *pa, const void *pb)
{
    uint64_t a = *(const uint64_t *)pa, b = *(const uint64_t *)pb;
    int best = -1;
    uint32_t best_x = 0;
    for (uint32_t k = 0; k < g_order; ++k) {
        if (!((g_cmask >> k) & 1u)) continue;
        uint32_t x = g_inds[k][a] ^ g_inds[k][b];
        if (msb_less(best_x, x)) { best = (int)k; best_x = x; }
    }
    if (best >= 0) {
        uint32_t va = g_inds[best][a], vb = g_inds[best][b];
        return va < vb ? -1 : 1;
    }
    for (uint32_t k = 0; k < g_order; ++k) {
        if ((g_cmask >> k) & 1u) continue;
        uint32_t va = g_inds[k][a], vb = g_inds[k][b];
        if (va != vb) return va < vb ? -1 : 1;
    }
    return a < b ? -1 : (a > b ? 1 : 0);
}

int64_t oracle_coo_to_ghicoo(uint32_t order, uint64_t nnz, const uint32_t *const *inds,
                             const float *vals, uint32_t block_bits, uint32_t cmask,
                             uint64_t *bptr, uint32_t *const *binds, uint8_t *const *einds,
                             uint32_t *const *uinds, float *out_vals)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || block_bits < 1 || block_bits > 8) return -1;
    if (cmask == 0 || (cmask >> order) != 0) return -1;
    uint64_t *perm = (uint64_t *)malloc((nnz ? nnz : 1) * sizeof(uint64_t));
    if (!perm) return -2;
    for (uint64_t x = 0; x < nnz; ++x) perm[x] = x;
    g_order = order; g_inds = inds; g_cmask = cmask;
    qsort(perm, nnz, sizeof(uint64_t), cmp_ghicoo);
    uint32_t emask = (1u << block_bits) - 1u;
    int64_t nb = 0;
    for (uint64_t x = 0; x < nnz; ++x) {
        uint64_t p = perm[x];
        int new_block = (x == 0);
        if (!new_block) {
            uint64_t q = perm[x - 1];
            for (uint32_t k = 0; k < order; ++k)
                if (((cmask >> k) & 1u) && (inds[k][p] >> block_bits) != (inds[k][q] >> block_bits))
                    new_block = 1;
        }
        if (new_block) {
            bptr[nb] = x;
            for (uint32_t k = 0; k < order; ++k)
                if ((cmask >> k) & 1u) binds[k][nb] = inds[k][p] >> block_bits;
            ++nb;
        }
        for (uint32_t k = 0; k < order; ++k) {
            if ((cmask >> k) & 1u) einds[k][x] = (uint8_t)(inds[k][p] & emask);
            else uinds[k][x] = inds[k][p];
        }
        out_vals[x] = vals[p];
    }
    bptr[nb] = nnz;
    free(perm);
    return nb;
}

/* O-gHiCOO-MTTKRP: Alg. 3 with the block rebasing applied to the     */
/* compressed modes only: i_k = binds_k(b)*B + einds_k(x) if k is compressed, */
/* else i_k = inds_k(x); then the accumulation of O-MTTKRP.                   */
int oracle_mttkrp_ghicoo(uint32_t order, const uint32_t *dims, uint32_t block_bits, uint32_t cmask,
                         uint64_t nblocks, const uint64_t *bptr, const uint32_t *const *binds,
                         const uint8_t *const *einds, const uint32_t *const *uinds,
                         const float *vals, uint32_t mode, const float *const *factors,
                         uint32_t R, double *Mref, double *Aref)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || mode >= order || R < 1) return -1;
    uint64_t B = 1ull << block_bits;
    uint64_t rows = dims[mode];
    uint64_t ik[ORACLE_MAX_ORDER];
    for (uint64_t e = 0; e < rows * R; ++e) { Mref[e] = 0.0; Aref[e] = 0.0; }
    for (uint64_t b = 0; b < nblocks; ++b) {
        for (uint64_t x = bptr[b]; x < bptr[b + 1]; ++x) {
            for (uint32_t k = 0; k < order; ++k)
                ik[k] = ((cmask >> k) & 1u) ? (uint64_t)binds[k][b] * B + einds[k][x]
                                            : (uint64_t)uinds[k][x];
            for (uint32_t r = 0; r < R; ++r) {
                double t = (double)vals[x];
                for (uint32_t k = 0; k < order; ++k) {
                    if (k == mode) continue;
                    t *= (double)factors[k][ik[k] * R + r];
                }
                Mref[ik[mode] * R + r] += t;
                Aref[ik[mode] * R + r] += fabs(t);
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------- */
/* O-TS / O-TEW.  The paper fixes single precision   */
/* (P:109): each result is the fp64 operation rounded once to fp32, which    */
/* equals the correctly rounded fp32 operation (53 >= 2*24 + 2).             */
/*   op: 0 add, 1 sub, 2 mul, 3 div.                                          */
/* ------------------------------------------------------------------------- */
static float ew_apply(uint32_t op, float a, float b)
{
    double x = (double)a, y = (double)b, z;
    if (op == 0) z = x + y;
    else if (op == 1) z = x - y;
    else if (op == 2) z = x * y;
    else z = x / y;
    return (float)z;
}

/* TS: out[i] = vals[i] op s. */
int oracle_ts(uint64_t n, const float *vals, uint32_t op, float s, float *out)
{
    if (op > 3) return -1;
    for (uint64_t i = 0; i < n; ++i) out[i] = ew_apply(op, vals[i], s);
    return 0;
}

/* TEW with identical non-zero patterns: out[i] = a[i] op b[i]. */
int oracle_tew_same(uint64_t n, const float *a, const float *b, uint32_t op, float *out)
{
    if (op > 3) return -1;
    for (uint64_t i = 0; i < n; ++i) out[i] = ew_apply(op, a[i], b[i]);
    return 0;
}

/* TEW with different patterns (R#31): Z(c) = X(c) op Y(c) over the union of  */
/* the patterns for add/sub (a missing operand: z = x, or z = 0 - y) and over their */
/* intersection for mul/div; output in lexicographic order.  Entries of X and Y are */
/* merged by sorting (coords, source); a coordinate repeated inside one input is an */
/* error (-4).  Returns the output nnz (capacity Mx + My), or < 0.                  */
typedef struct { uint32_t c[ORACLE_MAX_ORDER]; int src; float v; } ew_rec;
static uint32_t g_ew_order;
static int cmp_ew(const void *pa, const void *pb)
{
    const ew_rec *a = (const ew_rec *)pa, *b = (const ew_rec *)pb;
    for (uint32_t k = 0; k < g_ew_order; ++k)
        if (a->c[k] != b->c[k]) return a->c[k] < b->c[k] ? -1 : 1;
    return a->src - b->src;
}

int64_t oracle_tew_merge(uint32_t order, uint64_t Mx, const uint32_t *const *ix, const float *vx,
                         uint64_t My, const uint32_t *const *iy, const float *vy, uint32_t op,
                         uint32_t *const *out_inds, float *out_vals)
{
    if (order < 1 || order > ORACLE_MAX_ORDER || op > 3) return -1;
    uint64_t T = Mx + My;
    ew_rec *r = (ew_rec *)malloc((T ? T : 1) * sizeof(ew_rec));
    if (!r) return -2;
    for (uint64_t i = 0; i < T; ++i) {
        memset(&r[i], 0, sizeof(ew_rec));
        for (uint32_t k = 0; k < order; ++k) r[i].c[k] = i < Mx ? ix[k][i] : iy[k][i - Mx];
        r[i].src = i < Mx ? 0 : 1;
        r[i].v = i < Mx ? vx[i] : vy[i - Mx];
    }
    g_ew_order = order;
    qsort(r, T, sizeof(ew_rec), cmp_ew);
    int64_t nz = 0;
    uint64_t i = 0;
    while (i < T) {
        uint64_t j = i + 1;
        while (j < T && memcmp(r[i].c, r[j].c, sizeof(r[i].c)) == 0) ++j; /* same coordinate */
        if (j - i > 2 || (j - i == 2 && r[i].src == r[i + 1].src)) { free(r); return -4; }
        int hx = r[i].src == 0 || (j - i == 2);
        int hy = r[j - 1].src == 1;
        float xv = r[i].src == 0 ? r[i].v : 0.0f, yv = r[j - 1].src == 1 ? r[j - 1].v : 0.0f;
        int keep = (op <= 1) ? 1 : (hx && hy);
        if (keep) {
            float z;
            if (hx && hy) z = ew_apply(op, xv, yv);
            else if (hx) z = xv;
            else z = (op == 1) ? ew_apply(1, 0.0f, yv) : yv;
            for (uint32_t k = 0; k < order; ++k) out_inds[k][nz] = r[i].c[k];
            out_vals[nz] = z;
            ++nz;
        }
        i = j;
    }
    free(r);
    return nz;
}

/* ------------------------------------------------------------------------------ */
/* Label permutation of the synthetic generators (R#22, permute = 1): mode k's      */
/* indices are relabelled by a bijection pi_k of [0, I_k) derived from the seed:     */
/*   L = ceil(log2 I_k), m = 2^L - 1, K = mix64(seed ^ 0xA0761D6478BD642F ^ k);      */
/*   f(v): three rounds r of  v = (v * (((K >> 16r) & 0xFFFF) | 1)) & m;              */
/*                            v ^= v >> ceil(L / 2)  (L >= 2);                         */
/*                            v = (v + ((K >> (32 + 8r)) & 0xFFFFFF)) & m;           */
/*   pi_k(v) = first f^j(v), j >= 1, below I_k (cycle walking: a bijection of [0, I_k) */
/*   because f permutes [0, 2^L)).  Each step is written out below.                   */
/* ------------------------------------------------------------------------------ */
static uint64_t relabel_round(uint64_t v, uint64_t key, uint32_t L, uint64_t m)
{
    for (int r = 0; r < 3; ++r) {
        uint64_t mul = ((key >> (16 * r)) & 0xFFFFull) | 1ull;  /* odd: a bijection mod 2^L */
        v = (v * mul) & m;
        if (L >= 2) v ^= v >> ((L + 1) / 2);                    /* xor-shift: a bijection */
        uint64_t add = (key >> (32 + 8 * r)) & 0xFFFFFFull;
        v = (v + add) & m;                                       /* translation mod 2^L */
    }
    return v;
}

uint32_t oracle_relabel_index(uint32_t v, uint32_t dim, uint64_t seed, uint32_t k)
{
    uint32_t L = 0;
    while (L < 32 && (1ull << L) < (uint64_t)dim) ++L;
    uint64_t m = (L >= 64) ? ~0ull : ((1ull << L) - 1ull);
    uint64_t key = mix64(seed ^ 0xA0761D6478BD642Full ^ (uint64_t)k);
    uint64_t y = v;
    do { y = relabel_round(y, key, L, m); } while (y >= dim);
    return (uint32_t)y;
}

/* in place: inds[k][x] = pi_k(inds[k][x]) for every mode and nonzero */
int oracle_relabel(uint32_t order, const uint32_t *dims, uint64_t nnz, uint64_t seed, uint32_t *const *inds)
{
    if (order < 1 || order > ORACLE_MAX_ORDER) return -1;
    for (uint32_t k = 0; k < order; ++k)
        for (uint64_t x = 0; x < nnz; ++x) inds[k][x] = oracle_relabel_index(inds[k][x], dims[k], seed, k);
    return 0;
}
