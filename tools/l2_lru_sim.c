// tools/l2_lru_sim.c -- host simulation of the COO MTTKRP factor gathers of H (mode 0, two gathered
// factors, product-form Kronecker indices, L = 23, M = 1e8) through a set-associative LRU of
// 128-B lines (SECT=1: 64-B halves filled separately, as a sectored L2 does; STREAM=1: the
// 16 B/nonzero stream; OUT=1: output rows).  Compares the packed hot-row tier (LAYOUT=0) with a
// heat-ordered relabelling of every factor (LAYOUT=1).  Not part of the library.
//   gcc -O2 -o /tmp/lru tools/l2_lru_sim.c && SECT=1 STREAM=1 OUT=1 /tmp/lru 23 100000000 <cache MB> <tier MB>
// LRU simulation of the gathers of H mode 0 (two factors), 128-B lines, set-associative.
// layout 0: hot tier packed (top T rows jointly by count) + cold rows at natural addresses
// layout 1: every factor relabelled by descending count (rank order), rows contiguous
#include <stdio.h>
#include <stdlib.h>
#include <stdint.h>
#include <string.h>
static uint64_t s0 = 0x9E3779B97F4A7C15ull;
static inline uint64_t rnd(void) { uint64_t z = (s0 += 0x9E3779B97F4A7C15ull); z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull; z = (z ^ (z >> 27)) * 0x94d049bb133111ebull; return z ^ (z >> 31); }
static inline uint32_t draw(int L) { return (uint32_t)(rnd() & rnd()) & ((1u << L) - 1); }
#define WAYS 16
typedef struct { uint64_t tag[WAYS]; uint32_t age[WAYS]; uint8_t valid[WAYS]; } Set;
static Set *sets; static uint64_t nsets; static uint32_t clk;
static int SECT = 0;
// addr64 = 64-B unit index; line = addr64 >> 1; SECT: 64-B halves filled separately
static int access64(uint64_t a64) {
  uint64_t line = a64 >> 1; uint8_t bit = SECT ? (uint8_t)(1u << (a64 & 1)) : 3;
  Set *s = &sets[line % nsets]; clk++;
  int lru = 0;
  for (int w = 0; w < WAYS; ++w) {
    if (s->tag[w] == line + 1) { s->age[w] = clk; if (s->valid[w] & bit) return 1; s->valid[w] |= bit; return 0; }
    if (s->age[w] < s->age[lru]) lru = w;
  }
  s->tag[lru] = line + 1; s->age[lru] = clk; s->valid[lru] = bit; return 0;
}
static int access_line(uint64_t line) { return access64(line << 1); }
static int cmpdesc(const void *a, const void *b) { uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b; return x < y ? 1 : x > y ? -1 : 0; }
int main(int argc, char **argv) {
  SECT = getenv("SECT") != 0;
  int L = atoi(argv[1]); uint64_t M = strtoull(argv[2], 0, 10); double cache_mb = atof(argv[3]); double tier_mb = atof(argv[4]);
  uint64_t I = 1ull << L;
  uint32_t *a = malloc(M * 4), *b = malloc(M * 4);
  uint32_t *ca = calloc(I, 4), *cb = calloc(I, 4);
  for (uint64_t x = 0; x < M; ++x) { draw(L); a[x] = draw(L); b[x] = draw(L); ca[a[x]]++; cb[b[x]]++; }
  // (order of processing: random stream of nonzeros; mode-0 sort makes a, b independent of time)
  // ranks: per factor, count desc
  uint64_t *ka = malloc(I * 8), *kb = malloc(I * 8);
  for (uint64_t r = 0; r < I; ++r) { ka[r] = ((uint64_t)ca[r] << 32) | (0xFFFFFFFFu - r); kb[r] = ((uint64_t)cb[r] << 32) | (0xFFFFFFFFu - r); }
  qsort(ka, I, 8, cmpdesc); qsort(kb, I, 8, cmpdesc);
  uint32_t *ra = malloc(I * 4), *rb = malloc(I * 4);
  for (uint64_t i = 0; i < I; ++i) { ra[0xFFFFFFFFu - (uint32_t)ka[i]] = i; rb[0xFFFFFFFFu - (uint32_t)kb[i]] = i; }
  uint64_t tier_rows = (uint64_t)(tier_mb * 1048576 / 64), smem_rows = 256;  // per factor: half each
  nsets = (uint64_t)(cache_mb * 1048576 / 128) / WAYS; sets = calloc(nsets, sizeof(Set));
  for (int layout = atoi(getenv("LAYOUT") ? getenv("LAYOUT") : "0"); layout < 1 + atoi(getenv("LAYOUT") ? getenv("LAYOUT") : "0"); ++layout) {
    memset(sets, 0, nsets * sizeof(Set)); clk = 0;
    uint64_t miss = 0, acc = 0, smem = 0;
    for (uint64_t x = 0; x < M; ++x) {
      if (getenv("STREAM") && (x % 32) == 0)  // 4 arrays x 128 B per 32 nonzeros, no reuse
        for (int q = 0; q < 4; ++q) access_line((((uint64_t)3 + q) << 44) / 128 + x / 32);
      if (getenv("OUT") && (x % 26) == 0) access_line(((uint64_t)9 << 44) / 128 + x / 26 / 2);
      for (int f = 0; f < 2; ++f) {
        uint32_t row = f ? b[x] : a[x], rk = f ? rb[row] : ra[row];
        if (rk < smem_rows) { smem++; continue; }
        uint64_t addr;
        if (layout == 0) addr = rk < smem_rows + tier_rows / 2 ? ((uint64_t)1 << 40) + ((uint64_t)f * tier_rows / 2 + rk) * 64 : ((uint64_t)f << 36) + (uint64_t)row * 64;
        else addr = ((uint64_t)f << 36) + (uint64_t)rk * 64;
        acc++; miss += !access64(addr >> 6);
      }
    }
    printf("L=%d M=%llu cache %.0f MB tier %.0f MB layout %d: L2 accesses %llu misses %llu (%.1f%%) smem %llu -> miss bytes %.2f GB (64 B/miss)\n",
           L, (unsigned long long)M, cache_mb, tier_mb, layout, (unsigned long long)acc, (unsigned long long)miss, 100.0 * miss / acc, (unsigned long long)smem, miss * 64 / 1e9);
  }
}
