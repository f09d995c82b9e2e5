// tools/l2_twopass_sim.c (not part of the library): the sectored-LRU model of tools/l2_lru_sim.c
// applied to a two-pass COO schedule of H mode 0.  Pass 1 = the nonzeros whose two gathered rows
// are both in the hot tiers (shared-memory tier or the packed L2 tier), pass 2 = the rest; each
// pass in output-row order.  Pass 1 stores every touched output row once; pass 2 read-modify-
// writes its rows (a red at L2: a miss reads 64 B; every touched row is written back).  Stream
// lines (16 B per nonzero) go through the cache with no reuse.  One pass = the current kernel.
//   gcc -O2 -o /tmp/twopass tools/l2_twopass_sim.c && SECT=1 /tmp/twopass 23 100000000 32 64
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
static uint64_t s0 = 0x9E3779B97F4A7C15ull;
static inline uint64_t rnd(void) { uint64_t z = (s0 += 0x9E3779B97F4A7C15ull); z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ull; z = (z ^ (z >> 27)) * 0x94d049bb133111ebull; return z ^ (z >> 31); }
static inline uint32_t draw(int L) { return (uint32_t)(rnd() & rnd()) & ((1u << L) - 1); }
#define WAYS 16
typedef struct { uint64_t tag[WAYS]; uint32_t age[WAYS]; uint8_t valid[WAYS]; } Set;
static Set *sets; static uint64_t nsets; static uint32_t clk; static int SECT = 0;
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
static int cmpdesc(const void *a, const void *b) { uint64_t x = *(const uint64_t *)a, y = *(const uint64_t *)b; return x < y ? 1 : x > y ? -1 : 0; }
typedef struct { uint32_t row, a, b, pass; } E;
static int cmpE(const void *p, const void *q) {
  const E *x = p, *y = q;
  if (x->pass != y->pass) return x->pass < y->pass ? -1 : 1;
  return x->row < y->row ? -1 : x->row > y->row;
}
int main(int argc, char **argv) {
  SECT = getenv("SECT") != 0;
  int L = atoi(argv[1]); uint64_t M = strtoull(argv[2], 0, 10); double cache_mb = atof(argv[3]); double tier_mb = atof(argv[4]);
  uint64_t I = 1ull << L;
  E *e = malloc(M * sizeof(E));
  uint32_t *ca = calloc(I, 4), *cb = calloc(I, 4);
  for (uint64_t x = 0; x < M; ++x) { e[x].row = draw(L); e[x].a = draw(L); e[x].b = draw(L); ca[e[x].a]++; cb[e[x].b]++; }
  uint64_t *ka = malloc(I * 8), *kb = malloc(I * 8);
  for (uint64_t r = 0; r < I; ++r) { ka[r] = ((uint64_t)ca[r] << 32) | (0xFFFFFFFFu - r); kb[r] = ((uint64_t)cb[r] << 32) | (0xFFFFFFFFu - r); }
  qsort(ka, I, 8, cmpdesc); qsort(kb, I, 8, cmpdesc);
  uint32_t *ra = malloc(I * 4), *rb = malloc(I * 4);
  for (uint64_t i = 0; i < I; ++i) { ra[0xFFFFFFFFu - (uint32_t)ka[i]] = i; rb[0xFFFFFFFFu - (uint32_t)kb[i]] = i; }
  const uint64_t tier_rows = (uint64_t)(tier_mb * 1048576 / 64), smem_rows = 256, hot = smem_rows + tier_rows / 2;
  nsets = (uint64_t)(cache_mb * 1048576 / 128) / WAYS; sets = calloc(nsets, sizeof(Set));
  for (int passes = 1; passes <= 2; ++passes) {
    uint64_t n1 = 0;
    for (uint64_t x = 0; x < M; ++x) {
      e[x].pass = passes == 2 && !(ra[e[x].a] < hot && rb[e[x].b] < hot);
      n1 += !e[x].pass;
    }
    qsort(e, M, sizeof(E), cmpE);
    memset(sets, 0, nsets * sizeof(Set)); clk = 0;
    uint64_t gmiss = 0, omiss = 0, owrite = 0;
    uint32_t prow = 0xFFFFFFFFu, ppass = 9;
    for (uint64_t x = 0; x < M; ++x) {
      if ((x % 32) == 0) for (int q = 0; q < 4; ++q) access64((((uint64_t)3 + q) << 44) / 64 + x / 16 * 2);
      if (e[x].row != prow || e[x].pass != ppass) {
        const int hit = access64((((uint64_t)9 << 44) >> 6) + e[x].row);
        if (e[x].pass == 1 && !hit) omiss++;  // pass 2 reads the row written by pass 1
        owrite++;
        prow = e[x].row; ppass = e[x].pass;
      }
      for (int f = 0; f < 2; ++f) {
        uint32_t row = f ? e[x].b : e[x].a, rk = f ? rb[row] : ra[row];
        if (rk < smem_rows) continue;
        uint64_t addr = rk < hot ? ((uint64_t)1 << 40) + ((uint64_t)f * tier_rows / 2 + rk) * 64 : ((uint64_t)f << 36) + (uint64_t)row * 64;
        gmiss += !access64(addr >> 6);
      }
    }
    printf("passes %d (pass 1: %.1f%% of the nonzeros), cache %.0f MB%s, tier %.0f MB: gather misses %.1fM (%.2f GB), "
           "output reads %.2f GB + writes %.2f GB, total %.2f GB + stream 1.6 GB\n",
           passes, 100.0 * n1 / M, cache_mb, SECT ? " sectored" : "", tier_mb, gmiss / 1e6, gmiss * 64 / 1e9, omiss * 64 / 1e9,
           owrite * 64 / 1e9, (gmiss + omiss + owrite) * 64 / 1e9);
  }
}
