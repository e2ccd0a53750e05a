/* oracle_sweep.c — TEST HARNESS (not product code): the oracle's three checkers against each other on a large
 * number of small random traces (SURVEY §4.2 "brute == count on >= 1e5 random small traces").
 *
 *   oracle_check_brute        every pair (the definition itself, O(n^2))
 *   oracle_check_grouped      counting by inclusion-exclusion per location (O(n log n))
 *   oracle_check_partitioned  the grouped checker on T threads over a hash partition of the locations
 *
 * Traces come from the seeded counter-based generator of sesagen (gen_common.h rnd_record); per trace the
 * structure parameters (blocks, threads, intervals, words, spaces, sizes, atomics/writes, values, order) and the
 * config (warp size, lockstep, granularity, benign reporting) are drawn from the trace seed, so that dense
 * collisions, partial overlaps, mixed sizes, all access kinds and every ordering rule are exercised.  Every fifth
 * trace is a multi-launch trace (NEXT-4) with per-record launch ids (the *_ep checkers).
 *
 *   oracle_sweep <first_seed> <count>      -> prints "traces=... racy=... races=..." and exits 0, or 1 on the
 *                                             first disagreement (printing the seed and config).           */
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include "gen_common.h"

typedef struct {
  uint64_t addr, first, second;
  uint32_t block, interval;
  uint8_t space, kind;
  uint8_t reserved[2];
  uint32_t epoch;
} race_t;

int oracle_check_brute(const void *r, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls, uint32_t G,
                       uint32_t flags, race_t *out, uint64_t cap, uint64_t *nout);
int oracle_check_grouped(const void *r, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls, uint32_t G,
                         uint32_t flags, race_t *out, uint64_t cap, uint64_t *nout);
int oracle_check_partitioned(const void *r, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls, uint32_t G,
                             uint32_t flags, uint32_t T, race_t *out, uint64_t cap, uint64_t *nout);
int oracle_check_brute_ep(const void *r, const uint32_t *ep, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls,
                          uint32_t G, uint32_t flags, race_t *out, uint64_t cap, uint64_t *nout);
int oracle_check_grouped_ep(const void *r, const uint32_t *ep, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls,
                            uint32_t G, uint32_t flags, race_t *out, uint64_t cap, uint64_t *nout);
int oracle_check_partitioned_ep(const void *r, const uint32_t *ep, uint64_t n, uint64_t base, uint32_t ws,
                                uint32_t ls, uint32_t G, uint32_t flags, uint32_t T, race_t *out, uint64_t cap,
                                uint64_t *nout);

#define CAP 200000

int main(int argc, char **argv) {
  const uint64_t s0 = argc > 1 ? strtoull(argv[1], NULL, 10) : 0;
  const uint64_t cnt = argc > 2 ? strtoull(argv[2], NULL, 10) : 1000;
  static const uint32_t WS[] = {32, 32, 4, 1, 2, 8, 32, 3};
  static const uint32_t LS[] = {0, 1, 1, 1, 0, 1, 1, 1};
  static const uint32_t GR[] = {4, 4, 1, 2, 8, 16, 64, 4};
  static const uint16_t SZ[][4] = {{4, 4, 4, 4}, {1, 2, 4, 8}, {1, 1, 2, 2}, {4, 8, 16, 3}, {8, 8, 1, 4}};
  race_t *a = malloc(CAP * sizeof(race_t)), *b = malloc(CAP * sizeof(race_t)), *c = malloc(CAP * sizeof(race_t));
  grec *recs = malloc(4096 * sizeof(grec));
  uint32_t *ep = malloc(4096 * sizeof(uint32_t));
  uint64_t racy = 0, total = 0, kinds[4] = {0, 0, 0, 0};
  for (uint64_t s = s0; s < s0 + cnt; s++) {
    const uint64_t h = gmix(0xC0FFEE00ull ^ s);
    rndcfg R;
    memset(&R, 0, sizeof R);
    R.seed = gmix(h + 11);
    R.n = 1 + (h % 97 == 0 ? gmix(h + 1) % 400 : gmix(h + 1) % 72);
    R.blocks = 1 + (uint32_t)(gmix(h + 2) % 4);
    R.threads = 1 + (uint32_t)(gmix(h + 3) % 80);
    R.intervals = 1 + (uint32_t)(gmix(h + 4) % 4);
    R.words = 1 + (uint32_t)(gmix(h + 5) % 30);
    R.shared_pm = (uint32_t)(gmix(h + 6) % 3) * 500;
    R.atomic_pm = (uint32_t)(gmix(h + 7) % 4) * 80;
    R.write_pm = 100 + (uint32_t)(gmix(h + 8) % 5) * 120;
    R.values = 1 + (uint32_t)(gmix(h + 9) % 4);
    R.nsizes = 4;
    memcpy(R.sizes, SZ[gmix(h + 10) % 5], sizeof R.sizes);
    R.sorted = (uint32_t)(gmix(h + 12) % 3 != 0);
    R.unaligned = (uint32_t)(gmix(h + 13) % 2);
    R.gbase = 0x10000000000ull;
    for (uint64_t i = 0; i < R.n; i++) rnd_record(&R, i, &recs[i]);
    const int k = (int)(s % 8);
    const uint32_t flags = (gmix(h + 14) % 3 == 0) ? 1u : 0u; /* benign W/W reporting on a third */
    const uint32_t T = 1 + (uint32_t)(s % 4);
    const uint64_t base = (gmix(h + 15) % 5 == 0) ? (1ull << 33) : 0;
    uint64_t na = 0, nb = 0, nc = 0;
    int ra, rb, rc;
    if (s % 5 == 4) { /* multi-launch trace (NEXT-4): per-record launch ids, non-decreasing or arbitrary */
      const uint32_t E = 1 + (uint32_t)(gmix(h + 16) % 4);
      for (uint64_t i = 0; i < R.n; i++)
        ep[i] = (gmix(h + 17) & 1) ? (uint32_t)((i * E) / R.n) : (uint32_t)(gmix(h ^ (i + 99)) % E);
      ra = oracle_check_brute_ep(recs, ep, R.n, base, WS[k], LS[k], GR[k], flags, a, CAP, &na);
      rb = oracle_check_grouped_ep(recs, ep, R.n, base, WS[k], LS[k], GR[k], flags, b, CAP, &nb);
      rc = oracle_check_partitioned_ep(recs, ep, R.n, base, WS[k], LS[k], GR[k], flags, T, c, CAP, &nc);
    } else {
      ra = oracle_check_brute(recs, R.n, base, WS[k], LS[k], GR[k], flags, a, CAP, &na);
      rb = oracle_check_grouped(recs, R.n, base, WS[k], LS[k], GR[k], flags, b, CAP, &nb);
      rc = oracle_check_partitioned(recs, R.n, base, WS[k], LS[k], GR[k], flags, T, c, CAP, &nc);
    }
    if (ra || rb || rc || na != nb || na != nc || memcmp(a, b, na * sizeof(race_t)) ||
        memcmp(a, c, na * sizeof(race_t))) {
      printf("MISMATCH seed=%llu n=%llu ws=%u ls=%u G=%u flags=%u T=%u rc=%d/%d/%d races=%llu/%llu/%llu\n",
             (unsigned long long)s, (unsigned long long)R.n, WS[k], LS[k], GR[k], flags, T, ra, rb, rc,
             (unsigned long long)na, (unsigned long long)nb, (unsigned long long)nc);
      return 1;
    }
    racy += na > 0;
    total += na;
    for (uint64_t q = 0; q < na; q++) kinds[a[q].kind & 3]++;
  }
  printf("traces=%llu racy=%llu races=%llu rw=%llu ww=%llu benign=%llu\n", (unsigned long long)cnt,
         (unsigned long long)racy, (unsigned long long)total, (unsigned long long)kinds[1],
         (unsigned long long)kinds[2], (unsigned long long)kinds[3]);
  free(a); free(b); free(c); free(recs); free(ep);
  return 0;
}
