/* gen_host.c — host build of the C3-C5 generators (feeds the oracle and the CPU baseline). */
#include <stdlib.h>
#include <string.h>

#include "gen_common.h"

/* records [lo, hi) of C5 */
void gen_c5_host(const c5cfg *c, uint64_t lo, uint64_t hi, grec *out) {
  for (uint64_t i = lo; i < hi; i++) c5_record(c, i, &out[i - lo]);
}

uint64_t gen_c3_count_host(const c3cfg *c) {
  const uint64_t T = (uint64_t)c->blocks * c->threads;
  uint64_t n = 0;
  for (uint64_t g = 0; g < T; g++) n += c3_count(c, g);
  return n;
}

/* all records in order (out must hold gen_c3_count_host records) */
void gen_c3_host(const c3cfg *c, const uint64_t *cdf, grec *out) {
  const uint64_t T = (uint64_t)c->blocks * c->threads;
  uint64_t o = 0;
  for (uint64_t g = 0; g < T; g++) {
    c3_write(c, cdf, g, out + o);
    o += c3_count(c, g);
  }
}

/* per-node record counts and row offsets: rows[v] = sum of degrees before v (n+1 entries) */
uint64_t gen_c4_layout_host(const c4cfg *c, const uint64_t *dcdf, uint64_t *rows, uint64_t *counts) {
  const uint64_t N = 1ull << c->log2n;
  uint64_t r = 0, total = 0;
  for (uint64_t v = 0; v < N; v++) {
    rows[v] = r;
    r += c4_degree(c, dcdf, v);
  }
  rows[N] = r;
  for (uint64_t v = 0; v < N; v++) {
    counts[v] = c4_count(c, dcdf, v, rows[v]);
    total += counts[v];
  }
  return total;
}

void gen_c4_host(const c4cfg *c, const uint64_t *dcdf, const uint64_t *rows, const uint64_t *counts, grec *out) {
  const uint64_t N = 1ull << c->log2n;
  uint64_t o = 0;
  for (uint64_t v = 0; v < N; v++) {
    c4_write(c, dcdf, v, rows[v], out + o);
    o += counts[v];
  }
}

/* records [lo, hi) of a random trace */
void gen_random_host(const rndcfg *c, uint64_t lo, uint64_t hi, grec *out) {
  for (uint64_t i = lo; i < hi; i++) rnd_record(c, i, &out[i - lo]);
}

uint64_t gen_sizeof_rndcfg(void) { return sizeof(rndcfg); }
uint64_t gen_sizeof_c3cfg(void) { return sizeof(c3cfg); }
uint64_t gen_sizeof_c4cfg(void) { return sizeof(c4cfg); }
uint64_t gen_sizeof_c5cfg(void) { return sizeof(c5cfg); }
