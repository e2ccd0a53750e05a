/* gen_common.h — counter-based generators of the BASELINE configs C3-C5, shared by the host C
 * build (gen_host.c, feeds the oracle) and the CUDA build (gen_dev.cu, feeds the bench).  Each record is a pure
 * function of (config, seed, counter): both builds produce identical bytes (tests/test_generators.py).
 * No race-check arithmetic lives here. */
#ifndef SESAGEN_COMMON_H
#define SESAGEN_COMMON_H
#include <stdint.h>

#ifdef __CUDACC__
#define GEN_HD __host__ __device__ __forceinline__
#else
#define GEN_HD static inline
#endif

typedef struct {
  uint64_t addr, vh;
  uint32_t block, thread, interval;
  uint16_t size;
  uint8_t space, rw;
} grec;

enum { G_SHARED = 0, G_GLOBAL = 1, G_R = 0, G_W = 1, G_A = 2 };

GEN_HD uint64_t gmix(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

GEN_HD void gset(grec *r, uint64_t addr, uint64_t vh, uint32_t b, uint32_t t, uint32_t iv, uint16_t sz, uint8_t sp,
                 uint8_t rw) {
  r->addr = addr;
  r->vh = vh;
  r->block = b;
  r->thread = t;
  r->interval = iv;
  r->size = sz;
  r->space = sp;
  r->rw = rw;
}

/* first index i in [0, n) with u < cdf[i]; n - 1 if none (cdf[n-1] is 2^64 - 1) */
GEN_HD uint32_t ginv_cdf(const uint64_t *cdf, uint32_t n, uint64_t u) {
  uint32_t lo = 0, hi = n - 1;
  while (lo < hi) {
    uint32_t m = (lo + hi) >> 1;
    if (u < cdf[m]) hi = m; else lo = m + 1;
  }
  return lo;
}

/* ---------------------------------------------------------------------------------------------------- C5
 * n records; record i: block i/2048, interval (i/512)%4, thread i%512; global, 4 bytes at base + 4*pi(i) with
 * pi a 4-round Feistel bijection of [0, 2^30); R 70% / W 25% / A 5%; W value = gmix(seed^0x57 ^ i).
 * Injection: K = max(1, n/10000) strata of S = n/K records; victim v = k*S + h(k) % (S/2), partner p = v + S/2
 * gets v's address; (R,R)/(A,A) -> partner becomes W; (W,W) -> partner's value ^= 1.  Every stratum is one
 * race: RW if either is R else WW, witness (v, p). */
typedef struct {
  uint64_t seed, n, base;
} c5cfg;

GEN_HD uint32_t c5_perm(uint64_t seed, uint32_t x) {
  uint32_t L = x >> 15, R = x & 0x7FFF;
  for (uint32_t r = 0; r < 4; r++) {
    uint32_t F = (uint32_t)(gmix(seed ^ ((uint64_t)r << 40) ^ R) & 0x7FFF);
    uint32_t nl = R, nr = L ^ F;
    L = nl;
    R = nr;
  }
  return (L << 15) | R;
}

GEN_HD uint8_t c5_base_rw(uint64_t seed, uint64_t i) {
  uint64_t u = gmix(seed ^ 0x5A5A0000ull ^ i) % 100;
  return u < 70 ? G_R : (u < 95 ? G_W : G_A);
}

GEN_HD uint64_t c5_base_vh(uint64_t seed, uint64_t i) { return gmix(seed ^ 0x57ull ^ (i << 8)); }

GEN_HD void c5_record(const c5cfg *c, uint64_t i, grec *r) {
  const uint64_t K = c->n / 10000 ? c->n / 10000 : 1, S = c->n / K;
  uint64_t a = i;            /* address owner */
  uint8_t rw = c5_base_rw(c->seed, i);
  uint64_t vh = rw == G_W ? c5_base_vh(c->seed, i) : 0;
  const uint64_t k = i / S;
  if (k < K && S >= 2) {
    const uint64_t half = S / 2;
    const uint64_t v = k * S + gmix(c->seed ^ 0x1A1Aull ^ k) % half, p = v + half;
    if (i == p) {
      a = v;
      const uint8_t rv = c5_base_rw(c->seed, v);
      if ((rv == G_R && rw == G_R) || (rv == G_A && rw == G_A)) {
        rw = G_W;
        vh = c5_base_vh(c->seed, i);
      } else if (rv == G_W && rw == G_W) {
        vh = c5_base_vh(c->seed, v) ^ 1ull;
      }
    }
  }
  gset(r, c->base + 4ull * c5_perm(c->seed, (uint32_t)a), vh, (uint32_t)(i / 2048), (uint32_t)(i % 512),
       (uint32_t)((i / 512) % 4), 4, G_GLOBAL, rw);
}

/* ---------------------------------------------------------------------------------------------------- C3
 * Parboil-histo-shaped: blocks x threads; thread gtid handles pixels p = k*(blocks*threads) + gtid, k < ppt:
 * R img[p]; if guarded (1 in 64, hash of p): R bins[b]; ATOMIC bins[b], b = Zipf(s=1) over nbins (cdf table). */
typedef struct {
  uint64_t seed;
  uint32_t blocks, threads, ppt, nbins;
  uint64_t img_base, bins_base;
} c3cfg;

GEN_HD uint32_t c3_bin(const c3cfg *c, const uint64_t *cdf, uint64_t p) {
  return ginv_cdf(cdf, c->nbins, gmix(c->seed ^ 0xB1Bull ^ (p << 4)));
}
GEN_HD int c3_guard(const c3cfg *c, uint64_t p) { return (gmix(c->seed ^ 0x6A6Aull ^ (p << 4)) & 63) == 0; }

GEN_HD uint32_t c3_count(const c3cfg *c, uint64_t gtid) {
  const uint64_t T = (uint64_t)c->blocks * c->threads;
  uint32_t s = 0;
  for (uint32_t k = 0; k < c->ppt; k++) s += 2 + c3_guard(c, k * T + gtid);
  return s;
}

GEN_HD void c3_write(const c3cfg *c, const uint64_t *cdf, uint64_t gtid, grec *out) {
  const uint64_t T = (uint64_t)c->blocks * c->threads;
  const uint32_t b = (uint32_t)(gtid / c->threads), t = (uint32_t)(gtid % c->threads);
  uint64_t o = 0;
  for (uint32_t k = 0; k < c->ppt; k++) {
    const uint64_t p = k * T + gtid;
    const uint32_t bin = c3_bin(c, cdf, p);
    gset(&out[o++], c->img_base + 4 * p, 0, b, t, 0, 4, G_GLOBAL, G_R);
    if (c3_guard(c, p)) gset(&out[o++], c->bins_base + 4ull * bin, 0, b, t, 0, 4, G_GLOBAL, G_R);
    gset(&out[o++], c->bins_base + 4ull * bin, 0, b, t, 0, 4, G_GLOBAL, G_A);
  }
}

/* ---------------------------------------------------------------------------------------------------- C4
 * Lonestar-bfs-shaped (one BFS level): 2^log2n nodes, thread v = node v (512 per block), one interval.
 * degree = power law (alpha 2.1, d in [4, 1024], cdf table, mean ~16.8); node class by hash: 45% frontier,
 * 5% visited, 50% unvisited; edge e = row[v] + j has dst = R-MAT column bits (P(bit) = 61/256 per level).
 * Every thread: R dist[v].  Frontier: R row[v], R row[v+1], per edge: R col[e], R dist[dst]; dst unvisited:
 * W dist[dst] (value of the next level) and W changed (value 1). */
typedef struct {
  uint64_t seed;
  uint32_t log2n, dmin, ndeg, pad;
  uint64_t dist_base, row_base, col_base, changed_base;
} c4cfg;

GEN_HD uint32_t c4_degree(const c4cfg *c, const uint64_t *dcdf, uint64_t v) {
  return c->dmin + ginv_cdf(dcdf, c->ndeg, gmix(c->seed ^ 0xDE6ull ^ (v << 3)));
}
GEN_HD uint32_t c4_class(const c4cfg *c, uint64_t v) { /* 0 frontier, 1 visited, 2 unvisited */
  const uint64_t u = gmix(c->seed ^ 0xC1A55ull ^ (v << 3)) % 100;
  return u < 45 ? 0 : (u < 50 ? 1 : 2);
}
GEN_HD uint64_t c4_dst(const c4cfg *c, uint64_t e) {
  uint64_t d = 0;
  for (uint32_t l = 0; l < c->log2n; l++) {
    const uint64_t h = gmix(c->seed ^ 0xE06Eull ^ (e << 6) ^ (uint64_t)(l >> 3));
    const uint32_t byte = (uint32_t)((h >> (8 * (l & 7))) & 0xFF);
    d = (d << 1) | (byte < 61 ? 1u : 0u);
  }
  return d;
}

GEN_HD uint32_t c4_count(const c4cfg *c, const uint64_t *dcdf, uint64_t v, uint64_t row) {
  if (c4_class(c, v) != 0) return 1;
  const uint32_t deg = c4_degree(c, dcdf, v);
  uint32_t s = 3;
  for (uint32_t j = 0; j < deg; j++) s += 2 + (c4_class(c, c4_dst(c, row + j)) == 2 ? 2 : 0);
  return s;
}

GEN_HD void c4_write(const c4cfg *c, const uint64_t *dcdf, uint64_t v, uint64_t row, grec *out) {
  const uint32_t b = (uint32_t)(v >> 9), t = (uint32_t)(v & 511);
  uint64_t o = 0;
  gset(&out[o++], c->dist_base + 4 * v, 0, b, t, 0, 4, G_GLOBAL, G_R);
  if (c4_class(c, v) != 0) return;
  gset(&out[o++], c->row_base + 4 * v, 0, b, t, 0, 4, G_GLOBAL, G_R);
  gset(&out[o++], c->row_base + 4 * (v + 1), 0, b, t, 0, 4, G_GLOBAL, G_R);
  const uint32_t deg = c4_degree(c, dcdf, v);
  const uint64_t level_vh = gmix(c->seed ^ 0x1E7E1ull), one_vh = gmix(1);
  for (uint32_t j = 0; j < deg; j++) {
    const uint64_t e = row + j, dst = c4_dst(c, e);
    gset(&out[o++], c->col_base + 4 * e, 0, b, t, 0, 4, G_GLOBAL, G_R);
    gset(&out[o++], c->dist_base + 4 * dst, 0, b, t, 0, 4, G_GLOBAL, G_R);
    if (c4_class(c, dst) == 2) {
      gset(&out[o++], c->dist_base + 4 * dst, level_vh, b, t, 0, 4, G_GLOBAL, G_W);
      gset(&out[o++], c->changed_base, one_vh, b, t, 0, 4, G_GLOBAL, G_W);
    }
  }
}
/* ------------------------------------------------------------------------------------------------ random
 * Random traces for property sweeps (oracle self-consistency, GPU parity).  Record i is a pure function of
 * (cfg, i): block / interval either from the position (sorted = 1: (block, interval) ascending, the canonical
 * schedule of P:257) or hashed; thread, space, access kind, size, word (+ in-word offset) and value from
 * independent hashes.  Dense collisions come from a small `words`.  No race-check arithmetic. */
typedef struct {
  uint64_t seed, n;
  uint32_t blocks, threads, intervals, words;
  uint32_t shared_pm, atomic_pm, write_pm; /* per mille */
  uint32_t values;                         /* value hashes in [0, values) */
  uint32_t nsizes, sorted, unaligned, pad;
  uint16_t sizes[4];
  uint64_t gbase;                          /* global addresses: gbase + 4 * word + offset */
} rndcfg;

GEN_HD void rnd_record(const rndcfg *c, uint64_t i, grec *r) {
  const uint64_t h = gmix(c->seed ^ gmix(i));
  const uint64_t h1 = gmix(h + 1), h2 = gmix(h + 2), h3 = gmix(h + 3), h4 = gmix(h + 4), h5 = gmix(h + 5),
                 h6 = gmix(h + 6), h7 = gmix(h + 7);
  uint32_t b, iv;
  if (c->sorted) {
    const uint64_t cells = (uint64_t)c->blocks * c->intervals;
    const uint64_t bi = c->n ? (uint64_t)(((unsigned __int128)i * cells) / c->n) : 0;
    b = (uint32_t)(bi / c->intervals);
    iv = (uint32_t)(bi % c->intervals);
  } else {
    b = (uint32_t)(h1 % c->blocks);
    iv = (uint32_t)((h1 >> 32) % c->intervals);
  }
  const uint32_t t = (uint32_t)(h2 % c->threads);
  const uint8_t sp = (h3 % 1000) < c->shared_pm ? G_SHARED : G_GLOBAL;
  const uint32_t u = (uint32_t)(h4 % 1000);
  const uint8_t rw = u < c->atomic_pm ? G_A : u < c->atomic_pm + c->write_pm ? G_W : G_R;
  const uint16_t sz = c->sizes[h5 % c->nsizes];
  const uint64_t w = h6 % c->words, off = c->unaligned ? (h6 >> 40) % 4 : 0;
  const uint64_t addr = sp == G_GLOBAL ? c->gbase + 4 * w + off : 4 * w + off;
  gset(r, addr, h7 % c->values, b, t, iv, sz, sp, rw);
}

#endif
