/*
 * sesa_oracle.c — CPU ORACLE for the concrete race check.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may load this.
 * It shares no code, header, table or helper with the CUDA path (paper_conf_sc_lilg14_b200/csrc); every
 * struct below is declared here independently from the paper's problem statement.
 *
 * Paper: Li, Li, Gopalakrishnan, "Practical Symbolic Race Checking of GPU Programs", SC'14.
 * "P:<line>" = /root/reference/PAPER.md line.
 *
 * What is computed (plain definition):
 *   A data race = two threads make a happens-before-unordered access to the same memory location and one
 *   access is a write (§I).  Per barrier interval, read and write sets are instantiated for two
 *   different threads t1 != t2 and compared address by address (WW and WR checks, §II; P:263-269
 *   §IV-B).  Here the accesses are concrete records; the pair predicate P(r, s) is spelled out in
 *   oracle_pair_kind() below, rule by rule, with the reading each rule follows.
 *
 * Two independent checkers:
 *   oracle_check_brute   — every pair i < j, every common location: the definition itself, O(n^2).
 *   oracle_check_grouped — group entries by location (qsort), per location decide "has a partner of kind K"
 *                          by COUNTING partners (inclusion-exclusion over sorted tuples), then witness
 *                          x = min flagged index, y = min s with P(x, s) of kind K.  O(n log n).
 *   oracle_check_partitioned — checker 2 on T threads: locations partitioned by a hash of λ mod T (a race is a
 *                          property of one location, c.1), each thread runs the unchanged group algorithm on its
 *                          partition; byte-identical output (SURVEY §8c.3 "T-thread mode"; full-size parity).
 * With flag F_BENIGN all three also report benign W/W pairs as a third kind (oracle_benign_pair).
 * Precise warp model (NEXT-3): oracle_pair_kind_warp + oracle_check_warp_brute / oracle_check_warp_grouped, on
 * records with an instruction / divergence extension.
 * They agree on every input (tests/test_oracle.py); the GPU path uses neither method (it uses per-run
 * min/max summaries), so agreement of the GPU with this oracle is not circular.
 *
 * Also: oracle_validate (the record validity rules of include/sesa.h, re-stated) and oracle_expand (the
 * parametric-flow instantiation "replace i by j", §IV-A).
 */
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- independent declarations of the record / race / flow layouts (32 / 40 / 104 bytes) ---------------- */
typedef struct {
  uint64_t addr, value_hash;
  uint32_t block, thread, interval;
  uint16_t size;
  uint8_t space, rw;
} orec;

typedef struct {
  uint64_t addr, first, second;
  uint32_t block, interval;
  uint8_t space, kind;
  uint8_t reserved[2];
  uint32_t epoch; /* kernel launch of the location (multi-launch traces, NEXT-4); 0 for one launch */
} orace;

typedef struct {
  uint64_t base;
  int64_t bstride, tstride, istride;
  uint64_t value_seed;
  uint32_t block_lo, block_hi, nthreads, interval;
  uint32_t pmask, pval, pmod, prem, plo, phi;
  uint32_t fkind, fc, fm, count;
  uint16_t size;
  uint8_t space, rw;
  uint32_t flags;
} oflow;

enum { SH = 0, GL = 1 };            /* memory sorts: shared / global */
enum { RD = 0, WR = 1, AT = 2 };    /* load, store, atomic intrinsic */
enum { K_RW = 1, K_WW = 2, K_WWB = 3 }; /* the WR and WW checks of P:79; K_WWB = a benign W/W pair */
#define F_BENIGN 1u                 /* config flag: also report benign W/W pairs as kind K_WWB (NEXT-4) */
#define NOBI 0xFFFFFFFFu            /* block/interval of a GLOBAL location (not part of λ) */

/* ---- validity (the rules of include/sesa.h, independently restated) -------------------------------------
 * returns 0 if all valid, else 1 and *bad = lowest bad index.  */
int oracle_validate(const orec *r, uint64_t n, uint64_t *bad) {
  for (uint64_t i = 0; i < n; i++) {
    int ok = r[i].space <= 1 && r[i].rw <= 2 && r[i].size >= 1 &&
             r[i].addr <= UINT64_MAX - (uint64_t)(r[i].size - 1); /* addr + size - 1 must not wrap */
    if (!ok) {
      *bad = i;
      return 1;
    }
  }
  return 0;
}

int oracle_config_ok(uint32_t ws, uint32_t ls, uint32_t G) {
  if (ws < 1 || ls > 1 || G < 1 || G > 4096 || (G & (G - 1)) != 0) return 0;
  return 1;
}

/* ---- the pair predicate P(r, s) -------------------------------------------------------------------------
 * Precondition: r and s are different records that cover a common location λ (same space; if shared, same
 * block and same interval; a common granule).  Returns 0 (no race), K_RW or K_WW.                          */
int oracle_pair_kind(const orec *r, const orec *s, uint32_t ws, uint32_t ls) {
  /* (1) different threads: t1 != t2; a thread never races with itself (P:287 case 2) */
  if (r->block == s->block && r->thread == s->thread) return 0;
  /* (2) at least one write; an atomic is a write (read vs atomicAdd is a race) */
  if (r->rw == RD && s->rw == RD) return 0;
  /* (3) atomic-atomic pairs never race (north_star; P:573 and P:447 count only plain-vs-atomic) */
  if (r->rw == AT && s->rw == AT) return 0;
  /* (4) unordered: global memory of one block is ordered across __syncthreads (reading R2);
         different blocks are never ordered.  Shared λ already fixes block+interval. */
  if (r->space == GL && r->block == s->block && r->interval != s->interval) return 0;
  int kind = (r->rw == RD || s->rw == RD) ? K_RW : K_WW;
  /* (5) lockstep: intra-warp threads race only on simultaneous writes, so an intra-warp pair with a
         read is exempt (reading R6-R8); warp = thread / warp_size, groups of consecutive threads */
  if (ls && kind == K_RW && r->block == s->block && r->interval == s->interval &&
      r->thread / ws == s->thread / ws)
    return 0;
  /* (6) benign W/W: two plain writes of the same value (Table IV "W/W (Benign)") */
  if (r->rw == WR && s->rw == WR && r->value_hash == s->value_hash) return 0;
  return kind;
}

/* ---- the benign W/W pair B(r, s) (reported only with F_BENIGN) --------------------------------------------
 * Table IV reports "W/W (Benign)" verdicts (bfs, cutcp, spmv) and the conclusion "races later deemed to be
 * benign": a write/write conflict that rule (6) above removes from the race set because both threads
 * write the same value.  B(r, s) = both plain writes, equal value_hash, and every other condition of a W/W race:
 * different threads (1) and unordered (4).  Rules (2), (3) hold for two plain writes; (5) exempts only pairs
 * with a read.  Same precondition as oracle_pair_kind.                                                        */
int oracle_benign_pair(const orec *r, const orec *s) {
  if (r->rw != WR || s->rw != WR || r->value_hash != s->value_hash) return 0;
  if (r->block == s->block && r->thread == s->thread) return 0;                      /* (1) */
  if (r->space == GL && r->block == s->block && r->interval != s->interval) return 0; /* (4) */
  return 1;
}

/* granule range of a record: [addr/G, (addr+size-1)/G]  (reading R1: overlap at granularity G) */
static void granules(const orec *r, uint32_t G, uint64_t *lo, uint64_t *hi) {
  *lo = r->addr / G;
  *hi = (r->addr + (uint64_t)(r->size - 1)) / G;
}

/* λ of record r at granule g: (SHARED, block, interval, g) or (GLOBAL, -, -, g), in kernel launch `epoch`.
 * Multi-launch traces (reading R23): the launches of one trace run one after the
 * other (each kernel completes before the next starts on the stream), so accesses of different launches are
 * ordered — like accesses separated by a barrier — and never race: the launch is part of λ. */
typedef struct {
  uint32_t epoch, space, block, interval;
  uint64_t g;
} loc;

static loc loc_of(const orec *r, uint64_t g, uint32_t epoch) {
  loc L;
  L.epoch = epoch;
  L.space = r->space;
  L.block = r->space == SH ? r->block : NOBI;
  L.interval = r->space == SH ? r->interval : NOBI;
  L.g = g;
  return L;
}

static int loc_cmp(const loc *a, const loc *b) {
  if (a->epoch != b->epoch) return a->epoch < b->epoch ? -1 : 1;
  if (a->space != b->space) return a->space < b->space ? -1 : 1;
  if (a->block != b->block) return a->block < b->block ? -1 : 1;
  if (a->interval != b->interval) return a->interval < b->interval ? -1 : 1;
  if (a->g != b->g) return a->g < b->g ? -1 : 1;
  return 0;
}

/* ---- candidate list, sorted into the canonical output order ------------------------------------------- */
typedef struct {
  loc L;
  uint32_t kind;
  uint64_t i, j;
} cand;

static int cand_cmp(const void *pa, const void *pb) {
  const cand *a = (const cand *)pa, *b = (const cand *)pb;
  int c = loc_cmp(&a->L, &b->L);
  if (c) return c;
  if (a->kind != b->kind) return a->kind < b->kind ? -1 : 1;
  if (a->i != b->i) return a->i < b->i ? -1 : 1;
  if (a->j != b->j) return a->j < b->j ? -1 : 1;
  return 0;
}

typedef struct {
  cand *v;
  uint64_t n, cap;
} cvec;

static int cpush(cvec *c, cand x) {
  if (c->n == c->cap) {
    uint64_t nc = c->cap ? c->cap * 2 : 1024;
    cand *nv = (cand *)realloc(c->v, nc * sizeof(cand));
    if (!nv) return -1;
    c->v = nv;
    c->cap = nc;
  }
  c->v[c->n++] = x;
  return 0;
}

/* sorted candidates -> one race per (λ, kind), the first (= lexicographically smallest (i, j)) of each */
static int emit_sorted(cvec *c, uint32_t G, uint64_t base, orace *out, uint64_t cap, uint64_t *nout) {
  qsort(c->v, c->n, sizeof(cand), cand_cmp);
  uint64_t k = 0;
  for (uint64_t a = 0; a < c->n; a++) {
    if (a > 0 && loc_cmp(&c->v[a].L, &c->v[a - 1].L) == 0 && c->v[a].kind == c->v[a - 1].kind) continue;
    if (k < cap) {
      orace *o = &out[k];
      memset(o, 0, sizeof(*o));
      o->addr = c->v[a].L.g * (uint64_t)G;
      o->first = base + c->v[a].i;
      o->second = base + c->v[a].j;
      o->block = c->v[a].L.block;
      o->interval = c->v[a].L.interval;
      o->space = (uint8_t)c->v[a].L.space;
      o->kind = (uint8_t)c->v[a].kind;
      o->epoch = c->v[a].L.epoch;
    }
    k++;
  }
  *nout = k;
  return k > cap ? 7 : 0;
}

/* ---- checker 1: brute force over all pairs ---------------------------------------------------------------
 * return 0 ok, 1 invalid record (*nout = bad index), 2 bad config, 3 no memory, 7 truncated */
/* epoch: per-record kernel launch (NULL: one launch) */
#define EP(i) (epoch ? epoch[i] : 0u)
int oracle_check_brute_ep(const orec *r, const uint32_t *epoch, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls,
                          uint32_t G, uint32_t flags, orace *out, uint64_t cap, uint64_t *nout) {
  if (!oracle_config_ok(ws, ls, G) || (flags & ~F_BENIGN)) return 2;
  uint64_t bad;
  if (oracle_validate(r, n, &bad)) {
    *nout = bad;
    return 1;
  }
  cvec c = {0, 0, 0};
  for (uint64_t i = 0; i < n; i++) {
    uint64_t ilo, ihi;
    granules(&r[i], G, &ilo, &ihi);
    for (uint64_t j = i + 1; j < n; j++) {
      if (EP(i) != EP(j)) continue; /* different launches are ordered (reading R23) */
      if (r[i].space != r[j].space) continue;
      /* shared memory is per block and λ includes the interval */
      if (r[i].space == SH && (r[i].block != r[j].block || r[i].interval != r[j].interval)) continue;
      uint64_t jlo, jhi;
      granules(&r[j], G, &jlo, &jhi);
      uint64_t lo = ilo > jlo ? ilo : jlo, hi = ihi < jhi ? ihi : jhi;
      if (lo > hi) continue; /* no common granule */
      int kind = oracle_pair_kind(&r[i], &r[j], ws, ls);
      if (!kind && (flags & F_BENIGN) && oracle_benign_pair(&r[i], &r[j])) kind = K_WWB;
      if (!kind) continue;
      for (uint64_t g = lo; g <= hi; g++) {
        cand x;
        x.L = loc_of(&r[i], g, EP(i));
        x.kind = (uint32_t)kind;
        x.i = i;
        x.j = j;
        if (cpush(&c, x)) {
          free(c.v);
          return 3;
        }
      }
    }
  }
  int rc = emit_sorted(&c, G, base, out, cap, nout);
  free(c.v);
  return rc;
}

int oracle_check_brute(const orec *r, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls, uint32_t G,
                       uint32_t flags, orace *out, uint64_t cap, uint64_t *nout) {
  return oracle_check_brute_ep(r, NULL, n, base, ws, ls, G, flags, out, cap, nout);
}

/* ---- checker 2: group by location, count partners --------------------------------------------------------- */
typedef struct {
  loc L;
  uint64_t idx; /* record index */
} entry;

static int entry_cmp(const void *pa, const void *pb) {
  const entry *a = (const entry *)pa, *b = (const entry *)pb;
  int c = loc_cmp(&a->L, &b->L);
  if (c) return c;
  return a->idx < b->idx ? -1 : (a->idx > b->idx ? 1 : 0);
}

/* tuple of the fields the partner counts are keyed on */
typedef struct {
  uint64_t f[6];
} tup;
static int tup_cmp_n(const tup *a, const tup *b, int nf) {
  for (int k = 0; k < nf; k++)
    if (a->f[k] != b->f[k]) return a->f[k] < b->f[k] ? -1 : 1;
  return 0;
}
/* qsort has no context argument: one comparator per field count (no global state, so worker threads of
 * oracle_check_partitioned can sort concurrently) */
static int tup_cmp4(const void *pa, const void *pb) { return tup_cmp_n((const tup *)pa, (const tup *)pb, 4); }
static int tup_cmp5(const void *pa, const void *pb) { return tup_cmp_n((const tup *)pa, (const tup *)pb, 5); }

/* number of tuples in sorted array a[0..k) whose first nf fields equal q's */
static uint64_t count_prefix(const tup *a, uint64_t k, const tup *q, int nf) {
  uint64_t lo = 0, hi = k; /* lower bound */
  while (lo < hi) {
    uint64_t m = (lo + hi) / 2;
    if (tup_cmp_n(&a[m], q, nf) < 0) lo = m + 1; else hi = m;
  }
  uint64_t first = lo;
  hi = k; /* upper bound */
  while (lo < hi) {
    uint64_t m = (lo + hi) / 2;
    if (tup_cmp_n(&a[m], q, nf) <= 0) lo = m + 1; else hi = m;
  }
  return lo - first;
}

/* Per group (all entries at one λ), counts of partners of entry r by inclusion-exclusion:
 *   OB(X)  = #type-X entries in other blocks            = C[X] - C[X,b]         (0 for a shared λ: one block)
 *   ST(X)  = #type-X, same (block,interval), other thread = C[X,b,i] - C[X,b,i,t]
 *   SW(X)  = #type-X, same (block,interval), other warp   = C[X,b,i] - C[X,b,i,w]
 *   EQ     = #plain-W partners with the same value_hash that are otherwise unordered partners of r
 *          = (C[W,v] - C[W,v,b]) + (C[W,v,b,i] - C[W,v,b,i,t])
 * (same block, other interval is ordered for global memory and impossible for shared: never counted.)
 *   RW(r)  = r read:  Σ_{X∈{W,A}} OB(X) + (ls ? SW(X) : ST(X));  r write/atomic: OB(R) + (ls ? SW(R) : ST(R))
 *   WW(r)  = r write: OB(A)+ST(A) + OB(W)+ST(W) - EQ;  r atomic: OB(W)+ST(W);  r read: 0
 *   B(r)   = r write: EQ (its benign partners, oracle_benign_pair);  otherwise 0                              */
typedef struct {
  const orec *r;
  const entry *e;
  uint64_t k;
  uint32_t ws, ls;
  tup *A, *B, *V;
  uint8_t *flag_rw, *flag_ww, *flag_b;
  uint64_t a0, a1; /* entries this worker flags */
  tup *sort_arr;   /* sort worker: the array and its field count */
  int sort_nf;
} gjob;

/* the counts and flags of entries [a0, a1) of one group (A, B, V sorted) */
static void flags_range(const gjob *g) {
  const orec *r = g->r;
  const entry *e = g->e;
  const uint64_t k = g->k;
  const uint32_t ws = g->ws, ls = g->ls;
  const tup *A = g->A, *B = g->B, *V = g->V;
  for (uint64_t a = g->a0; a < g->a1; a++) {
    const orec *x = &r[e[a].idx];
    uint64_t OB[3], ST[3], SW[3];
    for (int X = 0; X < 3; X++) {
      tup q; memset(&q, 0, sizeof q);
      q.f[0] = (uint64_t)X; q.f[1] = x->block; q.f[2] = x->interval; q.f[3] = x->thread;
      uint64_t cX = count_prefix(A, k, &q, 1), cXb = count_prefix(A, k, &q, 2);
      uint64_t cXbi = count_prefix(A, k, &q, 3), cXbit = count_prefix(A, k, &q, 4);
      tup qw = q; qw.f[3] = x->thread / ws;
      uint64_t cXbiw = count_prefix(B, k, &qw, 4);
      OB[X] = cX - cXb;
      ST[X] = cXbi - cXbit;
      SW[X] = cXbi - cXbiw;
    }
    uint64_t rw = 0, ww = 0, eq = 0;
    if (x->rw == RD) {
      rw = OB[WR] + (ls ? SW[WR] : ST[WR]) + OB[AT] + (ls ? SW[AT] : ST[AT]);
    } else {
      rw = OB[RD] + (ls ? SW[RD] : ST[RD]);
    }
    if (x->rw == WR) {
      tup q; memset(&q, 0, sizeof q);
      q.f[0] = WR; q.f[1] = x->value_hash; q.f[2] = x->block; q.f[3] = x->interval; q.f[4] = x->thread;
      uint64_t cv = count_prefix(V, k, &q, 2), cvb = count_prefix(V, k, &q, 3);
      uint64_t cvbi = count_prefix(V, k, &q, 4), cvbit = count_prefix(V, k, &q, 5);
      eq = (cv - cvb) + (cvbi - cvbit);
      ww = OB[AT] + ST[AT] + OB[WR] + ST[WR] - eq;
    } else if (x->rw == AT) {
      ww = OB[WR] + ST[WR];
    }
    g->flag_rw[a] = rw > 0;
    g->flag_ww[a] = ww > 0;
    g->flag_b[a] = eq > 0;
  }
}

static void *flags_worker(void *arg) {
  flags_range((const gjob *)arg);
  return NULL;
}
static void *sort_worker(void *arg) {
  gjob *g = (gjob *)arg;
  qsort(g->sort_arr, g->k, sizeof(tup), g->sort_nf == 5 ? tup_cmp5 : tup_cmp4);
  return NULL;
}

/* Groups this large are sorted and counted by `par` threads (the arithmetic is unchanged: the three sorts
 * are independent and every entry's counts only read the sorted arrays). */
#define GROUP_PAR_MIN (1u << 20)

static int group_flags(const orec *r, const entry *e, uint64_t k, uint32_t ws, uint32_t ls, uint8_t *flag_rw,
                       uint8_t *flag_ww, uint8_t *flag_b, uint32_t par) {
  tup *A = (tup *)malloc(k * sizeof(tup)); /* (type, block, interval, thread) */
  tup *B = (tup *)malloc(k * sizeof(tup)); /* (type, block, interval, warp)   */
  tup *V = (tup *)malloc(k * sizeof(tup)); /* (type, value, block, interval, thread) */
  if (!A || !B || !V) {
    free(A); free(B); free(V);
    return 3;
  }
  for (uint64_t a = 0; a < k; a++) {
    const orec *x = &r[e[a].idx];
    memset(&A[a], 0, sizeof(tup));
    memset(&B[a], 0, sizeof(tup));
    memset(&V[a], 0, sizeof(tup));
    A[a].f[0] = x->rw; A[a].f[1] = x->block; A[a].f[2] = x->interval; A[a].f[3] = x->thread;
    B[a].f[0] = x->rw; B[a].f[1] = x->block; B[a].f[2] = x->interval; B[a].f[3] = x->thread / ws;
    V[a].f[0] = x->rw; V[a].f[1] = x->value_hash; V[a].f[2] = x->block; V[a].f[3] = x->interval;
    V[a].f[4] = x->thread;
  }
  gjob g;
  memset(&g, 0, sizeof g);
  g.r = r; g.e = e; g.k = k; g.ws = ws; g.ls = ls; g.A = A; g.B = B; g.V = V;
  g.flag_rw = flag_rw; g.flag_ww = flag_ww; g.flag_b = flag_b;
  if (par <= 1 || k < GROUP_PAR_MIN) {
    qsort(A, k, sizeof(tup), tup_cmp4);
    qsort(B, k, sizeof(tup), tup_cmp4);
    qsort(V, k, sizeof(tup), tup_cmp5);
    g.a0 = 0; g.a1 = k;
    flags_range(&g);
  } else {
    gjob s[3];
    pthread_t th[64];
    tup *arr[3] = {A, B, V};
    for (int q = 0; q < 3; q++) {
      s[q] = g;
      s[q].sort_arr = arr[q];
      s[q].sort_nf = q == 2 ? 5 : 4;
    }
    int ok[3];
    for (int q = 1; q < 3; q++) ok[q] = pthread_create(&th[q], NULL, sort_worker, &s[q]) == 0;
    sort_worker(&s[0]);
    for (int q = 1; q < 3; q++) {
      if (ok[q]) pthread_join(th[q], NULL);
      else sort_worker(&s[q]);
    }
    const uint32_t P = par > 64 ? 64 : par;
    gjob w[64];
    for (uint32_t t = 0; t < P; t++) {
      w[t] = g;
      w[t].a0 = k * t / P;
      w[t].a1 = k * (t + 1) / P;
    }
    int okw[64];
    for (uint32_t t = 1; t < P; t++) okw[t] = pthread_create(&th[t], NULL, flags_worker, &w[t]) == 0;
    flags_range(&w[0]);
    for (uint32_t t = 1; t < P; t++) {
      if (okw[t]) pthread_join(th[t], NULL);
      else flags_range(&w[t]);
    }
  }
  free(A); free(B); free(V);
  return 0;
}

/* Entries e[0..m) sorted by (λ, record index): per group (all entries at one λ) flags by counting, then the
 * canonical witness per kind; candidates are appended to *c.  Returns 0, 3 (no memory) or 9 (counting bug). */
static int process_groups(const orec *r, const entry *e, uint64_t m, uint32_t ws, uint32_t ls, uint32_t flags,
                          uint32_t par, cvec *c) {
  int rc = 0;
  uint8_t *frw = NULL, *fww = NULL, *fb = NULL;
  uint64_t fcap = 0;
  for (uint64_t a = 0; a < m && rc == 0;) {
    uint64_t b = a + 1;
    while (b < m && loc_cmp(&e[b].L, &e[a].L) == 0) b++;
    uint64_t k = b - a; /* group [a, b): every entry at one λ, ascending record index */
    if (k >= 2) {
      if (k > fcap) {
        free(frw); free(fww); free(fb);
        frw = (uint8_t *)malloc(k); fww = (uint8_t *)malloc(k); fb = (uint8_t *)malloc(k);
        fcap = k;
        if (!frw || !fww || !fb) { rc = 3; break; }
      }
      rc = group_flags(r, &e[a], k, ws, ls, frw, fww, fb, par);
      if (rc) break;
      const int kmax = (flags & F_BENIGN) ? K_WWB : K_WW;
      for (int K = K_RW; K <= kmax; K++) {
        const uint8_t *fl = K == K_RW ? frw : K == K_WW ? fww : fb;
        uint64_t xa = UINT64_MAX; /* x = min flagged record index (entries are index-ascending) */
        for (uint64_t q = 0; q < k; q++)
          if (fl[q]) { xa = q; break; }
        if (xa == UINT64_MAX) continue;
        const orec *x = &r[e[a + xa].idx];
        uint64_t y = UINT64_MAX; /* y = min partner of x of kind K */
        for (uint64_t q = 0; q < k; q++) {
          if (q == xa) continue;
          const orec *sq = &r[e[a + q].idx];
          if (K == K_WWB ? oracle_benign_pair(x, sq) : oracle_pair_kind(x, sq, ws, ls) == K) {
            y = e[a + q].idx;
            break;
          }
        }
        if (y == UINT64_MAX) { rc = 9; break; } /* a flag without a partner: counting bug */
        cand cd;
        cd.L = e[a].L;
        cd.kind = (uint32_t)K;
        cd.i = e[a + xa].idx < y ? e[a + xa].idx : y;
        cd.j = e[a + xa].idx < y ? y : e[a + xa].idx;
        if (cpush(c, cd)) { rc = 3; break; }
      }
    }
    a = b;
  }
  free(frw); free(fww); free(fb);
  return rc;
}

/* hash of a location λ (splitmix64 finaliser, the same mix as oracle_expand's value hash) */
static uint64_t mix(uint64_t x);
static uint64_t loc_hash(const loc *L) {
  return mix(mix(mix(mix(((uint64_t)L->space << 32) ^ L->block) ^ L->interval) ^ L->g) ^ L->epoch);
}

/* Entries of the records whose location hash falls in partition `part` of `nparts` (nparts == 1: every entry),
 * sorted by (λ, record index); *m_out = count.  NULL on no memory (*m_out = UINT64_MAX). */
static entry *collect_entries(const orec *r, const uint32_t *epoch, uint64_t n, uint32_t G, uint32_t part,
                              uint32_t nparts, uint64_t *m_out) {
  uint64_t m = 0;
  for (uint64_t i = 0; i < n; i++) {
    uint64_t lo, hi;
    granules(&r[i], G, &lo, &hi);
    for (uint64_t g = lo; g <= hi; g++) {
      if (nparts > 1) {
        loc L = loc_of(&r[i], g, EP(i));
        if (loc_hash(&L) % nparts != part) continue;
      }
      m++;
    }
  }
  entry *e = (entry *)malloc((m ? m : 1) * sizeof(entry));
  if (!e) {
    *m_out = UINT64_MAX;
    return NULL;
  }
  uint64_t p = 0;
  for (uint64_t i = 0; i < n; i++) {
    uint64_t lo, hi;
    granules(&r[i], G, &lo, &hi);
    for (uint64_t g = lo; g <= hi; g++) {
      loc L = loc_of(&r[i], g, EP(i));
      if (nparts > 1 && loc_hash(&L) % nparts != part) continue;
      e[p].L = L;
      e[p].idx = i;
      p++;
    }
  }
  qsort(e, m, sizeof(entry), entry_cmp);
  *m_out = m;
  return e;
}

int oracle_check_grouped_ep(const orec *r, const uint32_t *epoch, uint64_t n, uint64_t base, uint32_t ws,
                            uint32_t ls, uint32_t G, uint32_t flags, orace *out, uint64_t cap, uint64_t *nout) {
  if (!oracle_config_ok(ws, ls, G) || (flags & ~F_BENIGN)) return 2;
  uint64_t bad;
  if (oracle_validate(r, n, &bad)) {
    *nout = bad;
    return 1;
  }
  /* entries = (record, granule) pairs, grouped by location */
  uint64_t m = 0;
  entry *e = collect_entries(r, epoch, n, G, 0, 1, &m);
  if (!e) return 3;
  cvec c = {0, 0, 0};
  int rc = process_groups(r, e, m, ws, ls, flags, 1, &c);
  free(e);
  if (rc) {
    free(c.v);
    return rc;
  }
  rc = emit_sorted(&c, G, base, out, cap, nout);
  free(c.v);
  return rc;
}

int oracle_check_grouped(const orec *r, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls, uint32_t G,
                         uint32_t flags, orace *out, uint64_t cap, uint64_t *nout) {
  return oracle_check_grouped_ep(r, NULL, n, base, ws, ls, G, flags, out, cap, nout);
}

/* ---- checker 2, T threads: the locations are partitioned by loc_hash mod T (SURVEY §8c.3 "T-thread mode").
 * A race is a property of one location (c.1), so every group lands whole in one partition and each thread
 * runs the unchanged group algorithm on its partition; the candidate lists are concatenated and emitted in
 * the canonical order.  The result is byte-identical to oracle_check_grouped (tests/test_oracle.py).       */
typedef struct {
  const orec *r;
  const uint32_t *epoch;
  uint64_t n;
  uint32_t ws, ls, G, flags, part, nparts;
  cvec c;
  int rc;
} pjob;

static void *pworker(void *arg) {
  pjob *j = (pjob *)arg;
  uint64_t m = 0;
  entry *e = collect_entries(j->r, j->epoch, j->n, j->G, j->part, j->nparts, &m);
  if (!e) {
    j->rc = 3;
    return NULL;
  }
  j->rc = process_groups(j->r, e, m, j->ws, j->ls, j->flags, j->nparts, &j->c);
  free(e);
  return NULL;
}

int oracle_check_partitioned_ep(const orec *r, const uint32_t *epoch, uint64_t n, uint64_t base, uint32_t ws,
                                uint32_t ls, uint32_t G, uint32_t flags, uint32_t T, orace *out, uint64_t cap,
                                uint64_t *nout) {
  if (!oracle_config_ok(ws, ls, G) || (flags & ~F_BENIGN)) return 2;
  if (T < 1) T = 1;
  if (T > 1024) T = 1024;
  uint64_t bad;
  if (oracle_validate(r, n, &bad)) {
    *nout = bad;
    return 1;
  }
  pjob *jobs = (pjob *)calloc(T, sizeof(pjob));
  pthread_t *th = (pthread_t *)calloc(T, sizeof(pthread_t));
  if (!jobs || !th) {
    free(jobs); free(th);
    return 3;
  }
  for (uint32_t t = 0; t < T; t++) {
    jobs[t].r = r; jobs[t].epoch = epoch; jobs[t].n = n; jobs[t].ws = ws; jobs[t].ls = ls; jobs[t].G = G; jobs[t].flags = flags;
    jobs[t].part = t; jobs[t].nparts = T;
  }
  for (uint32_t t = 1; t < T; t++)
    if (pthread_create(&th[t], NULL, pworker, &jobs[t]) != 0) jobs[t].rc = -1;
  pworker(&jobs[0]);
  int rc = jobs[0].rc;
  for (uint32_t t = 1; t < T; t++) {
    if (jobs[t].rc == -1) { pworker(&jobs[t]); } /* thread creation failed: run it here */
    else pthread_join(th[t], NULL);
    if (jobs[t].rc && !rc) rc = jobs[t].rc;
  }
  cvec c = {0, 0, 0};
  for (uint32_t t = 0; t < T && !rc; t++)
    for (uint64_t q = 0; q < jobs[t].c.n && !rc; q++)
      if (cpush(&c, jobs[t].c.v[q])) rc = 3;
  for (uint32_t t = 0; t < T; t++) free(jobs[t].c.v);
  free(jobs); free(th);
  if (rc) {
    free(c.v);
    return rc;
  }
  rc = emit_sorted(&c, G, base, out, cap, nout);
  free(c.v);
  return rc;
}

int oracle_check_partitioned(const orec *r, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls, uint32_t G,
                             uint32_t flags, uint32_t T, orace *out, uint64_t cap, uint64_t *nout) {
  return oracle_check_partitioned_ep(r, NULL, n, base, ws, ls, G, flags, T, out, cap, nout);
}

/* ---- precise warp model (reading R24) -------------------------------------------
 * Each record carries an extension {pc, div}: pc = the static instruction that made the access; div = 0 when the
 * thread's warp was convergent at that instruction, else (branch instance << 1 | side) of the divergent branch
 * region containing it (innermost region).  P:281 (§IV-B): "threads within a warp are executed in a lock-step
 * manner: two intra-warp threads can race only if they simultaneously write to the same shared variable at the
 * same instruction.  In case of divergence, we execute the two sides sequentially ... the executor has to
 * enumerate both orders"; P:87 (§II): the divergent read/write of race() is a race "no matter whether t1 and t2
 * are within a warp".  So, with lockstep on, for two threads of one warp (same block, same interval):
 *   - on the two sides of one divergent branch instance: both orders of the sides occur -> unordered, rules 1-4
 *     and 6 decide as without lockstep ("both orders");
 *   - otherwise lockstep orders them, except two writes at the same instruction (simultaneous): then a
 *     W/W race (benign filter 6 still applies); every other intra-warp pair is exempt.
 * With lockstep off the extension is ignored.  With every pc equal and every div 0 this is exactly rule (5) of
 * oracle_pair_kind (intra-warp pairs with a read exempt, intra-warp writes kept).                            */
typedef struct {
  uint32_t pc, div;
} oext;

int oracle_pair_kind_warp(const orec *r, const orec *s, const oext *er, const oext *es, uint32_t ws, uint32_t ls) {
  if (r->block == s->block && r->thread == s->thread) return 0;                        /* (1) */
  if (r->rw == RD && s->rw == RD) return 0;                                            /* (2) */
  if (r->rw == AT && s->rw == AT) return 0;                                            /* (3) */
  if (r->space == GL && r->block == s->block && r->interval != s->interval) return 0;   /* (4) */
  int kind = (r->rw == RD || s->rw == RD) ? K_RW : K_WW;
  if (ls && r->block == s->block && r->interval == s->interval && r->thread / ws == s->thread / ws) {
    const int divergent = er->div != 0 && es->div != 0 && (er->div >> 1) == (es->div >> 1) &&
                          (er->div & 1) != (es->div & 1);
    if (!divergent && (kind == K_RW || er->pc != es->pc)) return 0;                    /* (5') */
  }
  if (r->rw == WR && s->rw == WR && r->value_hash == s->value_hash) return 0;           /* (6) */
  return kind;
}

/* brute force over all pairs (the definition); returns like oracle_check_brute (no benign flag) */
int oracle_check_warp_brute(const orec *r, const oext *ext, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls,
                            uint32_t G, orace *out, uint64_t cap, uint64_t *nout) {
  if (!oracle_config_ok(ws, ls, G)) return 2;
  uint64_t bad;
  if (oracle_validate(r, n, &bad)) {
    *nout = bad;
    return 1;
  }
  cvec c = {0, 0, 0};
  for (uint64_t i = 0; i < n; i++) {
    uint64_t ilo, ihi;
    granules(&r[i], G, &ilo, &ihi);
    for (uint64_t j = i + 1; j < n; j++) {
      if (r[i].space != r[j].space) continue;
      if (r[i].space == SH && (r[i].block != r[j].block || r[i].interval != r[j].interval)) continue;
      uint64_t jlo, jhi;
      granules(&r[j], G, &jlo, &jhi);
      uint64_t lo = ilo > jlo ? ilo : jlo, hi = ihi < jhi ? ihi : jhi;
      if (lo > hi) continue;
      const int kind = oracle_pair_kind_warp(&r[i], &r[j], &ext[i], &ext[j], ws, ls);
      if (!kind) continue;
      for (uint64_t g = lo; g <= hi; g++) {
        cand x;
        x.L = loc_of(&r[i], g, 0);
        x.kind = (uint32_t)kind;
        x.i = i;
        x.j = j;
        if (cpush(&c, x)) {
          free(c.v);
          return 3;
        }
      }
    }
  }
  int rc = emit_sorted(&c, G, base, out, cap, nout);
  free(c.v);
  return rc;
}

/* grouped by location, then every pair of the group in lexicographic (i, j) order: the first racing pair of a
 * kind is its witness (O(sum of group sizes squared); an independent organisation of the same definition) */
int oracle_check_warp_grouped(const orec *r, const oext *ext, uint64_t n, uint64_t base, uint32_t ws, uint32_t ls,
                              uint32_t G, orace *out, uint64_t cap, uint64_t *nout) {
  if (!oracle_config_ok(ws, ls, G)) return 2;
  uint64_t bad;
  if (oracle_validate(r, n, &bad)) {
    *nout = bad;
    return 1;
  }
  uint64_t m = 0;
  entry *e = collect_entries(r, NULL, n, G, 0, 1, &m);
  if (!e) return 3;
  cvec c = {0, 0, 0};
  int rc = 0;
  for (uint64_t a = 0; a < m && !rc;) {
    uint64_t b = a + 1;
    while (b < m && loc_cmp(&e[b].L, &e[a].L) == 0) b++;
    int found[3] = {0, 0, 0};
    for (uint64_t x = a; x < b && !(found[K_RW] && found[K_WW]) && !rc; x++)
      for (uint64_t y = x + 1; y < b; y++) {
        const uint64_t i = e[x].idx, j = e[y].idx;
        const int kind = oracle_pair_kind_warp(&r[i], &r[j], &ext[i], &ext[j], ws, ls);
        if (!kind || found[kind]) continue;
        found[kind] = 1;
        cand cd;
        cd.L = e[a].L;
        cd.kind = (uint32_t)kind;
        cd.i = i;
        cd.j = j;
        if (cpush(&c, cd)) { rc = 3; break; }
      }
    a = b;
  }
  free(e);
  if (rc) {
    free(c.v);
    return rc;
  }
  rc = emit_sorted(&c, G, base, out, cap, nout);
  free(c.v);
  return rc;
}

/* ---- parametric flow instantiation (replace thread id i by j in the race history) ---------- */
static uint64_t mix(uint64_t x) { /* splitmix64 finaliser, as documented in include/sesa.h */
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

static int flow_active(const oflow *f, uint32_t t) {
  if (t >= f->nthreads) return 0;
  if ((t & f->pmask) != f->pval) return 0;
  if (f->pmod != 0 && t % f->pmod != f->prem) return 0;
  if (t < f->plo || t >= f->phi) return 0;
  return 1;
}

static uint64_t flow_f(const oflow *f, uint32_t t) {
  switch (f->fkind) {
    case 0: return t;
    case 1: return ((uint64_t)t + f->fc) % f->fm;
    case 2: return (uint64_t)(t ^ f->fc);
    case 3: return (uint64_t)(t >> f->fc);
    default: return (uint64_t)(t >> f->fc) * f->fm + (uint64_t)(t & ((1u << f->fc) - 1u)); /* row-major 2-D */
  }
}

/* Writes up to cap records in canonical-schedule order (block, interval, thread, descriptor, k); returns the
 * total count (which may exceed cap: then only cap were written).  Returns UINT64_MAX on a bad descriptor
 * (fkind > 4, MODADD with fm == 0, SHR/ROW2D with fc >= 32). */
uint64_t oracle_expand(const oflow *fl, uint64_t nf, orec *out, uint64_t cap) {
  if (nf == 0) return 0;
  uint32_t bmin = UINT32_MAX, bmax = 0, tmax = 0;
  for (uint64_t d = 0; d < nf; d++) {
    if (fl[d].fkind > 4 || (fl[d].fkind == 1 && fl[d].fm == 0) || (fl[d].fkind >= 3 && fl[d].fc >= 32))
      return UINT64_MAX;
    if (fl[d].block_lo >= fl[d].block_hi) continue;
    if (fl[d].block_lo < bmin) bmin = fl[d].block_lo;
    if (fl[d].block_hi > bmax) bmax = fl[d].block_hi;
    if (fl[d].nthreads > tmax) tmax = fl[d].nthreads;
  }
  if (bmin >= bmax) return 0;
  /* distinct intervals, ascending */
  uint32_t *iv = (uint32_t *)malloc(nf * sizeof(uint32_t));
  uint64_t niv = 0;
  for (uint64_t d = 0; d < nf; d++) {
    uint64_t q = 0;
    while (q < niv && iv[q] != fl[d].interval) q++;
    if (q == niv) iv[niv++] = fl[d].interval;
  }
  for (uint64_t a = 1; a < niv; a++) /* insertion sort */
    for (uint64_t b = a; b > 0 && iv[b - 1] > iv[b]; b--) {
      uint32_t tmp = iv[b]; iv[b] = iv[b - 1]; iv[b - 1] = tmp;
    }
  uint64_t k = 0;
  for (uint64_t b = bmin; b < bmax; b++)
    for (uint64_t q = 0; q < niv; q++)
      for (uint32_t t = 0; t < tmax; t++)
        for (uint64_t d = 0; d < nf; d++) {
          const oflow *f = &fl[d];
          if (f->interval != iv[q] || b < f->block_lo || b >= f->block_hi || !flow_active(f, t)) continue;
          for (uint32_t c = 0; c < f->count; c++) {
            if (k < cap) {
              orec *o = &out[k];
              memset(o, 0, sizeof(*o));
              o->addr = f->base + (uint64_t)f->bstride * b + (uint64_t)f->tstride * flow_f(f, t) +
                        (uint64_t)f->istride * c;
              o->value_hash = f->rw != WR ? 0 : (f->flags & 1) ? f->value_seed : mix(mix(mix(f->value_seed ^ b) ^ t) ^ c);
              o->block = (uint32_t)b;
              o->thread = t;
              o->interval = f->interval;
              o->size = f->size;
              o->space = f->space;
              o->rw = f->rw;
            }
            k++;
          }
        }
  free(iv);
  return k;
}

/* sizes, so the Python loader can assert the layouts */
uint64_t oracle_sizeof_rec(void) { return sizeof(orec); }
uint64_t oracle_sizeof_race(void) { return sizeof(orace); }
uint64_t oracle_sizeof_flow(void) { return sizeof(oflow); }
