// k_conflict.cu — segmented conflict detection over the sorted entries (SURVEY §8a rows a5 + a6).
//
// After the sort, every location λ is one contiguous run ("group") of keys; for a global location the entries
// of one (block, interval) are a contiguous "sub-run".  The paper instantiates a barrier interval's read/write
// sets at two thread ids t1 != t2 and asks the solver whether an address can coincide.
// Concretely that is: does entry e have a partner s in its group with P(e, s) (include/sesa.h rules 1-6)?
// We answer it without enumerating pairs, from per-group and per-sub-run summaries ("Agg"):
//   per access type X in {READ, WRITE, ATOMIC}: min/max identity  (identity = thread in a sub-run, block in a
//   group) -> "exists an X with identity != mine" / "exists an X in another warp" (lockstep);
//   for plain writes: min and max value hash with the identity attaining them, plus the min (max) over the
//   OTHER identities -> "exists a write with identity != mine AND value != mine" (benign W/W filter).
// flag_K(e) = partner of kind K exists; witness x_K = min flagged position of the group, y_K = min position s
// with P(x_K, s) of kind K (lexicographic minimum, reading R12).
//
// A CTA owns a window of up to CT_TILE = 1536 sorted entries (below).  Summaries are computed with a per-thread fold
// over its CT_ITEMS = 6 entries
// plus block-wide segmented scans of the per-thread folds (warp shuffles), forward and backward, so each entry
// receives the total of its segment without storing per-entry summaries.  Runs that cross a tile boundary
// (hot locations: C3 bins, C4 `changed`) are completed in three extra steps:
//   mode 1 (every tile): internal groups -> races; crossing pieces -> per-tile partial summaries
//   carry  (k_carry)    : segmented scans over the tile partials -> full incoming/outgoing summaries
//   mode 2 (crossing tiles): exact flags of crossing entries -> atomicMin x into the owner tile's slot
//   mode 3 (crossing tiles): atomicMin y;  cross_emit: one race per (crossing group, kind)
// Only entries of groups with >= 2 entries gather their 32-byte record (by position); singletons — all but
// 2e5 of C5's 1e9 entries — cost 8 bytes of key traffic.
#include "kernels.cuh"

#ifndef CT_UNROLL
#define CT_UNROLL 1
#endif

namespace sesa {
constexpr int kCtUnroll = CT_UNROLL;

// ------------------------------------------------------------------------------------------------ summaries
__device__ __forceinline__ Agg agg_empty() {
  Agg r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = ~0u, r.mx[x] = 0u;
  r.i1 = r.i2 = ~0u;
  r.v1 = r.v1b = ~0ull;
  r.v2 = r.v2b = 0ull;
  return r;
}

// (per-type fields set by selects: an index by the runtime access type would put the summary in local memory)
__device__ __forceinline__ Agg agg_item(u32 rw, u32 id, u64 vh) {
  Agg r = agg_empty();
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = rw == (u32)x ? id : ~0u, r.mx[x] = rw == (u32)x ? id : 0u;
  if (rw == RW_WRITE) {
    r.v1 = r.v2 = vh;
    r.i1 = r.i2 = id;
  }
  return r;
}

__device__ __forceinline__ Agg agg_merge(const Agg& a, const Agg& b) {
  Agg r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = min(a.mn[x], b.mn[x]), r.mx[x] = max(a.mx[x], b.mx[x]);
  const bool ae = a.mn[RW_WRITE] > a.mx[RW_WRITE], be = b.mn[RW_WRITE] > b.mx[RW_WRITE];
  if (ae || be) {
    const Agg& s = ae ? b : a;
    r.i1 = s.i1, r.i2 = s.i2, r.v1 = s.v1, r.v1b = s.v1b, r.v2 = s.v2, r.v2b = s.v2b;
    return r;
  }
  if (b.v1 < a.v1) {
    r.v1 = b.v1, r.i1 = b.i1;
    r.v1b = min(b.v1b, a.i1 != b.i1 ? a.v1 : a.v1b);
  } else {
    r.v1 = a.v1, r.i1 = a.i1;
    r.v1b = min(a.v1b, b.i1 != a.i1 ? b.v1 : b.v1b);
  }
  if (b.v2 > a.v2) {
    r.v2 = b.v2, r.i2 = b.i2;
    r.v2b = max(b.v2b, a.i2 != b.i2 ? a.v2 : a.v2b);
  } else {
    r.v2 = a.v2, r.i2 = a.i2;
    r.v2b = max(a.v2b, b.i2 != a.i2 ? b.v2 : b.v2b);
  }
  return r;
}

// "exists an entry of type X with identity != id"
__device__ __forceinline__ bool ex_id(const Agg& S, int X, u32 id) { return S.mn[X] < id || S.mx[X] > id; }
// "exists an entry of type X in another warp" (warp = thread / ws)
__device__ __forceinline__ bool ex_warp(const Agg& S, int X, u32 w, u32 ws) {
  return S.mn[X] <= S.mx[X] && (S.mn[X] / ws < w || S.mx[X] / ws > w);
}
// "exists a plain write with identity != id and value != v"
__device__ __forceinline__ bool ex_wval(const Agg& S, u32 id, u64 v) {
  if (!ex_id(S, RW_WRITE, id)) return false;
  const u64 lo = S.i1 != id ? S.v1 : S.v1b;
  const u64 hi = S.i2 != id ? S.v2 : S.v2b;
  return lo != v || hi != v;
}

// tri-state "exists a plain write with identity != id and value != v": 0 no, 1 yes, 2 unknown (never for Agg)
__device__ __forceinline__ int wval3(const Agg& S, u32 id, u64 v) { return ex_wval(S, id, v) ? 1 : 0; }

struct OpAgg {
  __device__ __forceinline__ Agg operator()(const Agg& a, const Agg& b) const { return agg_merge(a, b); }
};

// ---- cheap summary (AggC): same identity fields, only min/max of the write values
__device__ __forceinline__ bool ex_id(const AggC& S, int X, u32 id) { return S.mn[X] < id || S.mx[X] > id; }
__device__ __forceinline__ bool ex_warp(const AggC& S, int X, u32 w, u32 ws) {
  return S.mn[X] <= S.mx[X] && (S.mn[X] / ws < w || S.mx[X] / ws > w);
}
__device__ __forceinline__ int wval3(const AggC& S, u32 id, u64 v) {
  if (!ex_id(S, RW_WRITE, id)) return 0;  // no writer with another identity
  if (S.vlo == S.vhi) return 0;           // every write of the set has one value, which is mine (I am a writer)
  return 2;                               // >= 2 identities and >= 2 values: needs the exact summary
}
struct OpAggC {
  __device__ __forceinline__ AggC operator()(const AggC& a, const AggC& b) const {
    AggC r;
#pragma unroll
    for (int x = 0; x < 3; x++) r.mn[x] = min(a.mn[x], b.mn[x]), r.mx[x] = max(a.mx[x], b.mx[x]);
    r.vlo = min(a.vlo, b.vlo);
    r.vhi = max(a.vhi, b.vhi);
    return r;
  }
};
template <class A>
__device__ __forceinline__ A agg_empty_t();
template <>
__device__ __forceinline__ Agg agg_empty_t<Agg>() { return agg_empty(); }
template <>
__device__ __forceinline__ AggC agg_empty_t<AggC>() {
  AggC r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = ~0u, r.mx[x] = 0u;
  r.vlo = ~0ull, r.vhi = 0ull;
  return r;
}
template <class A>
__device__ __forceinline__ A agg_item_t(u32 rw, u32 id, u64 vh);
template <>
__device__ __forceinline__ Agg agg_item_t<Agg>(u32 rw, u32 id, u64 vh) { return agg_item(rw, id, vh); }
template <>
__device__ __forceinline__ AggC agg_item_t<AggC>(u32 rw, u32 id, u64 vh) {
  AggC r = agg_empty_t<AggC>();
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = rw == (u32)x ? id : ~0u, r.mx[x] = rw == (u32)x ? id : 0u;
  if (rw == RW_WRITE) r.vlo = r.vhi = vh;
  return r;
}
template <class A>
struct OpOf;
template <>
struct OpOf<Agg> {
  typedef OpAgg type;
};
template <>
struct OpOf<AggC> {
  typedef OpAggC type;
};
template <class A>
struct QuadOf;
template <>
struct QuadOf<Agg> {
  typedef AggQuad type;
};
template <>
struct QuadOf<AggC> {
  typedef AggQuadC type;
};

struct X2 {
  u64 v[2];
};
struct OpX2 {
  __device__ __forceinline__ X2 operator()(const X2& a, const X2& b) const {
    X2 r;
    r.v[0] = min(a.v[0], b.v[0]);
    r.v[1] = min(a.v[1], b.v[1]);
    return r;
  }
};

// min of each 32-bit half independently (x in the low half, y in the high half)
struct OpXY {
  __device__ __forceinline__ X2 operator()(const X2& a, const X2& b) const {
    X2 r;
#pragma unroll
    for (int k = 0; k < 2; k++) {
      const u64 hi = min(a.v[k] >> 32, b.v[k] >> 32), lo = min(a.v[k] & 0xFFFFFFFFull, b.v[k] & 0xFFFFFFFFull);
      r.v[k] = (hi << 32) | lo;
    }
    return r;
  }
};

// ------------------------------------------------------------------------------------------------ shuffles
__device__ __forceinline__ u32 shfl(u32 v, int o, bool down) {
  return down ? __shfl_down_sync(~0u, v, o) : __shfl_up_sync(~0u, v, o);
}
__device__ __forceinline__ u64 shfl(u64 v, int o, bool down) {
  return down ? __shfl_down_sync(~0u, v, o) : __shfl_up_sync(~0u, v, o);
}
__device__ __forceinline__ Agg shfl(const Agg& a, int o, bool down) {
  Agg r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = shfl(a.mn[x], o, down), r.mx[x] = shfl(a.mx[x], o, down);
  r.i1 = shfl(a.i1, o, down), r.i2 = shfl(a.i2, o, down);
  r.v1 = shfl(a.v1, o, down), r.v1b = shfl(a.v1b, o, down);
  r.v2 = shfl(a.v2, o, down), r.v2b = shfl(a.v2b, o, down);
  return r;
}
__device__ __forceinline__ AggC shfl(const AggC& a, int o, bool down) {
  AggC r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = shfl(a.mn[x], o, down), r.mx[x] = shfl(a.mx[x], o, down);
  r.vlo = shfl(a.vlo, o, down), r.vhi = shfl(a.vhi, o, down);
  return r;
}
__device__ __forceinline__ X2 shfl(const X2& a, int o, bool down) {
  X2 r;
  r.v[0] = shfl(a.v[0], o, down);
  r.v[1] = shfl(a.v[1], o, down);
  return r;
}

// Block-wide exclusive segmented scan of per-thread (flag, value): flag = "a segment starts inside this
// thread's span" (in scan direction).  REV = backward (from the last thread).  carry seeds the first thread.
template <class T, class Op, bool REV, int THREADS>
__device__ __forceinline__ T block_seg_excl(bool flag, const T& val, const T& carry, Op op, T* s_wv, u8* s_wf) {
  constexpr int WARPS = THREADS / 32;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  bool f = flag;
  T v = val;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const bool f2 = __shfl_sync(~0u, (u32)f, REV ? lane + o : lane - o) != 0;
    const T v2 = shfl(v, o, REV);
    const bool has = REV ? lane + o < 32 : lane >= o;
    if (has) {
      if (!f) v = op(v2, v);
      f = f || f2;
    }
  }
  const bool fe = __shfl_sync(~0u, (u32)f, REV ? lane + 1 : lane - 1) != 0;
  const T ve = shfl(v, 1, REV);
  if (REV ? lane == 0 : lane == 31) {
    s_wv[warp] = v;
    s_wf[warp] = f;
  }
  __syncthreads();
  T wp = carry;
  if (!REV) {
    for (int w = 0; w < warp; w++) wp = s_wf[w] ? s_wv[w] : op(wp, s_wv[w]);
  } else {
    for (int w = WARPS - 1; w > warp; w--) wp = s_wf[w] ? s_wv[w] : op(wp, s_wv[w]);
  }
  const bool first = REV ? lane == 31 : lane == 0;
  T ex = first ? wp : (fe ? ve : op(wp, ve));
  __syncthreads();
  return ex;
}

// Segmented all-reduce over the tile (blocked: thread t owns items t*ITEMS .. t*ITEMS+ITEMS-1): calls
// cb(j, total of j's segment) for every item.  Segment starts/ends are bits hbit/tbit of fl[j].
template <class T, class Op, class ItemF, class CB>
__device__ __forceinline__ void tile_allreduce(const u8* fl, u8 hbit, u8 tbit, ItemF item, Op op, const T& ident,
                                               const T& carry_in, const T& carry_out, CB cb, T* s_wv, u8* s_wf) {
  const int j0 = threadIdx.x * CT_ITEMS;
  // per-thread folds: F = from the last head to the end, B = from the start to the first tail
  T F = ident, B = ident;
  bool ff = false, bf = false;
  // loops kept rolled (CT_UNROLL): the kernels are instruction-cache bound when every item is inlined
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = j0 + q;
    const T it = item(j);
    if (fl[j] & hbit) F = it, ff = true;
    else F = op(F, it);
  }
#pragma unroll kCtUnroll
  for (int q = CT_ITEMS - 1; q >= 0; q--) {
    const int j = j0 + q;
    const T it = item(j);
    if (fl[j] & tbit) B = it, bf = true;
    else B = op(it, B);
  }
  const T Ef = block_seg_excl<T, Op, false, CT_THREADS>(ff, F, carry_in, op, s_wv, s_wf);
  const T Eb = block_seg_excl<T, Op, true, CT_THREADS>(bf, B, carry_out, op, s_wv, s_wf);
  int q = 0;
  while (q < CT_ITEMS) {
    T tot = (q == 0 && !(fl[j0] & hbit)) ? Ef : ident;
    int e = q;
    while (true) {
      tot = op(tot, item(j0 + e));
      const bool t = fl[j0 + e] & tbit;
      e++;
      if (t || e == CT_ITEMS) break;
    }
    if (!(fl[j0 + e - 1] & tbit)) tot = op(tot, Eb);
    for (int r = q; r < e; r++) cb(j0 + r, tot);
    q = e;
  }
}

// ------------------------------------------------------------------------------------------------ pair rule
struct F5 {
  u32 block, interval, thread, rw;
  u64 vh;
};

// P(x, s) of include/sesa.h for two entries at the same location; 0 = no race
__device__ __forceinline__ u32 pair_kind(const F5& x, const F5& s, u32 ws, u32 ls) {
  if (x.block == s.block && x.thread == s.thread) return 0;                  // (1) t1 != t2
  if (x.rw == RW_READ && s.rw == RW_READ) return 0;                           // (2) a write
  if (x.rw == RW_ATOMIC && s.rw == RW_ATOMIC) return 0;                       // (3) not both atomic
  if (x.block == s.block && x.interval != s.interval) return 0;               // (4) ordered by a barrier
  const u32 kind = (x.rw == RW_READ || s.rw == RW_READ) ? KIND_RW : KIND_WW;
  if (ls && kind == KIND_RW && x.block == s.block && x.interval == s.interval && x.thread / ws == s.thread / ws)
    return 0;                                                                 // (5) lockstep warp
  if (x.rw == RW_WRITE && s.rw == RW_WRITE && x.vh == s.vh) return 0;         // (6) benign W/W
  return kind;
}

// ------------------------------------------------------------------------------------------------ tile state
enum : u8 { FL_GH = 1, FL_GT = 2, FL_SH = 4, FL_ST = 8, FL_INT = 16 };
enum : u8 { TF_GH = 1, TF_GT = 2, TF_SH = 4, TF_ST = 8, TF_CIN = 16, TF_COUT = 32 };

struct TileSmem {
  u64 key[CT_TILE + 2];  // [0] = previous entry, [j+1] = item j, [cnt+1] = next entry
  u32 blk[CT_TILE + 2];
  u32 ivl[CT_TILE + 2];
  u32 thr[CT_TILE];
  u64 vh[CT_TILE];
  u32 xy[CT_TILE][2];  // mode 1: x of tail items, then y candidates
  u8 rw[CT_TILE];
  u8 fl[CT_TILE];
  u8 gq[CT_TILE];
  u8 res[CT_TILE];
  Agg wv[CT_THREADS / 32];
  AggC wvc[CT_THREADS / 32];
  X2 wx[CT_THREADS / 32];
  u8 wf[CT_THREADS / 32];
  int any, first_gtail, last_ghead, unknown;
};

__device__ __forceinline__ u32 pos_of(const KeyLayout& L, u64 key) { return (u32)(key & lowmask(L.pos_bits)); }

// Tile windows.  Tiles step by CT_NOM entries; a tile also takes the rest of its last location run when that run
// ends within CT_EXT entries past the nominal end (and the next tile skips those entries), so that the short
// runs straddling a boundary — nearly every boundary in C2/C4, whose locations hold ~17 entries — are completed
// inside one tile instead of going through the crossing-run carries (modes 2/3).  Windows partition the entries:
// window(t) = [t*CT_NOM + skip(t*CT_NOM), (t+1)*CT_NOM + skip((t+1)*CT_NOM)) clipped to [0, m), <= CT_TILE long.
constexpr u32 CT_EXT = 256, CT_NOM = CT_TILE - CT_EXT;

// skip(b): entries from b on that belong to a run owned by the tile before boundary b (run head >= b - CT_NOM,
// i.e. inside that tile) and ending by b + CT_EXT; 0 if b starts a run or the run is long.  One warp per boundary
// (tile_starts_kernel, once per check): the conflict kernels read their windows instead of four dependent loads.
__device__ u32 window_skip_warp(const ConflictArgs& a, u64 b) {
  const KeyLayout& L = a.L;
  if (b == 0 || b >= a.m) return 0;
  const u64 g = group_of_hi(L, a.keys[b - 1] >> L.pos_bits);
  if (group_of_hi(L, a.keys[b] >> L.pos_bits) != g) return 0;  // b heads a run
  if (b >= (u64)CT_NOM + 1 && group_of_hi(L, a.keys[b - CT_NOM - 1] >> L.pos_bits) == g) return 0;  // long run
  const int lane = threadIdx.x & 31;
  for (u32 t0 = 0; t0 < CT_EXT; t0 += 32) {  // entries b + 1 .. b + CT_EXT: the first one outside the run
    const u64 i = b + 1 + t0 + lane;
    const u32 out = __ballot_sync(~0u, i >= a.m || group_of_hi(L, a.keys[i] >> L.pos_bits) != g);
    if (out) return t0 + __ffs(out);
  }
  return 0;  // the run is long
}

__global__ void tile_starts_kernel(ConflictArgs a, u32 ntiles, u32* __restrict__ ts) {
  const u32 t = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (t > ntiles) return;
  const u64 b = (u64)t * CT_NOM;
  const u32 sk = window_skip_warp(a, b);
  if ((threadIdx.x & 31) == 0) ts[t] = (u32)min((u64)a.m, b + sk);
}

void launch_tile_starts(const ConflictArgs& a, u32 ntiles, u32* tstart, cudaStream_t st) {
  const u64 threads = ((u64)ntiles + 1) * 32;
  tile_starts_kernel<<<(unsigned)((threads + 255) / 256), 256, 0, st>>>(a, ntiles, tstart);
}

// Tile windows: tile t owns entries [tstart[t], tstart[t+1]) — windows partition the entries, <= CT_TILE long;
// cnt = 0 for a tile whose entries all went to its predecessor
__device__ __forceinline__ void tile_window(const ConflictArgs& a, u32 tile, u64* tb, u32* cnt) {
  const u32 lo = a.tstart[tile], hi = a.tstart[tile + 1];
  *tb = lo;
  *cnt = hi - lo;
}

// the record of entry e (sorted/compacted entry index) with key `key`: by position in the caller's record array
// (single GPU), or entry-aligned records fetched from the owner ranks (distributed check)
// (tdiv > 1: the identity of a record is its warp thread / tdiv — the inter-warp half of the precise warp model)
// One 256-bit load per gathered record, cached in L2 only (.cg): the record is used once, and two 16-byte loads
// through L1 fetched ~3.5 sectors per record from L2 (ncu, C4) — measured 12.4 -> 11.5 -> 10.4 ms on C4's mode 1
// with the early gather and this load (vs 11.3 with L1-allocating 256-bit loads).
__device__ __forceinline__ Rec load_rec_gather(const Rec* p) {
  u32 w[8];
  asm("ld.global.cg.L2::64B.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(w[0]), "=r"(w[1]), "=r"(w[2]), "=r"(w[3]), "=r"(w[4]), "=r"(w[5]), "=r"(w[6]), "=r"(w[7])
      : "l"(p));
  Rec r;
  r.addr = (u64)w[0] | ((u64)w[1] << 32);
  r.vh = (u64)w[2] | ((u64)w[3] << 32);
  r.block = w[4];
  r.thread = w[5];
  r.interval = w[6];
  r.size = (u16)(w[7] & 0xFFFF);
  r.space = (u8)((w[7] >> 16) & 0xFF);
  r.rw = (u8)(w[7] >> 24);
  return r;
}
__device__ __forceinline__ Rec rec_at(const ConflictArgs& a, u64 e, u64 key) {
  Rec r = load_rec_gather(a.rec_entry ? a.rec_entry + e : a.rec + (pos_of(a.L, key) - a.rec_pos_base));
  if (a.tdiv > 1) r.thread /= a.tdiv;
  return r;
}

// Loads keys and group flags; with GATHER (mode 1) also every record — every entry of a compacted array has a
// partner candidate somewhere, so the record loads go out with the key loads — and the sub-run flags.  Modes 2/3
// gather only their crossing pieces afterwards (tile_gather).  Returns false if no entry of the tile has a
// partner candidate (all singletons).
template <bool GATHER>
__device__ bool tile_load(const ConflictArgs& a, TileSmem& s, u64 tb, u32 cnt) {
  const KeyLayout& L = a.L;
  const int tid = threadIdx.x;
  u64 k[CT_ITEMS];
#pragma unroll
  for (int q = 0; q < CT_ITEMS; q++) {  // compile-time trip count: all loads in flight
    const u32 j = q * CT_THREADS + tid;
    k[q] = j < cnt ? __ldcs(a.keys + tb + j) : 0ull;
  }
  constexpr int HALF = CT_ITEMS / 2;  // records in two batches of loads in flight (register budget)
#pragma unroll
  for (int h = 0; h < CT_ITEMS; h += HALF) {
    Rec r[HALF];
    if (GATHER) {
#pragma unroll
      for (int q = 0; q < HALF; q++)
        if ((h + q) * CT_THREADS + tid < (int)cnt) r[q] = rec_at(a, tb + (h + q) * CT_THREADS + tid, k[h + q]);
    }
#pragma unroll
    for (int q = 0; q < HALF; q++) {
      const u32 j = (h + q) * CT_THREADS + tid;
      if (j >= cnt) continue;
      s.key[j + 1] = k[h + q];
      if (GATHER) {
        s.blk[j + 1] = r[q].block;
        s.ivl[j + 1] = r[q].interval;
        s.thr[j] = r[q].thread;
        s.rw[j] = r[q].rw;
        s.vh[j] = r[q].vh;
      }
    }
  }
  if (tid == 0) {  // the entries just outside the window: key (and (block, interval))
    s.key[0] = 0ull;
    if (tb > 0) {
      s.key[0] = a.keys[tb - 1];
      if (GATHER) {
        const Rec r = rec_at(a, tb - 1, s.key[0]);
        s.blk[0] = r.block, s.ivl[0] = r.interval;
      }
    }
    s.any = 0;
    s.first_gtail = CT_TILE;
    s.last_ghead = -1;
  }
  if (tid == CT_THREADS - 1) {
    s.key[cnt + 1] = 0ull;
    if (tb + cnt < a.m) {
      s.key[cnt + 1] = a.keys[tb + cnt];
      if (GATHER) {
        const Rec r = rec_at(a, tb + cnt, s.key[cnt + 1]);
        s.blk[cnt + 1] = r.block, s.ivl[cnt + 1] = r.interval;
      }
    }
  }
  __syncthreads();
  const int j0 = tid * CT_ITEMS;
  bool any = false;
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = j0 + q;
    // items past the window's end carry no boundary flags: they are transparent to the segmented scans, so
    // the backward carry of a run crossing out of a short window reaches its last real item (cnt - 1)
    u8 f = j < (int)cnt ? (FL_GH | FL_GT) : 0;
    if (j < (int)cnt) {
      const u64 kj = s.key[j + 1];
      const bool sp = (j > 0 || tb > 0) && same_group(L, s.key[j], kj);
      const bool sn = (j + 1 < (int)cnt || tb + cnt < a.m) && same_group(L, kj, s.key[j + 2]);
      f = (sp ? 0 : FL_GH) | (sn ? 0 : FL_GT) | ((sp || sn) ? FL_INT : 0);
      any |= sp || sn;
      if (f & FL_GT) atomicMin(&s.first_gtail, j);
      if (f & FL_GH) atomicMax(&s.last_ghead, j);
    }
    s.fl[j] = f;
  }
  if (!__syncthreads_or(any)) return false;
  if (GATHER) {
    // sub-runs: a new (block, interval) inside a group (contiguous: input order is (block, interval) order)
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = j0 + q;
      u8 f = s.fl[j];
      if (f & FL_INT) {
        const bool sh = (f & FL_GH) || s.blk[j] != s.blk[j + 1] || s.ivl[j] != s.ivl[j + 1];
        const bool st = (f & FL_GT) || s.blk[j + 2] != s.blk[j + 1] || s.ivl[j + 2] != s.ivl[j + 1];
        f |= (sh ? FL_SH : 0) | (st ? FL_ST : 0);
      } else if (j < (int)cnt) {
        f |= FL_SH | FL_ST;
      }
      s.fl[j] = f;
    }
    __syncthreads();
  }
  return true;
}

// Modes 2/3: records and sub-run flags of the entries [lo, hi) (whole crossing pieces: a piece starting at 0
// needs the (block, interval) of the entry before the window, one ending at cnt that of the entry after it).
// All threads call.
__device__ void tile_gather(const ConflictArgs& a, TileSmem& s, u64 tb, u32 cnt, int lo, int hi) {
  const int tid = threadIdx.x;
  constexpr int B = 3;
  for (int j0 = lo; j0 < hi; j0 += B * CT_THREADS) {
    Rec r[B];
#pragma unroll
    for (int q = 0; q < B; q++) {
      const int j = j0 + q * CT_THREADS + tid;
      if (j < hi) r[q] = rec_at(a, tb + j, s.key[j + 1]);
    }
#pragma unroll
    for (int q = 0; q < B; q++) {
      const int j = j0 + q * CT_THREADS + tid;
      if (j >= hi) continue;
      s.blk[j + 1] = r[q].block;
      s.ivl[j + 1] = r[q].interval;
      s.thr[j] = r[q].thread;
      s.rw[j] = r[q].rw;
      s.vh[j] = r[q].vh;
    }
  }
  if (lo == 0 && tid == 0 && tb > 0) {
    const Rec r = rec_at(a, tb - 1, s.key[0]);
    s.blk[0] = r.block, s.ivl[0] = r.interval;
  }
  if (hi == (int)cnt && tid == CT_THREADS - 1 && tb + cnt < a.m) {
    const Rec r = rec_at(a, tb + cnt, s.key[cnt + 1]);
    s.blk[cnt + 1] = r.block, s.ivl[cnt + 1] = r.interval;
  }
  __syncthreads();
  for (int j = lo + tid; j < hi; j += CT_THREADS) {
    u8 f = s.fl[j];
    if (f & FL_INT) {
      const bool sh = (f & FL_GH) || s.blk[j] != s.blk[j + 1] || s.ivl[j] != s.ivl[j + 1];
      const bool st = (f & FL_GT) || s.blk[j + 2] != s.blk[j + 1] || s.ivl[j + 2] != s.ivl[j + 1];
      f |= (sh ? FL_SH : 0) | (st ? FL_ST : 0);
    } else {
      f |= FL_SH | FL_ST;
    }
    s.fl[j] = f;
  }
  __syncthreads();
}

// group- and sub-run-level summaries -> s.res[j] = bit0 RW partner, bit1 WW partner.  In mode 1 also returns
// the tile-edge partial summaries (P = item 0's segment, S = item cnt-1's segment) per level.  With the cheap
// summary (A = AggC) a benign query that cannot be decided sets s.unknown (the check is then redone exactly).
template <class A>
__device__ A* scan_scratch(TileSmem& s);
template <>
__device__ __forceinline__ Agg* scan_scratch<Agg>(TileSmem& s) { return s.wv; }
template <>
__device__ __forceinline__ AggC* scan_scratch<AggC>(TileSmem& s) { return s.wvc; }

template <class A>
__device__ void tile_flags(const ConflictArgs& a, TileSmem& s, u32 cnt, const A cin[2], const A cout[2],
                           A* part /* [4] or null */, bool one_group = false) {
  typedef typename OpOf<A>::type Op;
  const u32 ws = a.ws, ls = a.ls;
  const A E = agg_empty_t<A>();
  // group level (identity = block): "another block" queries -> s.gq (bit3: benign query yes, bit4: unknown)
  auto gitem = [&](int j) { return (s.fl[j] & FL_INT) ? agg_item_t<A>(s.rw[j], s.blk[j + 1], s.vh[j]) : E; };
  auto gcb = [&](int j, const A& R) {
    if (part && j == 0) part[0] = R;
    if (part && j == (int)cnt - 1) part[1] = R;
    if (!(s.fl[j] & FL_INT)) return;
    const u32 b = s.blk[j + 1];
    u8 g = (ex_id(R, RW_READ, b) ? 1 : 0) | (ex_id(R, RW_WRITE, b) ? 2 : 0) | (ex_id(R, RW_ATOMIC, b) ? 4 : 0);
    if (s.rw[j] == RW_WRITE) {
      const int q = wval3(R, b, s.vh[j]);
      g |= q == 1 ? 8 : q == 2 ? 16 : 0;
    }
    s.gq[j] = g;
  };
  // a shared location fixes its block, so "another block" never holds for shared entries: a tile of shared
  // locations only (e.g. most of C2) skips the run-level scan
  bool my_g = false;
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = threadIdx.x * CT_ITEMS + q;
    if (j < (int)cnt && (s.fl[j] & FL_INT)) my_g |= space_of_hi(a.L, s.key[j + 1] >> a.L.pos_bits) == SP_GLOBAL;
  }
  if (!__syncthreads_or(my_g)) {
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = threadIdx.x * CT_ITEMS + q;
      if (j < (int)cnt) s.gq[j] = 0;
    }
    if (part) {
      // the carries (and the crossing-mode skips) still need the first / last run pieces: two masked reductions
      const int ft = s.first_gtail, lh = s.last_ghead;
      A p0 = E, p1 = E;
#pragma unroll kCtUnroll
      for (int q = 0; q < CT_ITEMS; q++) {
        const int j = threadIdx.x * CT_ITEMS + q;
        if (j >= (int)cnt) continue;
        const A it = gitem(j);
        if (j <= ft) p0 = Op()(p0, it);
        if (j >= lh) p1 = Op()(p1, it);
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) p0 = Op()(p0, shfl(p0, o, true)), p1 = Op()(p1, shfl(p1, o, true));
      A* wv = scan_scratch<A>(s);
      for (int r = 0; r < 2; r++) {
        if ((threadIdx.x & 31) == 0) wv[threadIdx.x >> 5] = r ? p1 : p0;
        __syncthreads();
        if (threadIdx.x == 0) {
          A t = wv[0];
          for (int w = 1; w < CT_THREADS / 32; w++) t = Op()(t, wv[w]);
          part[r] = t;
        }
        __syncthreads();
      }
    }
  } else if (one_group) {
    // the window is one piece of one run: its summary is carry in + a plain block reduction + carry out
    A v = E;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = threadIdx.x * CT_ITEMS + q;
      if (j < (int)cnt) v = Op()(v, gitem(j));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = Op()(v, shfl(v, o, true));
    A* wv = scan_scratch<A>(s);
    __shared__ A s_run;
    if ((threadIdx.x & 31) == 0) wv[threadIdx.x >> 5] = v;
    __syncthreads();
    if (threadIdx.x == 0) {
      A t = cin[0];
      for (int w = 0; w < CT_THREADS / 32; w++) t = Op()(t, wv[w]);
      s_run = Op()(t, cout[0]);
    }
    __syncthreads();
    const A R = s_run;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = threadIdx.x * CT_ITEMS + q;
      if (j < (int)cnt) gcb(j, R);
    }
  } else {
    tile_allreduce<A>(s.fl, FL_GH, FL_GT, gitem, Op(), E, cin[0], cout[0], gcb, scan_scratch<A>(s), s.wf);
  }
  __syncthreads();
  // sub-run level (identity = thread): same block and interval
  tile_allreduce<A>(
      s.fl, FL_SH, FL_ST,
      [&](int j) { return (s.fl[j] & FL_INT) ? agg_item_t<A>(s.rw[j], s.thr[j], s.vh[j]) : E; }, Op(), E, cin[1],
      cout[1],
      [&](int j, const A& S) {
        if (part && j == 0) part[2] = S;
        if (part && j == (int)cnt - 1) part[3] = S;
        if (!(s.fl[j] & FL_INT)) return;
        const u32 t = s.thr[j], w = t / ws, rw = s.rw[j];
        const u8 g = s.gq[j];
        bool frw, fww;
        if (rw == RW_READ) {
          frw = (ls ? (ex_warp(S, RW_WRITE, w, ws) || ex_warp(S, RW_ATOMIC, w, ws))
                    : (ex_id(S, RW_WRITE, t) || ex_id(S, RW_ATOMIC, t))) ||
                (g & 6);
          fww = false;
        } else {
          frw = (ls ? ex_warp(S, RW_READ, w, ws) : ex_id(S, RW_READ, t)) || (g & 1);
          if (rw == RW_WRITE) {
            const int q = wval3(S, t, s.vh[j]);
            fww = ex_id(S, RW_ATOMIC, t) || (g & 4) || q == 1 || (g & 8);
            if (!fww && (q == 2 || (g & 16))) s.unknown = 1;  // undecidable with the cheap summary
          } else {
            fww = ex_id(S, RW_WRITE, t) || (g & 2);
          }
        }
        s.res[j] = (frw ? 1 : 0) | (fww ? 2 : 0);
      },
      scan_scratch<A>(s), s.wf);
  __syncthreads();
}

__device__ __forceinline__ F5 fields(const TileSmem& s, int j) {
  F5 f;
  f.block = s.blk[j + 1], f.interval = s.ivl[j + 1], f.thread = s.thr[j], f.rw = s.rw[j], f.vh = s.vh[j];
  return f;
}

__device__ void emit_race(const ConflictArgs& a, u64 head_hi, u32 kind, u32 x, u32 y, u32 hb, u32 hi_) {
  const KeyLayout& L = a.L;
  const u32 idx = atomicAdd(a.race_count, 1u);
  if (idx >= a.race_cap) return;
  RaceOut r;
  const u32 sp = space_of_hi(L, head_hi);
  r.addr = granule_of_hi(L, head_hi) << L.log2G;
  r.first = a.index_base + x;
  r.second = a.index_base + y;
  r.block = sp == SP_SHARED ? hb : NOBI;
  r.interval = sp == SP_SHARED ? hi_ : NOBI;
  r.space = (u8)sp;
  r.kind = (u8)kind;
  r.reserved[0] = r.reserved[1] = 0;
  r.epoch = 0;
  a.races[idx] = r;
  a.race_keys[idx] = (group_of_hi(L, head_hi) << 2) | (kind - 1);  // 2 kind bits: RW, WW, benign WW
  a.race_vals[idx] = idx;
}

// A location whose whole summary shows no possible pair of either kind: no RW (no read, or no write/atomic) and
// no WW (no write, or no atomic and every write of one value — benign).  C4's `changed` run (60 M same-valued
// writes) is one; its middle tiles skip the crossing modes entirely.
// no_rw / no_ww: the summary of a whole run rules out every pair of that kind
__device__ __forceinline__ void cannot_race(const AggC& g, bool* no_rw, bool* no_ww) {
  const bool noR = g.mn[RW_READ] > g.mx[RW_READ], noW = g.mn[RW_WRITE] > g.mx[RW_WRITE];
  const bool noA = g.mn[RW_ATOMIC] > g.mx[RW_ATOMIC];
  *no_rw = noR || (noW && noA);
  *no_ww = noW || (noA && g.vlo == g.vhi);
}
__device__ __forceinline__ void cannot_race(const Agg& g, bool* no_rw, bool* no_ww) {
  const bool noR = g.mn[RW_READ] > g.mx[RW_READ], noW = g.mn[RW_WRITE] > g.mx[RW_WRITE];
  const bool noA = g.mn[RW_ATOMIC] > g.mx[RW_ATOMIC];
  *no_rw = noR || (noW && noA);
  *no_ww = noW || (noA && g.v1 == g.v2);
}
__device__ __forceinline__ u64 ld_volatile(const u64* p) { return *reinterpret_cast<const volatile u64*>(p); }

// ------------------------------------------------------------------------------------------------ internal groups
// Mode 1 fast path for the groups that lie wholly inside the window.  The witness of (λ, K) needs only x_K (the
// lowest flagged position) and y_K (the lowest partner of x_K), not every entry's flag: per group, one exact
// summary G with identity = block decides "a partner in another block" for any entry in O(1); a partner in the
// entry's own (block, interval) sub-run is found pair by pair (sub-runs are short: the tile takes the scan path
// if an internal sub-run exceeds SR_MAX entries).  With position-ordered runs (lowG == 0) the x and y searches
// stop at the first hit — usually within the first few entries.  Groups of up to GR_SEQ entries: one thread each;
// longer groups: one warp each (lane-strided summary + butterfly merge, 32 candidates per step, ballots).
constexpr int GR_SEQ = 16;
constexpr int SR_MAX = 64;

__device__ __forceinline__ Agg shfl_x(const Agg& a, int o) {
  Agg r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = __shfl_xor_sync(~0u, a.mn[x], o), r.mx[x] = __shfl_xor_sync(~0u, a.mx[x], o);
  r.i1 = __shfl_xor_sync(~0u, a.i1, o), r.i2 = __shfl_xor_sync(~0u, a.i2, o);
  r.v1 = __shfl_xor_sync(~0u, a.v1, o), r.v1b = __shfl_xor_sync(~0u, a.v1b, o);
  r.v2 = __shfl_xor_sync(~0u, a.v2, o), r.v2b = __shfl_xor_sync(~0u, a.v2b, o);
  return r;
}

__device__ __forceinline__ AggC shfl_x(const AggC& a, int o) {
  AggC r;
#pragma unroll
  for (int x = 0; x < 3; x++) r.mn[x] = __shfl_xor_sync(~0u, a.mn[x], o), r.mx[x] = __shfl_xor_sync(~0u, a.mx[x], o);
  r.vlo = __shfl_xor_sync(~0u, a.vlo, o), r.vhi = __shfl_xor_sync(~0u, a.vhi, o);
  return r;
}

// The group summary is built cheap first (per type min/max identity, min/max write value): it decides "a plain
// write of another identity with another value" (false) whenever all plain writes share one value or come from one
// identity; only otherwise is the exact summary built.
__device__ __forceinline__ bool cheap_decides(const AggC& G) {
  return G.vlo == G.vhi || !(G.mn[RW_WRITE] < G.mx[RW_WRITE]);
}
__device__ __forceinline__ bool wval_other(const Agg& G, u32 b, u64 v) { return ex_wval(G, b, v); }
__device__ __forceinline__ bool wval_other(const AggC&, u32, u64) { return false; }  // (cheap_decides holds)

// a partner of e in another block (G: the group's summary, identity = block): RW / WW
template <class S>
__device__ __forceinline__ void flags_other_block(const S& G, const F5& e, bool* rwf, bool* wwf) {
  const u32 b = e.block;
  if (e.rw == RW_READ) {
    *rwf = ex_id(G, RW_WRITE, b) || ex_id(G, RW_ATOMIC, b);
    *wwf = false;
  } else {
    *rwf = ex_id(G, RW_READ, b);
    *wwf = e.rw == RW_WRITE ? (ex_id(G, RW_ATOMIC, b) || wval_other(G, b, e.vh)) : ex_id(G, RW_WRITE, b);
  }
}

// a partner of item j in its sub-run [sh, st] (same block and interval): rules 1-6 pair by pair
__device__ __forceinline__ void flags_subrun(const TileSmem& s, int j, int sh, int st, const F5& me, u32 ws, u32 ls,
                                             bool* f0, bool* f1) {
  for (int q = sh; q <= st && !(*f0 && *f1); q++) {
    if (q == j) continue;
    const u32 k = pair_kind(me, fields(s, q), ws, ls);
    *f0 = *f0 || k == KIND_RW;
    *f1 = *f1 || k == KIND_WW;
  }
}

__device__ __forceinline__ void emit_group(const ConflictArgs& a, const TileSmem& s, int t, u32 kind, u32 x, u32 y) {
  emit_race(a, s.key[t + 1] >> a.L.pos_bits, kind, x, y, s.blk[t + 1], s.ivl[t + 1]);
}

// one thread: group [h, t] (>= 2 entries, all gathered), given its summary G
template <class S>
__device__ void group_thread_search(const ConflictArgs& a, const TileSmem& s, int h, int t, const S& G) {
  const KeyLayout& L = a.L;
  bool no0, no1;
  cannot_race(G, &no0, &no1);
  if (no0 && no1) return;
  const bool ordered = L.lowG == 0;
  bool need0 = !no0, need1 = !no1;
  u32 xp0 = ~0u, xp1 = ~0u;
  int xj0 = -1, xj1 = -1, sh = h, st = h;
  for (int j = h; j <= t && (need0 || need1); j++) {
    if (s.fl[j] & FL_SH) {
      sh = st = j;
      while (!(s.fl[st] & FL_ST)) st++;
    }
    const F5 me = fields(s, j);
    bool f0, f1;
    flags_other_block(G, me, &f0, &f1);
    f0 = f0 && need0, f1 = f1 && need1;
    if (st > sh && (need0 != f0 || need1 != f1)) {
      flags_subrun(s, j, sh, st, me, a.ws, a.ls, &f0, &f1);
      f0 = f0 && need0, f1 = f1 && need1;
    }
    const u32 p = pos_of(L, s.key[j + 1]);
    if (f0 && p < xp0) xp0 = p, xj0 = j, need0 = !ordered;
    if (f1 && p < xp1) xp1 = p, xj1 = j, need1 = !ordered;
  }
#pragma unroll 1
  for (int k = 0; k < 2; k++) {
    const int xj = k ? xj1 : xj0;
    if (xj < 0) continue;
    const F5 X = fields(s, xj);
    u32 y = ~0u;
    for (int q = h; q <= t; q++) {
      if (pair_kind(X, fields(s, q), a.ws, a.ls) != (u32)(k + 1)) continue;
      y = min(y, pos_of(L, s.key[q + 1]));
      if (ordered) break;
    }
    emit_group(a, s, t, (u32)(k + 1), k ? xp1 : xp0, y);
  }
}

__device__ void group_thread(const ConflictArgs& a, const TileSmem& s, int h, int t) {
  AggC C = agg_empty_t<AggC>();
  for (int j = h; j <= t; j++) C = OpAggC()(C, agg_item_t<AggC>(s.rw[j], s.blk[j + 1], s.vh[j]));
  if (cheap_decides(C)) {
    group_thread_search(a, s, h, t, C);
  } else {
    Agg G = agg_empty();
    for (int j = h; j <= t; j++) G = agg_merge(G, agg_item(s.rw[j], s.blk[j + 1], s.vh[j]));
    group_thread_search(a, s, h, t, G);
  }
}

// one warp: group [h, t], given its summary G (in every lane)
template <class S>
__device__ void group_warp_search(const ConflictArgs& a, const TileSmem& s, int h, int t, const S& G) {
  const KeyLayout& L = a.L;
  const int lane = threadIdx.x & 31;
  bool no0, no1;
  cannot_race(G, &no0, &no1);
  if (no0 && no1) return;
  const bool ordered = L.lowG == 0;
  bool need0 = !no0, need1 = !no1;
  u32 xp[2] = {~0u, ~0u};
  int xj[2] = {-1, -1};
  for (int c = h; c <= t && (need0 || need1); c += 32) {
    const int j = c + lane;
    bool f0 = false, f1 = false;
    u32 p = ~0u;
    if (j <= t) {
      const F5 me = fields(s, j);
      flags_other_block(G, me, &f0, &f1);
      f0 = f0 && need0, f1 = f1 && need1;
      if (need0 != f0 || need1 != f1) {
        const u8 fj = s.fl[j];
        if (!((fj & FL_SH) && (fj & FL_ST))) {
          int sh = j, st = j;
          while (!(s.fl[sh] & FL_SH)) sh--;
          while (!(s.fl[st] & FL_ST)) st++;
          flags_subrun(s, j, sh, st, me, a.ws, a.ls, &f0, &f1);
          f0 = f0 && need0, f1 = f1 && need1;
        }
      }
      p = pos_of(L, s.key[j + 1]);
    }
#pragma unroll
    for (int k = 0; k < 2; k++) {
      const bool f = k ? f1 : f0;
      const u32 m = __reduce_min_sync(~0u, f ? p : ~0u);
      if (m < xp[k]) {
        xp[k] = m;
        xj[k] = c + __ffs(__ballot_sync(~0u, f && p == m)) - 1;
        if (ordered) (k ? need1 : need0) = false;
      }
    }
  }
#pragma unroll
  for (int k = 0; k < 2; k++) {
    if (xj[k] < 0) continue;
    const F5 X = fields(s, xj[k]);
    u32 y = ~0u;
    for (int c = h; c <= t; c += 32) {
      const int j = c + lane;
      const bool hit = j <= t && pair_kind(X, fields(s, j), a.ws, a.ls) == (u32)(k + 1);
      y = min(y, __reduce_min_sync(~0u, hit ? pos_of(L, s.key[j + 1]) : ~0u));
      if (ordered && y != ~0u) break;
    }
    if (lane == 0) emit_group(a, s, t, (u32)(k + 1), xp[k], y);
  }
}

__device__ void group_warp(const ConflictArgs& a, const TileSmem& s, int h, int t) {
  const int lane = threadIdx.x & 31;
  AggC C = agg_empty_t<AggC>();
  for (int j = h + lane; j <= t; j += 32) C = OpAggC()(C, agg_item_t<AggC>(s.rw[j], s.blk[j + 1], s.vh[j]));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) C = OpAggC()(C, shfl_x(C, o));
  if (cheap_decides(C)) {  // (warp-uniform: every lane holds the whole summary)
    group_warp_search(a, s, h, t, C);
  } else {
    Agg G = agg_empty();
    for (int j = h + lane; j <= t; j += 32) G = agg_merge(G, agg_item(s.rw[j], s.blk[j + 1], s.vh[j]));
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) G = agg_merge(G, shfl_x(G, o));
    group_warp_search(a, s, h, t, G);
  }
}

// exclusive block-wide sum of v (CT_THREADS threads); *total = the sum over the block
__device__ __forceinline__ u32 block_excl_sum(u32 v, u32* s_w, u32* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  u32 x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u32 y = __shfl_up_sync(~0u, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[warp] = x;
  __syncthreads();
  u32 off = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < CT_THREADS / 32; w++) {
    const u32 sw = s_w[w];
    off += w < warp ? sw : 0u;
    tot += sw;
  }
  __syncthreads();
  *total = tot;
  return off + x - v;
}

// Does an internal group of the tile (entries [lo, hi)) hold a sub-run longer than SR_MAX?  (all threads call)
__device__ __forceinline__ bool long_subrun(const TileSmem& s, int lo, int hi) {
  bool lsr = false;
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = threadIdx.x * CT_ITEMS + q;
    const u8 f = s.fl[j];
    if (j < lo || j >= hi || !(f & FL_INT) || !(f & FL_SH) || (f & FL_ST)) continue;
    int e = j + 1;
    while (!(s.fl[e] & FL_ST) && e - j < SR_MAX) e++;
    lsr = lsr || !(s.fl[e] & FL_ST);
  }
  return __syncthreads_or(lsr) != 0;
}

// races of the internal groups (entries [lo, hi)): group list by a block scan, then threads / warps
__device__ void internal_groups(const ConflictArgs& a, TileSmem& s, int lo, int hi) {
  __shared__ u32 s_w[CT_THREADS / 32];
  unsigned short* gh = reinterpret_cast<unsigned short*>(&s.xy[0][0]);
  unsigned short* gt = gh + CT_TILE / 2 + 8;
  u32 nh = 0, nt = 0;
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = threadIdx.x * CT_ITEMS + q;
    const u8 f = s.fl[j];
    if (j < lo || j >= hi || !(f & FL_INT)) continue;
    nh += (f & FL_GH) ? 1u : 0u;
    nt += (f & FL_GT) ? 1u : 0u;
  }
  u32 tot;
  const u32 ex = block_excl_sum(nh | (nt << 16), s_w, &tot);
  u32 oh = ex & 0xFFFFu, ot = ex >> 16;
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = threadIdx.x * CT_ITEMS + q;
    const u8 f = s.fl[j];
    if (j < lo || j >= hi || !(f & FL_INT)) continue;
    if (f & FL_GH) gh[oh++] = (unsigned short)j;
    if (f & FL_GT) gt[ot++] = (unsigned short)j;
  }
  __syncthreads();
  const int ng = (int)(tot & 0xFFFFu);
  for (int g = threadIdx.x; g < ng; g += CT_THREADS)
    if (gt[g] - gh[g] < GR_SEQ) group_thread(a, s, gh[g], gt[g]);
  for (int g = threadIdx.x >> 5; g < ng; g += CT_THREADS / 32)
    if (gt[g] - gh[g] >= GR_SEQ) group_warp(a, s, gh[g], gt[g]);
}

// the tile-edge pieces for the carries without the segmented scans: part[0] / part[1] = run-level summaries of
// [0, first run tail] / [last run head, cnt), part[2] / part[3] = sub-run-level ones of [0, first sub-run tail] /
// [last sub-run head, cnt) — what tile_flags hands the carries
template <class A>
__device__ void tile_parts(const TileSmem& s, u32 cnt, A* part) {
  typedef typename OpOf<A>::type Op;
  __shared__ int s_fst, s_lsh;
  __shared__ A s_red[2][CT_THREADS / 32];
  if (threadIdx.x == 0) s_fst = (int)cnt - 1, s_lsh = 0;
  __syncthreads();
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = threadIdx.x * CT_ITEMS + q;
    if (j >= (int)cnt) continue;
    if (s.fl[j] & FL_ST) atomicMin(&s_fst, j);
    if (s.fl[j] & FL_SH) atomicMax(&s_lsh, j);
  }
  __syncthreads();
  const int ft = s.first_gtail, lh = s.last_ghead, fst = s_fst, lsh = s_lsh;
  const A E = agg_empty_t<A>();
#pragma unroll 1
  for (int r = 0; r < 2; r++) {
    A p0 = E, p1 = E;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = threadIdx.x * CT_ITEMS + q;
      if (j >= (int)cnt || !(s.fl[j] & FL_INT)) continue;
      const A it = agg_item_t<A>(s.rw[j], r ? s.thr[j] : s.blk[j + 1], s.vh[j]);
      if (j <= (r ? fst : ft)) p0 = Op()(p0, it);
      if (j >= (r ? lsh : lh)) p1 = Op()(p1, it);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) p0 = Op()(p0, shfl(p0, o, true)), p1 = Op()(p1, shfl(p1, o, true));
    if ((threadIdx.x & 31) == 0) s_red[0][threadIdx.x >> 5] = p0, s_red[1][threadIdx.x >> 5] = p1;
    __syncthreads();
    if (threadIdx.x < 2) {
      A t = s_red[threadIdx.x][0];
      for (int w = 1; w < CT_THREADS / 32; w++) t = Op()(t, s_red[threadIdx.x][w]);
      part[2 * r + threadIdx.x] = t;
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------------------------------------------ mode 2 fast
// Mode 2 without the segmented scans: a crossing piece only needs its lowest flagged position per kind (x into
// the owner's slot), and an entry's flag follows from the run summary R (carries + the piece's part, identity =
// block: "a partner in another block"), the summary S of its sub-run if that sub-run continues across the
// window's edge (carries + part, identity = thread), or pair by pair inside a sub-run within the window.  Only
// the pieces' records are gathered; with position-ordered runs the search stops at the first chunk that flags.
// Returns false (nothing done) when an inner sub-run is longer than SR_MAX: the caller takes the scan path.
template <class A>
__device__ bool cross_pieces_fast(const ConflictArgs& a, TileSmem& s, u32 tile, u64 tb, u32 cnt, bool cin,
                                  bool cout, const u8 (*need)[2]) {
  typedef typename OpOf<A>::type Op;
  typedef typename QuadOf<A>::type Q;
  const int tid = threadIdx.x;
  const int ftail = s.first_gtail, lhead = s.last_ghead;
  const bool pa = cin && a.phase != 1 && (need[0][0] || need[0][1]);
  const bool pb = cout && lhead >= 0 && a.phase != 2 && (need[1][0] || need[1][1]);
  const int aend = min(ftail, (int)cnt - 1);
  if (pa) tile_gather(a, s, tb, cnt, 0, aend + 1);
  if (pb) tile_gather(a, s, tb, cnt, lhead, (int)cnt);
  __shared__ int s_fst, s_lsh;
  __shared__ A s_R[2], s_S[2];
  __shared__ unsigned long long s_min[4];
  if (tid == 0) s_fst = (int)cnt - 1, s_lsh = 0;
  if (tid < 4) s_min[tid] = ~0ull;
  __syncthreads();
  auto in_piece = [&](int j) { return (pa && j <= aend) || (pb && j >= lhead && j < (int)cnt); };
  // the edge sub-runs: the first one of piece A (if it continues in from the previous window) and the last one
  // of the piece that ends the window (B, or A when the window lies inside one run) if it continues out
  const bool middle = cin && cout && lhead < 0;
  const bool lastp = pb || (pa && middle);  // the window's last entry belongs to a processed piece
  const int llo = pb ? lhead : 0;
  for (int j = tid; j < (int)cnt; j += CT_THREADS) {
    if (pa && j <= aend && (s.fl[j] & FL_ST)) atomicMin(&s_fst, j);
    if (lastp && j >= llo && (s.fl[j] & FL_SH)) atomicMax(&s_lsh, j);
  }
  __syncthreads();
  const int fst = s_fst, lsh = s_lsh;
  const bool cinS = pa && !(s.fl[0] & FL_SH), coutS = lastp && !(s.fl[cnt - 1] & FL_ST);
  // inner sub-runs (not continuing across an edge) longer than SR_MAX: the scan path
  bool lng = false;
  for (int j = tid; j < (int)cnt; j += CT_THREADS) {
    if (!in_piece(j) || !(s.fl[j] & FL_SH) || (s.fl[j] & FL_ST) || (coutS && j == lsh)) continue;
    int e = j + 1;
    while (e < (int)cnt - 1 && !(s.fl[e] & FL_ST) && e - j < SR_MAX) e++;
    lng = lng || !(s.fl[e] & FL_ST);
  }
  if (tid == 0) {
    const A* c = reinterpret_cast<const Q*>(a.carry)[tile].a;  // [grp In, grp Out, sub In, sub Out]
    const A* pp = reinterpret_cast<const Q*>(a.part)[tile].a;  // [grp P, grp S, sub P, sub S]
    const A E = agg_empty_t<A>();  // (only the summaries a piece uses: the others are not written this check)
    if (pa) s_R[0] = middle ? Op()(Op()(c[0], pp[0]), c[1]) : Op()(c[0], pp[0]);
    if (pb) s_R[1] = Op()(pp[1], c[1]);
    if (cinS) s_S[0] = Op()(Op()(c[2], pp[2]), (fst == (int)cnt - 1 && coutS) ? c[3] : E);
    if (coutS) s_S[1] = Op()(Op()((lsh == 0 && cinS) ? c[2] : E, pp[3]), c[3]);
  }
  if (__syncthreads_or(lng)) return false;
  const bool ordered = a.L.lowG == 0;
  const u32 ws = a.ws, ls = a.ls;
#pragma unroll 1
  for (int P = 0; P < 2; P++) {
    if (!(P ? pb : pa)) continue;
    const int lo = P ? lhead : 0, hi = P ? (int)cnt - 1 : aend;
    bool n0 = need[P][0], n1 = need[P][1];
    for (int c0 = lo; c0 <= hi && (n0 || n1); c0 += CT_THREADS) {
      const int j = c0 + tid;
      bool f0 = false, f1 = false, unk = false;
      if (j <= hi && (s.fl[j] & FL_INT)) {
        const F5 me = fields(s, j);
        const A& R = s_R[P];
        const u32 b = me.block, t = me.thread;
        int qg = 0, qs = 0;
        if (me.rw == RW_READ) {
          f0 = ex_id(R, RW_WRITE, b) || ex_id(R, RW_ATOMIC, b);
        } else {
          f0 = ex_id(R, RW_READ, b);
          if (me.rw == RW_WRITE) qg = wval3(R, b, me.vh), f1 = ex_id(R, RW_ATOMIC, b) || qg == 1;
          else f1 = ex_id(R, RW_WRITE, b);
        }
        const bool inF = cinS && j <= fst, inL = coutS && j >= lsh;
        if (inF || inL) {
          const A& S = s_S[inF ? 0 : 1];
          const u32 w = t / ws;
          if (me.rw == RW_READ) {
            f0 = f0 || (ls ? (ex_warp(S, RW_WRITE, w, ws) || ex_warp(S, RW_ATOMIC, w, ws))
                           : (ex_id(S, RW_WRITE, t) || ex_id(S, RW_ATOMIC, t)));
          } else {
            f0 = f0 || (ls ? ex_warp(S, RW_READ, w, ws) : ex_id(S, RW_READ, t));
            if (me.rw == RW_WRITE) qs = wval3(S, t, me.vh), f1 = f1 || ex_id(S, RW_ATOMIC, t) || qs == 1;
            else f1 = f1 || ex_id(S, RW_WRITE, t);
          }
        } else if ((n0 && !f0) || (n1 && !f1)) {
          const u8 fj = s.fl[j];
          if (!((fj & FL_SH) && (fj & FL_ST))) {
            int sh = j, st = j;
            while (!(s.fl[sh] & FL_SH)) sh--;
            while (!(s.fl[st] & FL_ST)) st++;
            flags_subrun(s, j, sh, st, me, ws, ls, &f0, &f1);
          }
        }
        f0 = f0 && n0, f1 = f1 && n1;
        unk = n1 && !f1 && (qg == 2 || qs == 2);
      }
      if (__syncthreads_or(unk)) {  // a benign query the cheap summary cannot decide: the host reruns exactly
        if (tid == 0) atomicOr(a.need_exact, 1u);
        return true;
      }
      const unsigned long long p = ((unsigned long long)pos_of(a.L, s.key[j + 1]) << 32) | (u32)(tb + j);
      if (f0) atomicMin(&s_min[2 * P], p);
      if (f1) atomicMin(&s_min[2 * P + 1], p);
      __syncthreads();
      if (ordered) n0 = n0 && s_min[2 * P] == ~0ull, n1 = n1 && s_min[2 * P + 1] == ~0ull;
      __syncthreads();
    }
  }
  if (tid == 0) {
    if (pa) {
      Slot* sl = &a.slots[a.owner[tile]];
      if (s_min[0] != ~0ull) atomicMin((unsigned long long*)&sl->x[0], s_min[0]);
      if (s_min[1] != ~0ull) atomicMin((unsigned long long*)&sl->x[1], s_min[1]);
    }
    if (pb) {
      Slot* sl = &a.slots[tile];
      if (s_min[2] != ~0ull) atomicMin((unsigned long long*)&sl->x[0], s_min[2]);
      if (s_min[3] != ~0ull) atomicMin((unsigned long long*)&sl->x[1], s_min[3]);
    }
  }
  // Position-ordered runs: piece B is the run's first entries, so an x found there is final, and so is the lowest
  // partner y found there (any other entry lies later) — search it now, while the records are in shared memory;
  // mode 3 then skips the run (mode3_any).
  if (ordered && pb) {
    __shared__ unsigned long long s_y[2];
    __shared__ F5 s_X[2];
    if (tid < 2) {
      s_y[tid] = ~0ull;
      if (s_min[2 + tid] != ~0ull) s_X[tid] = fields(s, (int)((u32)s_min[2 + tid] - (u32)tb));
    }
    __syncthreads();
#pragma unroll 1
    for (int k = 0; k < 2; k++) {
      if (s_min[2 + k] == ~0ull) continue;
      for (int c0 = lhead; c0 < (int)cnt; c0 += CT_THREADS) {
        const int j = c0 + tid;
        const bool hit = j < (int)cnt && (s.fl[j] & FL_INT) && pair_kind(s_X[k], fields(s, j), ws, ls) == (u32)(k + 1);
        if (hit) atomicMin(&s_y[k], ((unsigned long long)pos_of(a.L, s.key[j + 1]) << 32) | (u32)(tb + j));
        if (__syncthreads_or(hit)) break;
      }
    }
    if (tid < 2 && s_y[tid] != ~0ull) atomicMin((unsigned long long*)&a.slots[tile].y[tid], s_y[tid]);
  }
  return true;
}

// ------------------------------------------------------------------------------------------------ mode 1 / 2
// Mode 2: which crossing pieces of a tile can still lower a witness x.  A crossing piece matters for a kind K
// only if its run's whole summary allows a K pair and — for the piece a run crosses IN with (its head lies in an
// earlier tile), in position-ordered runs (lowG == 0) — no entry before this tile is flagged K yet: x_K is a
// minimum position.  need[piece][kind] (piece 0 = crossing in, 1 = crossing out); returns true if nothing is
// needed (C4's `changed`, the far tiles of C3's hot bins, the second tile of a crossing dist[v]).
template <class A>
__device__ bool mode2_skip(const ConflictArgs& a, u32 tile, u8 need[2][2]) {
  typedef typename OpOf<A>::type Op;
  typedef typename QuadOf<A>::type Q;
  need[0][0] = need[0][1] = need[1][0] = need[1][1] = 0;
  const u8 tf = a.tile_flags[tile];
  const A* c = reinterpret_cast<const Q*>(a.carry)[tile].a;    // [grp In, grp Out, ...]
  const A* pp = reinterpret_cast<const Q*>(a.part)[tile].a;    // [grp P, grp S, ...]
  const bool middle = (tf & TF_CIN) && (tf & TF_COUT) && !(tf & TF_GH);
  bool skip = true;
  if ((tf & TF_CIN) && a.phase != 1) {  // piece A: the run crossing in (the whole tile if middle)
    bool done[2];
    const A run = middle ? Op()(Op()(c[0], pp[0]), c[1]) : Op()(c[0], pp[0]);
    cannot_race(run, &done[0], &done[1]);
    if (a.L.lowG == 0) {  // the window starts at the nominal start: the run crossing there is long
      const u64 first = pos_of(a.L, a.keys[(u64)tile * CT_NOM]);
      const Slot* sl = &a.slots[a.owner[tile]];
      for (int k = 0; k < 2; k++) {
        const u64 x = ld_volatile(&sl->x[k]);
        done[k] = done[k] || (x != ~0ull && (x >> 32) < first);
      }
    }
    skip = skip && done[0] && done[1];
    need[0][0] = !done[0], need[0][1] = !done[1];
  }
  if ((tf & TF_COUT) && (tf & TF_GH) && a.phase != 2) {  // piece B: a run starting here and crossing out
    bool done[2];
    cannot_race(Op()(pp[1], c[1]), &done[0], &done[1]);
    skip = skip && done[0] && done[1];
    need[1][0] = !done[0], need[1][1] = !done[1];
  }
  return skip;
}

// Mode 3: does a crossing run this tile takes part in have a witness x (and, position-ordered, no partner y
// before this tile yet)?
__device__ bool mode3_any(const ConflictArgs& a, u32 tile) {
  const u8 tf = a.tile_flags[tile];
  bool any = false;
  if ((tf & TF_CIN) && a.phase != 1) {
    const Slot& sl = a.slots[a.owner[tile]];
    if (a.L.lowG == 0) {
      const u64 first = pos_of(a.L, a.keys[(u64)tile * CT_NOM]);
      for (int k = 0; k < 2; k++) {
        const u64 y = ld_volatile(&sl.y[k]);
        any |= sl.x[k] != ~0ull && !(y != ~0ull && (y >> 32) < first);
      }
    } else {
      any |= sl.x[0] != ~0ull || sl.x[1] != ~0ull;
    }
  }
  if ((tf & TF_COUT) && (tf & TF_GH) && a.phase != 2) {  // (position-ordered: mode 2 found y with x in this piece)
    const Slot& sl = a.slots[tile];
    for (int k = 0; k < 2; k++) any |= sl.x[k] != ~0ull && !(a.L.lowG == 0 && sl.y[k] != ~0ull);
  }
  return any;
}

// Modes 2/3 run persistent CTAs over a worklist of the crossing tiles that still have work (one thread per
// crossing tile decides): skipped tiles cost no CTA launch (C4: 133 K crossing tiles, most skipped in phase 2).
template <class A>
__global__ void cross_filter_kernel(ConflictArgs a, u32 ncross, int mode) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= ncross) return;
  const u32 tile = a.cross_list[i];
  u8 need[2][2];
  const bool keep = mode == 2 ? !mode2_skip<A>(a, tile, need) : mode3_any(a, tile);
  if (keep) a.work[atomicAdd(a.work_count, 1u)] = tile;
}

template <int MODE, class A>
__device__ void conflict_tile(const ConflictArgs& a, TileSmem& s, u32 tile) {
  typedef typename QuadOf<A>::type Q;
  __shared__ u8 s_need[2][2];  // mode 2: piece (A = crossing in, B = crossing out) x kind (RW, WW) can lower x
  if (MODE == 2) {
    __shared__ int s_skip;
    if (threadIdx.x == 0) s_skip = mode2_skip<A>(a, tile, s_need);
    __syncthreads();
    if (s_skip) return;
  }
  u64 tb;
  u32 cnt;
  tile_window(a, tile, &tb, &cnt);
  const KeyLayout& L = a.L;
  const int tid = threadIdx.x;

  if (cnt == 0 || !tile_load<MODE == 1>(a, s, tb, cnt)) {
    if (MODE == 1 && tid == 0) a.tile_flags[tile] = TF_GH | TF_GT | TF_SH | TF_ST;
    return;
  }
  const bool cin = !(s.fl[0] & FL_GH), cout = !(s.fl[cnt - 1] & FL_GT);
  A ci[2], co[2];
  ci[0] = ci[1] = co[0] = co[1] = agg_empty_t<A>();
  if (tid == 0) s.unknown = 0;
  if (MODE == 2) {
    if (cross_pieces_fast<A>(a, s, tile, tb, cnt, cin, cout, s_need)) return;
    tile_gather(a, s, tb, cnt, 0, (int)cnt);  // the scan path: every record
  }
  if (MODE == 2) {
    const A* c = reinterpret_cast<const Q*>(a.carry)[tile].a;  // [grp In, grp Out, sub In, sub Out]
    if (cin) ci[0] = c[0];
    if (cout) co[0] = c[1];
    if (!(s.fl[0] & FL_SH)) ci[1] = c[2];
    if (!(s.fl[cnt - 1] & FL_ST)) co[1] = c[3];
  }
  __shared__ A s_part[4];
  if (MODE == 1 && cin && cout && s.last_ghead < 0) {
    // a window inside one crossing run: mode 1 only owes the carries their pieces (the run-level summary and the
    // first / last sub-run pieces) — plain block reductions; modes 2/3 decide its entries
    typedef typename OpOf<A>::type Op;
    __shared__ int s_fst, s_lsh;
    if (tid == 0) s_fst = (int)cnt - 1, s_lsh = 0;
    __syncthreads();
    bool sh = false, st = false;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = tid * CT_ITEMS + q;
      if (j >= (int)cnt) continue;
      if (s.fl[j] & FL_ST) atomicMin(&s_fst, j), st = true;
      if (s.fl[j] & FL_SH) atomicMax(&s_lsh, j), sh = true;
    }
    const bool any_sh = __syncthreads_or(sh), any_st = __syncthreads_or(st);
    const int fst = s_fst, lsh = s_lsh;
    const A E = agg_empty_t<A>();
    A g = E, p = E, q2 = E;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = tid * CT_ITEMS + q;
      if (j >= (int)cnt) continue;
      g = Op()(g, agg_item_t<A>(s.rw[j], s.blk[j + 1], s.vh[j]));
      const A it = agg_item_t<A>(s.rw[j], s.thr[j], s.vh[j]);
      if (j <= fst) p = Op()(p, it);
      if (j >= lsh) q2 = Op()(q2, it);
    }
    A* wv = scan_scratch<A>(s);  // [WARPS]
    const A red[3] = {g, p, q2};
    for (int r = 0; r < 3; r++) {
      A v = red[r];
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v = Op()(v, shfl(v, o, true));
      if ((tid & 31) == 0) wv[tid >> 5] = v;
      __syncthreads();
      if (tid == 0) {
        A t = wv[0];
        for (int w = 1; w < CT_THREADS / 32; w++) t = Op()(t, wv[w]);
        if (r == 0) s_part[0] = s_part[1] = t;
        else s_part[r + 1] = t;
      }
      __syncthreads();
    }
    if (tid == 0) {
      a.tile_flags[tile] = (any_sh ? TF_SH : 0) | (any_st ? TF_ST : 0) | TF_CIN | TF_COUT;
      for (int i = 0; i < 4; i++) reinterpret_cast<Q*>(a.part)[tile].a[i] = s_part[i];
      a.cross_list[atomicAdd(a.cross_count, 1u)] = tile;
    }
    return;
  }
  // mode 1: the groups wholly inside the window [ilo, ihi) take the fast path (internal_groups) unless one of
  // their sub-runs is long; the crossing pieces only owe the carries their edge summaries (tile_parts)
  const int ilo = cin ? s.first_gtail + 1 : 0, ihi = cout ? s.last_ghead : (int)cnt;
  const bool fast = MODE == 1 && !long_subrun(s, ilo, ihi);
  if (fast) {
    if (cin || cout) tile_parts<A>(s, cnt, s_part);
  } else {
    tile_flags<A>(a, s, cnt, ci, co, MODE == 1 ? s_part : nullptr, MODE == 2 && cin && cout && s.last_ghead < 0);
  }
  const int ftail = s.first_gtail, lhead = s.last_ghead;
  if (s.unknown) {  // a benign query the cheap summary cannot decide: the host reruns with exact summaries
    if (tid == 0) atomicOr(a.need_exact, 1u);
    if (MODE == 1 && tid == 0) a.tile_flags[tile] = TF_GH | TF_GT | TF_SH | TF_ST;
    return;
  }

  if (MODE == 1) {
    // does the tile hold a sub-run head / tail anywhere? (block-wide votes over each thread's items)
    bool my_sh = false, my_st = false;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const u32 j = tid * CT_ITEMS + q;
      if (j < cnt) my_sh |= (s.fl[j] & FL_SH) != 0, my_st |= (s.fl[j] & FL_ST) != 0;
    }
    const bool sh = __syncthreads_or(my_sh), st = __syncthreads_or(my_st);
    if (tid == 0) {
      u8 tf = 0;
      if (lhead >= 0) tf |= TF_GH;
      if (ftail < (int)cnt) tf |= TF_GT;
      if (sh) tf |= TF_SH;
      if (st) tf |= TF_ST;
      if (cin) tf |= TF_CIN;
      if (cout) tf |= TF_COUT;
      a.tile_flags[tile] = tf;
      if (cin || cout) {
        for (int i = 0; i < 4; i++) reinterpret_cast<Q*>(a.part)[tile].a[i] = s_part[i];
        a.cross_list[atomicAdd(a.cross_count, 1u)] = tile;
      }
      if (cout && lhead >= 0) {  // this tile owns the group that crosses out
        Slot sl;
        sl.x[0] = sl.x[1] = sl.y[0] = sl.y[1] = ~0ull;
        sl.head_key = s.key[lhead + 1];
        sl.hblock = s.blk[lhead + 1];
        sl.hinterval = s.ivl[lhead + 1];
        a.slots[tile] = sl;
      }
    }
    if (fast) {
      internal_groups(a, s, ilo, ihi);
      return;
    }
    // no flagged entry in a group internal to the tile (every internal group race-free, e.g. all of C2; or only
    // crossing pieces, e.g. the middle tiles of C3's hot bins — modes 2/3 own those): nothing to emit here
    bool my_res = false;
#pragma unroll kCtUnroll
    for (int q = 0; q < CT_ITEMS; q++) {
      const int j = tid * CT_ITEMS + q;
      if (j < (int)cnt && !(cin && j <= ftail) && !(cout && j >= lhead))
        my_res |= s.res[j] != 0 && (s.fl[j] & FL_INT);
    }
    if (!__syncthreads_or(my_res)) return;
    // x per group: min flagged (position << 11 | item) per kind; every entry then tests P(x, entry)
    const X2 XE = {{~0ull, ~0ull}};
    tile_allreduce<X2>(
        s.fl, FL_GH, FL_GT,
        [&](int j) {
          X2 r = XE;
          if (s.fl[j] & FL_INT) {
            const u64 v = ((u64)pos_of(L, s.key[j + 1]) << 11) | (u64)j;
            if (s.res[j] & 1) r.v[0] = v;
            if (s.res[j] & 2) r.v[1] = v;
          }
          return r;
        },
        OpX2(), XE, XE, XE,
        [&](int j, const X2& X) {
          if (!(s.fl[j] & FL_INT)) return;
          const F5 me = fields(s, j);
#pragma unroll
          for (int k = 0; k < 2; k++) {
            u32 yc = ~0u;
            if (X.v[k] != ~0ull) {
              const int jx = (int)(X.v[k] & 2047);
              if (pair_kind(fields(s, jx), me, a.ws, a.ls) == (u32)(k + 1)) yc = pos_of(L, s.key[j + 1]);
            }
            s.xy[j][k] = yc;  // y candidate of this entry
          }
        },
        s.wx, s.wf);
    __syncthreads();
    // per group: low half = min flagged position (x), high half = min y candidate (y); emit at the tail
    tile_allreduce<X2>(
        s.fl, FL_GH, FL_GT,
        [&](int j) {
          X2 r = XE;
          if (s.fl[j] & FL_INT) {
            const u32 p = pos_of(L, s.key[j + 1]);
            r.v[0] = ((u64)s.xy[j][0] << 32) | ((s.res[j] & 1) ? p : 0xFFFFFFFFu);
            r.v[1] = ((u64)s.xy[j][1] << 32) | ((s.res[j] & 2) ? p : 0xFFFFFFFFu);
          }
          return r;
        },
        OpXY(), XE, XE, XE,
        [&](int j, const X2& T) {
          if (!(s.fl[j] & FL_INT) || !(s.fl[j] & FL_GT)) return;
          if ((cin && j <= ftail) || (cout && j >= lhead)) return;  // crossing groups: modes 2/3
#pragma unroll
          for (int k = 0; k < 2; k++) {
            const u32 x = (u32)(T.v[k] & 0xFFFFFFFFull), y = (u32)(T.v[k] >> 32);
            if (x == 0xFFFFFFFFu) continue;
            // every entry of a group has the group's (space, granule) and, for shared memory, its (block,
            // interval): the tail entry describes the location
            emit_race(a, s.key[j + 1] >> L.pos_bits, (u32)(k + 1), x, y, s.blk[j + 1], s.ivl[j + 1]);
          }
        },
        s.wx, s.wf);
    return;
  }

  // MODE 2: exact flags of the crossing pieces -> x candidates into the owner's slot
  // pieces: [0, ftail] if cin (owner = a.owner[tile]); [lhead, cnt-1] if cout (owner = tile, or a.owner[tile]
  // when the whole tile is one group)
  __shared__ unsigned long long s_min[4];
  if (tid < 4) s_min[tid] = ~0ull;
  __syncthreads();
  const int j0 = tid * CT_ITEMS;
#pragma unroll kCtUnroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = j0 + q;
    if (j >= (int)cnt || !(s.fl[j] & FL_INT)) continue;
    // (position, entry index): the witness is the min POSITION (with an unsorted-input layout, entries of a run
    // are ordered by (block, interval) first); the entry index locates its record in mode 3
    const unsigned long long p = ((unsigned long long)pos_of(L, s.key[j + 1]) << 32) | (u32)(tb + j);
    const bool A = cin && j <= ftail && a.phase != 1, B = cout && j >= lhead && a.phase != 2;
    if (A) {
      if (s.res[j] & 1) atomicMin(&s_min[0], p);
      if (s.res[j] & 2) atomicMin(&s_min[1], p);
    }
    if (B && !A) {
      if (s.res[j] & 1) atomicMin(&s_min[2], p);
      if (s.res[j] & 2) atomicMin(&s_min[3], p);
    }
  }
  __syncthreads();
  if (tid == 0) {
    if (cin) {
      Slot* sl = &a.slots[a.owner[tile]];
      if (s_min[0] != ~0ull) atomicMin((unsigned long long*)&sl->x[0], s_min[0]);
      if (s_min[1] != ~0ull) atomicMin((unsigned long long*)&sl->x[1], s_min[1]);
    }
    if (cout && lhead >= 0 && !(cin && lhead <= ftail)) {
      Slot* sl = &a.slots[tile];
      if (s_min[2] != ~0ull) atomicMin((unsigned long long*)&sl->x[0], s_min[2]);
      if (s_min[3] != ~0ull) atomicMin((unsigned long long*)&sl->x[1], s_min[3]);
    }
  }
}

template <int MODE, class A>
// mode 1 at 3 CTAs/SM (the shared-memory limit): up to 80 registers, no spills; mode 2 at 2 (128 registers)
__global__ void __launch_bounds__(CT_THREADS, MODE == 1 ? 3 : 2) conflict_kernel(ConflictArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  TileSmem& s = *reinterpret_cast<TileSmem*>(smem_raw);
  if (MODE == 1) {
    conflict_tile<MODE, A>(a, s, blockIdx.x);
  } else {
    const u32 nw = *a.work_count;
    for (u32 w = blockIdx.x; w < nw; w += gridDim.x) {
      conflict_tile<MODE, A>(a, s, a.work[w]);
      __syncthreads();
    }
  }
}

// ------------------------------------------------------------------------------------------------ mode 3: y
__device__ void y_tile(const ConflictArgs& a, TileSmem& s, u32 tile) {
  {
    // nothing to do unless a crossing run this tile takes part in has a witness x (re-checked: other tiles of
    // the phase may have lowered y since the worklist was made)
    __shared__ int s_any;
    if (threadIdx.x == 0) s_any = mode3_any(a, tile);
    __syncthreads();
    if (!s_any) return;
  }
  u64 tb;
  u32 cnt;
  tile_window(a, tile, &tb, &cnt);
  const KeyLayout& L = a.L;
  const int tid = threadIdx.x;
  if (cnt == 0 || !tile_load<false>(a, s, tb, cnt)) return;
  const bool cin = !(s.fl[0] & FL_GH), cout = !(s.fl[cnt - 1] & FL_GT);
  const int ftail = s.first_gtail, lhead = s.last_ghead;
  __shared__ F5 s_x[2][2];
  __shared__ u32 s_has[2][2];
  __shared__ unsigned long long s_min[2][2];
  __shared__ u32 s_owner[2];
  if (tid == 0) {
    s_owner[0] = cin && a.phase != 1 ? a.owner[tile] : ~0u;
    s_owner[1] = (cout && lhead >= 0 && !(cin && lhead <= ftail)) && a.phase != 2 ? tile : ~0u;
  }
  __syncthreads();
  if (tid < 4) {
    const int g = tid >> 1, k = tid & 1;
    s_has[g][k] = 0;
    s_min[g][k] = ~0ull;
    if (s_owner[g] != ~0u) {
      const u64 xp = a.slots[s_owner[g]].x[k];
      if (xp != ~0ull) {
        const u32 x = (u32)(xp & 0xFFFFFFFFull);
        const Rec r = rec_at(a, x, a.keys[x]);
        F5 f;
        f.block = r.block, f.interval = r.interval, f.thread = r.thread, f.rw = r.rw, f.vh = r.vh;
        s_x[g][k] = f;
        s_has[g][k] = 1;
      }
    }
  }
  __syncthreads();
  // records of the pieces only
  if (s_owner[0] != ~0u && (s_has[0][0] || s_has[0][1])) tile_gather(a, s, tb, cnt, 0, min(ftail, (int)cnt - 1) + 1);
  if (s_owner[1] != ~0u && (s_has[1][0] || s_has[1][1])) tile_gather(a, s, tb, cnt, lhead, (int)cnt);
  const int j0 = tid * CT_ITEMS;
#pragma unroll
  for (int q = 0; q < CT_ITEMS; q++) {
    const int j = j0 + q;
    if (j >= (int)cnt || !(s.fl[j] & FL_INT)) continue;
    const bool A = cin && j <= ftail && s_owner[0] != ~0u, B = cout && j >= lhead && s_owner[1] != ~0u;
    const int g = A ? 0 : (B ? 1 : -1);
    if (g < 0) continue;
    const F5 me = fields(s, j);
    const unsigned long long p = ((unsigned long long)pos_of(L, s.key[j + 1]) << 32) | (u32)(tb + j);
    for (int k = 0; k < 2; k++)
      if (s_has[g][k] && pair_kind(s_x[g][k], me, a.ws, a.ls) == (u32)(k + 1)) atomicMin(&s_min[g][k], p);
  }
  __syncthreads();
  if (tid < 4) {
    const int g = tid >> 1, k = tid & 1;
    if (s_owner[g] != ~0u && s_min[g][k] != ~0ull)
      atomicMin((unsigned long long*)&a.slots[s_owner[g]].y[k], s_min[g][k]);
  }
}

__global__ void __launch_bounds__(CT_THREADS) conflict_y_kernel(ConflictArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  TileSmem& s = *reinterpret_cast<TileSmem*>(smem_raw);
  const u32 nw = *a.work_count;
  for (u32 w = blockIdx.x; w < nw; w += gridDim.x) {
    y_tile(a, s, a.work[w]);
    __syncthreads();
  }
}

// one race per (crossing group, kind) with a witness; owner tiles are the crossing tiles with TF_COUT whose
// last group head lies inside the tile
__global__ void cross_emit_kernel(ConflictArgs a, u32 ncross) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= ncross) return;
  const u32 tile = a.cross_list[i];
  if (!(a.tile_flags[tile] & TF_COUT) || !(a.tile_flags[tile] & TF_GH)) return;
  // the crossing-out group's head is in this tile only if the tile has a group head (TF_GH) — then the last
  // head is the crossing group's head (slots[tile] was written by mode 1)
  const Slot sl = a.slots[tile];
  for (int k = 0; k < 2; k++)
    if (sl.x[k] != ~0ull)  // (position << 32 | entry): report positions
      emit_race(a, sl.head_key >> a.L.pos_bits, (u32)(k + 1), (u32)(sl.x[k] >> 32), (u32)(sl.y[k] >> 32), sl.hblock,
                sl.hinterval);
}

__global__ void races_set_epoch_kernel(const RaceOut* __restrict__ in, u32 nr, u32 e, RaceOut* __restrict__ out) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < nr) {
    RaceOut r = in[i];
    r.epoch = e;
    out[i] = r;
  }
}

void launch_races_set_epoch(const RaceOut* in, u32 nr, u32 e, RaceOut* out, cudaStream_t st) {
  if (nr) races_set_epoch_kernel<<<(nr + 255) / 256, 256, 0, st>>>(in, nr, e, out);
}

// ------------------------------------------------------------------------------------------------ precise warps
// SURVEY §8f NEXT-3 (reading R24).  With lockstep on, records extended with {pc, div}:
// intra-warp pairs race only on the two sides of one divergent branch instance (any kind) or as two writes at
// one instruction (W/W).  The per-location witness is the lexicographic minimum over the union of
//   (A) the pairs of different warps (or blocks): the ordinary conflict tiles with identity = warp (tdiv = ws,
//       lockstep off) — two records of one warp then look like one thread (rule 1) — and
//   (B) the pairs inside one (location, block, interval, warp) group, checked pair by pair (such groups hold at
//       most 32 threads' accesses): entries regrouped by a sort on (run ordinal, hash of (block, interval, warp)).
// Both halves fold their pairs into one atomicMin slot per (run, kind) as (position << 32 | position).
__device__ __forceinline__ u32 warp_hash(u32 b, u32 i, u32 w) {
  return (u32)(sesa_mix(((u64)b << 32) ^ ((u64)i << 20) ^ (u64)w) >> 32);
}

// run heads and the (block, interval, warp) hash of every compacted entry
__global__ void warp_key_kernel(const u64* __restrict__ comp, u32 m2, KeyLayout L, const Rec* __restrict__ rec,
                                u32 ws, u32* __restrict__ head, u32* __restrict__ hkey) {
  const u32 j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= m2) return;
  const u64 k = comp[j];
  head[j] = (j == 0 || group_of_hi(L, k >> L.pos_bits) != group_of_hi(L, comp[j - 1] >> L.pos_bits)) ? 1u : 0u;
  const Rec r = load_rec(rec + pos_of(L, k));
  hkey[j] = warp_hash(r.block, r.interval, r.thread / ws);
}

__global__ void warp_key2_kernel(const u32* __restrict__ head, const u32* __restrict__ hscan,
                                 const u32* __restrict__ hkey, u32 m2, u64* __restrict__ key2, u32* __restrict__ val) {
  const u32 j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= m2) return;
  key2[j] = ((u64)(hscan[j] + head[j] - 1) << 32) | hkey[j];
  val[j] = j;
}

// (B): thread p checks its entry against the later entries of its (run, hash) segment, pair by pair
__global__ void warp_pairs_kernel(const u64* __restrict__ comp, KeyLayout L, const Rec* __restrict__ rec,
                                  const uint2* __restrict__ ext, u32 ws, const u64* __restrict__ key2,
                                  const u32* __restrict__ order, u32 m2, unsigned long long* __restrict__ slot) {
  const u32 p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= m2) return;
  const u64 kk = key2[p];
  if (p + 1 >= m2 || key2[p + 1] != kk) return;
  const u32 x = order[p], px = pos_of(L, comp[x]);
  const Rec X = load_rec(rec + px);
  const uint2 ex = ext[px];
  const u32 gid = (u32)(kk >> 32);
  for (u32 q = p + 1; q < m2 && key2[q] == kk; q++) {
    const u32 py = pos_of(L, comp[order[q]]);
    const Rec Y = load_rec(rec + py);
    if (X.block != Y.block || X.interval != Y.interval || X.thread / ws != Y.thread / ws) continue;  // hash twin
    if (X.thread == Y.thread) continue;                                                      // (1)
    if (X.rw == RW_READ && Y.rw == RW_READ) continue;                                        // (2)
    if (X.rw == RW_ATOMIC && Y.rw == RW_ATOMIC) continue;                                    // (3)
    const u32 kind = (X.rw == RW_READ || Y.rw == RW_READ) ? KIND_RW : KIND_WW;
    const uint2 ey = ext[py];
    const bool divergent = ex.y != 0 && ey.y != 0 && (ex.y >> 1) == (ey.y >> 1) && ((ex.y ^ ey.y) & 1u);
    if (!divergent && (kind == KIND_RW || ex.x != ey.x)) continue;                           // (5')
    if (X.rw == RW_WRITE && Y.rw == RW_WRITE && X.vh == Y.vh) continue;                      // (6)
    const u32 lo = min(px, py), hi = max(px, py);
    atomicMin(&slot[2 * (u64)gid + kind - 1], ((unsigned long long)lo << 32) | hi);
  }
}

// (A): the inter-warp races of the ordinary conflict tiles, folded into the slots of their runs
__global__ void warp_fold_kernel(const u64* __restrict__ rkeys, const RaceOut* __restrict__ races, u32 nr,
                                 const u64* __restrict__ comp, u32 m2, KeyLayout L, const u32* __restrict__ hscan,
                                 u64 index_base, unsigned long long* __restrict__ slot) {
  const u32 r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= nr) return;
  const u64 hk = rkeys[r] >> 2;
  const u32 kind = (u32)(rkeys[r] & 3) + 1;
  u32 lo = 0, hi = m2;  // first entry of the run: lower bound of its group key
  while (lo < hi) {
    const u32 mid = (lo + hi) >> 1;
    if (group_of_hi(L, comp[mid] >> L.pos_bits) < hk) lo = mid + 1;
    else hi = mid;
  }
  const RaceOut x = races[r];
  atomicMin(&slot[2 * (u64)hscan[lo] + kind - 1],
            ((unsigned long long)(x.first - index_base) << 32) | (unsigned long long)(x.second - index_base));
}

__global__ void warp_emit_kernel(ConflictArgs a, const u32* __restrict__ head, const u32* __restrict__ hscan,
                                 const unsigned long long* __restrict__ slot) {
  const u32 j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= a.m || !head[j]) return;
  const u32 gid = hscan[j];
  const u64 k = a.keys[j];
  for (u32 kind = KIND_RW; kind <= KIND_WW; kind++) {
    const unsigned long long v = slot[2 * (u64)gid + kind - 1];
    if (v == ~0ull) continue;
    const Rec r = load_rec(a.rec + pos_of(a.L, k));
    emit_race(a, k >> a.L.pos_bits, kind, (u32)(v >> 32), (u32)v, r.block, r.interval);
  }
}

void launch_warp_keys(const u64* comp, u32 m2, const KeyLayout& L, const Rec* rec, u32 ws, u32* head, u32* hkey,
                      cudaStream_t st) {
  if (m2) warp_key_kernel<<<(m2 + 255) / 256, 256, 0, st>>>(comp, m2, L, rec, ws, head, hkey);
}
void launch_warp_key2(const u32* head, const u32* hscan, const u32* hkey, u32 m2, u64* key2, u32* val, cudaStream_t st) {
  if (m2) warp_key2_kernel<<<(m2 + 255) / 256, 256, 0, st>>>(head, hscan, hkey, m2, key2, val);
}
void launch_warp_pairs(const u64* comp, const KeyLayout& L, const Rec* rec, const void* ext, u32 ws, const u64* key2,
                       const u32* order, u32 m2, unsigned long long* slot, cudaStream_t st) {
  if (m2)
    warp_pairs_kernel<<<(m2 + 255) / 256, 256, 0, st>>>(comp, L, rec, (const uint2*)ext, ws, key2, order, m2, slot);
}
void launch_warp_fold(const u64* rkeys, const RaceOut* races, u32 nr, const u64* comp, u32 m2, const KeyLayout& L,
                      const u32* hscan, u64 index_base, unsigned long long* slot, cudaStream_t st) {
  if (nr) warp_fold_kernel<<<(nr + 255) / 256, 256, 0, st>>>(rkeys, races, nr, comp, m2, L, hscan, index_base, slot);
}
void launch_warp_emit(const ConflictArgs& a, const u32* head, const u32* hscan, const unsigned long long* slot,
                      cudaStream_t st) {
  if (a.m) warp_emit_kernel<<<(a.m + 255) / 256, 256, 0, st>>>(a, head, hscan, slot);
}

u32 conflict_tiles(u64 m) { return (u32)((m + CT_NOM - 1) / CT_NOM); }

template <int MODE, class A>
static void launch_ck(const ConflictArgs& a, u32 nblocks, cudaStream_t st) {
  const size_t sm = sizeof(TileSmem);
  smem_optin((const void*)conflict_kernel<MODE, A>, sm);
  conflict_kernel<MODE, A><<<nblocks, CT_THREADS, sm, st>>>(a);
}

// modes 2/3: nblocks = crossing tiles; a filter kernel makes the worklist, persistent CTAs (one full wave) take it
void launch_conflict(int mode, bool exact, const ConflictArgs& a, u32 nblocks, cudaStream_t st) {
  if (!nblocks) return;
  const size_t sm = sizeof(TileSmem);
  if (mode == 1) {
    if (exact) launch_ck<1, Agg>(a, nblocks, st);
    else launch_ck<1, AggC>(a, nblocks, st);
    return;
  }
  cudaMemsetAsync(a.work_count, 0, 4, st);
  if (exact) cross_filter_kernel<Agg><<<(nblocks + 255) / 256, 256, 0, st>>>(a, nblocks, mode);
  else cross_filter_kernel<AggC><<<(nblocks + 255) / 256, 256, 0, st>>>(a, nblocks, mode);
  const void* k = mode == 3 ? (const void*)conflict_y_kernel
                            : exact ? (const void*)conflict_kernel<2, Agg> : (const void*)conflict_kernel<2, AggC>;
  smem_optin(k, sm);
  const u32 wave = (u32)(dev_sm_count() * std::max(1, blocks_per_sm(k, CT_THREADS, sm)));
  const u32 grid = std::min(nblocks, wave);
  if (mode == 3) conflict_y_kernel<<<grid, CT_THREADS, sm, st>>>(a);
  else if (exact) conflict_kernel<2, Agg><<<grid, CT_THREADS, sm, st>>>(a);
  else conflict_kernel<2, AggC><<<grid, CT_THREADS, sm, st>>>(a);
}

void launch_cross_emit(const ConflictArgs& a, u32 ncross, cudaStream_t st) {
  if (ncross) cross_emit_kernel<<<(ncross + 255) / 256, 256, 0, st>>>(a, ncross);
}

// ------------------------------------------------------------------------------------------------ carries
// Segmented scans over tiles: for level L in {group, sub-run}:
//   In_L[j+1]  = (tile j has an L-head) ? S_L[j] : In_L[j] (+) S_L[j]     (forward)
//   Out_L[j-1] = (tile j has an L-tail) ? P_L[j] : P_L[j] (+) Out_L[j]    (backward)
//   owner[j+1] = (tile j has a group head) ? j : owner[j]
// computed in chunks of 1024 tiles (one CTA each), chunk carries by one CTA, then applied.
constexpr int CARRY_T = 1024;

template <class A>
struct CarryEl {
  A a;
  u32 owner;
  u32 pad;  // explicit (always 0): stored with the struct, so global copies carry no uninitialised bytes
};

template <class A>
struct OpCarry {
  __device__ __forceinline__ CarryEl<A> operator()(const CarryEl<A>& x, const CarryEl<A>& y) const {
    CarryEl<A> r;
    r.a = typename OpOf<A>::type()(x.a, y.a);
    r.owner = max(x.owner, y.owner);
    r.pad = 0;
    return r;
  }
};
template <class A>
__device__ __forceinline__ CarryEl<A> shfl(const CarryEl<A>& c, int o, bool down) {
  CarryEl<A> r;
  r.a = shfl(c.a, o, down);
  r.owner = shfl(c.owner, o, down);
  r.pad = 0;
  return r;
}

// scan direction d: 0 grp fwd, 1 grp bwd, 2 sub fwd, 3 sub bwd
template <class A>
__device__ __forceinline__ void carry_element(const ConflictArgs& a, u32 j, u32 ntiles, int d, bool& f,
                                              CarryEl<A>& e) {
  typedef typename QuadOf<A>::type Q;
  e.a = agg_empty_t<A>();
  e.owner = 0;
  e.pad = 0;
  f = true;
  if (j >= ntiles) return;
  const u8 tf = a.tile_flags[j];
  const bool crossing = tf & (TF_CIN | TF_COUT);
  const u8 bit = d == 0 ? TF_GH : d == 1 ? TF_GT : d == 2 ? TF_SH : TF_ST;
  f = (tf & bit) != 0;
  const int pi = d == 0 ? 1 : d == 1 ? 0 : d == 2 ? 3 : 2;  // fwd uses S (last piece), bwd uses P (first piece)
  if (crossing) e.a = reinterpret_cast<const Q*>(a.part)[j].a[pi];
  e.owner = (d == 0 && f) ? j : 0;
}

template <class A, bool REV>
__device__ CarryEl<A> carry_block_scan(bool f, const CarryEl<A>& v, const CarryEl<A>& seed, CarryEl<A>* s_wv,
                                       u8* s_wf) {
  // inclusive = exclusive (+) own
  CarryEl<A> ex = block_seg_excl<CarryEl<A>, OpCarry<A>, REV, CARRY_T>(f, v, seed, OpCarry<A>(), s_wv, s_wf);
  return f ? v : OpCarry<A>()(ex, v);
}

template <class A>
__global__ void __launch_bounds__(CARRY_T) carry_chunk_kernel(ConflictArgs a, u32 ntiles, CarryEl<A>* chunk_tot,
                                                              u8* chunk_f) {
  __shared__ CarryEl<A> s_wv[CARRY_T / 32];
  __shared__ u8 s_wf[CARRY_T / 32];
  const u32 j = blockIdx.x * CARRY_T + threadIdx.x;
  for (int d = 0; d < 4; d++) {
    bool f;
    CarryEl<A> e;
    carry_element<A>(a, j, ntiles, d, f, e);
    CarryEl<A> seed;
    seed.a = agg_empty_t<A>(), seed.owner = 0, seed.pad = 0;
    const bool rev = d & 1;
    CarryEl<A> inc = rev ? carry_block_scan<A, true>(f, e, seed, s_wv, s_wf)
                         : carry_block_scan<A, false>(f, e, seed, s_wv, s_wf);
    const bool flag_any = __syncthreads_or(f);
    // chunk total = inclusive value at the chunk's last (fwd) / first (bwd) thread
    if ((!rev && threadIdx.x == CARRY_T - 1) || (rev && threadIdx.x == 0)) {
      chunk_tot[blockIdx.x * 4 + d] = inc;
      chunk_f[blockIdx.x * 4 + d] = flag_any;
    }
    __syncthreads();
  }
}

template <class A>
__global__ void __launch_bounds__(CARRY_T) carry_top_kernel(u32 nchunks, CarryEl<A>* chunk_tot, u8* chunk_f,
                                                            CarryEl<A>* chunk_carry) {
  __shared__ CarryEl<A> s_wv[CARRY_T / 32];
  __shared__ u8 s_wf[CARRY_T / 32];
  const u32 c = threadIdx.x;
  for (int d = 0; d < 4; d++) {
    CarryEl<A> e;
    bool f = true;
    e.a = agg_empty_t<A>(), e.owner = 0, e.pad = 0;
    if (c < nchunks) e = chunk_tot[c * 4 + d], f = chunk_f[c * 4 + d];
    CarryEl<A> seed;
    seed.a = agg_empty_t<A>(), seed.owner = 0, seed.pad = 0;
    CarryEl<A> ex =
        (d & 1) ? block_seg_excl<CarryEl<A>, OpCarry<A>, true, CARRY_T>(f, e, seed, OpCarry<A>(), s_wv, s_wf)
                : block_seg_excl<CarryEl<A>, OpCarry<A>, false, CARRY_T>(f, e, seed, OpCarry<A>(), s_wv, s_wf);
    if (c < nchunks) chunk_carry[c * 4 + d] = ex;
  }
}

template <class A>
__global__ void __launch_bounds__(CARRY_T) carry_apply_kernel(ConflictArgs a, u32 ntiles,
                                                              const CarryEl<A>* chunk_carry) {
  typedef typename QuadOf<A>::type Q;
  __shared__ CarryEl<A> s_wv[CARRY_T / 32];
  __shared__ u8 s_wf[CARRY_T / 32];
  const u32 j = blockIdx.x * CARRY_T + threadIdx.x;
  for (int d = 0; d < 4; d++) {
    bool f;
    CarryEl<A> e;
    carry_element<A>(a, j, ntiles, d, f, e);
    const bool rev = d & 1;
    const CarryEl<A> seed = chunk_carry[blockIdx.x * 4 + d];
    CarryEl<A> inc = rev ? carry_block_scan<A, true>(f, e, seed, s_wv, s_wf)
                         : carry_block_scan<A, false>(f, e, seed, s_wv, s_wf);
    // fwd inclusive at j feeds tile j+1; bwd inclusive at j feeds tile j-1
    const long long tgt = rev ? (long long)j - 1 : (long long)j + 1;
    if (j < ntiles && tgt >= 0 && tgt < (long long)ntiles) {
      const u8 tt = a.tile_flags[tgt];
      const bool need = rev ? (tt & TF_COUT) : (tt & TF_CIN);
      if (need) {
        reinterpret_cast<Q*>(a.carry)[tgt].a[d] = inc.a;
        if (d == 0) a.owner[tgt] = inc.owner;
      }
    }
  }
}

size_t carry_temp_bytes(u32 ntiles) {
  const u32 nch = (ntiles + CARRY_T - 1) / CARRY_T;
  return (size_t)nch * 4 * sizeof(CarryEl<Agg>) * 2 + (size_t)nch * 4 + 256;
}

template <class A>
static void launch_carry_t(const ConflictArgs& a, u32 ntiles, void* temp, cudaStream_t st) {
  const u32 nch = (ntiles + CARRY_T - 1) / CARRY_T;
  CarryEl<A>* tot = reinterpret_cast<CarryEl<A>*>(temp);
  CarryEl<A>* car = tot + (size_t)nch * 4;
  u8* fl = reinterpret_cast<u8*>(car + (size_t)nch * 4);
  carry_chunk_kernel<A><<<nch, CARRY_T, 0, st>>>(a, ntiles, tot, fl);
  carry_top_kernel<A><<<1, CARRY_T, 0, st>>>(nch, tot, fl, car);
  carry_apply_kernel<A><<<nch, CARRY_T, 0, st>>>(a, ntiles, car);
}

void launch_carry(bool exact, const ConflictArgs& a, u32 ntiles, void* temp, cudaStream_t st) {
  if (exact) launch_carry_t<Agg>(a, ntiles, temp, st);
  else launch_carry_t<AggC>(a, ntiles, temp, st);
}

// canonical sort key of a race record (as emitted by emit_race) rebuilt from its fields (rank-0 merge)
__global__ void race_rekey_kernel(const RaceOut* __restrict__ r, u64 n, KeyLayout L, u64* __restrict__ keys,
                                  u32* __restrict__ vals) {
  const u64 i = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const RaceOut x = r[i];
  // global races carry block = interval = NOBI: use the layout minima so the (masked) low fields stay zero
  const bool glob = x.space == SP_GLOBAL;
  const u64 hi = key_hi_of(L, x.space, glob ? L.bminG : x.block, glob ? L.iminG : x.interval, x.addr >> L.log2G);
  keys[i] = (group_of_hi(L, hi) << 2) | (u64)(x.kind - 1);
  vals[i] = (u32)i;
}

void race_rekey_launch(const RaceOut* r, u64 n, const KeyLayout& L, u64* keys, u32* vals, cudaStream_t st) {
  if (n) race_rekey_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(r, n, L, keys, vals);
}

__global__ void permute_races_kernel(const RaceOut* __restrict__ in, const u32* __restrict__ order,
                                     RaceOut* __restrict__ out, u32 nr) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < nr) out[i] = in[order[i]];
}

void launch_permute_races(const RaceOut* in, const u32* order, RaceOut* out, u32 nr, cudaStream_t st) {
  if (nr) permute_races_kernel<<<(nr + 255) / 256, 256, 0, st>>>(in, order, out, nr);
}


// ------------------------------------------------------------------------------------------------ benign W/W
// SURVEY §8f NEXT-4 (Table IV "W/W (Benign)" P:467): with SESA_FLAG_REPORT_BENIGN every location holding a
// benign pair — two plain writes of one value by different threads, unordered — gets one kind-3 record.  "Exists
// a plain write with another identity AND the same value" is not a min/max summary query, so the plain writes
// of multi-entry locations are regrouped by (location, value) (sort by value, then stable by location ordinal)
// and become a DERIVED trace: one plain write per entry, location = its (location, value) run, distinct values.
// A W/W race of the derived trace (the ordinary pipeline, rule (6) never fires) is exactly a benign pair of the
// original, and because a run lists its entries in original position order the derived witness maps to the
// original lexicographic minimum; the minimum over a location's runs is taken with one atomicMin per race.

// The record of compacted entry j: by its position (single GPU), or entry-aligned (rec_entry: the distributed
// check fetches the records of multi-entry locations from their owner ranks, dist.cu)
__device__ __forceinline__ Rec benign_rec(const Rec* rec, const Rec* rec_entry, const KeyLayout& L, const u64* comp,
                                          u32 j) {
  return rec_entry ? load_rec(rec_entry + j) : load_rec(rec + pos_of(L, comp[j]));
}

// head flag (first entry of a location run) and plain-write flag of every compacted entry
__global__ void benign_mark_kernel(const u64* __restrict__ comp, u32 m2, KeyLayout L, const Rec* __restrict__ rec, const Rec* __restrict__ rec_entry,
                                   u32* __restrict__ head, u32* __restrict__ wflag) {
  const u32 j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= m2) return;
  const u64 k = comp[j];
  head[j] = (j == 0 || group_of_hi(L, k >> L.pos_bits) != group_of_hi(L, comp[j - 1] >> L.pos_bits)) ? 1u : 0u;
  wflag[j] = benign_rec(rec, rec_entry, L, comp, j).rw == RW_WRITE ? 1u : 0u;
}

// plain writes -> (value, entry) pairs at their exclusive write rank; location ordinal of every entry
__global__ void benign_gather_kernel(const u64* __restrict__ comp, u32 m2, KeyLayout L, const Rec* __restrict__ rec, const Rec* __restrict__ rec_entry,
                                     const u32* __restrict__ head, const u32* __restrict__ hscan,
                                     const u32* __restrict__ wflag, const u32* __restrict__ wscan,
                                     u32* __restrict__ gid, u64* __restrict__ vkey, u32* __restrict__ vidx) {
  const u32 j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= m2) return;
  gid[j] = hscan[j] + head[j] - 1;
  if (wflag[j]) {
    vkey[wscan[j]] = benign_rec(rec, rec_entry, L, comp, j).vh;
    vidx[wscan[j]] = j;
  }
}

// sort keys of the plain-write list (entry vidx[i]): 0 = original position, 1 = value hash, 2 = location ordinal
__global__ void benign_keys_kernel(const u64* __restrict__ comp, KeyLayout L, const Rec* __restrict__ rec, const Rec* __restrict__ rec_entry,
                                   const u32* __restrict__ vidx, u32 m3, const u32* __restrict__ gid, int what,
                                   u64* __restrict__ keys) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m3) return;
  const u32 j = vidx[i];
  keys[i] = what == 2 ? (u64)gid[j] : what == 0 ? (u64)pos_of(L, comp[j]) : benign_rec(rec, rec_entry, L, comp, j).vh;
}

// run heads of the (location, value) order
__global__ void benign_runs_kernel(const u64* __restrict__ comp, KeyLayout L, const Rec* __restrict__ rec, const Rec* __restrict__ rec_entry,
                                   const u32* __restrict__ gid, const u32* __restrict__ order, u32 m3,
                                   u32* __restrict__ rhead) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m3) return;
  const u32 j = order[i];
  bool h = i == 0;
  if (!h) {
    const u32 jp = order[i - 1];
    h = gid[jp] != gid[j] || benign_rec(rec, rec_entry, L, comp, jp).vh != benign_rec(rec, rec_entry, L, comp, j).vh;
  }
  rhead[i] = h ? 1u : 0u;
}

// derived trace: record i = plain write of entry order[i] at location (its space, block, interval, run id) with
// granularity 1 and the distinct value i + 1; dpos[i] = original position, dj[i] = entry
__global__ void benign_derive_kernel(const u64* __restrict__ comp, KeyLayout L, const Rec* __restrict__ rec, const Rec* __restrict__ rec_entry,
                                     const u32* __restrict__ order, const u32* __restrict__ rhead,
                                     const u32* __restrict__ rscan, u32 m3, Rec* __restrict__ out,
                                     u32* __restrict__ dpos, u32* __restrict__ dj) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= m3) return;
  const u32 j = order[i];
  const u32 p = pos_of(L, comp[j]);
  const Rec r = benign_rec(rec, rec_entry, L, comp, j);
  Rec d = r;
  d.addr = rscan[i] + rhead[i] - 1;
  d.vh = (u64)i + 1;
  d.size = 1;
  d.rw = RW_WRITE;
  out[i] = d;
  dpos[i] = p;
  dj[i] = j;
}

// child W/W races -> per location the lexicographic minimum (first << 32 | second) of original positions
__global__ void benign_min_kernel(const RaceOut* __restrict__ cr, u32 nc, const u32* __restrict__ dpos,
                                  const u32* __restrict__ dj, const u32* __restrict__ gid,
                                  unsigned long long* __restrict__ slot) {
  const u32 c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= nc) return;
  const RaceOut x = cr[c];
  const unsigned long long v = ((unsigned long long)dpos[x.first] << 32) | dpos[x.second];
  atomicMin(&slot[gid[dj[x.first]]], v);
}

__global__ void benign_emit_kernel(ConflictArgs a, const RaceOut* __restrict__ cr, u32 nc,
                                   const u32* __restrict__ dpos, const u32* __restrict__ dj,
                                   const u32* __restrict__ gid, const unsigned long long* __restrict__ slot) {
  const u32 c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= nc) return;
  const RaceOut x = cr[c];
  const u32 j = dj[x.first];
  const unsigned long long v = ((unsigned long long)dpos[x.first] << 32) | dpos[x.second];
  if (slot[gid[j]] != v) return;  // pairs are unique per location: exactly one child race wins
  const u64 k = a.keys[j];
  const Rec r = benign_rec(a.rec, a.rec_entry, a.L, a.keys, j);
  emit_race(a, k >> a.L.pos_bits, KIND_WWB, dpos[x.first], dpos[x.second], r.block, r.interval);
}

void launch_benign_mark(const u64* comp, u32 m2, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, u32* head, u32* wflag,
                        cudaStream_t st) {
  if (m2) benign_mark_kernel<<<(m2 + 255) / 256, 256, 0, st>>>(comp, m2, L, rec, rec_entry, head, wflag);
}
void launch_benign_gather(const u64* comp, u32 m2, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* head,
                          const u32* hscan, const u32* wflag, const u32* wscan, u32* gid, u64* vkey, u32* vidx,
                          cudaStream_t st) {
  if (m2)
    benign_gather_kernel<<<(m2 + 255) / 256, 256, 0, st>>>(comp, m2, L, rec, rec_entry, head, hscan, wflag, wscan, gid, vkey,
                                                           vidx);
}
void launch_benign_keys(const u64* comp, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* vidx, u32 m3, const u32* gid,
                        int what, u64* keys, cudaStream_t st) {
  if (m3) benign_keys_kernel<<<(m3 + 255) / 256, 256, 0, st>>>(comp, L, rec, rec_entry, vidx, m3, gid, what, keys);
}
void launch_benign_runs(const u64* comp, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* gid, const u32* order,
                        u32 m3, u32* rhead, cudaStream_t st) {
  if (m3) benign_runs_kernel<<<(m3 + 255) / 256, 256, 0, st>>>(comp, L, rec, rec_entry, gid, order, m3, rhead);
}
void launch_benign_derive(const u64* comp, const KeyLayout& L, const Rec* rec, const Rec* rec_entry, const u32* order, const u32* rhead,
                          const u32* rscan, u32 m3, Rec* out, u32* dpos, u32* dj, cudaStream_t st) {
  if (m3)
    benign_derive_kernel<<<(m3 + 255) / 256, 256, 0, st>>>(comp, L, rec, rec_entry, order, rhead, rscan, m3, out, dpos, dj);
}
void launch_benign_min_emit(const ConflictArgs& a, const RaceOut* cr, u32 nc, const u32* dpos, const u32* dj,
                            const u32* gid, unsigned long long* slot, cudaStream_t st) {
  if (!nc) return;
  benign_min_kernel<<<(nc + 255) / 256, 256, 0, st>>>(cr, nc, dpos, dj, gid, slot);
  benign_emit_kernel<<<(nc + 255) / 256, 256, 0, st>>>(a, cr, nc, dpos, dj, gid, slot);
}

}  // namespace sesa
