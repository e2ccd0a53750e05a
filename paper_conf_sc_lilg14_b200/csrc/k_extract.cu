// k_extract.cu — record validation + extents and key extraction with upfront digit
// histograms (row a2).  Both are HBM-streaming passes over the 32-byte records: one 32-byte sector per record,
// read with two 16-byte vector loads, grid sized to a multiple of the 148 SMs.
#include <algorithm>
#include <cstdlib>

#include "kernels.cuh"

namespace sesa {

// ------------------------------------------------------------------------------------------------------------
// extents: per record check validity (include/sesa.h: space <= 1, rw <= 2, size >= 1, addr + size - 1 does not
// wrap — the bounds P:73 and the memory sorts of Fig. 3), and reduce per space: min/max granule,
// block, interval; count entries (granules) and multi-granule records; detect (block, interval) order.
// ------------------------------------------------------------------------------------------------------------
constexpr int EX_STAGES = 4, EX_CHUNK = 16384, EX_RECS = EX_CHUNK / 32;

// Per-space extents in granule units (the block-level reduction format written to Summary).
struct SpaceAcc {
  u64 cnt, gmin, gmax;
  u32 bmin, bmax, imin, imax;
  __device__ __forceinline__ void init() { cnt = 0, gmin = ~0ull, gmax = 0, bmin = ~0u, bmax = 0, imin = ~0u, imax = 0; }
  __device__ __forceinline__ void add(u64 glo, u64 ghi, u32 b, u32 i) {
    cnt++;
    gmin = min(gmin, glo), gmax = max(gmax, ghi);
    bmin = min(bmin, b), bmax = max(bmax, b);
    imin = min(imin, i), imax = max(imax, i);
  }
  __device__ __forceinline__ void warp_reduce() {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      cnt += __shfl_xor_sync(~0u, cnt, o);
      gmin = min(gmin, __shfl_xor_sync(~0u, gmin, o));
      gmax = max(gmax, __shfl_xor_sync(~0u, gmax, o));
      bmin = min(bmin, __shfl_xor_sync(~0u, bmin, o));
      bmax = max(bmax, __shfl_xor_sync(~0u, bmax, o));
      imin = min(imin, __shfl_xor_sync(~0u, imin, o));
      imax = max(imax, __shfl_xor_sync(~0u, imax, o));
    }
  }
};

// extents2: warp w streams the contiguous record range [w*rw, (w+1)*rw) in rows of 32 (U rows in
// flight), all index arithmetic in 32 bits (n < 2^31, include/sesa.h).  Per record only what the layout needs:
// min address and max last byte per space (granule = address >> log2G commutes with min/max, so the shifts
// happen once per thread), block/interval min/max, the extra-granule count from the in-granule offset (32-bit),
// validity, and (block, interval) order against the predecessor (previous lane, or the previous row's lane 31).
struct SpaceAcc2 {
  u32 cnt, bmin, bmax, imin, imax;
  u64 amin, amax;
  __device__ __forceinline__ void init() { cnt = 0, amin = ~0ull, amax = 0, bmin = ~0u, bmax = 0, imin = ~0u, imax = 0; }
  __device__ __forceinline__ void add_a(u64 a, u64 last) {  // address extents only
    cnt++;
    amin = min(amin, a), amax = max(amax, last);
  }
  __device__ __forceinline__ void add(u64 a, u64 last, u32 b, u32 i) {
    cnt++;
    amin = min(amin, a), amax = max(amax, last);
    bmin = min(bmin, b), bmax = max(bmax, b);
    imin = min(imin, i), imax = max(imax, i);
  }
  __device__ __forceinline__ SpaceAcc to_acc(u32 log2G) const {
    SpaceAcc A;
    A.init();
    if (cnt) {
      A.cnt = cnt, A.gmin = amin >> log2G, A.gmax = amax >> log2G;
      A.bmin = bmin, A.bmax = bmax, A.imin = imin, A.imax = imax;
    }
    return A;
  }
};

// With tile_hist != null the warp ranges are whole tiles of FUSED_TILE records and each warp also writes, per
// tile, the histogram of the raw low granule byte (addr >> log2G) & 255: once the extents fix gmin, these are the
// tile histograms of the first sort digit ((g - gmin) & 255 is a rotation of g & 255), which lets the fused
// extract + first sort pass place every tile without a look-back (k_fused.cu).
// block reduction of one CTA's extents (warp shuffles, then one atomic per field per CTA) into the Summary
template <int THREADS>
__device__ __forceinline__ void flush_summary(u64 bad64, u64 ent, u64 mul, u32 unsorted, const SpaceAcc2& A0,
                                              const SpaceAcc2& A1, u32 log2G, Summary* __restrict__ out) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  SpaceAcc S0 = A0.to_acc(log2G), S1 = A1.to_acc(log2G);
  __shared__ SpaceAcc sa[THREADS / 32][2];
  __shared__ u64 s64[THREADS / 32][3];
  __shared__ u32 s_uns[THREADS / 32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    bad64 = min(bad64, __shfl_xor_sync(~0u, bad64, o));
    ent += __shfl_xor_sync(~0u, ent, o);
    mul += __shfl_xor_sync(~0u, mul, o);
    unsorted |= __shfl_xor_sync(~0u, unsorted, o);
  }
  S0.warp_reduce();
  S1.warp_reduce();
  if (lane == 0) {
    s64[warp][0] = bad64, s64[warp][1] = ent, s64[warp][2] = mul;
    sa[warp][0] = S0, sa[warp][1] = S1;
    s_uns[warp] = unsorted;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < THREADS / 32; w++) {
      s64[0][0] = min(s64[0][0], s64[w][0]);
      s64[0][1] += s64[w][1];
      s64[0][2] += s64[w][2];
      s_uns[0] |= s_uns[w];
      for (int x = 0; x < 2; x++) {
        SpaceAcc& d = sa[0][x];
        const SpaceAcc& e = sa[w][x];
        d.cnt += e.cnt;
        d.gmin = min(d.gmin, e.gmin), d.gmax = max(d.gmax, e.gmax);
        d.bmin = min(d.bmin, e.bmin), d.bmax = max(d.bmax, e.bmax);
        d.imin = min(d.imin, e.imin), d.imax = max(d.imax, e.imax);
      }
    }
    if (s64[0][0] != ~0ull) atomicMin(&out->bad_index, (unsigned long long)s64[0][0]);
    if (s64[0][1]) atomicAdd(&out->entries, (unsigned long long)s64[0][1]);
    if (s64[0][2]) atomicAdd(&out->multi, (unsigned long long)s64[0][2]);
    for (int x = 0; x < 2; x++) {
      const SpaceAcc& d = sa[0][x];
      if (!d.cnt) continue;
      atomicAdd(&out->count[x], (unsigned long long)d.cnt);
      atomicMin(&out->gmin[x], (unsigned long long)d.gmin);
      atomicMax(&out->gmax[x], (unsigned long long)d.gmax);
      atomicMin(&out->bmin[x], d.bmin);
      atomicMax(&out->bmax[x], d.bmax);
      atomicMin(&out->imin[x], d.imin);
      atomicMax(&out->imax[x], d.imax);
    }
    if (s_uns[0]) atomicOr(&out->unsorted, 1u);
  }
}

template <int U>
// With regions (nreg > 0; sorted by (space, base), non-overlapping, space s in [rs[s], rs[s+1])), every valid
// record of a space with regions is also checked for containment (OOB, NEXT-1): binary search for the last
// region starting at or below addr, then addr + size <= end.
// With gout != null the low 32 bits of the granule index addr >> log2G of every record are also written (4 bytes
// per record,
// coalesced): the fused pass then reads 8 bytes per record instead of the record's 32-byte sector.
// With wout != null (and tile_hist) bit (i & 31) of wout[i >> 5] is set iff record i writes (WRITE or ATOMIC):
// the fused pass puts it into the key (KeyLayout::wbit).
// With tile_hist2 != null (large traces: candidates for the bucket path, k_bucket.cu) each warp also writes the
// per-tile histograms of the raw digit (g >> HYB_LO) & 255, and the CTA the histogram of (g >> (HYB_LO + 8)) & 255
// (bhist[3]): the two global digits of the bucket path.
__global__ void __launch_bounds__(256) extents2_kernel(const Rec* __restrict__ rec, u32 n, u32 log2G, u32 rw,
                                                       Summary* __restrict__ out, u32* __restrict__ tile_hist,
                                                       const Region* __restrict__ regs, uint3 rs,
                                                       u32* __restrict__ gout, u32* __restrict__ tile_hist2,
                                                       u32* __restrict__ wout) {
  __shared__ u32 s_th[8][RADIX];
  __shared__ u32 s_th2[8][RADIX];
  __shared__ u32 s_hb[4][RADIX];  // raw granule bytes 1..3 (with tile_hist), bits 22..29 (with tile_hist2)
  extern __shared__ Region s_reg[];  // [rs.z]
  for (u32 i = threadIdx.x; i < rs.z; i += 256) s_reg[i] = regs[i];
  if (tile_hist)
    for (u32 i = threadIdx.x; i < 4 * RADIX; i += 256) (&s_hb[0][0])[i] = 0;
  if (rs.z || tile_hist) __syncthreads();
  constexpr int THREADS = 256;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const u32 gw = (blockIdx.x * THREADS + threadIdx.x) >> 5;
  const u64 start64 = (u64)gw * rw;
  const u32 start = (u32)min(start64, (u64)n), end = (u32)min((u64)n, start64 + rw);
  const u32 gmask = (1u << log2G) - 1u;
  u32 bad = ~0u, extra = 0, multi = 0, unsorted = 0, oobc = 0, oobf = ~0u;
  SpaceAcc2 A0, A1;
  A0.init();
  A1.init();
  const uint4* q = reinterpret_cast<const uint4*>(rec);
  u64 prev_bi = 0;  // (block << 32 | interval) of the record before the current row's lane 0
  if (start > 0 && start < end) {
    const uint4 p = __ldg(q + 2 * (u64)(start - 1) + 1);
    prev_bi = ((u64)p.x << 32) | p.z;
  }
  u32* th = s_th[warp];
  u32* th2 = s_th2[warp];
  const u32 seg = tile_hist ? (u32)FUSED_TILE : rw;  // records between histogram flushes
  u32 wacc = 0;  // write bits of row (32 * group + lane) (wout)
  for (u32 t0 = start; t0 < end; t0 += seg) {
  const u32 tend = min(end, t0 + seg);
  if (tile_hist) {
#pragma unroll
    for (int q = 0; q < RADIX / 32; q++) th[q * 32 + lane] = 0;
    if (tile_hist2)
#pragma unroll
      for (int q = 0; q < RADIX / 32; q++) th2[q * 32 + lane] = 0;
    __syncwarp();
  }
  for (u32 r0 = t0; r0 < tend; r0 += 32 * U) {
    uint4 a[U], b[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 i = r0 + u * 32 + lane;
      if (i < tend) a[u] = __ldcs(q + 2 * (u64)i), b[u] = __ldcs(q + 2 * (u64)i + 1);
      else a[u] = make_uint4(0, 0, 0, 0), b[u] = make_uint4(0, 0, 0, 0);
    }
    bool ok[U];
    bool allg = true, alls = true;
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 i = r0 + u * 32 + lane;
      const u64 bi = ((u64)b[u].x << 32) | b[u].z;
      const u64 up = __shfl_up_sync(~0u, bi, 1);
      const u64 pbi = lane ? up : prev_bi;
      prev_bi = __shfl_sync(~0u, bi, 31);
      const u32 size = b[u].w & 0xFFFFu, sp = (b[u].w >> 16) & 0xFFu, rwv = b[u].w >> 24;
      const u64 addr = ((u64)a[u].y << 32) | a[u].x;
      const bool in = i < tend;
      ok[u] = in && sp <= 1u && rwv <= 2u && size >= 1u && addr + (u64)size - 1ull >= addr;
      bad = (in && !ok[u]) ? min(bad, i) : bad;
      const u32 e = ((a[u].x & gmask) + size - 1u) >> log2G;  // granules beyond the first
      extra += ok[u] ? e : 0u;
      multi += (ok[u] && e != 0u) ? 1u : 0u;
      unsorted |= (ok[u] && bi < pbi) ? 1u : 0u;
      allg = allg && (!ok[u] || sp == SP_GLOBAL);
      alls = alls && (!ok[u] || sp == SP_SHARED);
    }
    if (rs.z) {  // OOB: containment in a registered region of the record's space
#pragma unroll
      for (int u = 0; u < U; u++) {
        if (!ok[u]) continue;
        const u32 sp = (b[u].w >> 16) & 0xFFu;
        int lo = sp ? (int)rs.x : 0, hi = sp ? (int)rs.z : (int)rs.x;
        if (lo >= hi) continue;  // no regions registered for this space: not checked
        const u64 addr = ((u64)a[u].y << 32) | a[u].x;
        const u64 last = addr + (u64)(b[u].w & 0xFFFFu) - 1ull;
        while (hi - lo > 1) {
          const int mid = (lo + hi) >> 1;
          if (s_reg[mid].base <= addr) lo = mid;
          else hi = mid;
        }
        if (!(s_reg[lo].base <= addr && last < s_reg[lo].end)) oobc++, oobf = min(oobf, r0 + u * 32 + lane);
      }
    }
    // one space decision per batch (traces are mostly single-space)
    const bool bg = __all_sync(~0u, allg), bs = !bg && __all_sync(~0u, alls);
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u64 addr = ((u64)a[u].y << 32) | a[u].x;
      const u64 last = addr + (u64)(b[u].w & 0xFFFFu) - 1ull;
      const bool glob = bg || (!bs && ((b[u].w >> 16) & 0xFFu) == SP_GLOBAL);
      if (ok[u]) {
        if (glob) A1.add(addr, last, b[u].x, b[u].z);
        else A0.add(addr, last, b[u].x, b[u].z);
        if (tile_hist) {
          const u64 g = addr >> log2G;
          atomicAdd(&th[(u32)g & (RADIX - 1)], 1u);
          atomicAdd(&s_hb[0][(u32)(g >> 8) & (RADIX - 1)], 1u);
          atomicAdd(&s_hb[1][(u32)(g >> 16) & (RADIX - 1)], 1u);
          atomicAdd(&s_hb[2][(u32)(g >> 24) & (RADIX - 1)], 1u);
          if (tile_hist2) {
            atomicAdd(&th2[(u32)(g >> HYB_LO) & (RADIX - 1)], 1u);
            atomicAdd(&s_hb[3][(u32)(g >> (HYB_LO + RADIX_BITS)) & (RADIX - 1)], 1u);
          }
        }
      }
      if (gout && r0 + u * 32 + lane < tend) __stcs(gout + r0 + u * 32 + lane, (u32)(addr >> log2G));
    }
    if (wout) {  // one bit per record: it writes.  Rows of 32 records are 32-aligned (warp ranges are whole
                 // tiles of 6 x 32 rows); lane j collects row j of each group of 32 rows, written as one 128-B line
#pragma unroll
      for (int u = 0; u < U; u++) {
        const unsigned wm = __ballot_sync(~0u, ok[u] && (b[u].w >> 24) != RW_READ);
        if (((((r0 + u * 32) >> 5) & 31u) == (u32)lane) && r0 + u * 32 < tend) wacc = wm;
      }
      const u32 lastR = (min(r0 + 32 * U, tend) - 1) >> 5, g0 = lastR & ~31u;
      if ((lastR & 31u) == 31u || r0 + 32 * U >= tend)
        if (g0 + lane <= lastR) wout[g0 + lane] = wacc;
    }
  }
  if (tile_hist) {
    __syncwarp();
    u32* dst = tile_hist + (u64)(t0 / FUSED_TILE) * RADIX;
#pragma unroll
    for (int q = 0; q < RADIX / 32; q++) dst[q * 32 + lane] = th[q * 32 + lane];
    if (tile_hist2) {
      u32* dst2 = tile_hist2 + (u64)(t0 / FUSED_TILE) * RADIX;
#pragma unroll
      for (int q = 0; q < RADIX / 32; q++) dst2[q * 32 + lane] = th2[q * 32 + lane];
    }
    __syncwarp();
  }
  }
  // block reduction (warp shuffles, then one atomic per field per CTA)
  u64 bad64 = bad == ~0u ? ~0ull : (u64)bad, ent = (u64)extra + A0.cnt + A1.cnt, mul = multi;
  if (rs.z) {
    u64 oc = oobc, of = oobf == ~0u ? ~0ull : (u64)oobf;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) oc += __shfl_xor_sync(~0u, oc, o), of = min(of, __shfl_xor_sync(~0u, of, o));
    if (lane == 0 && oc) atomicAdd(&out->oob_count, (unsigned long long)oc), atomicMin(&out->oob_first, (unsigned long long)of);
  }
  if (tile_hist) {
    __syncthreads();
    for (u32 i = threadIdx.x; i < (tile_hist2 ? 4u : 3u) * RADIX; i += 256) {
      const u32 v = (&s_hb[0][0])[i];
      if (v) atomicAdd(&(&out->bhist[0][0])[i], v);
    }
  }
  flush_summary<THREADS>(bad64, ent, mul, unsorted, A0, A1, log2G, out);
}

// ------------------------------------------------------------------------------------------------------------
// Extents fused with the bucket path's first partition (k_bucket.cu; C5-like traces, chosen by a sample of the
// records before any pass).  The bucket path's first digit is key_hi bits [HYB_LO, HYB_LO + 8) with gmin aligned
// down to 2^(HYB_LO + 16), i.e. the RAW granule bits [14, 22): known while the records stream by, before gmin
// is.  So one pass validates, reduces the extents and writes every record's key into the region of its digit —
// keys carry the raw low 30 granule bits (key_hi = g - G0 follows modulo 2^30 once G0 is known; the second
// partition pass rebases them) — instead of an extents pass writing a 4-byte granule array that a fused pass
// reads back (C5: 36 + 12 GB -> 40 GB of traffic).  Order inside a region does not matter on the bucket path
// (each chunk's survivors are sorted by full key), so a CTA takes slots of region d in windows of XP_WIN
// reserved by one global atomic, and a tile's keys, grouped by digit in shared memory, leave in coalesced runs.
// Window remainders are filled with ~0 sentinels, which the second pass skips.  A region that would pass its
// capacity sets *overflow (the host then runs the ordinary path: the result never depends on this pass's
// speculation).  Per tile of XP_TILE records: (1) load the next tile's records into registers (in flight during
// the rest), (2) validate + extents + count atomics (rank = return value), (3) digit bases + windows (thread d),
// (4) keys into shared memory by digit, (5) coalesced write-out.
// ------------------------------------------------------------------------------------------------------------
#ifndef XP_THREADS_
#define XP_THREADS_ 768
#endif
#ifndef XP_ROWS_
#define XP_ROWS_ 3
#endif
#ifndef XP_STAGES_
#define XP_STAGES_ 2
#endif
#ifndef XP_CPP_
#define XP_CPP_ 4
#endif
// XP_TILE records per ring chunk; XP_CPP chunks per partition round (XP_KT keys)
constexpr int XP_THREADS = XP_THREADS_, XP_ROWS = XP_ROWS_, XP_TILE = XP_THREADS * XP_ROWS, XP_STAGES = XP_STAGES_;
constexpr int XP_CPP = XP_CPP_, XP_KT = XP_TILE * XP_CPP;
#ifndef XP_WIN_
#define XP_WIN_ 128
#endif
constexpr u32 XP_WIN = XP_WIN_;
// dynamic shared memory: the record ring, then the stage of a round's keys (static shared memory stops at 48 KB)
constexpr size_t XP_RING = (size_t)XP_STAGES * XP_TILE * 32, XP_SMEM = XP_RING + (size_t)XP_KT * 8;

// The tiles' records arrive by TMA bulk copies into a ring of XP_STAGES tiles (192 KB in flight per SM without
// registers: one CTA of 512 threads per SM would otherwise hold one tile in flight and stall on every barrier).
__global__ void __launch_bounds__(XP_THREADS, 1) extents_part_kernel(XPArgs A) {
  constexpr int THREADS = XP_THREADS, U = XP_ROWS;
  extern __shared__ __align__(128) unsigned char xp_ring[];
  __shared__ u64 bars[XP_STAGES];
  u64* stage = reinterpret_cast<u64*>(xp_ring + XP_RING);  // [XP_KT]
  __shared__ u32 s_cnt[RADIX], s_base[RADIX], s_hb[RADIX];
  __shared__ uint4 s_wo[RADIX];  // per digit: {d1, split, d2, -} (write-out deltas)
  __shared__ u32 s_tot;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  for (int i = tid; i < RADIX; i += THREADS) s_cnt[i] = 0, s_hb[i] = 0;
  u32 wpos = 0, wend = 0;  // thread d < RADIX: its CTA's current window of region d
  u32 nstart = 0;          // and the next one, reserved ahead
  bool nvalid = false;
  const u32 n = A.n, log2G = A.log2G, gmask = (1u << log2G) - 1u;
  const uint4* q = reinterpret_cast<const uint4*>(A.rec);
  u32 bad = ~0u, extra = 0, multi = 0, unsorted = 0;
  SpaceAcc2 A0, A1;
  A0.init();
  A1.init();
  BulkRing<XP_STAGES> ring(xp_ring, bars, XP_TILE * 32);
  ring.start(A.rec, (u64)n * 32);  // (contains __syncthreads)
  for (u64 j0 = 0; ring.next(j0); j0 += XP_CPP) {
  u64 key[XP_CPP * U];
  u32 rk[XP_CPP * U];
#pragma unroll
  for (int cc = 0; cc < XP_CPP; cc++) {
    const u64 j = j0 + cc;
    if (!ring.next(j)) {  // (CTA-uniform)
#pragma unroll
      for (int u = 0; u < U; u++) rk[cc * U + u] = ~0u;
      continue;
    }
    const u32 tile = (u32)ring.chunk_index(j);
    const u32 tb = tile * XP_TILE, r0 = tb + warp * 32 * U;
    // the (block, interval) before the warp's first row: in the ring, or (warp 0) the previous tile's last record
    uint4 pv = make_uint4(0, 0, 0, 0);
    if (warp == 0 && tb > 0) pv = __ldg(q + 2 * (u64)(tb - 1) + 1);
    const uint4* R = reinterpret_cast<const uint4*>(ring.wait(j));
    if (warp > 0) pv = R[2 * (warp * 32 * U - 1) + 1];
    u64 prev_bi = ((u64)pv.x << 32) | pv.z;
#pragma unroll
    for (int uu = 0; uu < U; uu++) {
      const int u = cc * U + uu;
      const u32 i = r0 + uu * 32 + lane, li = warp * 32 * U + uu * 32 + lane;
      const bool in = i < n;
      const uint4 ca = in ? R[2 * li] : make_uint4(0, 0, 0, 0), cb = in ? R[2 * li + 1] : make_uint4(0, 0, 0, 0);
      const u64 bi = ((u64)cb.x << 32) | cb.z;
      const u64 up = __shfl_up_sync(~0u, bi, 1);
      const u64 pbi = lane ? up : prev_bi;
      prev_bi = __shfl_sync(~0u, bi, 31);
      const u32 size = cb.w & 0xFFFFu, sp = (cb.w >> 16) & 0xFFu, rwv = cb.w >> 24;
      const u64 addr = ((u64)ca.y << 32) | ca.x;
      const bool ok = in && sp <= 1u && rwv <= 2u && size >= 1u && addr + (u64)size - 1ull >= addr;
      bad = (in && !ok) ? min(bad, i) : bad;
      const u32 e = ((ca.x & gmask) + size - 1u) >> log2G;
      extra += ok ? e : 0u;
      multi += (ok && e != 0u) ? 1u : 0u;
      unsorted |= (ok && i > 0 && bi < pbi) ? 1u : 0u;
      const u64 last = addr + (u64)size - 1ull;
      // (block / interval extents are not kept: the fused path needs them only for unsorted or shared traces,
      // which go back to the ordinary path)
      if (ok) {
        if (sp == SP_GLOBAL) A1.add_a(addr, last);
        else A0.cnt++;
      }
      const u64 g = addr >> log2G;
      key[u] = ((g & ((1ull << 30) - 1ull)) << A.pos_bits) | (u64)i;
      rk[u] = ~0u;
      if (ok) {
        atomicAdd(&s_hb[(u32)(g >> (HYB_LO + RADIX_BITS)) & (RADIX - 1)], 1u);
        rk[u] = atomicAdd(&s_cnt[(u32)(g >> HYB_LO) & (RADIX - 1)], 1u);
      }
    }
    ring.release(j);  // (contains __syncthreads: the slot is refilled with tile j + XP_STAGES)
  }
    // Thread d < RADIX (warps 0-7): the digit's stage base — the counts of the warps before it by one warp
    // reduction each (redux), its own warp by a shuffle scan: no block scan, one barrier less — and this tile's
    // slots in the CTA's windows.  The next window is reserved ahead (its atomic's result is first needed a tile
    // or more later, so its latency is off the critical path); a run longer than a window reserves at once.
    if (tid < RADIX) {
      u32 before = 0;
#pragma unroll
      for (int w2 = 0; w2 < RADIX / 32 - 1; w2++)  // (independent loads and reductions: no dependent chain)
        before += __reduce_add_sync(~0u, w2 < warp ? s_cnt[w2 * 32 + lane] : 0u);
      const u32 c = s_cnt[tid];
      u32 x = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const u32 y = __shfl_up_sync(~0u, x, o);
        if (lane >= o) x += y;
      }
      const u32 base = before + x - c;
      s_base[tid] = base;
      if (tid == RADIX - 1) s_tot = before + x;
      const u32 avail = wend - wpos, seg1 = min(c, avail);
      // stage slot jj of this digit -> window slot jj + d1 (jj < split) or jj + d2 (modular u32 deltas)
      uint4 wo = make_uint4(wpos - base, base + seg1, 0u, 0u);
      wpos += seg1;
      if (c > seg1) {
        const u32 rest = c - seg1;
        u32 st, res;
        if (nvalid && rest <= XP_WIN) {
          st = nstart, res = XP_WIN, nvalid = false;
        } else {
          res = max(XP_WIN, (rest + 31u) & ~31u);
          st = atomicAdd(&A.gfill[tid], res);
        }
        if ((u64)st + res > A.cap) atomicOr(A.overflow, 1u);
        wo.z = st - (base + seg1);
        wpos = st + rest;
        wend = st + res;
      }
      s_wo[tid] = wo;
      if (!nvalid && wend - wpos < XP_WIN / 2) nstart = atomicAdd(&A.gfill[tid], XP_WIN), nvalid = true;
    }
    __syncthreads();
    if (tid < RADIX) s_cnt[tid] = 0;  // (every count was read before the barrier)
#pragma unroll
    for (int u = 0; u < XP_CPP * U; u++)
      if (rk[u] != ~0u) stage[s_base[(u32)(key[u] >> (A.pos_bits + HYB_LO)) & (RADIX - 1)] + rk[u]] = key[u];
    __syncthreads();
    // coalesced runs: stage slot jj of digit d goes to its window slot
    const u32 tot = s_tot;
    for (u32 jj = tid; jj < tot; jj += THREADS) {
      const u64 k = stage[jj];
      const uint4 wo = s_wo[(u32)(k >> (A.pos_bits + HYB_LO)) & (RADIX - 1)];
      const u32 dst = jj + (jj < wo.y ? wo.x : wo.z), d = (u32)(k >> (A.pos_bits + HYB_LO)) & (RADIX - 1);
      // (plain stores: a run's partial edge sectors wait in L2 for the CTA's next run of the digit; streaming
      // stores evicted them half-written)
      if (dst < A.cap) A.kout[(u64)d * A.cap + dst] = k;
    }
    // (the next tile's first barrier, in ring.release, orders these reads of the tables before they change)
  }
  // window remainders (and a reserved next window) -> sentinels
  if (tid < RADIX) {
    for (u32 jj = wpos; jj < wend && jj < A.cap; jj++) A.kout[(u64)tid * A.cap + jj] = ~0ull;
    if (nvalid) {
      if ((u64)nstart + XP_WIN > A.cap) atomicOr(A.overflow, 1u);
      for (u32 jj = nstart; jj < nstart + XP_WIN && jj < A.cap; jj++) A.kout[(u64)tid * A.cap + jj] = ~0ull;
    }
  }
  __syncthreads();
  for (int i = tid; i < RADIX; i += THREADS)
    if (s_hb[i]) atomicAdd(&A.out->bhist[3][i], s_hb[i]);
  const u64 bad64 = bad == ~0u ? ~0ull : (u64)bad, ent = (u64)extra + A0.cnt + A1.cnt;
  flush_summary<THREADS>(bad64, ent, (u64)multi, unsorted, A0, A1, log2G, A.out);
}

void launch_extents_part(const XPArgs& A, cudaStream_t st) {
  const u32 T = (A.n + XP_TILE - 1) / XP_TILE;
  const u32 grid = std::min<u32>(T, (u32)dev_sm_count());
  smem_optin((const void*)extents_part_kernel, XP_SMEM);
  extents_part_kernel<<<grid, XP_THREADS, XP_SMEM, st>>>(A);
}

u64 extents_part_cap(u64 n) {
  // per region: the mean, 1/8 more, a window per CTA and a tile of slack, in whole 32-key rows
  // (a multiple of the second pass's tile: its tiles read whole tiles inside a region)
  const u64 mean = (n + RADIX - 1) / RADIX;
  const u64 c = mean + mean / 8 + 2 * (u64)XP_WIN * (u64)dev_sm_count() + XP_KT;
  return (c + PART_TILE_KEYS - 1) / PART_TILE_KEYS * PART_TILE_KEYS;
}

// ---- record sample predicting the fused path (before any pass) -----------------------------------------------
// every stride-th record: flags bit 0 = a sampled record is invalid, shared, spans two granules or sits below
// its predecessor in (block, interval) order; min / max granule; histogram of the absolute chunk index g >> 15
// modulo 2^15 (G0 is a multiple of 2^15, so these are the bucket path's chunks; folding can only raise the max)
__global__ void presample_kernel(const Rec* __restrict__ rec, u32 n, u32 stride, u32 log2G, u32* __restrict__ hist,
                                 unsigned long long* __restrict__ ext /* [0] flags, [1] gmin, [2] gmax */) {
  const u64 step = (u64)gridDim.x * blockDim.x * stride;
  u64 gmn = ~0ull, gmx = 0;
  u32 flags = 0;
  for (u64 i0 = (u64)(blockIdx.x * blockDim.x + (threadIdx.x & ~31u)) * stride; i0 < n; i0 += step) {
    const u64 i = i0 + (u64)(threadIdx.x & 31) * stride;
    u32 c = ~0u;
    if (i < n) {
      const Rec r = load_rec(rec + i);
      const u64 g = r.addr >> log2G, gl = (r.addr + (u64)r.size - 1ull) >> log2G;
      const bool ok = r.space == SP_GLOBAL && r.rw <= 2 && r.size >= 1 && r.addr + (u64)r.size - 1ull >= r.addr && g == gl;
      if (!ok) flags |= 1u;
      if (i > 0) {
        const Rec p = load_rec(rec + i - 1);
        if (((u64)r.block << 32 | r.interval) < ((u64)p.block << 32 | p.interval)) flags |= 1u;
      }
      gmn = min(gmn, g), gmx = max(gmx, g);
      c = (u32)(g >> HYB_CHUNK) & ((1u << 15) - 1u);
    }
    const unsigned peers = __match_any_sync(~0u, c);
    if (c != ~0u && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&hist[c], (u32)__popc(peers));
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    flags |= __shfl_xor_sync(~0u, flags, o);
    gmn = min(gmn, __shfl_xor_sync(~0u, gmn, o));
    gmx = max(gmx, __shfl_xor_sync(~0u, gmx, o));
  }
  if ((threadIdx.x & 31) == 0) {
    if (flags) atomicOr(&ext[0], (unsigned long long)flags);
    atomicMin(&ext[1], gmn);
    atomicMax(&ext[2], gmx);
  }
}

__global__ void presample_max_kernel(const u32* __restrict__ hist, unsigned long long* __restrict__ ext) {
  u32 mx = 0;
  for (u32 c = blockIdx.x * blockDim.x + threadIdx.x; c < (1u << 15); c += gridDim.x * blockDim.x) mx = max(mx, hist[c]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(~0u, mx, o));
  if ((threadIdx.x & 31) == 0) atomicMax(&ext[3], (unsigned long long)mx);
}

// temp: >= presample_temp_bytes(); h_ext (host, valid after a sync): flags, gmin, gmax, max chunk count; *samples
size_t presample_temp_bytes() { return (1u << 15) * 4 + 64; }
void launch_presample(const Rec* rec, u32 n, u32 log2G, u32 want, void* temp, unsigned long long* h_ext,
                      u32* samples, cudaStream_t st) {
  u32* hist = reinterpret_cast<u32*>(temp);
  unsigned long long* ext = reinterpret_cast<unsigned long long*>(hist + (1u << 15));
  const u32 stride = std::max<u32>(1, n / want);
  *samples = (n + stride - 1) / stride;
  cudaMemsetAsync(hist, 0, (1u << 15) * 4 + 32, st);
  const unsigned long long init[4] = {0ull, ~0ull, 0ull, 0ull};
  cudaMemcpyAsync(ext, init, 32, cudaMemcpyHostToDevice, st);
  const u32 grid = (u32)std::min<u64>(((u64)*samples + 255) / 256, (u64)dev_sm_count() * 8);
  presample_kernel<<<grid, 256, 0, st>>>(rec, n, stride, log2G, hist, ext);
  presample_max_kernel<<<32, 256, 0, st>>>(hist, ext);
  cudaMemcpyAsync(h_ext, ext, 32, cudaMemcpyDeviceToHost, st);
}

static int ring_grid(const void* kern, int threads, size_t smem) {
  return dev_sm_count() * blocks_per_sm(kern, threads, smem);
}

void launch_extents(const Rec* rec, u64 n, u32 log2G, Summary* d_sum, u32* tile_hist, const Region* regs, u32 nreg,
                    u32 nreg_shared, int grid, cudaStream_t st, u32* gout, u32* tile_hist2, u32* wout) {
  // extents2: contiguous warp ranges, one full wave of resident warps (the round-1 grid-stride kernel took
  // 7.7 ms on C5: 132 instructions per record, 64-bit index math and local-memory accumulators; this one 4.6 ms)
  const int sms = dev_sm_count(), per = blocks_per_sm((const void*)extents2_kernel<4>, 256, 0);
  smem_optin((const void*)extents2_kernel<4>, MAX_REGIONS * sizeof(Region));
  const u64 warps = (u64)sms * per * 8;
  const u64 gran = tile_hist ? FUSED_TILE : 128;  // warp ranges: whole tiles when tile histograms are wanted
  u64 rw = (n + warps - 1) / warps;
  rw = std::max<u64>(gran, (rw + gran - 1) / gran * gran);
  const u64 nw = (n + rw - 1) / rw;
  extents2_kernel<4><<<(unsigned)((nw + 7) / 8), 256, nreg * sizeof(Region), st>>>(
      rec, (u32)n, log2G, (u32)rw, d_sum, tile_hist, regs, make_uint3(nreg_shared, 0u, nreg), gout,
      tile_hist ? tile_hist2 : nullptr, tile_hist ? wout : nullptr);
  (void)grid;
}

// ------------------------------------------------------------------------------------------------------------
// key extraction, 1 entry per record (every record within one granule): key = key_hi << pos_bits | pos, plus
// the histogram of every radix digit the sort will use (onesweep's upfront histogram), accumulated per CTA in
// shared memory with warp-aggregated (ballot-matched) increments and flushed with one global atomic per bin.
// ------------------------------------------------------------------------------------------------------------
template <int THREADS, int RB>
__global__ void __launch_bounds__(THREADS) extract_1to1_kernel(const Rec* __restrict__ rec, u64 n, KeyLayout L,
                                                                u32 npass, u64* __restrict__ keys,
                                                                u32* __restrict__ hist /* [npass][1<<RB] */,
                                                                u64 pos_base) {
  constexpr int RADIX = 1 << RB;
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ u64 bars[EX_STAGES];
  u32* sh = reinterpret_cast<u32*>(smem + (size_t)EX_STAGES * EX_CHUNK);  // [warps][npass][RADIX]
  const u32 nsh = npass * RADIX * (THREADS / 32);
  for (u32 i = threadIdx.x; i < nsh; i += THREADS) sh[i] = 0;
  u32* wsh = sh + (threadIdx.x >> 5) * npass * RADIX;  // per-warp private sub-histograms: plain smem atomics
  BulkRing<EX_STAGES> ring(smem, bars, EX_CHUNK);
  ring.start(rec, n * 32);  // (contains __syncthreads)
  for (u64 j = 0; ring.next(j); j++) {
    const Rec* R = reinterpret_cast<const Rec*>(ring.wait(j));
    const u64 c0 = ring.chunk_index(j) * EX_RECS;
    const u32 nr = ring.chunk_bytes(j) / 32;
#pragma unroll
    for (int h = 0; h < EX_RECS / THREADS; h++) {
      const u32 t = h * THREADS + threadIdx.x;
      if (t >= nr) continue;
      const Rec& x = R[t];
      // (with KeyLayout::wbit the write bit sits below the position)
      const u64 key = (key_hi_of(L, x.space, x.block, x.interval, x.addr >> L.log2G) << (L.pos_bits + L.wbit)) |
                      ((pos_base + c0 + t) << L.wbit) | (L.wbit && x.rw != RW_READ ? 1ull : 0ull);
      __stcs(keys + c0 + t, key);
      for (u32 p = 0; p < npass; p++)
        atomicAdd(&wsh[p * RADIX + ((key >> (L.pos_bits + L.wbit + p * RB)) & (RADIX - 1))], 1u);
    }
    ring.release(j);
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS) {
    u32 v = 0;
    for (int w = 0; w < THREADS / 32; w++) v += sh[w * npass * RADIX + i];
    if (v) atomicAdd(&hist[i], v);
  }
}

void launch_extract_1to1(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, u64* keys, u32* hist, u64 pos_base,
                         int, cudaStream_t st) {
  const size_t sm = (size_t)EX_STAGES * EX_CHUNK + (size_t)npass * 8 * RADIX * 4;  // ring + npass x 8 warps hist
  const int grid = ring_grid((const void*)extract_1to1_kernel<256, RADIX_BITS>, 256, sm);
  const u64 chunks = (n * 32 + EX_CHUNK - 1) / EX_CHUNK;
  extract_1to1_kernel<256, RADIX_BITS><<<(unsigned)std::min<u64>(chunks, (u64)grid), 256, sm, st>>>(rec, n, L, npass,
                                                                                                   keys, hist, pos_base);
}

// ------------------------------------------------------------------------------------------------------------
// multi-granule path: entries per record = granules it covers (reading R1: byte ranges compared at granule G).
// count -> exclusive scan (offsets) -> expand.  Entry order = record order, then ascending granule.
// ------------------------------------------------------------------------------------------------------------
__global__ void entry_count_kernel(const Rec* __restrict__ rec, u64 n, u32 log2G, u32* __restrict__ cnt) {
  u64 k = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  Rec r = load_rec(rec + k);
  u64 glo = r.addr >> log2G, ghi = (r.addr + (u64)(r.size - 1)) >> log2G;
  cnt[k] = (u32)(ghi - glo + 1);
}

template <int THREADS, int RB>
__global__ void __launch_bounds__(THREADS) extract_multi_kernel(const Rec* __restrict__ rec, u64 n, KeyLayout L,
                                                                 u32 npass, const u32* __restrict__ off,
                                                                 u64* __restrict__ keys, u32* __restrict__ hist,
                                                                 u64 pos_base) {
  constexpr int RADIX = 1 << RB;
  extern __shared__ u32 sh[];
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS) sh[i] = 0;
  __syncthreads();
  const u64 stride = (u64)gridDim.x * THREADS;
  for (u64 k = (u64)blockIdx.x * THREADS + threadIdx.x; k < n; k += stride) {
    Rec r = load_rec(rec + k);
    u64 glo = r.addr >> L.log2G, ghi = (r.addr + (u64)(r.size - 1)) >> L.log2G;
    u64 o = off[k];
    for (u64 g = glo; g <= ghi; g++, o++) {
      u64 key = (key_hi_of(L, r.space, r.block, r.interval, g) << (L.pos_bits + L.wbit)) | ((pos_base + k) << L.wbit) |
                (L.wbit && r.rw != RW_READ ? 1ull : 0ull);
      keys[o] = key;
      for (u32 p = 0; p < npass; p++)
        atomicAdd(&sh[p * RADIX + ((key >> (L.pos_bits + L.wbit + p * RB)) & (RADIX - 1))], 1u);
    }
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS)
    if (sh[i]) atomicAdd(&hist[i], sh[i]);
}

void launch_entry_count(const Rec* rec, u64 n, u32 log2G, u32* cnt, cudaStream_t st) {
  entry_count_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(rec, n, log2G, cnt);
}

void launch_extract_multi(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, const u32* off, u64* keys,
                          u32* hist, u64 pos_base, int grid, cudaStream_t st) {
  size_t smem = (size_t)npass * (1 << RADIX_BITS) * sizeof(u32);
  extract_multi_kernel<256, RADIX_BITS><<<grid, 256, smem, st>>>(rec, n, L, npass, off, keys, hist, pos_base);
}

}  // namespace sesa
