// k_sort.cu — hand-written onesweep LSD radix sort pass for sm_100a (the dominant step).
//
// One pass = one kernel: a CTA takes the next tile in launch order (atomic tile counter, so every predecessor
// tile is resident or done: forward progress for the look-back), loads 16 keys per thread warp-striped
// (coalesced 256-byte rows), ranks them per warp with ballot bit-matching (stable: item-major, lane-minor),
// publishes its per-digit counts, obtains the exclusive per-digit prefix of all earlier tiles by decoupled
// look-back (Merrill & Garland single-pass scan, one 64-bit status word per (tile, digit) tagged with a pass
// epoch so the array never needs clearing), scatters the tile into shared memory in digit order, and writes it
// out so that each digit's run of the tile lands contiguously (coalesced stores).  Traffic per pass: 8 B read +
// 8 B written per key (+4 + 4 with values); the look-back words add 8 B x 256 per 4096-key tile (~0.5 B/key).
#include <algorithm>

#include "kernels.cuh"

namespace sesa {

static constexpr u64 LB_AGG = 1ull << 62, LB_PREFIX = 2ull << 62;
static constexpr u64 LB_VAL = (1ull << 54) - 1;

__device__ __forceinline__ u64 lb_pack(u64 status, u32 epoch, u64 v) { return status | ((u64)epoch << 54) | v; }

__device__ __forceinline__ void st_relaxed(u64* p, u64 v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ u64 ld_relaxed(const u64* p) {
  u64 v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}


// global exclusive prefix of each pass's digit histogram -> bin_base[pass][digit]
__global__ void bin_base_kernel(const u32* __restrict__ hist, u64* __restrict__ base) {
  __shared__ u64 s[RADIX];
  const u32 p = blockIdx.x, d = threadIdx.x;
  s[d] = hist[p * RADIX + d];
  __syncthreads();
  if (d == 0) {
    u64 acc = 0;
    for (int i = 0; i < RADIX; i++) {
      u64 c = s[i];
      s[i] = acc;
      acc += c;
    }
  }
  __syncthreads();
  base[p * RADIX + d] = s[d];
}

void launch_bin_base(const u32* hist, u64* bin_base, u32 npass, cudaStream_t st) {
  if (npass) bin_base_kernel<<<npass, RADIX, 0, st>>>(hist, bin_base);
}

// Key/value onesweep (race lists and the benign regrouping: short arrays).  One tile (body templated on FULL:
// full tiles skip every validity test).  Per item the digit (9 bits; invalid items of a partial tile use digit
// RADIX) and later its rank are packed into one register: rd = rank << 9 | d.  Peer sets come from per-warp
// shared-memory masks (each lane sets its bit in its digit's word).
constexpr int KV_THREADS = 256, KV_ITEMS = 16, KV_MINB = 3, KV_LBW = 4;

template <bool FULL>
__device__ __forceinline__ void onesweep_kv_tile(const u64* __restrict__ kin, u64* __restrict__ kout,
                                                 const u32* __restrict__ vin, u32* __restrict__ vout, u32 m, u32 shift,
                                                 const u64* __restrict__ bin_base, u64* __restrict__ lookback,
                                                 u32 epoch, u32 tile, unsigned char* smem) {
  constexpr int THREADS = KV_THREADS, ITEMS = KV_ITEMS, LBW = KV_LBW;
  constexpr int WARPS = THREADS / 32;
  constexpr int TILE = THREADS * ITEMS;
  u64* keys_s = reinterpret_cast<u64*>(smem);                                  // [TILE]
  u32* vals_s = reinterpret_cast<u32*>(keys_s + TILE);                          // [TILE]
  u32* whist = vals_s + TILE;                                                   // [WARPS][RADIX]
  u32* bin_start = whist + WARPS * RADIX;                                       // [RADIX]
  long long* glob = reinterpret_cast<long long*>(bin_start + RADIX);            // [RADIX] (8-byte slots)
  u32* globu = reinterpret_cast<u32*>(glob);                                    // u32 view of the same slots
  u32* scratch = reinterpret_cast<u32*>(glob + RADIX);                          // [WARPS + 1]
  u32* wmask = scratch + WARPS + 1;                                             // [WARPS][RADIX + 1]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const u64 tbase = (u64)tile * TILE;
  const u64 wbase = tbase + (u64)warp * 32 * ITEMS + lane;
  // number of valid items of this thread (items i < nv are inside the array)
  const int nv = FULL ? ITEMS : (int)(wbase < m ? min((u64)ITEMS, ((u64)m - wbase + 31) / 32) : 0ull);
  u64 k[ITEMS];
  u32 v[ITEMS];
  u32 rd[ITEMS];
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    if (FULL || i < nv) {
      k[i] = __ldcs(kin + wbase + (u64)i * 32);  // streaming: each key is read once per pass
      v[i] = __ldcs(vin + wbase + (u64)i * 32);
    }
  }
#pragma unroll
  for (int i = 0; i < ITEMS; i++) rd[i] = (FULL || i < nv) ? (u32)((k[i] >> shift) & (RADIX - 1)) : (u32)RADIX;
  u32* wh = whist + warp * RADIX;
  // (1) early counts: per-warp digit histogram with shared-memory atomics (no ordering needed for counts)
#pragma unroll
  for (int i = 0; i < ITEMS; i++)
    if (FULL || i < nv) atomicAdd(&wh[rd[i]], 1u);
  __syncthreads();
  // (2) per-digit tile totals -> publish the tile aggregate BEFORE ranking, so that successor tiles find it
  //     during their look-back; per-warp counts become exclusive offsets across warps
  u32 tot = 0;
  if (tid < RADIX) {
#pragma unroll
    for (int w = 0; w < WARPS; w++) {
      const u32 c = whist[w * RADIX + tid];
      whist[w * RADIX + tid] = tot;
      tot += c;
    }
    st_relaxed(lookback + (u64)tile * RADIX + tid, lb_pack(tile == 0 ? LB_PREFIX : LB_AGG, epoch, tot));
  }
  const u32 bs = block_excl_sum<THREADS>(tid < RADIX ? tot : 0u, scratch);  // (contains __syncthreads)
  if (tid < RADIX) bin_start[tid] = bs;
  // (3) look-back for the exclusive prefix of every digit over earlier tiles; each bin-owner thread inspects LBW
  //     predecessors per L2 round trip and backs off while they are unpublished
  if (tid < RADIX) {
    u64 excl = 0;
    if (tile > 0) {
      long long p = (long long)tile - 1;
      int spins = 0;
      while (true) {
        u64 w[LBW];
#pragma unroll
        for (int q = 0; q < LBW; q++) w[q] = p - q >= 0 ? ld_relaxed(lookback + (u64)(p - q) * RADIX + tid) : 0ull;
        int q = 0;
        bool done = false;
#pragma unroll
        for (int qq = 0; qq < LBW; qq++) {
          if (done || q != qq || p - qq < 0) continue;
          const u32 e = (u32)((w[qq] >> 54) & 0xFF);
          const u64 st = w[qq] & (3ull << 62);
          if (e != epoch || st == 0) continue;
          excl += w[qq] & LB_VAL;
          q = qq + 1;
          if (st == LB_PREFIX) done = true;
        }
        if (done) break;
        if (q == 0) __nanosleep(++spins < 4 ? 32 : 128);
        p -= q;
      }
      st_relaxed(lookback + (u64)tile * RADIX + tid, lb_pack(LB_PREFIX, epoch, excl + tot));
    }
    globu[tid] = (u32)(bin_base[tid] + excl) - bs;  // positions < m < 2^32: modular u32 offsets
  }
  // (4) stable warp-level ranking: running per-warp digit counter (starts at the warp's offset) + lower peers
  u32* wm = wmask + warp * (RADIX + 1);
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    const u32 d = rd[i];
    atomicOr(&wm[d], 1u << lane);
    __syncwarp();
    // the peer word and the running counter are read together: one shared-memory round trip per item
    const unsigned peers = wm[d];
    const u32 c = (FULL || d < RADIX) ? wh[d] : 0u;  // (invalid items of a partial tile: digit RADIX, no counter)
    __syncwarp();
    const bool leader = lane == 31 - __clz(peers);
    rd[i] |= (c + __popc(peers & lanemask_lt())) << 9;
    if (leader) {
      wm[d] = 0;
      if (FULL || d < RADIX) wh[d] = c + __popc(peers);
    }
    __syncwarp();
  }
  __syncthreads();
  // (5) scatter into shared memory in (digit, stable) order, then coalesced stores of each digit's run
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    if (FULL || i < nv) {
      const u32 pos = bin_start[rd[i] & 511] + (rd[i] >> 9);
      keys_s[pos] = k[i];
      vals_s[pos] = v[i];
    }
  }
  __syncthreads();
  const u32 tcount = FULL ? (u32)TILE : (u32)min((u64)TILE, (u64)m - tbase);
#pragma unroll 4
  for (u32 j = tid; j < tcount; j += THREADS) {
    const u64 key = keys_s[j];
    const u32 d = (u32)((key >> shift) & (RADIX - 1));
    const u32 dst = globu[d] + j;
    __stcs(kout + dst, key);
    __stcs(vout + dst, vals_s[j]);
  }
}

__global__ void __launch_bounds__(KV_THREADS, KV_MINB) onesweep_kv_kernel(
    const u64* __restrict__ kin, u64* __restrict__ kout, const u32* __restrict__ vin, u32* __restrict__ vout, u32 m,
    u32 shift, const u64* __restrict__ bin_base, u64* __restrict__ lookback, u32* __restrict__ tile_ctr, u32 epoch) {
  constexpr int WARPS = KV_THREADS / 32;
  constexpr int TILE = KV_THREADS * KV_ITEMS;
  static_assert(RADIX <= KV_THREADS, "one bin per thread");
  extern __shared__ __align__(16) unsigned char smem[];
  u32* whist = reinterpret_cast<u32*>(smem) + 3 * TILE;
  u32* wmask = whist + WARPS * RADIX + RADIX + 2 * RADIX + WARPS + 1;
  __shared__ u32 s_tile;
  const int tid = threadIdx.x;
  // one tile per CTA; tile ids from an atomic counter = execution order (blockIdx order measured 45% slower:
  // a tile whose predecessor was dispatched later spins in the look-back)
  if (tid == 0) s_tile = atomicAdd(tile_ctr, 1u);
  for (int i = tid; i < WARPS * RADIX; i += KV_THREADS) whist[i] = 0;
  for (int i = tid; i < WARPS * (RADIX + 1); i += KV_THREADS) wmask[i] = 0;
  __syncthreads();
  const u32 tile = s_tile;
  if ((u64)(tile + 1) * TILE <= m)
    onesweep_kv_tile<true>(kin, kout, vin, vout, m, shift, bin_base, lookback, epoch, tile, smem);
  else
    onesweep_kv_tile<false>(kin, kout, vin, vout, m, shift, bin_base, lookback, epoch, tile, smem);
}

static size_t onesweep_kv_smem() {
  constexpr int WARPS = KV_THREADS / 32, TILE = KV_THREADS * KV_ITEMS;
  return (size_t)TILE * 12 + (size_t)WARPS * RADIX * 4 + RADIX * 4 + RADIX * 8 + (WARPS + 1) * 4 +
         (size_t)WARPS * (RADIX + 1) * 4;
}

// ------------------------------------------------------------------------------------------------------------
// onesweep2 (keys only; the sort passes of the check): the tile-local position of every key is known once the
// tile's digit counts are (bin start + the warp's offset within the bin + its stable rank in the warp), so
// ranking writes each key straight into its shared-memory slot and keeps no per-item rank registers; the global
// offsets from the look-back are only needed by the final coalesced write-out, so the look-back is walked after
// ranking (predecessors have had the ranking time to publish their inclusive prefixes).  The tile (256 threads x
// 32 keys) arrives by TMA bulk copies issued in the kernel prologue, right after the tile id.  Peer sets: every
// 4th item by 8 ballots (ALU pipe), the others by shared-memory masks (LSU pipe, the binding one) — measured
// against all-masks, all-ballots, every 2nd/3rd item by ballots and MATCH.
// ------------------------------------------------------------------------------------------------------------
#ifndef OS_ITEMS_
#define OS_ITEMS_ 32
#endif
#ifndef OS_MINB_
#define OS_MINB_ 2
#endif
constexpr int OS_THREADS = 256, OS_ITEMS = OS_ITEMS_, OS_MINB = OS_MINB_, OS_LBW = 4, OS_TILE = OS_THREADS * OS_ITEMS;

__device__ __forceinline__ u64 gtime() {
  u64 t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
// Per-tile phase stamps for diagnosis (never set by the library: always null).  Its runtime checks at the phase
// boundaries also shape ptxas's schedule: compiled without them the pass spills 68 instead of 20 bytes per thread
// and runs 3% slower (4.94 vs 4.80 ms per 1e9 keys, measured).
__device__ unsigned long long* g_prof = nullptr;

// UNST == 3 (the second partition pass after the fused extents + first partition, k_extract.cu): the input is
// RADIX regions of cap keys, region r holding fill[r] keys (sentinel-padded); tiles never straddle regions
// (tile t belongs to region t / tpr: no lookup before the tile's bulk copy, which reads a whole tile; the keys past
// the fill are not used), and each key is rebased on load from raw low-30 granule bits to key_hi =
// (raw - g0) mod 2^30 (sentinels stay ~0)
struct MapArgs {
  const u32* fill;     // [RADIX]
  u64 cap;
  u32 tpr;             // tiles per region (a tile past a region's fill is empty or partial)
  u32 pos_bits, g0;    // rebase: pos_bits of the layout, low 30 bits of G0
};

template <int THREADS, int ITEMS, int LBW, bool FULL, bool LATE_LB, int S, bool BAL, int TMA, int MIX = 0,
          int UNST = 0>
__device__ __forceinline__ void onesweep2_tile(const u64* __restrict__ kin, u64* __restrict__ kout, u32 m, u32 shift,
                                               const u64* __restrict__ bin_base, u64* __restrict__ lookback,
                                               u32 epoch, u32 tile, unsigned char* smem, unsigned long long* prof,
                                               u64* ebar, const MapArgs& mp) {
  constexpr int WARPS = THREADS / 32;
  constexpr int TILE = THREADS * ITEMS;
  constexpr int IPS = ITEMS / S;  // items per rank stream
  static_assert(ITEMS % S == 0, "streams split the items evenly");
  u64* keys_s = reinterpret_cast<u64*>(smem);                    // [TILE]
  u32* whist = reinterpret_cast<u32*>(keys_s + TILE);             // [WARPS*S][RADIX]: counts -> tile-local bases
  u32* globu = whist + WARPS * S * RADIX;                        // [RADIX]
  u32* scratch = globu + RADIX;                                  // [WARPS + 1]
  u32* wmask = scratch + WARPS + 1;                              // [WARPS*S][RADIX + 1]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const u64 tbase = (u64)tile * TILE;
  const u64 wbase = tbase + (u64)warp * 32 * ITEMS + lane;
  const int nv = FULL ? ITEMS : (int)(wbase < m ? min((u64)ITEMS, ((u64)m - wbase + 31) / 32) : 0ull);
  u64 k[ITEMS];
  if (TMA) {
    // the tile arrives by bulk copies straight into shared memory (no L1 miss tracking, no registers in flight),
    // then each thread takes its warp-striped keys (conflict-free rows); the scatter below overwrites keys_s.
    // TMA == 2: the copies were issued in the kernel prologue, right after the tile id arrived.
    __shared__ u64 tbar;
    u64& bar = TMA == 2 ? *ebar : tbar;
    if (TMA == 1 && tid == 0) {
      mbar_init(&bar, 1);
      fence_mbar_init();
      const u32 cnt = FULL ? (u32)TILE : (u32)min((u64)TILE, (u64)m - tbase);
      const u32 bytes = (cnt * 8 + 15) & ~15u;  // key buffers carry >= 16 bytes of slack
      mbar_expect_tx(&bar, bytes);
      for (u32 off = 0; off < bytes; off += 16384)
        bulk_g2s(reinterpret_cast<unsigned char*>(keys_s) + off, reinterpret_cast<const unsigned char*>(kin + tbase) + off,
                 min(16384u, bytes - off), &bar);
    }
    if (TMA == 1) __syncthreads();
    mbar_wait(&bar, 0);
#pragma unroll
    for (int i = 0; i < ITEMS; i++)
      if (FULL || i < nv) k[i] = keys_s[warp * 32 * ITEMS + i * 32 + lane];
    if (UNST == 3) {
      const u64 pm = (1ull << mp.pos_bits) - 1ull;
#pragma unroll
      for (int i = 0; i < ITEMS; i++)
        if ((FULL || i < nv) && k[i] != ~0ull)
          k[i] = ((((k[i] >> mp.pos_bits) - (u64)mp.g0) & ((1ull << 30) - 1ull)) << mp.pos_bits) | (k[i] & pm);
    }
    __syncthreads();
  } else {
#pragma unroll
    for (int i = 0; i < ITEMS; i++)
      if (FULL || i < nv) k[i] = __ldcs(kin + wbase + (u64)i * 32);
  }
  // (UNST = 0: stable pass; 1: unstable pass on the TOP digit whose input carries ~0 sentinels — padding of
  //  32-aligned digit runs: nothing lies above the top digit, so a sentinel is the only key whose shifted value is
  //  >= RADIX; 2: unstable pass on any digit, no sentinels)
  auto digit = [&](int i) -> u32 {
    if (!(FULL || i < nv)) return (u32)RADIX;
    if (UNST == 1 || UNST == 3) { const u32 d9 = (u32)(k[i] >> shift) & (2 * RADIX - 1); return d9 < RADIX ? d9 : (u32)RADIX; }
    return (u32)((k[i] >> shift) & (RADIX - 1));
  };
  // rank streams: items [s*IPS, (s+1)*IPS) of a warp form stream s (stable order = warp, stream, item, lane),
  // each with its own counters and peer masks, so that S items are ranked per shared-memory round trip
  u32* wh = whist + warp * S * RADIX;
  if (prof) {
    __syncthreads();
    if (tid == 0) prof[1] = gtime();
  }
  // (1) per-(warp, stream) digit counts.  UNST (the bucket path's partition passes, which need no stable order):
  //     the count atomic's return value is the key's rank within its (warp, digit) group — no ranking loop
  u32 rk[UNST ? (ITEMS + 1) / 2 : 1];
  if (UNST)
#pragma unroll
    for (int i = 0; i < (ITEMS + 1) / 2; i++) rk[i] = 0;
#pragma unroll
  for (int i = 0; i < ITEMS; i++)
    if ((FULL || i < nv) && (!UNST || digit(i) < RADIX)) {
      const u32 r = atomicAdd(&wh[(i / IPS) * RADIX + digit(i)], 1u);
      if (UNST) rk[i / 2] |= r << (16 * (i & 1));
    }
  __syncthreads();
  // (2) tile totals -> publish the aggregate; per-(warp, stream, digit) tile-local base = bin start + offset
  u32 tot = 0;
  if (tid < RADIX) {
#pragma unroll
    for (int w = 0; w < WARPS * S; w++) {
      const u32 c = whist[w * RADIX + tid];
      whist[w * RADIX + tid] = tot;
      tot += c;
    }
    st_relaxed(lookback + (u64)tile * RADIX + tid, lb_pack(tile == 0 ? LB_PREFIX : LB_AGG, epoch, tot));
  }
  const u32 bs = block_excl_sum<THREADS>(tid < RADIX ? tot : 0u, scratch);  // (contains __syncthreads)
  if (tid < RADIX) {
#pragma unroll
    for (int w = 0; w < WARPS * S; w++) whist[w * RADIX + tid] += bs;
  }
  __shared__ u32 s_real;  // UNST: keys of the tile (sentinels excluded)
  if (UNST && tid == RADIX - 1) s_real = bs + tot;
  auto look_back = [&]() {
    if (tid < RADIX) {
      u64 excl = 0;
      if (tile > 0) {
        long long p = (long long)tile - 1;
        int spins = 0;
        while (true) {
          constexpr int LW = LBW;
          u64 w[LW];
#pragma unroll
          for (int q = 0; q < LW; q++) w[q] = p - q >= 0 ? ld_relaxed(lookback + (u64)(p - q) * RADIX + tid) : 0ull;
          int q = 0;
          bool done = false;
#pragma unroll
          for (int qq = 0; qq < LW; qq++) {
            if (done || q != qq || p - qq < 0) continue;
            const u32 e = (u32)((w[qq] >> 54) & 0xFF);
            const u64 st = w[qq] & (3ull << 62);
            if (e != epoch || st == 0) continue;
            excl += w[qq] & LB_VAL;
            q = qq + 1;
            if (st == LB_PREFIX) done = true;
          }
          if (done) break;
          if (q == 0) __nanosleep(++spins < 4 ? 32 : 128);
          p -= q;
        }
        if (prof && tid == 0) prof[7] = ((u64)(tile - p) << 32) | (u64)spins;
        st_relaxed(lookback + (u64)tile * RADIX + tid, lb_pack(LB_PREFIX, epoch, excl + tot));
      }
      globu[tid] = (u32)(bin_base[tid] + excl) - bs;  // positions < m < 2^32: modular u32 offsets
    }
  };
  if (!LATE_LB) look_back();
  __syncthreads();
  if (prof && tid == 0) prof[2] = gtime();
  if (UNST) {
    // (3') each key straight to its slot: (warp, digit) base + its count-atomic rank
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
      const u32 d = digit(i);
      if (d < RADIX) keys_s[wh[d] + ((rk[i / 2] >> (16 * (i & 1))) & 0xFFFFu)] = k[i];
    }
  } else {
  // (3) stable warp ranking, each key stored straight into its tile-local slot
  u32* wm = wmask + warp * S * (RADIX + 1);
  const unsigned lt = lanemask_lt();
#pragma unroll
  for (int i = 0; i < IPS; i++) {
    // peer sets: shared-memory masks (LSU), ballots per digit bit (BAL, ALU) or, with MIX, odd items by ballots
    // (MIX 1) or by MATCH (MIX 2, ADU) so that two pipes share the work
    const bool bal = BAL || (MIX == 1 && (i & 1)) || (MIX == 3 && i % 3 == 0) || (MIX == 4 && i % 4 == 0) ||
                     (MIX == 5 && i % 4 != 0);
    const bool mat = MIX == 2 && (i & 1);
    const bool msk = !bal && !mat;
    u32 d[S];
#pragma unroll
    for (int q = 0; q < S; q++) {
      d[q] = digit(q * IPS + i);
      if (msk) atomicOr(&wm[q * (RADIX + 1) + d[q]], 1u << lane);
    }
    if (msk) __syncwarp();
    unsigned peers[S];
    u32 c[S];
#pragma unroll
    for (int q = 0; q < S; q++) {
      peers[q] = bal ? (FULL ? peers_of<RADIX_BITS>(d[q]) : peers_of<RADIX_BITS + 1>(d[q]))
                     : mat ? __match_any_sync(~0u, d[q]) : wm[q * (RADIX + 1) + d[q]];
      c[q] = (FULL || d[q] < RADIX) ? wh[q * RADIX + d[q]] : 0u;  // (invalid items: digit RADIX, no counter)
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < S; q++) {
      const bool leader = lane == 31 - __clz(peers[q]);
      if (FULL || d[q] < RADIX) keys_s[c[q] + __popc(peers[q] & lt)] = k[q * IPS + i];
      if (leader) {
        if (msk) wm[q * (RADIX + 1) + d[q]] = 0;
        if (FULL || d[q] < RADIX) wh[q * RADIX + d[q]] = c[q] + __popc(peers[q]);
      }
    }
    __syncwarp();
  }
  }
  if (prof && tid == 0) prof[3] = gtime();
  if (LATE_LB) look_back();
  __syncthreads();
  if (prof && tid == 0) prof[4] = gtime();
  // (4) coalesced write-out of each digit's run
  if (FULL && (!UNST || s_real == (u32)TILE)) {  // (the common case: a full tile without sentinels)
#pragma unroll 4
    for (u32 j = tid; j < (u32)TILE; j += THREADS) {
      const u64 key = keys_s[j];
      const u32 d = (u32)((key >> shift) & (RADIX - 1));
      __stcs(kout + (globu[d] + j), key);
    }
  } else {
    const u32 tcount = UNST ? s_real : FULL ? (u32)TILE : (u32)min((u64)TILE, (u64)m - tbase);
#pragma unroll 4
    for (u32 j = tid; j < tcount; j += THREADS) {
      const u64 key = keys_s[j];
      const u32 d = (u32)((key >> shift) & (RADIX - 1));
      __stcs(kout + (globu[d] + j), key);
    }
  }
  if (prof) {
    __syncthreads();
    if (tid == 0) prof[5] = gtime(), prof[6] = (u64)blockIdx.x;
  }
}

template <int THREADS, int ITEMS, int MINB, int LBW, bool LATE_LB, int S, bool BAL, int TMA, int MIX = 0,
          int UNST = 0>
__global__ void __launch_bounds__(THREADS, MINB) onesweep2_kernel(const u64* __restrict__ kin, u64* __restrict__ kout,
                                                                  u32 m, u32 shift, const u64* __restrict__ bin_base,
                                                                  u64* __restrict__ lookback,
                                                                  u32* __restrict__ tile_ctr, u32 epoch,
                                                                  MapArgs mp) {
  constexpr int WARPS = THREADS / 32;
  constexpr int TILE = THREADS * ITEMS;
  static_assert(RADIX <= THREADS, "one bin per thread");
  extern __shared__ __align__(16) unsigned char smem[];
  u32* whist = reinterpret_cast<u32*>(smem) + 2 * TILE;
  u32* wmask = whist + WARPS * S * RADIX + RADIX + WARPS + 1;
  __shared__ u32 s_tile, s_mcnt;
  __shared__ u64 ebar, s_msrc;
  const int tid = threadIdx.x;
  if (tid == 0) {
    const u32 t = atomicAdd(tile_ctr, 1u);
    s_tile = t;
    u64 tb = (u64)t * TILE;
    u32 cnt = (u32)min((u64)TILE, (u64)m - tb);
    u32 rf = 0, o = 0;
    if (UNST == 3) {  // region t / tpr; the whole tile is copied, its key count is known when the fill arrives
      const u32 r = t / mp.tpr;
      o = (t - r * mp.tpr) * TILE;
      tb = (u64)r * mp.cap + o;
      cnt = TILE;
      rf = mp.fill[r];  // (in flight with the bulk copy)
    }
    if (TMA == 2) {  // start the tile's bulk copies before the counter arrays are cleared
      const u32 bytes = (cnt * 8 + 15) & ~15u;  // key buffers carry >= 16 bytes of slack
      mbar_init(&ebar, 1);
      fence_mbar_init();
      mbar_expect_tx(&ebar, bytes);
      for (u32 off = 0; off < bytes; off += 16384)
        bulk_g2s(smem + off, reinterpret_cast<const unsigned char*>(kin + tb) + off, min(16384u, bytes - off), &ebar);
    }
    if (UNST == 3) s_msrc = tb, s_mcnt = rf > o ? min((u32)TILE, rf - o) : 0u;
  }
  for (int i = tid; i < WARPS * S * RADIX; i += THREADS) whist[i] = 0;
  if (!BAL && !UNST)
    for (int i = tid; i < WARPS * S * (RADIX + 1); i += THREADS) wmask[i] = 0;
  __syncthreads();
  const u32 tile = s_tile;
  unsigned long long* prof = g_prof ? g_prof + (u64)tile * 8 : nullptr;
  if (prof && tid == 0) prof[0] = gtime();
  if (UNST == 3) {  // the tile as a tile of a virtual array: kin + tile * TILE = its keys, m = its end
    kin = reinterpret_cast<const u64*>(reinterpret_cast<uintptr_t>(kin) + (s_msrc - (u64)tile * TILE) * 8);
    m = tile * TILE + s_mcnt;
  }
  if ((u64)(tile + 1) * TILE <= m)
    onesweep2_tile<THREADS, ITEMS, LBW, true, LATE_LB, S, BAL, TMA, MIX, UNST>(kin, kout, m, shift, bin_base, lookback,
                                                                             epoch, tile, smem, prof, &ebar, mp);
  else
    onesweep2_tile<THREADS, ITEMS, LBW, false, LATE_LB, S, BAL, TMA, MIX, UNST>(kin, kout, m, shift, bin_base, lookback,
                                                                              epoch, tile, smem, prof, &ebar, mp);
}

// the measured configuration: 256 x 32 keys, 2 CTAs/SM, look-back after ranking, one rank stream,
// prologue bulk copies (TMA 2), every 4th item's peers by ballots (MIX 4)
#define OS_CFG OS_THREADS, OS_ITEMS, OS_MINB, OS_LBW, true, 1, false, 2, 4
// the bucket path's partition passes (no stable order needed): on the top digit with sentinels (1), on a lower
// digit of a key array (2)
// (measured on C5, per 1e9 keys: 256 x 32 at 2 CTAs/SM 4.09 ms; 256 x 24 at 3: 4.21; 256 x 20 at 3: 4.36;
// 512 x 16 at 2: 4.44; 256 x 16 at 4: 4.69)
constexpr int PT_THREADS = 256, PT_ITEMS = 32, PT_MINB = 2;
#define OS_UCFG PT_THREADS, PT_ITEMS, PT_MINB, OS_LBW, true, 1, false, 2, 4, 1
#define OS_UCFG2 PT_THREADS, PT_ITEMS, PT_MINB, OS_LBW, true, 1, false, 2, 4, 2
#define OS_UCFG3 R3_THREADS_, R3_ITEMS_, R3_MINB_, OS_LBW, true, 1, false, 2, 4, 3

static size_t onesweep2_smem() {
  constexpr int WARPS = OS_THREADS / 32;
  return (size_t)OS_TILE * 8 + (size_t)WARPS * RADIX * 4 + RADIX * 4 + (WARPS + 1) * 4 +
         (size_t)WARPS * (RADIX + 1) * 4;
}

u32 sort_tile_keys() { return OS_TILE; }

// unstable partition pass (the bucket path: chunk order only, survivors are sorted per chunk afterwards);
// top = the pass's digit is the key's top digit and its input may hold ~0 sentinels
void launch_partition_pass(const u64* kin, u64* kout, u32 m, u32 shift, const u64* bin_base, u64* lookback,
                           u32* tile_ctr, u32 epoch, cudaStream_t st, bool top) {
  if (!m) return;
  constexpr int WARPS = PT_THREADS / 32, TILE = PT_THREADS * PT_ITEMS;
  const size_t sm = (size_t)TILE * 8 + (size_t)WARPS * RADIX * 4 + RADIX * 4 + (WARPS + 1) * 4;
  const u32 tiles = (u32)((m + TILE - 1) / TILE);
  if (top) {
    smem_optin((const void*)onesweep2_kernel<OS_UCFG>, sm);
    onesweep2_kernel<OS_UCFG><<<tiles, PT_THREADS, sm, st>>>(kin, kout, m, shift, bin_base, lookback, tile_ctr, epoch,
                                                              MapArgs{});
  } else {
    smem_optin((const void*)onesweep2_kernel<OS_UCFG2>, sm);
    onesweep2_kernel<OS_UCFG2><<<tiles, PT_THREADS, sm, st>>>(kin, kout, m, shift, bin_base, lookback, tile_ctr, epoch,
                                                               MapArgs{});
  }
}

// the second partition pass over the fused extents pass's regions (UNST 3): tiles = tprefix[RADIX] (host)
void launch_partition_regions(const u64* kin, u64* kout, u32 tpr, u32 shift, const u64* bin_base, u64* lookback,
                              u32* tile_ctr, u32 epoch, const u32* fill, u64 cap, u32 pos_bits, u32 g0,
                              cudaStream_t st) {
  const u32 tiles = tpr * RADIX;
  if (!tiles) return;
  constexpr int WARPS = R3_THREADS_ / 32, TILE = R3_THREADS_ * R3_ITEMS_;
  const size_t sm = (size_t)TILE * 8 + (size_t)WARPS * RADIX * 4 + RADIX * 4 + (WARPS + 1) * 4;
  smem_optin((const void*)onesweep2_kernel<OS_UCFG3>, sm);
  MapArgs mp{fill, cap, tpr, pos_bits, g0};
  onesweep2_kernel<OS_UCFG3><<<tiles, R3_THREADS_, sm, st>>>(kin, kout, (u32)((u64)tiles * TILE), shift, bin_base,
                                                            lookback, tile_ctr, epoch, mp);
}

// bin bases of a digit histogram with every run padded to a multiple of 32 (the bucket path's first pass on a key
// array); the pad slots of kout get ~0 sentinels; *mpad = padded length
__global__ void padded_bin_base_kernel(const u32* __restrict__ hist, u64* __restrict__ base, u64* __restrict__ kout,
                                       u32* __restrict__ mpad) {
  __shared__ u32 s[RADIX];
  const u32 d = threadIdx.x, c = hist[d];
  s[d] = (c + 31u) & ~31u;
  __syncthreads();
  if (d == 0) {
    u32 acc = 0;
    for (int i = 0; i < RADIX; i++) {
      const u32 v = s[i];
      s[i] = acc;
      acc += v;
    }
    *mpad = acc;
  }
  __syncthreads();
  base[d] = s[d];
  for (u32 q = s[d] + c; q < s[d] + ((c + 31u) & ~31u); q++) kout[q] = ~0ull;
}

void launch_padded_bin_base(const u32* hist, u64* base, u64* kout, u32* mpad, cudaStream_t st) {
  padded_bin_base_kernel<<<1, RADIX, 0, st>>>(hist, base, kout, mpad);
}

void launch_onesweep(const u64* kin, u64* kout, const u32* vin, u32* vout, u32 m, u32 shift, const u64* bin_base,
                     u64* lookback, u32* tile_ctr, u32 epoch, cudaStream_t st) {
  if (!m) return;
  if (vin) {  // key/value (race lists, benign regrouping)
    const size_t sm = onesweep_kv_smem();
    smem_optin((const void*)onesweep_kv_kernel, sm);
    const u32 tiles = (u32)((m + KV_THREADS * KV_ITEMS - 1) / (KV_THREADS * KV_ITEMS));
    onesweep_kv_kernel<<<tiles, KV_THREADS, sm, st>>>(kin, kout, vin, vout, m, shift, bin_base, lookback, tile_ctr,
                                                       epoch);
  } else {
    const size_t sm = onesweep2_smem();
    smem_optin((const void*)onesweep2_kernel<OS_CFG>, sm);
    const u32 tiles = (u32)((m + OS_TILE - 1) / OS_TILE);
    onesweep2_kernel<OS_CFG><<<tiles, OS_THREADS, sm, st>>>(kin, kout, m, shift, bin_base, lookback, tile_ctr, epoch,
                                                             MapArgs{});
  }
}

// digit histograms of plain keys: npass 8-bit digits from bit `shift` (race lists: 0; exchanged keys: pos_bits)
__global__ void hist_keys_kernel(const u64* __restrict__ keys, u32 m, u32 npass, u32 shift, u32* __restrict__ hist) {
  extern __shared__ u32 sh[];
  for (u32 i = threadIdx.x; i < npass * RADIX; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  for (u32 k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) {
    u64 key = keys[k];
    for (u32 p = 0; p < npass; p++) atomicAdd(&sh[p * RADIX + ((key >> (shift + p * RADIX_BITS)) & (RADIX - 1))], 1u);
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += blockDim.x)
    if (sh[i]) atomicAdd(&hist[i], sh[i]);
}

void launch_hist_keys_shift(const u64* keys, u32 m, u32 npass, u32 shift, u32* hist, cudaStream_t st) {
  if (!m || !npass) return;
  u32 grid = min((m + 255) / 256, 1184u);
  hist_keys_kernel<<<grid, 256, npass * RADIX * 4, st>>>(keys, m, npass, shift, hist);
}

void launch_hist_keys(const u64* keys, u32 m, u32 npass, u32* hist, cudaStream_t st) {
  launch_hist_keys_shift(keys, m, npass, 0, hist, st);
}

}  // namespace sesa
