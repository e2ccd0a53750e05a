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
#include <cstdlib>

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

// Lanes holding the same digit (stable peers) without __match_any_sync: MATCH runs on the slow ADU pipe on
// sm_100 (ncu: 65-96% ADU busy), ballots run on the ALU pipe.  NB = digit bits to compare.
template <int NB>
__device__ __forceinline__ unsigned peers_of(u32 d) {
  unsigned p = ~0u;
#pragma unroll
  for (int b = 0; b < NB; b++) {
    const bool bit = (d >> b) & 1u;
    const unsigned m = __ballot_sync(~0u, bit);
    p &= bit ? m : ~m;
  }
  return p;
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

// block-wide exclusive sum over THREADS values (one per thread)
template <int THREADS>
__device__ __forceinline__ u32 block_excl_sum(u32 v, u32* scratch /* [THREADS/32 + 1] */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  u32 x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    u32 y = __shfl_up_sync(~0u, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) scratch[warp] = x;
  __syncthreads();
  if (threadIdx.x == 0) {
    u32 acc = 0;
    for (int w = 0; w < THREADS / 32; w++) {
      u32 c = scratch[w];
      scratch[w] = acc;
      acc += c;
    }
  }
  __syncthreads();
  return scratch[warp] + x - v;
}

template <int THREADS, int ITEMS, bool VALS, int MATCH>
__global__ void __launch_bounds__(THREADS, 3) onesweep_kernel(const u64* __restrict__ kin, u64* __restrict__ kout,
                                                           const u32* __restrict__ vin, u32* __restrict__ vout,
                                                           u32 m, u32 shift, const u64* __restrict__ bin_base,
                                                           u64* __restrict__ lookback, u32* __restrict__ tile_ctr,
                                                           u32 epoch) {
  constexpr int WARPS = THREADS / 32;
  constexpr int TILE = THREADS * ITEMS;
  static_assert(RADIX <= THREADS, "one bin per thread");
  extern __shared__ __align__(16) unsigned char smem[];
  u64* keys_s = reinterpret_cast<u64*>(smem);                                  // [TILE]
  u32* vals_s = reinterpret_cast<u32*>(keys_s + TILE);                          // [TILE] if VALS
  u32* whist = VALS ? vals_s + TILE : reinterpret_cast<u32*>(keys_s + TILE);    // [WARPS][RADIX]
  u32* bin_start = whist + WARPS * RADIX;                                       // [RADIX]
  long long* glob = reinterpret_cast<long long*>(bin_start + RADIX);            // [RADIX]
  u32* scratch = reinterpret_cast<u32*>(glob + RADIX);                          // [WARPS + 1]
  u32* wmask = scratch + WARPS + 1;                                             // [WARPS][RADIX + 1] (MATCH 1)
  __shared__ u32 s_tile;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_tile = atomicAdd(tile_ctr, 1u);
  for (int i = tid; i < WARPS * RADIX; i += THREADS) whist[i] = 0;
  if (MATCH == 1)
    for (int i = tid; i < WARPS * (RADIX + 1); i += THREADS) wmask[i] = 0;
  __syncthreads();
  const u32 tile = s_tile;
  const u64 tbase = (u64)tile * TILE;

  u64 k[ITEMS];
  u32 v[ITEMS];
  u32 rk[ITEMS];
  const u64 wbase = tbase + (u64)warp * 32 * ITEMS + lane;
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    u64 idx = wbase + (u64)i * 32;
    if (idx < m) {
      k[i] = __ldcs(kin + idx);  // streaming: each key is read once per pass
      if (VALS) v[i] = __ldcs(vin + idx);
    } else {
      k[i] = ~0ull;
    }
  }
  u32* wh = whist + warp * RADIX;
  const bool full = tbase + TILE <= m;
  // (1) early counts: per-warp digit histogram with shared-memory atomics (no ordering needed for counts)
#pragma unroll
  for (int i = 0; i < ITEMS; i++)
    if (full || wbase + (u64)i * 32 < m) atomicAdd(&wh[(u32)((k[i] >> shift) & (RADIX - 1))], 1u);
  __syncthreads();
  // (2) per-digit tile totals -> publish the tile aggregate BEFORE ranking, so that successor tiles find it
  //     during their look-back; per-warp counts become exclusive offsets across warps
  u32 tot = 0;
  if (tid < RADIX) {
#pragma unroll
    for (int w = 0; w < WARPS; w++) {
      u32 c = whist[w * RADIX + tid];
      whist[w * RADIX + tid] = tot;
      tot += c;
    }
    st_relaxed(lookback + (u64)tile * RADIX + tid, lb_pack(tile == 0 ? LB_PREFIX : LB_AGG, epoch, tot));
  }
  const u32 bs = block_excl_sum<THREADS>(tid < RADIX ? tot : 0u, scratch);  // (contains __syncthreads)
  if (tid < RADIX) bin_start[tid] = bs;
  // (3) stable warp-level ranking: running per-warp digit counter (starts at the warp's offset) + lower peers
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    const bool valid = full || wbase + (u64)i * 32 < m;
    const u32 d = valid ? (u32)((k[i] >> shift) & (RADIX - 1)) : (u32)RADIX;
    unsigned peers;
    if (MATCH == 0) {
      peers = full ? peers_of<RADIX_BITS>(d) : peers_of<RADIX_BITS + 1>(d);
    } else {
      // each lane sets its bit in its digit's word of a per-warp mask array: the word becomes the peer set
      u32* wm = wmask + warp * (RADIX + 1);
      atomicOr(&wm[d], 1u << lane);
      __syncwarp();
      peers = wm[d];
      __syncwarp();
      if (lane == 31 - __clz(peers)) wm[d] = 0;
    }
    u32 c = valid ? wh[d] : 0u;
    rk[i] = c + __popc(peers & lanemask_lt());
    __syncwarp();
    if (valid && lane == 31 - __clz(peers)) wh[d] = c + __popc(peers);
    __syncwarp();
  }
  // (4) look-back for the exclusive prefix of every digit over earlier tiles (by now mostly published)
  if (tid < RADIX) {
    u64 excl = 0;
    if (tile > 0) {
      long long p = (long long)tile - 1;
      while (true) {
        const u64 w = ld_relaxed(lookback + (u64)p * RADIX + tid);
        const u32 e = (u32)((w >> 54) & 0xFF);
        const u64 st = w & (3ull << 62);
        if (e != epoch || st == 0) continue;  // predecessor has not published yet: spin
        excl += w & LB_VAL;
        if (st == LB_PREFIX) break;
        p--;
      }
      st_relaxed(lookback + (u64)tile * RADIX + tid, lb_pack(LB_PREFIX, epoch, excl + tot));
    }
    glob[tid] = (long long)(bin_base[tid] + excl) - (long long)bs;
  }
  __syncthreads();
  // scatter into shared memory in (digit, stable) order
#pragma unroll
  for (int i = 0; i < ITEMS; i++) {
    if (wbase + (u64)i * 32 < m) {
      const u32 d = (u32)((k[i] >> shift) & (RADIX - 1));
      const u32 pos = bin_start[d] + rk[i];
      keys_s[pos] = k[i];
      if (VALS) vals_s[pos] = v[i];
    }
  }
  __syncthreads();
  const u32 tcount = (u32)min((u64)TILE, (u64)m - tbase);
#pragma unroll 4
  for (u32 j = tid; j < tcount; j += THREADS) {
    const u64 key = keys_s[j];
    const u32 d = (u32)((key >> shift) & (RADIX - 1));
    const u64 dst = (u64)(glob[d] + (long long)j);
    __stcs(kout + dst, key);
    if (VALS) __stcs(vout + dst, vals_s[j]);
  }
}

template <bool VALS>
static size_t onesweep_smem() {
  constexpr int WARPS = SORT_THREADS / 32;
  return (size_t)SORT_TILE * 8 + (VALS ? (size_t)SORT_TILE * 4 : 0) + (size_t)WARPS * RADIX * 4 + RADIX * 4 +
         RADIX * 8 + (WARPS + 1) * 4 + (size_t)WARPS * (RADIX + 1) * 4;
}

int sort_variant() {  // SESA_SORT_MATCH=0 ballots, 1 atomicOr masks (default)
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("SESA_SORT_MATCH");
    v = e ? atoi(e) : 1;
  }
  return v;
}

template <bool VALS, int MATCH>
static void launch_os(const u64* kin, u64* kout, const u32* vin, u32* vout, u32 m, u32 shift, const u64* bin_base,
                      u64* lookback, u32* tile_ctr, u32 epoch, cudaStream_t st) {
  auto kern = onesweep_kernel<SORT_THREADS, SORT_ITEMS, VALS, MATCH>;
  const size_t sm = onesweep_smem<VALS>();
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    set = true;
  }
  kern<<<sort_tiles(m), SORT_THREADS, sm, st>>>(kin, kout, vin, vout, m, shift, bin_base, lookback, tile_ctr, epoch);
}

void launch_onesweep(const u64* kin, u64* kout, const u32* vin, u32* vout, u32 m, u32 shift, const u64* bin_base,
                     u64* lookback, u32* tile_ctr, u32 epoch, cudaStream_t st) {
  if (!sort_tiles(m)) return;
  const bool ballot = sort_variant() == 0;
  if (vin) {
    if (ballot) launch_os<true, 0>(kin, kout, vin, vout, m, shift, bin_base, lookback, tile_ctr, epoch, st);
    else launch_os<true, 1>(kin, kout, vin, vout, m, shift, bin_base, lookback, tile_ctr, epoch, st);
  } else {
    if (ballot) launch_os<false, 0>(kin, kout, nullptr, nullptr, m, shift, bin_base, lookback, tile_ctr, epoch, st);
    else launch_os<false, 1>(kin, kout, nullptr, nullptr, m, shift, bin_base, lookback, tile_ctr, epoch, st);
  }
}

// digit histograms of plain keys (race list sort): npass 8-bit digits from bit 0
__global__ void hist_keys_kernel(const u64* __restrict__ keys, u32 m, u32 npass, u32* __restrict__ hist) {
  extern __shared__ u32 sh[];
  for (u32 i = threadIdx.x; i < npass * RADIX; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  for (u32 k = blockIdx.x * blockDim.x + threadIdx.x; k < m; k += gridDim.x * blockDim.x) {
    u64 key = keys[k];
    for (u32 p = 0; p < npass; p++) atomicAdd(&sh[p * RADIX + ((key >> (p * RADIX_BITS)) & (RADIX - 1))], 1u);
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += blockDim.x)
    if (sh[i]) atomicAdd(&hist[i], sh[i]);
}

void launch_hist_keys(const u64* keys, u32 m, u32 npass, u32* hist, cudaStream_t st) {
  if (!m || !npass) return;
  u32 grid = min((m + 255) / 256, 1184u);
  hist_keys_kernel<<<grid, 256, npass * RADIX * 4, st>>>(keys, m, npass, hist);
}

}  // namespace sesa
