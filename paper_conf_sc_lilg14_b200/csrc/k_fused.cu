// k_fused.cu — key extraction fused with the first LSD sort pass (SURVEY §8a rows a2 + a4), for the common
// layout: one space (global), records already in (block, interval) order, one granule per record — C3, C4, C5.
//
// The first sort digit of an entry is d = (g - gmin) & 255 with g = addr >> log2G.  Modulo 256 that is a
// rotation of the raw byte g & 255, whose per-tile histograms the extents pass already produced (k_extract.cu)
// before gmin was known.  From them three small kernels compute, for every tile t of FUSED_TILE records and
// digit d, the exact output offset of the tile's digit-d run (bin base + the digit-d counts of all earlier
// tiles).  The fused kernel then reads each record's address once (the key never makes the round trip through
// HBM that a separate extract kernel + first pass costs: 32 B read + 8 B written per record instead of
// 32 + 8 + 8 + 8), ranks the tile stably by d exactly like a onesweep tile (k_sort.cu) and writes each digit run
// to its precomputed offset — no decoupled look-back, so CTAs are persistent and take tiles in any order.  It
// also accumulates the histograms of the remaining digits (the upfront histograms of the later passes).
#include <algorithm>
#include <cstdlib>

#include "kernels.cuh"

namespace sesa {

// ---- tile offsets from the raw per-tile histograms H[t][r] (r = g & 255), r0 = gmin & 255, digit(r) = r - r0 --
// (1) per chunk of tiles: column sums P[c][r]
__global__ void tile_col_reduce_kernel(const u32* __restrict__ H, u32 T, u32 tpc, u32* __restrict__ P) {
  const u32 c = blockIdx.x, r = threadIdx.x;
  const u32 t0 = c * tpc, t1 = min(T, t0 + tpc);
  u32 s = 0;
#pragma unroll 8
  for (u32 t = t0; t < t1; t++) s += H[(u64)t * RADIX + r];
  P[(u64)c * RADIX + r] = s;
}

// (2) one CTA: exclusive prefix over chunks per raw byte, plus the bin base of each digit (rotated order)
// pad32 (the bucket path): every digit run is padded to a multiple of 32 slots with ~0 sentinels (written here,
// into kout), so that no 32-key row of the next, unstable pass holds two digit values (k_bucket.cu); *mtot = the
// padded length
__global__ void tile_col_scan_kernel(u32* __restrict__ P, u32 C, u32 r0, u64* __restrict__ kout,
                                     u32* __restrict__ mtot) {
  __shared__ u32 s_tot[RADIX], s_w[RADIX / 32 + 1];
  const u32 r = threadIdx.x, lane = r & 31, warp = r >> 5;
  u32 run = 0;
  for (u32 c0 = 0; c0 < C; c0 += 16) {  // 16 independent loads per round trip
    u32 v[16];
#pragma unroll
    for (int q = 0; q < 16; q++) v[q] = c0 + q < C ? P[(u64)(c0 + q) * RADIX + r] : 0u;
#pragma unroll
    for (int q = 0; q < 16; q++)
      if (c0 + q < C) P[(u64)(c0 + q) * RADIX + r] = run, run += v[q];
  }
  const u32 d = (r - r0) & (RADIX - 1);
  const u32 real = run;
  s_tot[d] = kout ? (run + 31u) & ~31u : run;
  __syncthreads();
  // exclusive scan over digits d (thread d holds s_tot[d])
  const u32 v = s_tot[r];
  u32 x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u32 y = __shfl_up_sync(~0u, x, o);
    if (lane >= (u32)o) x += y;
  }
  if (lane == 31) s_w[warp] = x;
  __syncthreads();
  if (r == 0) {
    u32 acc = 0;
    for (int w = 0; w < RADIX / 32; w++) {
      const u32 c = s_w[w];
      s_w[w] = acc;
      acc += c;
    }
  }
  __syncthreads();
  s_tot[r] = s_w[warp] + x - v;  // bin base of digit r
  if (kout && r == RADIX - 1) *mtot = s_w[warp] + x;
  __syncthreads();
  const u32 base = s_tot[d];
  if (kout)  // sentinels after the run's real keys
    for (u32 q = base + real; q < ((base + real + 31u) & ~31u); q++) kout[q] = ~0ull;
  for (u32 c = 0; c < C; c++) P[(u64)c * RADIX + r] += base;
}

// (3) per chunk: O[t][digit] = offset of tile t's digit run
__global__ void tile_col_down_kernel(const u32* __restrict__ H, u32 T, u32 tpc, const u32* __restrict__ P, u32 r0,
                                     u32* __restrict__ O) {
  const u32 c = blockIdx.x, r = threadIdx.x;
  const u32 t0 = c * tpc, t1 = min(T, t0 + tpc);
  const u32 d = (r - r0) & (RADIX - 1);
  u32 run = P[(u64)c * RADIX + r];
#pragma unroll 8
  for (u32 t = t0; t < t1; t++) {
    O[(u64)t * RADIX + d] = run;
    run += H[(u64)t * RADIX + r];
  }
}

size_t fused_temp_bytes(u64 n) {
  const u64 T = (n + FUSED_TILE - 1) / FUSED_TILE;
  return (T * RADIX * 4 + 255) / 256 * 256 + (u64)1024 * RADIX * 4;
}

// ---- the fused kernel -------------------------------------------------------------------------------------------
struct FusedArgs {
  const u32* gran;  // low 32 bits of every record's granule index (written by the extents pass)
  u32 n, log2G, pos_bits, npass;
  u32 dsh;          // the pass's digit is key_hi bits [dsh, dsh + 8): 0, or HYB_LO on the bucket path
  u64 gmin;
  const u32* toff;  // [T][RADIX] output offset of each tile's digit run
  u64* kout;
  u32* hist;        // [npass][RADIX] global digit histograms (rows 1.. are accumulated here)
  const u32* wbits; // with wbit: bit (i & 31) of wbits[i >> 5] = record i writes (extents pass)
  u32 wbit;         // 1: key = key_hi << pos_bits | pos << 1 | w (pos_bits here includes the bit)
};

// Persistent CTAs, software-pipelined in registers: right after a tile's digit counts (when its addresses have
// become 32-bit key parts), the CTA issues the loads of its NEXT tile's addresses into the freed registers, so
// they are in flight during the ranking and write-out of the current tile — the CTA's HBM reads never pause.
// UNST (the bucket path, which needs no stable order within a digit): the count atomic's return value is the
// key's rank within its (warp, digit) group, and the ranking loop is skipped.
template <int NP, bool UNST = false>
__global__ void __launch_bounds__(FUSED_THREADS, UNST ? FUSED_UMINB : FUSED_MINB) fused_extract_pass0_kernel(FusedArgs A) {
  constexpr int THREADS = FUSED_THREADS, ITEMS = FUSED_ITEMS, WARPS = THREADS / 32, TILE = FUSED_TILE;
  extern __shared__ __align__(16) unsigned char smem[];
  u64* keys_s = reinterpret_cast<u64*>(smem);              // [TILE]
  u32* whist = reinterpret_cast<u32*>(keys_s + TILE);       // [WARPS][RADIX]
  u32* globu = whist + WARPS * RADIX;                      // [RADIX]
  u32* scratch = globu + RADIX;                            // [WARPS + 1]
  u32* wmask = scratch + WARPS + 1;                        // [WARPS][RADIX + 1]
  u32* hrest = wmask + WARPS * (RADIX + 1);                // [NP - 1][RADIX]
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  constexpr u32 nrest = (NP - 1) * RADIX;
  for (u32 i = tid; i < WARPS * (RADIX + 1); i += THREADS) wmask[i] = 0;
  for (u32 i = tid; i < nrest; i += THREADS) hrest[i] = 0;
  const u32 T = (A.n + TILE - 1) / TILE;
  u32* wh = whist + warp * RADIX;
  u32* wm = wmask + warp * (RADIX + 1);
  const unsigned lt = lanemask_lt();
  // (0) granule indices of a tile's records (low 32 bits: 4 bytes per record, coalesced), from the extents pass;
  //     on this path the span is < 2^32, so key_hi = g - gmin = (low32(g) - low32(gmin)) mod 2^32
  u32 a[ITEMS];
  u32 wq = 0;  // with wbit: lane i < ITEMS holds the write bits of the warp's row i (32 records)
  auto issue = [&](u32 t) {
    const u32 wb = t * TILE + warp * 32 * ITEMS + lane;
    const u32* gp = A.gran + wb;
#pragma unroll
    for (int i = 0; i < ITEMS; i++)
      if (wb + i * 32 < A.n) a[i] = __ldcs(gp + i * 32);
    if (!UNST && A.wbit && lane < ITEMS && wb - lane + lane * 32 < A.n) wq = __ldcs(A.wbits + ((wb - lane) >> 5) + lane);
  };
  u32 tile = blockIdx.x;
  if (tile < T) issue(tile);
  while (tile < T) {
    const u32 tbase = tile * TILE;
    const u32 wbase = tbase + warp * 32 * ITEMS + lane;
    const int nv = wbase < A.n ? (int)min((u32)ITEMS, (A.n - wbase + 31) / 32) : 0;
    // only key_hi = g - gmin (< 2^32 on this path) is kept per item: the position part of the key is the item's
    // record index, known from (tile, warp, item, lane)
    u32 kh[ITEMS];
#pragma unroll
    for (int i = 0; i < ITEMS; i++) kh[i] = i < nv ? a[i] - (u32)A.gmin : 0u;
    const u32 wcur = wq;  // (the prefetch below overwrites wq)
    // the low part of item i's key: its position (and, with wbit, its write bit below it)
    auto low = [&](int i) -> u64 {
      const u64 pos = (u64)(wbase + i * 32);
      if (UNST || !A.wbit) return pos;
      return (pos << 1) | (u64)((__shfl_sync(~0u, wcur, i) >> lane) & 1u);
    };
    auto digit = [&](int i) -> u32 { return i < nv ? ((kh[i] >> A.dsh) & (RADIX - 1)) : (u32)RADIX; };
    for (u32 i = tid; i < WARPS * RADIX; i += THREADS) whist[i] = 0;
    __syncthreads();
    // (1) per-warp counts of the digit (UNST: with the ranks)
    u32 rk[UNST ? (ITEMS + 1) / 2 : 1];
    if (UNST)
#pragma unroll
      for (int i = 0; i < (ITEMS + 1) / 2; i++) rk[i] = 0;
#pragma unroll
    for (int i = 0; i < ITEMS; i++)
      if (i < nv) {
        const u32 r = atomicAdd(&wh[digit(i)], 1u);
        if (UNST) rk[i / 2] |= r << (16 * (i & 1));
      }
    __syncthreads();
    // (2) tile-local bases = bin start + warp offset; global write offsets from the precomputed table
    u32 tot = 0;
    if (tid < RADIX) {
#pragma unroll
      for (int w = 0; w < WARPS; w++) {
        const u32 c = whist[w * RADIX + tid];
        whist[w * RADIX + tid] = tot;
        tot += c;
      }
    }
    const u32 bs = block_excl_sum<THREADS>(tid < RADIX ? tot : 0u, scratch);  // (contains __syncthreads)
    if (tid < RADIX) {
#pragma unroll
      for (int w = 0; w < WARPS; w++) whist[w * RADIX + tid] += bs;
      globu[tid] = A.toff[(u64)tile * RADIX + tid] - bs;
    }
    __syncthreads();
    const u32 next = tile + gridDim.x;
    if (next < T) issue(next);  // prefetch: in flight during ranking and write-out
    if (UNST) {
      // (3') each key straight to its slot: (warp, digit) base + its count-atomic rank
#pragma unroll
      for (int i = 0; i < ITEMS; i++) {
        const u32 d = digit(i);
        if (d < RADIX)
          keys_s[wh[d] + ((rk[i / 2] >> (16 * (i & 1))) & 0xFFFFu)] = ((u64)kh[i] << A.pos_bits) | low(i);
      }
    } else {
    // (3) stable warp ranking (peer masks by shared-memory atomicOr), each key stored into its tile slot
#pragma unroll
    for (int i = 0; i < ITEMS; i++) {
      // every 4th item's peer set by ballots (ALU pipe) instead of shared-memory masks (LSU pipe, the binding one)
      const bool bal = (i & 3) == 0;
      const u32 d = digit(i);
      const u64 lo = low(i);  // (warp-wide shuffle: before any lane diverges)
      if (!bal) {
        atomicOr(&wm[d], 1u << lane);
        __syncwarp();
      }
      const unsigned peers = bal ? peers_of<RADIX_BITS + 1>(d) : wm[d];
      const u32 c = d < RADIX ? wh[d] : 0u;  // (invalid items: digit RADIX, no counter)
      __syncwarp();
      if (d < RADIX) keys_s[c + __popc(peers & lt)] = ((u64)kh[i] << A.pos_bits) | lo;
      if (lane == 31 - __clz(peers)) {
        if (!bal) wm[d] = 0;
        if (d < RADIX) wh[d] = c + __popc(peers);
      }
      __syncwarp();
    }
        }
    __syncthreads();
    // (4) coalesced write-out of each digit run, and the CTA histograms of the later digits
    const u32 tcount = min((u32)TILE, A.n - tbase);
#pragma unroll 4
    for (u32 j = tid; j < tcount; j += THREADS) {
      const u64 key = keys_s[j];
      const u32 d = (u32)((key >> (A.pos_bits + A.dsh)) & (RADIX - 1));
      __stcs(A.kout + (globu[d] + j), key);
#pragma unroll
      for (int p = 1; p < NP; p++)
        atomicAdd(&hrest[(p - 1) * RADIX + (u32)((key >> (A.pos_bits + p * RADIX_BITS)) & (RADIX - 1))], 1u);
    }
    __syncthreads();  // shared memory is reused by the next tile
    tile = next;
  }
  for (u32 i = tid; i < nrest; i += THREADS)
    if (hrest[i]) atomicAdd(&A.hist[RADIX + i], hrest[i]);
}

static size_t fused_smem(u32 npass) {
  constexpr int WARPS = FUSED_THREADS / 32;
  return (size_t)FUSED_TILE * 8 + (size_t)WARPS * RADIX * 4 + RADIX * 4 + (WARPS + 1) * 4 +
         (size_t)WARPS * (RADIX + 1) * 4 + (size_t)(npass > 0 ? npass - 1 : 0) * RADIX * 4;
}

bool fused_supported(u32 npass) { return npass >= 1 && npass <= 4; }  // sort_bits <= 32 on this path

// tile offsets O[t][d] into temp (fused_temp_bytes(n)) from the extents' raw per-tile histograms
void launch_tile_offsets(u64 n, const KeyLayout& L, const u32* tile_hist, void* temp, cudaStream_t st, u32 dsh,
                         u64* pad_kout, u32* mtot) {
  if (!n) return;
  const u32 T = (u32)((n + FUSED_TILE - 1) / FUSED_TILE);
  u32* O = reinterpret_cast<u32*>(temp);
  u32* P = reinterpret_cast<u32*>(reinterpret_cast<char*>(temp) + ((u64)T * RADIX * 4 + 255) / 256 * 256);
  const u32 C = std::min<u32>(T, 1024), tpc = (T + C - 1) / C, Cu = (T + tpc - 1) / tpc;
  const u32 r0 = (u32)((L.gminG >> dsh) & (RADIX - 1));
  tile_col_reduce_kernel<<<Cu, RADIX, 0, st>>>(tile_hist, T, tpc, P);
  tile_col_scan_kernel<<<1, RADIX, 0, st>>>(P, Cu, r0, pad_kout, mtot);
  tile_col_down_kernel<<<Cu, RADIX, 0, st>>>(tile_hist, T, tpc, P, r0, O);
}

// temp: holds the tile offsets (launch_tile_offsets); hist: [npass][RADIX] zeroed (rows >= 1 filled)
void launch_fused_extract_pass0(const u32* gran, u64 n, const KeyLayout& L, u32 npass, void* temp, u64* kout,
                                u32* hist, cudaStream_t st, u32 dsh, bool unstable, const u32* wbits) {
  if (!n) return;
  const u32 T = (u32)((n + FUSED_TILE - 1) / FUSED_TILE);
  u32* O = reinterpret_cast<u32*>(temp);
  const void* ks[4] = {(const void*)fused_extract_pass0_kernel<1>, (const void*)fused_extract_pass0_kernel<2>,
                       (const void*)fused_extract_pass0_kernel<3>, (const void*)fused_extract_pass0_kernel<4>};
  const size_t sm = fused_smem(npass);
  // persistent CTAs: one full wave at the occupancy of the largest variant
  const int grid = dev_sm_count() * (unstable ? blocks_per_sm((const void*)fused_extract_pass0_kernel<1, true>,
                                                               FUSED_THREADS, fused_smem(1))
                                              : blocks_per_sm(ks[3], FUSED_THREADS, fused_smem(4)));
  smem_optin(ks[std::min<u32>(npass, 4) - 1], sm);
  FusedArgs A;
  A.gran = gran;
  A.n = (u32)n;
  A.log2G = L.log2G;
  A.wbit = unstable ? 0u : L.wbit;
  A.wbits = wbits;
  A.pos_bits = L.pos_bits + A.wbit;
  A.npass = npass;
  A.dsh = dsh;
  A.gmin = L.gminG;
  A.toff = O;
  A.kout = kout;
  A.hist = hist;
  const u32 g = std::min<u32>(T, (u32)grid);
  if (unstable) {  // the bucket path: one digit, no later-digit histograms
    smem_optin((const void*)fused_extract_pass0_kernel<1, true>, sm);
    fused_extract_pass0_kernel<1, true><<<g, FUSED_THREADS, sm, st>>>(A);
    return;
  }
  switch (npass) {
    case 1: fused_extract_pass0_kernel<1><<<g, FUSED_THREADS, sm, st>>>(A); break;
    case 2: fused_extract_pass0_kernel<2><<<g, FUSED_THREADS, sm, st>>>(A); break;
    case 3: fused_extract_pass0_kernel<3><<<g, FUSED_THREADS, sm, st>>>(A); break;
    default: fused_extract_pass0_kernel<4><<<g, FUSED_THREADS, sm, st>>>(A); break;
  }
}

}  // namespace sesa
