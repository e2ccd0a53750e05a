// k_compact.cu — ordered stream compaction of the sorted keys down to entries whose location is touched by
// at least two entries ("compaction").  A location touched once cannot race (P:43 needs two
// accesses), so singletons — all but ~2e5 of C5's 1e9 entries — never reach the conflict tiles.
//
// Register-only and barrier-free: a warp owns a chunk of 512 consecutive keys (16 coalesced rows of 32), finds
// neighbours with shuffles and output slots with ballots.  Two streaming passes — per-chunk counts, exclusive
// scan of the counts (k_util), write — instead of a decoupled look-back (measured latency-bound) and instead of
// a shared-memory tile (the blocked layout gave 16-way bank conflicts: 53% short-scoreboard stalls in ncu).
// Order — and therefore location runs and their (block, interval) sub-runs — is preserved.
#include <algorithm>

#include "kernels.cuh"

namespace sesa {

// ------------------------------------------------------------------------------------------------------------
// Single-read compaction (default).  Warp w owns the contiguous key range [w*rw, (w+1)*rw) and streams it in
// rows of 32 coalesced keys (U = 12 rows in flight: 1.24 ms per 1e9 keys, at the HBM peak; U = 8: 1.49, 16: 1.50), comparing each key's location-run key with its predecessor's
// (shuffle; the previous row's lane 31 for lane 0) — per 32 keys one shuffle pair, one compare, one ballot.
// Kept keys go, in order, to the warp's own segment seg[w*rw ...); a tiny gather then concatenates the
// segments (exclusive scan of the per-warp counts).  Traffic: one 8-byte read per key plus 3 x 8 bytes per KEPT
// key, instead of two full reads — C5 keeps 2e5 of 1e9.
// G32: single space and the run key (key >> sh) fits 32 bits -> 32-bit run keys; else 64-bit masked keys.
// ------------------------------------------------------------------------------------------------------------
template <bool G32>
struct RunKey {
  u32 sh32;
  u64 mask_s, mask_g, mask_fixed;
  bool both;
  u32 sbit;
  __device__ __forceinline__ auto of(u64 k) const {
    if constexpr (G32) {
      return (u32)(k >> sh32);
    } else {
      const u64 mk = both ? (((k >> sbit) & 1ull) ? mask_g : mask_s) : mask_fixed;
      return k & mk;
    }
  }
};

template <int U, bool G32>
__global__ void __launch_bounds__(256, 4) compact_seg_kernel(const u64* __restrict__ keys, u32 m, RunKey<G32> R, u32 rw,
                                                          u64* __restrict__ seg, u32* __restrict__ wcnt) {
  const int lane = threadIdx.x & 31;
  const u32 w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const u64 start64 = (u64)w * rw;
  if (start64 >= m) return;
  const u32 start = (u32)start64, end = (u32)min((u64)m, start64 + rw);
  using G = decltype(R.of(0ull));
  G prevg;
  unsigned succ;  // the range's last key is in the same run as the next range's first key
  {
    const G g0 = R.of(keys[start]), gl = R.of(keys[end - 1]);
    prevg = start > 0 ? R.of(keys[start - 1]) : (G)(g0 ^ (G)1);  // array start: a differing sentinel
    succ = end < m ? (R.of(keys[end]) == gl ? 1u : 0u) : 0u;
  }
  const unsigned lt = lanemask_lt();
  u32 out = start;  // next free slot of this warp's segment
  // keep = same as predecessor, or same as successor (= the predecessor bit of the next lane / next row)
  auto finalize = [&](u64 key, unsigned sp, unsigned extra) {
    const unsigned keep = sp | (sp >> 1) | extra;
    if (keep) {  // warp-uniform
      if ((keep >> lane) & 1u) seg[out + __popc(keep & lt)] = key;
      out += __popc(keep);
    }
  };
  u64 pk = 0;  // a batch's last row waits for the next batch's first predecessor bit
  unsigned psp = 0;
  bool pending = false;
  for (u32 r0 = start; r0 < end; r0 += 32 * U) {
    u64 k[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 i = r0 + u * 32 + lane;
      k[u] = i < end ? __ldcs(keys + i) : 0ull;
    }
    unsigned sp[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 i = r0 + u * 32 + lane;
      const G g = R.of(k[u]);
      const G up = __shfl_up_sync(~0u, g, 1);
      const G p = lane ? up : prevg;
      sp[u] = __ballot_sync(~0u, i < end && p == g);
      prevg = __shfl_sync(~0u, g, 31);
    }
    if (pending) finalize(pk, psp, (sp[0] & 1u) << 31), pending = false;
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 rb = r0 + u * 32;
      if (rb >= end) break;
      if (rb + 32 < end) {
        if (u + 1 < U) finalize(k[u], sp[u], (sp[u + 1 < U ? u + 1 : u] & 1u) << 31);
        else pk = k[u], psp = sp[u], pending = true;
      } else {
        finalize(k[u], sp[u], succ << (end - 1 - rb));  // last row of the range
      }
    }
  }
  wcnt[w] = out - start;
}

// concatenate the warp segments: warp w copies its wcnt[w] keys to out[woff[w] ...)
__global__ void compact_gather_kernel(const u64* __restrict__ seg, u32 rw, u32 nw, const u32* __restrict__ wcnt,
                                      const u32* __restrict__ woff, u64* __restrict__ out) {
  const u32 w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (w >= nw) return;
  const u32 c = wcnt[w], o = woff[w];
  const u64* src = seg + (u64)w * rw;
  for (u32 i = lane; i < c; i += 32) out[o + i] = src[i];
}

static u32 compact_warps(u64 m, u32* rw_out) {
  // resident warps of one full wave on this device (both variants: the smaller occupancy)
  const int a = blocks_per_sm((const void*)compact_seg_kernel<12, true>, 256, 0);
  const int b = blocks_per_sm((const void*)compact_seg_kernel<8, false>, 256, 0);
  const u64 target = (u64)dev_sm_count() * 8 * (u64)std::max(1, std::min(a, b));
  u64 rw = (m + target - 1) / target;
  rw = std::max<u64>(256, (rw + 255) / 256 * 256);
  *rw_out = (u32)rw;
  return (u32)((m + rw - 1) / rw);
}

__global__ void add_u32_kernel(const u32* a, const u32* b, u32* c) { *c = *a + *b; }

size_t compact_temp_bytes(u64 m) {
  u32 rw;
  const u64 nw = compact_warps(m, &rw);
  return ((nw * 8 + 255) / 256) * 256 + scan_u32_temp_bytes(nw) + 256;
}

u64* launch_compact_multi(const u64* keys, u32 m, const KeyLayout& L, u64* seg, u64* out, void* temp, u32* total,
                          cudaStream_t st) {
  if (!m) return out;
  u32 rw;
  const u32 nw = compact_warps(m, &rw);
  u32* cnt = reinterpret_cast<u32*>(temp);
  u32* off = cnt + nw;
  void* stemp = reinterpret_cast<char*>(temp) + (((u64)nw * 8 + 255) / 256) * 256;
  const u32 grid = (nw + 7) / 8;
  const u32 sh_shared = L.pos_bits, sh_global = L.pos_bits + L.lowG;
  const u32 sh_fixed = L.single_space == SP_GLOBAL ? sh_global : sh_shared;
  if (!L.both && L.sort_bits + L.pos_bits - sh_fixed <= 32) {
    RunKey<true> R;
    R.sh32 = sh_fixed;
    compact_seg_kernel<12, true><<<grid, 256, 0, st>>>(keys, m, R, rw, seg, cnt);
  } else {
    RunKey<false> R;
    R.both = L.both != 0;
    R.sbit = L.space_shift + L.pos_bits;
    R.mask_s = ~((sh_shared >= 64) ? ~0ull : ((1ull << sh_shared) - 1ull));
    R.mask_g = ~((sh_global >= 64) ? ~0ull : ((1ull << sh_global) - 1ull));
    R.mask_fixed = L.single_space == SP_GLOBAL ? R.mask_g : R.mask_s;
    compact_seg_kernel<8, false><<<grid, 256, 0, st>>>(keys, m, R, rw, seg, cnt);
  }
  launch_scan_exclusive_u32(cnt, off, nw, stemp, st);
  compact_gather_kernel<<<grid, 256, 0, st>>>(seg, rw, nw, cnt, off, out);
  add_u32_kernel<<<1, 1, 0, st>>>(off + nw - 1, cnt + nw - 1, total);
  return out;
}

}  // namespace sesa
