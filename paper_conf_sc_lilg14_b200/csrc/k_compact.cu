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
                                                          u64* __restrict__ seg, u32* __restrict__ wcnt, u32 wb) {
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
      if ((keep >> lane) & 1u) seg[out + __popc(keep & lt)] = key >> wb;  // (wb: strip the write bit)
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

// ------------------------------------------------------------------------------------------------------------
// The same with the write bit (KeyLayout::wbit, the key's bit 0): a location whose entries all read cannot race
// (one of the two accesses writes), so its run is dropped as well, and kept keys are written without the
// bit (key >> 1: the plain layout).  Per row of 32 keys (warp-uniform masks: S = same run as the predecessor,
// W = writes) each lane forms the OR of W over its run: forward from the run's head (F, carried over rows) and
// backward to the run's end (B, carried from the next row).  What a warp cannot see — a run continuing into the
// previous or next warp range, or past the batch of U rows held in registers — counts as "has a write": such
// runs are kept, which is always safe (the conflict stage finds nothing in a read-only run).  The last row of a
// batch is finalised with the next batch, like above, once that batch's backward pass is known.
// ------------------------------------------------------------------------------------------------------------
#ifndef COMPACT_W_U
#define COMPACT_W_U 8
#endif
#ifndef COMPACT_W_MINB
#define COMPACT_W_MINB 4
#endif

template <int U, bool G32>
__global__ void __launch_bounds__(256, COMPACT_W_MINB) compact_seg_w_kernel(const u64* __restrict__ keys, u32 m, RunKey<G32> R,
                                                            u32 rw, u64* __restrict__ seg, u32* __restrict__ wcnt) {
  const int lane = threadIdx.x & 31;
  const u32 w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const u64 start64 = (u64)w * rw;
  if (start64 >= m) return;
  const u32 start = (u32)start64, end = (u32)min((u64)m, start64 + rw);
  using G = decltype(R.of(0ull));
  G prevg;
  unsigned succ;
  unsigned fcar;  // forward OR of the run holding the previous key (1 = unknown: it started in another range)
  {
    const G g0 = R.of(keys[start]), gl = R.of(keys[end - 1]);
    prevg = start > 0 ? R.of(keys[start - 1]) : (G)(g0 ^ (G)1);
    succ = end < m ? (R.of(keys[end]) == gl ? 1u : 0u) : 0u;
    fcar = prevg == g0 ? 1u : 0u;
  }
  const unsigned lt = lanemask_lt(), le = lt | (1u << lane), ge = ~lt, gt = ~le;
  u32 out = start;
  auto write = [&](u64 key, unsigned keep) {
    if (keep) {  // warp-uniform
      if ((keep >> lane) & 1u) seg[out + __popc(keep & lt)] = key >> 1;
      out += __popc(keep);
    }
  };
  // lane's forward OR: W over [its run's head in this row, lane], or over [0, lane] plus the carry if the run
  // began in an earlier row.  Branch-free: hb = the highest head at or below the lane (0: none).
  auto fwd = [&](unsigned S, unsigned Wm, unsigned carry) -> bool {
    const unsigned hl = ~S & le;
    const unsigned hb = hl ? (0x80000000u >> __clz(hl)) : 0u;
    const unsigned rng = hb ? (le & ~(hb - 1u)) : le;
    return ((Wm & rng) != 0u) | ((hb == 0u) & (carry != 0u));
  };
  // lane's backward OR: W over [lane, the lane before the next head in this row], or to lane 31 plus the carry
  auto bwd = [&](unsigned S, unsigned Wm, unsigned V, unsigned carry) -> bool {
    const unsigned hn = ~S & V & gt;
    const unsigned ln = hn & (0u - hn);  // the next head (lowest set bit; 0: none)
    const unsigned rng = ln ? (ge & (ln - 1u)) : ge;
    return ((Wm & rng) != 0u) | ((ln == 0u) & (carry != 0u));
  };
  u64 pk = 0;  // pending last row of the previous batch: key, S, W, F masks
  unsigned psp = 0, pwm = 0, pfm = 0;
  bool pending = false;
  for (u32 r0 = start; r0 < end; r0 += 32 * U) {
    u64 k[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 i = r0 + u * 32 + lane;
      k[u] = i < end ? __ldcs(keys + i) : 0ull;
    }
    unsigned sp[U], wm[U], kp[U];
#pragma unroll
    for (int u = 0; u < U; u++) {
      const u32 i = r0 + u * 32 + lane;
      const G g = R.of(k[u]);
      const G up = __shfl_up_sync(~0u, g, 1);
      const G p = lane ? up : prevg;
      sp[u] = __ballot_sync(~0u, i < end && p == g);
      wm[u] = __ballot_sync(~0u, i < end && (k[u] & 1ull));
      prevg = __shfl_sync(~0u, g, 31);
      // F masks (kp reused for the keep masks below)
      kp[u] = __ballot_sync(~0u, fwd(sp[u], wm[u], fcar));
      fcar = kp[u] >> 31;
    }
    const unsigned fl = kp[U - 1];  // F mask of the batch's last row (it may become the pending row)
    // candidates (touched >= 2 times) per row; a candidate whose run has a write at or before it (F) is kept
    // without the backward pass: only if some candidate lacks F does the batch run it (C3: rarely; C4: mostly)
    auto cand_of = [&](int u) -> unsigned {
      const u32 rb = r0 + u * 32;
      if (rb >= end) return 0u;
      const bool last = rb + 32 >= end;
      const unsigned nxt = last ? (succ << (end - 1 - rb)) : (u + 1 < U ? (sp[u + 1 < U ? u + 1 : u] & 1u) << 31 : 0u);
      return sp[u] | (sp[u] >> 1) | nxt;
    };
    const unsigned pcand = psp | (psp >> 1) | ((sp[0] & 1u) << 31);
    const bool np = r0 + (U - 1) * 32 < end && r0 + U * 32 < end;  // the batch's last row waits for the next
    unsigned need = pending ? (pcand & ~pfm) : 0u;
#pragma unroll
    for (int u = 0; u < U; u++)
      if (!(np && u == U - 1)) need |= cand_of(u) & ~kp[u];
    unsigned bnext = 0u;  // B carry into the row from the right (1 = unknown: the next batch)
    if (need) {
      bnext = 1u;
      // backward: keep masks, last row first
#pragma unroll
      for (int u = U - 1; u >= 0; u--) {
        const u32 rb = r0 + u * 32;
        if (rb >= end) {  // empty row
          kp[u] = 0;
          bnext = 0;
          continue;
        }
        const bool last = rb + 32 >= end;  // holds the range's last key
        const unsigned V = (last && end - rb < 32) ? ((1u << (end - rb)) - 1u) : ~0u;
        const unsigned car = last ? succ : bnext;
        // (the lanes past the range's end are no heads: the last run's carry is succ)
        const unsigned bm = __ballot_sync(~0u, bwd(sp[u], wm[u], V, car));
        kp[u] = cand_of(u) & (kp[u] | bm);
        bnext = sp[u] & bm & 1u;
      }
    } else {
#pragma unroll
      for (int u = 0; u < U; u++) kp[u] = cand_of(u);
    }
    if (pending) {  // the previous batch's last row: its run's backward carry is this batch's row-0 carry
      unsigned bm = 0u;
      if (pcand & ~pfm) bm = __ballot_sync(~0u, bwd(psp, pwm, ~0u, bnext));
      write(pk, pcand & (pfm | bm));
    }
#pragma unroll
    for (int u = 0; u < U; u++)
      if (!(np && u == U - 1)) write(k[u], kp[u]);
    pending = np;
    if (np) pk = k[U - 1], psp = sp[U - 1], pwm = wm[U - 1], pfm = fl;
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

// Is the write-bit filter worth its cost?  A warp per sampled row of 32 sorted keys counts the candidates
// (entries whose run, as far as the row shows, holds >= 2 entries) and those of them in runs that lie wholly in
// the row and hold no write — what the filter would drop there.  cnt[0] += candidates, cnt[1] += droppable.
template <bool G32>
__global__ void wbit_sample_kernel(const u64* __restrict__ keys, u32 m, RunKey<G32> R, u32 nsamp,
                                   unsigned long long* __restrict__ cnt) {
  const int lane = threadIdx.x & 31;
  const u32 s = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const u32 rows = m / 32;
  if (s >= nsamp || rows == 0) return;
  const u32 i = (u32)(((u64)s * rows / nsamp) * 32) + lane;
  const u64 k = keys[i];
  const auto g = R.of(k);
  const auto up = __shfl_up_sync(~0u, g, 1);
  const unsigned sp = __ballot_sync(~0u, lane > 0 && up == g), wm = __ballot_sync(~0u, (k & 1ull) != 0ull);
  const unsigned cand = sp | (sp >> 1);
  const unsigned lt = lanemask_lt(), le = lt | (1u << lane), gt = ~le;
  const unsigned hl = ~sp & le, hn = ~sp & gt;  // (lane 0 is a head: hl != 0)
  const unsigned hb = 0x80000000u >> __clz(hl), ln = hn & (0u - hn);
  const unsigned run = (hn ? (ln - 1u) : 0u) & ~(hb - 1u);  // the lane's run if it ends inside the row
  // (a run starting at lane 0 may have begun in the previous row: not counted)
  const bool drop = ((cand >> lane) & 1u) && hb != 1u && hn != 0u && (wm & run) == 0u;
  const unsigned dm = __ballot_sync(~0u, drop);
  if (lane == 0) {
    atomicAdd(&cnt[0], (unsigned long long)__popc(cand));
    atomicAdd(&cnt[1], (unsigned long long)__popc(dm));
  }
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

// host: sample (one sync) whether the write-bit filter pays on these sorted keys (L.wbit set)
bool compact_filter_pays(const u64* keys, u32 m, const KeyLayout& L, void* temp, cudaStream_t st) {
  if (!L.wbit || m < 32 * 4096) return L.wbit != 0;
  const u32 sh_shared = L.pos_bits, sh_global = L.pos_bits + L.lowG;
  const u32 sh_fixed = L.single_space == SP_GLOBAL ? sh_global : sh_shared;
  unsigned long long* c = reinterpret_cast<unsigned long long*>(temp);
  cudaMemsetAsync(c, 0, 16, st);
  const u32 nsamp = 16384;
  if (!L.both && L.sort_bits + L.pos_bits - sh_fixed <= 32) {
    RunKey<true> R;
    R.sh32 = sh_fixed + 1;
    wbit_sample_kernel<true><<<nsamp / 8, 256, 0, st>>>(keys, m, R, nsamp, c);
  } else {
    RunKey<false> R;
    R.both = L.both != 0;
    R.sbit = L.space_shift + L.pos_bits + 1;
    R.mask_s = ~((1ull << (sh_shared + 1)) - 1ull);
    R.mask_g = ~((sh_global + 1 >= 64) ? ~0ull : ((1ull << (sh_global + 1)) - 1ull));
    R.mask_fixed = L.single_space == SP_GLOBAL ? R.mask_g : R.mask_s;
    wbit_sample_kernel<false><<<nsamp / 8, 256, 0, st>>>(keys, m, R, nsamp, c);
  }
  unsigned long long h[2] = {0, 0};
  if (cudaMemcpyAsync(h, c, 16, cudaMemcpyDeviceToHost, st) != cudaSuccess || cudaStreamSynchronize(st) != cudaSuccess)
    return true;  // (the error resurfaces at the next sync; the filter is always correct)
  // the filter kernel costs ~0.3 ns per key more than the plain one and saves a ~25 ns record gather per dropped
  // entry in the conflict stage: worth it from ~2% droppable candidates
  return (double)h[1] > 0.02 * (double)h[0];
}

u64* launch_compact_multi(const u64* keys, u32 m, const KeyLayout& L, u64* seg, u64* out, void* temp, u32* total,
                          cudaStream_t st, bool filter) {
  if (!m) return out;
  u32 rw;
  const u32 nw = compact_warps(m, &rw);
  u32* cnt = reinterpret_cast<u32*>(temp);
  u32* off = cnt + nw;
  void* stemp = reinterpret_cast<char*>(temp) + (((u64)nw * 8 + 255) / 256) * 256;
  const u32 grid = (nw + 7) / 8;
  const u32 sh_shared = L.pos_bits, sh_global = L.pos_bits + L.lowG;
  const u32 sh_fixed = L.single_space == SP_GLOBAL ? sh_global : sh_shared;
  const u32 wb = L.wbit ? 1u : 0u;  // the write bit below the position: every shift moves up by one
  filter = filter && wb;             // (else the plain kernel strips the bit)
  if (!L.both && L.sort_bits + L.pos_bits - sh_fixed <= 32) {
    RunKey<true> R;
    R.sh32 = sh_fixed + wb;
    if (filter) compact_seg_w_kernel<COMPACT_W_U, true><<<grid, 256, 0, st>>>(keys, m, R, rw, seg, cnt);
    else compact_seg_kernel<12, true><<<grid, 256, 0, st>>>(keys, m, R, rw, seg, cnt, wb);
  } else {
    RunKey<false> R;
    R.both = L.both != 0;
    R.sbit = L.space_shift + L.pos_bits + wb;
    R.mask_s = ~((sh_shared + wb >= 64) ? ~0ull : ((1ull << (sh_shared + wb)) - 1ull));
    R.mask_g = ~((sh_global + wb >= 64) ? ~0ull : ((1ull << (sh_global + wb)) - 1ull));
    R.mask_fixed = L.single_space == SP_GLOBAL ? R.mask_g : R.mask_s;
    if (filter) compact_seg_w_kernel<COMPACT_W_U, false><<<grid, 256, 0, st>>>(keys, m, R, rw, seg, cnt);
    else compact_seg_kernel<8, false><<<grid, 256, 0, st>>>(keys, m, R, rw, seg, cnt, wb);
  }
  launch_scan_exclusive_u32(cnt, off, nw, stemp, st);
  compact_gather_kernel<<<grid, 256, 0, st>>>(seg, rw, nw, cnt, off, out);
  add_u32_kernel<<<1, 1, 0, st>>>(off + nw - 1, cnt + nw - 1, total);
  return out;
}

}  // namespace sesa
