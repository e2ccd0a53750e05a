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

// Keys stream through a 4-stage TMA ring of 16 KB chunks (2048 keys); warp w owns keys [256w, 256w + 256) of a
// chunk as 8 rows of 32 (conflict-free shared-memory reads); neighbours by shuffles, the chunk edges from global.
constexpr int CP_STAGES = 4, CP_CHUNK_BYTES = 16384, CP_CHUNK = CP_CHUNK_BYTES / 8, CP_THREADS = 256;
constexpr int CP_ROWS = CP_CHUNK / CP_THREADS;  // 8 rows per warp

// Per key one comparison with its predecessor (sp); "same as successor" is the next lane's sp (row ballot shifted
// by one, lane 31 takes bit 0 of the next row).  Keys outside [0, m) and the array edges use sentinel neighbours
// whose top bit differs, so no 64-bit bounds tests are needed in the inner loop.
template <bool WRITE>
__global__ void __launch_bounds__(CP_THREADS) compact_kernel(const u64* __restrict__ keys, u32 m, KeyLayout L,
                                                             u32* __restrict__ chunk_cnt,
                                                             const u32* __restrict__ chunk_off, u64* __restrict__ out) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ u64 bars[CP_STAGES];
  __shared__ u32 s_w[CP_THREADS / 32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  // run key shift: constant unless both spaces are present (then it depends on the key's space bit)
  const u32 sh_shared = L.pos_bits, sh_global = L.pos_bits + L.lowG;
  const u32 sh_fixed = L.both ? 0u : (L.single_space == SP_GLOBAL ? sh_global : sh_shared);
  const u32 sbit = L.space_shift + L.pos_bits;
  BulkRing<CP_STAGES> ring(smem, bars, CP_CHUNK_BYTES);
  ring.start(keys, (u64)m * 8);
  for (u64 j = 0; ring.next(j); j++) {
    const u64* K = reinterpret_cast<const u64*>(ring.wait(j));
    const u64 c = ring.chunk_index(j), base = c * CP_CHUNK;
    const u32 nk = ring.chunk_bytes(j) / 8;
    const u32 w0 = warp * 32 * CP_ROWS;
    u64 k[CP_ROWS];
#pragma unroll
    for (int r = 0; r < CP_ROWS; r++) {
      const u32 t = w0 + r * 32 + lane;
      // past the end: a sentinel that differs from every real key in the top bit (and from each other's groups:
      // those lanes are masked out of the ballots below anyway)
      k[r] = t < nk ? K[t] : ~0ull;
    }
    const u64 first_key = __shfl_sync(~0u, k[0], 0);
    u64 before = w0 > 0 ? K[w0 - 1] : (base > 0 ? keys[base - 1] : first_key ^ (1ull << 63));
    const u32 wend = w0 + 32 * CP_ROWS;
    const u64 last_key = __shfl_sync(~0u, k[CP_ROWS - 1], 31);
    const u64 after = wend < nk ? K[wend] : (base + wend < m ? keys[base + wend] : last_key ^ (1ull << 63));
    unsigned bsp[CP_ROWS], vm[CP_ROWS];  // ballot of "same group as predecessor" (valid lanes only)
#pragma unroll
    for (int r = 0; r < CP_ROWS; r++) {
      const u32 valid_rows = nk > w0 + r * 32 ? nk - (w0 + r * 32) : 0u;
      vm[r] = valid_rows >= 32 ? ~0u : ((1u << valid_rows) - 1u);
      const u64 up = __shfl_up_sync(~0u, k[r], 1);
      const u64 prev = lane > 0 ? up : before;
      const u32 sh = L.both ? ((k[r] >> sbit) & 1ull ? sh_global : sh_shared) : sh_fixed;
      bsp[r] = __ballot_sync(~0u, ((k[r] ^ prev) >> sh) == 0) & vm[r];
      before = __shfl_sync(~0u, k[r], 31);
    }
    // same as successor: bit (lane+1) of this row's sp ballot; lane 31 uses bit 0 of the next row (or `after`)
    const u32 sh_last = L.both ? ((last_key >> sbit) & 1ull ? sh_global : sh_shared) : sh_fixed;
    const bool last_sn = ((last_key ^ after) >> sh_last) == 0;
    u32 cnt = 0;
    unsigned keep[CP_ROWS];
#pragma unroll
    for (int r = 0; r < CP_ROWS; r++) {
      const unsigned nxt = r + 1 < CP_ROWS ? (bsp[r + 1 < CP_ROWS ? r + 1 : r] & 1u) : (last_sn ? 1u : 0u);
      const unsigned bsn = (bsp[r] >> 1) | (nxt << 31);
      keep[r] = (bsp[r] | bsn) & vm[r];
      cnt += __popc(keep[r]);
    }
    if (lane == 0) s_w[warp] = cnt;
    __syncthreads();
    if (!WRITE) {
      if (threadIdx.x == 0) {
        u32 t = 0;
        for (int w = 0; w < CP_THREADS / 32; w++) t += s_w[w];
        chunk_cnt[c] = t;
      }
    } else {
      u32 slot = chunk_off[c];
      for (int w = 0; w < warp; w++) slot += s_w[w];
#pragma unroll
      for (int r = 0; r < CP_ROWS; r++) {
        if (keep[r] & (1u << lane)) out[slot + __popc(keep[r] & lanemask_lt())] = k[r];
        slot += __popc(keep[r]);
      }
    }
    ring.release(j);  // (contains __syncthreads: s_w may be rewritten next chunk)
  }
}

__global__ void add_u32_kernel(const u32* a, const u32* b, u32* c) { *c = *a + *b; }

size_t compact_temp_bytes(u64 m) {
  const u64 n = (m + CP_CHUNK - 1) / CP_CHUNK;  // chunks
  return ((n * 8 + 255) / 256) * 256 + scan_u32_temp_bytes(n) + 256;
}

void launch_compact_multi(const u64* keys, u32 m, const KeyLayout& L, u64* out, void* temp, u32* total,
                          cudaStream_t st) {
  if (!m) return;
  const u32 n = (m + CP_CHUNK - 1) / CP_CHUNK;
  u32* cnt = reinterpret_cast<u32*>(temp);
  u32* off = cnt + n;
  void* stemp = reinterpret_cast<char*>(temp) + ((n * 8 + 255) / 256) * 256;
  static int grid = 0;
  const size_t sm = (size_t)CP_STAGES * CP_CHUNK_BYTES;
  if (!grid) {
    int dev = 0, sms = 148, per = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaFuncSetAttribute(compact_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaFuncSetAttribute(compact_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, compact_kernel<true>, CP_THREADS, sm);
    grid = sms * std::max(per, 1);
  }
  const u32 g = std::min<u32>((u32)grid, n);
  compact_kernel<false><<<g, CP_THREADS, sm, st>>>(keys, m, L, cnt, nullptr, nullptr);
  launch_scan_exclusive_u32(cnt, off, n, stemp, st);
  compact_kernel<true><<<g, CP_THREADS, sm, st>>>(keys, m, L, nullptr, off, out);
  add_u32_kernel<<<1, 1, 0, st>>>(off + n - 1, cnt + n - 1, total);  // total = off[last] + cnt[last]
}

}  // namespace sesa
