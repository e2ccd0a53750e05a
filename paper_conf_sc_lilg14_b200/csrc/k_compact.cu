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

template <bool WRITE>
__global__ void __launch_bounds__(CP_THREADS) compact_kernel(const u64* __restrict__ keys, u32 m, KeyLayout L,
                                                             u32* __restrict__ chunk_cnt,
                                                             const u32* __restrict__ chunk_off, u64* __restrict__ out) {
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ u64 bars[CP_STAGES];
  __shared__ u32 s_w[CP_THREADS / 32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
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
      k[r] = t < nk ? K[t] : 0ull;
    }
    // neighbours of the warp's first / last key: inside the chunk from shared memory, else from global
    const u64 before = w0 > 0 ? K[w0 - 1] : (base > 0 ? keys[base - 1] : 0ull);
    const u32 wend = w0 + 32 * CP_ROWS;
    const u64 after = wend < nk ? K[wend] : (base + wend < m ? keys[base + wend] : 0ull);
    u32 cnt = 0, slot = 0;
    if (WRITE) {  // this warp's output offset: chunk offset + counts of the chunk's earlier warps
      slot = chunk_off[c];
    }
    unsigned ball[CP_ROWS];
#pragma unroll
    for (int r = 0; r < CP_ROWS; r++) {
      const u64 i = base + w0 + r * 32 + lane;
      const u64 up = __shfl_up_sync(~0u, k[r], 1), dn = __shfl_down_sync(~0u, k[r], 1);
      const u64 pl = __shfl_sync(~0u, r > 0 ? k[r > 0 ? r - 1 : 0] : before, 31);
      const u64 nf = __shfl_sync(~0u, r + 1 < CP_ROWS ? k[r + 1 < CP_ROWS ? r + 1 : r] : after, 0);
      const u64 prev = lane > 0 ? up : (r > 0 ? pl : before);
      const u64 next = lane < 31 ? dn : (r + 1 < CP_ROWS ? nf : after);
      const bool valid = i < m;
      const bool sp = valid && i > 0 && same_group(L, k[r], prev);
      const bool sn = valid && i + 1 < m && same_group(L, k[r], next);
      ball[r] = __ballot_sync(~0u, sp || sn);
      cnt += __popc(ball[r]);
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
      for (int w = 0; w < warp; w++) slot += s_w[w];
#pragma unroll
      for (int r = 0; r < CP_ROWS; r++) {
        if (ball[r] & (1u << lane)) out[slot + __popc(ball[r] & lanemask_lt())] = k[r];
        slot += __popc(ball[r]);
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
