// k_compact.cu — ordered stream compaction of the sorted keys down to entries whose location is touched by
// at least two entries ("compaction").  A location touched once cannot race (P:43 needs two
// accesses), so singletons — all but ~2e5 of C5's 1e9 entries — never reach the conflict tiles.  Single pass:
// tiles of 2048 keys in acquisition order, block scan of per-thread counts, decoupled look-back for the global
// offset, output staged through shared memory so the writes are coalesced.  Order (and therefore location runs
// and their (block, interval) sub-runs) is preserved.
#include "kernels.cuh"

namespace sesa {

constexpr int CP_THREADS = 256, CP_ITEMS = 8, CP_TILE = CP_THREADS * CP_ITEMS;

__global__ void __launch_bounds__(CP_THREADS) compact_multi_kernel(const u64* __restrict__ keys, u32 m, KeyLayout L,
                                                                   u64* __restrict__ out, u64* __restrict__ lb,
                                                                   u32* __restrict__ ctr, u32* __restrict__ total) {
  __shared__ u64 sk[CP_TILE + 2];
  __shared__ u64 so[CP_TILE];
  __shared__ u32 s_tile, s_w[CP_THREADS / 32];
  __shared__ u64 s_base;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_tile = atomicAdd(ctr, 1u);
  __syncthreads();
  const u32 tile = s_tile;
  const u64 tb = (u64)tile * CP_TILE;
  const u32 cnt = (u32)min((u64)CP_TILE, (u64)m - tb);
#pragma unroll
  for (int q = 0; q < CP_ITEMS; q++) {  // compile-time trip count: all 8 loads in flight
    const u32 j = q * CP_THREADS + tid;
    if (j < cnt) sk[j + 1] = __ldcs(keys + tb + j);
  }
  if (tid == 0) {
    sk[0] = tb > 0 ? keys[tb - 1] : 0ull;
    sk[cnt + 1] = tb + cnt < m ? keys[tb + cnt] : 0ull;
  }
  __syncthreads();
  u32 flags = 0, c = 0;
#pragma unroll
  for (int q = 0; q < CP_ITEMS; q++) {
    const u32 j = tid * CP_ITEMS + q;
    if (j < cnt) {
      const u64 g = group_of_hi(L, sk[j + 1] >> L.pos_bits);
      const bool sp = (tb + j > 0) && group_of_hi(L, sk[j] >> L.pos_bits) == g;
      const bool sn = (tb + j + 1 < m) && group_of_hi(L, sk[j + 2] >> L.pos_bits) == g;
      if (sp || sn) flags |= 1u << q, c++;
    }
  }
  // block exclusive scan of per-thread counts
  u32 x = c;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const u32 y = __shfl_up_sync(~0u, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[warp] = x;
  __syncthreads();
  if (warp == 0) {
    u32 acc = 0;
    if (lane == 0) {
      for (int w = 0; w < CP_THREADS / 32; w++) {
        const u32 t = s_w[w];
        s_w[w] = acc;
        acc += t;
      }
    }
    acc = __shfl_sync(~0u, acc, 0);
    const u64 ex = warp_lookback(lb, tile, acc);
    if (lane == 0) {
      s_base = ex;
      if (tb + cnt >= m) *total = (u32)(ex + acc);  // the last tile publishes the count
    }
  }
  __syncthreads();
  u32 o = s_w[warp] + x - c;
#pragma unroll
  for (int q = 0; q < CP_ITEMS; q++)
    if (flags & (1u << q)) so[o++] = sk[tid * CP_ITEMS + q + 1];
  __syncthreads();
  // the tile's compacted count = exclusive offset of the (virtual) thread after the last one
  __shared__ u32 s_cnt;
  if (tid == CP_THREADS - 1) s_cnt = o;
  __syncthreads();
  const u64 base = s_base;
  for (u32 j = tid; j < s_cnt; j += CP_THREADS) out[base + j] = so[j];
}

size_t compact_temp_bytes(u64 m) { return ((m + CP_TILE - 1) / CP_TILE + 1) * 8 + 64; }

void launch_compact_multi(const u64* keys, u32 m, const KeyLayout& L, u64* out, void* temp, u32* total,
                          cudaStream_t st) {
  if (!m) return;
  const u32 tiles = (m + CP_TILE - 1) / CP_TILE;
  u32* ctr = reinterpret_cast<u32*>(temp);
  u64* lb = reinterpret_cast<u64*>(reinterpret_cast<char*>(temp) + 64);
  cudaMemsetAsync(temp, 0, compact_temp_bytes(m), st);
  compact_multi_kernel<<<tiles, CP_THREADS, 0, st>>>(keys, m, L, out, lb, ctr, total);
}

}  // namespace sesa
