// k_util.cu — single-pass exclusive scan of u32 counts (decoupled look-back), used for entry offsets of
// multi-granule records and for flow-expansion offsets.  Offsets are u32: callers guarantee totals < 2^32.
#include "kernels.cuh"

namespace sesa {

constexpr int SCAN_THREADS = 256, SCAN_ITEMS = 16, SCAN_TILE = SCAN_THREADS * SCAN_ITEMS;

__global__ void __launch_bounds__(SCAN_THREADS) scan_u32_kernel(const u32* __restrict__ in, u32* __restrict__ out,
                                                                u64 n, u64* __restrict__ lb, u32* __restrict__ ctr) {
  __shared__ u32 s_tile, s_w[SCAN_THREADS / 32];
  __shared__ u64 s_prefix;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) s_tile = atomicAdd(ctr, 1u);
  __syncthreads();
  const u32 tile = s_tile;
  const u64 base = (u64)tile * SCAN_TILE + (u64)tid * SCAN_ITEMS;
  u32 v[SCAN_ITEMS], sum = 0;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; i++) {
    v[i] = base + i < n ? in[base + i] : 0u;
    sum += v[i];
  }
  u32 x = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    u32 y = __shfl_up_sync(~0u, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) s_w[warp] = x;
  __syncthreads();
  if (warp == 0) {
    u32 acc = 0;
    if (lane == 0) {
      for (int w = 0; w < SCAN_THREADS / 32; w++) {
        u32 c = s_w[w];
        s_w[w] = acc;
        acc += c;
      }
    }
    acc = __shfl_sync(~0u, acc, 0);
    const u64 ex = warp_lookback(lb, tile, acc);
    if (lane == 0) s_prefix = ex;
  }
  __syncthreads();
  u32 run = (u32)s_prefix + s_w[warp] + x - sum;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; i++) {
    if (base + i < n) out[base + i] = run;
    run += v[i];
  }
}

size_t scan_u32_temp_bytes(u64 n) { return ((n + SCAN_TILE - 1) / SCAN_TILE + 1) * 8 + 64; }

void launch_scan_exclusive_u32(const u32* in, u32* out, u64 n, void* temp, cudaStream_t st) {
  if (!n) return;
  const u64 tiles = (n + SCAN_TILE - 1) / SCAN_TILE;
  u32* ctr = reinterpret_cast<u32*>(temp);
  u64* lb = reinterpret_cast<u64*>(reinterpret_cast<char*>(temp) + 64);
  cudaMemsetAsync(temp, 0, scan_u32_temp_bytes(n), st);
  scan_u32_kernel<<<(unsigned)tiles, SCAN_THREADS, 0, st>>>(in, out, n, lb, ctr);
}

}  // namespace sesa
