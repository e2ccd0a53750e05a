// k_util.cu — single-pass exclusive scan of u32 counts (decoupled look-back), used for entry offsets of
// multi-granule records and for flow-expansion offsets.  Offsets are u32: callers guarantee totals < 2^32.
#include <algorithm>
#include <map>
#include <mutex>
#include <tuple>

#include "kernels.cuh"

namespace sesa {

// ---- per-device launch properties ----------------------------------------------------------------------------
// The dynamic shared-memory opt-in of a kernel is stored per device context, and SM counts / occupancy are
// properties of the device: cache them per (kernel, device) under a lock, so that handles on several devices
// of one process (and host threads making their first call at the same time) each get a valid configuration.
static std::mutex g_props_mu;

static int current_device() {
  int dev = 0;
  cudaGetDevice(&dev);
  return dev;
}

int dev_sm_count() {
  static std::map<int, int> sms;
  const int dev = current_device();
  std::lock_guard<std::mutex> lk(g_props_mu);
  auto it = sms.find(dev);
  if (it != sms.end()) return it->second;
  int v = 0;
  if (cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || v <= 0) {
    cudaGetLastError();
    v = 148;
  }
  sms[dev] = v;
  return v;
}

static void smem_optin_locked(const void* kern, size_t bytes, int dev) {
  static std::map<std::pair<const void*, int>, size_t> done;
  auto it = done.find(std::make_pair(kern, dev));
  if (it != done.end() && it->second >= bytes) return;  // never lowered
  if (cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes) != cudaSuccess) {
    cudaGetLastError();  // the launch reports the error
    return;
  }
  done[std::make_pair(kern, dev)] = bytes;
}

void smem_optin(const void* kern, size_t bytes) {
  const int dev = current_device();
  std::lock_guard<std::mutex> lk(g_props_mu);
  smem_optin_locked(kern, bytes, dev);
}

int blocks_per_sm(const void* kern, int threads, size_t smem) {
  static std::map<std::tuple<const void*, int, int, size_t>, int> occ;
  const int dev = current_device();
  std::lock_guard<std::mutex> lk(g_props_mu);
  const auto key = std::make_tuple(kern, dev, threads, smem);
  auto it = occ.find(key);
  if (it != occ.end()) return it->second;
  smem_optin_locked(kern, smem, dev);
  int per = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, threads, smem) != cudaSuccess || per <= 0) {
    cudaGetLastError();
    per = 1;
  }
  occ[key] = per;
  return per;
}

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
