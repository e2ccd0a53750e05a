// k_extract.cu — record validation + extents and key extraction with upfront digit
// histograms (row a2).  Both are HBM-streaming passes over the 32-byte records: one 32-byte sector per record,
// read with two 16-byte vector loads, grid sized to a multiple of the 148 SMs.
#include <algorithm>
#include <cstdlib>

#include "kernels.cuh"

namespace sesa {

// ------------------------------------------------------------------------------------------------------------
// extents: per record check validity (include/sesa.h: space <= 1, rw <= 2, size >= 1, addr + size - 1 does not
// wrap — the bounds P:73 and the memory sorts of Fig. 3), and reduce per space: min/max granule,
// block, interval; count entries (granules) and multi-granule records; detect (block, interval) order.
// ------------------------------------------------------------------------------------------------------------
constexpr int EX_STAGES = 4, EX_CHUNK = 16384, EX_RECS = EX_CHUNK / 32;

// Register version (measured faster than a TMA ring here: the per-record reductions are ALU-heavy and the ring's
// strided shared-memory reads and barriers cost more than they save).  Scalar accumulators per space (arrays
// indexed by the record's space spilled to local memory), warp votes only in convergent code, and a warp-uniform
// single-space fast path (traces are mostly single-space).
struct SpaceAcc {
  u64 cnt, gmin, gmax;
  u32 bmin, bmax, imin, imax;
  __device__ __forceinline__ void init() { cnt = 0, gmin = ~0ull, gmax = 0, bmin = ~0u, bmax = 0, imin = ~0u, imax = 0; }
  __device__ __forceinline__ void add(u64 glo, u64 ghi, u32 b, u32 i) {
    cnt++;
    gmin = min(gmin, glo), gmax = max(gmax, ghi);
    bmin = min(bmin, b), bmax = max(bmax, b);
    imin = min(imin, i), imax = max(imax, i);
  }
  __device__ __forceinline__ void warp_reduce() {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      cnt += __shfl_xor_sync(~0u, cnt, o);
      gmin = min(gmin, __shfl_xor_sync(~0u, gmin, o));
      gmax = max(gmax, __shfl_xor_sync(~0u, gmax, o));
      bmin = min(bmin, __shfl_xor_sync(~0u, bmin, o));
      bmax = max(bmax, __shfl_xor_sync(~0u, bmax, o));
      imin = min(imin, __shfl_xor_sync(~0u, imin, o));
      imax = max(imax, __shfl_xor_sync(~0u, imax, o));
    }
  }
};

template <int THREADS, int U, int MINB>
__global__ void __launch_bounds__(THREADS, MINB) extents_kernel(const Rec* __restrict__ rec, u64 n, u32 log2G,
                                                          Summary* __restrict__ out) {
  u64 bad = ~0ull, ent = 0, multi = 0;
  SpaceAcc A0, A1;  // shared, global
  A0.init();
  A1.init();
  u32 unsorted = 0;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const u64 stride = (u64)gridDim.x * THREADS, gt = (u64)blockIdx.x * THREADS + threadIdx.x;
  const u64 rounds = (n + stride * U - 1) / (stride * U);
  for (u64 it = 0; it < rounds; it++) {
    Rec r[U];
#pragma unroll
    for (int j = 0; j < U; j++) {  // U independent 32-byte loads in flight per thread
      const u64 k = (it * U + j) * stride + gt;
      if (k < n) r[j] = load_rec(rec + k);
    }
#pragma unroll
    for (int j = 0; j < U; j++) {
      const u64 k = (it * U + j) * stride + gt;
      const bool in = k < n;
      // (block, interval) of record k-1: held by the previous lane, or loaded for lane 0 (convergent shuffles)
      u32 pb = __shfl_up_sync(~0u, in ? r[j].block : 0u, 1), pi = __shfl_up_sync(~0u, in ? r[j].interval : 0u, 1);
      if (lane == 0 && in && k > 0) {
        const uint4 q = __ldg(reinterpret_cast<const uint4*>(rec + k - 1) + 1);
        pb = q.x, pi = q.z;
      }
      const Rec& x = r[j];
      const bool ok = in && x.space <= 1 && x.rw <= 2 && x.size >= 1 && x.addr <= ~0ull - (u64)(x.size - 1);
      if (in && !ok) bad = min(bad, k);
      const u64 glo = x.addr >> log2G, ghi = (x.addr + (u64)(x.size - 1)) >> log2G;
      if (ok) {
        if (k > 0 && (x.block < pb || (x.block == pb && x.interval < pi))) unsorted = 1;
        ent += ghi - glo + 1;
        multi += ghi != glo;
      }
      const bool all_glob = __all_sync(~0u, !ok || x.space == SP_GLOBAL);
      if (all_glob) {
        if (ok) A1.add(glo, ghi, x.block, x.interval);
      } else if (__all_sync(~0u, !ok || x.space == SP_SHARED)) {
        if (ok) A0.add(glo, ghi, x.block, x.interval);
      } else if (ok) {
        if (x.space == SP_GLOBAL) A1.add(glo, ghi, x.block, x.interval);
        else A0.add(glo, ghi, x.block, x.interval);
      }
    }
  }
  // block reduction through warp shuffles then one atomic per field per CTA
  __shared__ SpaceAcc sa[THREADS / 32][2];
  __shared__ u64 s64[THREADS / 32][3];
  __shared__ u32 s_uns[THREADS / 32];
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    bad = min(bad, __shfl_xor_sync(~0u, bad, o));
    ent += __shfl_xor_sync(~0u, ent, o);
    multi += __shfl_xor_sync(~0u, multi, o);
    unsorted |= __shfl_xor_sync(~0u, unsorted, o);
  }
  A0.warp_reduce();
  A1.warp_reduce();
  if (lane == 0) {
    s64[warp][0] = bad, s64[warp][1] = ent, s64[warp][2] = multi;
    sa[warp][0] = A0, sa[warp][1] = A1;
    s_uns[warp] = unsorted;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < THREADS / 32; w++) {
      s64[0][0] = min(s64[0][0], s64[w][0]);
      s64[0][1] += s64[w][1];
      s64[0][2] += s64[w][2];
      s_uns[0] |= s_uns[w];
      for (int sp = 0; sp < 2; sp++) {
        SpaceAcc& d = sa[0][sp];
        const SpaceAcc& e = sa[w][sp];
        d.cnt += e.cnt;
        d.gmin = min(d.gmin, e.gmin), d.gmax = max(d.gmax, e.gmax);
        d.bmin = min(d.bmin, e.bmin), d.bmax = max(d.bmax, e.bmax);
        d.imin = min(d.imin, e.imin), d.imax = max(d.imax, e.imax);
      }
    }
    if (s64[0][0] != ~0ull) atomicMin(&out->bad_index, (unsigned long long)s64[0][0]);
    if (s64[0][1]) atomicAdd(&out->entries, (unsigned long long)s64[0][1]);
    if (s64[0][2]) atomicAdd(&out->multi, (unsigned long long)s64[0][2]);
    for (int sp = 0; sp < 2; sp++) {
      const SpaceAcc& d = sa[0][sp];
      if (!d.cnt) continue;
      atomicAdd(&out->count[sp], (unsigned long long)d.cnt);
      atomicMin(&out->gmin[sp], (unsigned long long)d.gmin);
      atomicMax(&out->gmax[sp], (unsigned long long)d.gmax);
      atomicMin(&out->bmin[sp], d.bmin);
      atomicMax(&out->bmax[sp], d.bmax);
      atomicMin(&out->imin[sp], d.imin);
      atomicMax(&out->imax[sp], d.imax);
    }
    if (s_uns[0]) atomicOr(&out->unsorted, 1u);
  }
}

static int ring_grid(const void* kern, int threads, size_t smem, size_t smem_max) {
  int dev = 0, sms = 148, per = 1;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_max);  // never lowered
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, threads, smem);
  return sms * (per > 0 ? per : 1);
}

void launch_extents(const Rec* rec, u64 n, u32 log2G, Summary* d_sum, int grid, cudaStream_t st) {
  static int v = -1;
  if (v < 0) {
    const char* e = getenv("SESA_EXT_CFG");
    v = e ? atoi(e) : 1;  // measured best on C5: U=4 records in flight, 64 registers, 4 CTAs/SM
  }
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const unsigned g = (unsigned)std::min<u64>((n + 255) / 256, (u64)sms * 8);
  switch (v) {
    case 1: extents_kernel<256, 4, 4><<<g, 256, 0, st>>>(rec, n, log2G, d_sum); break;
    case 2: extents_kernel<256, 8, 2><<<g, 256, 0, st>>>(rec, n, log2G, d_sum); break;
    case 3: extents_kernel<256, 2, 6><<<g, 256, 0, st>>>(rec, n, log2G, d_sum); break;
    case 4: extents_kernel<256, 8, 3><<<g, 256, 0, st>>>(rec, n, log2G, d_sum); break;
    default: extents_kernel<256, 4, 1><<<g, 256, 0, st>>>(rec, n, log2G, d_sum); break;
  }
  (void)grid;
}

// ------------------------------------------------------------------------------------------------------------
// key extraction, 1 entry per record (every record within one granule): key = key_hi << pos_bits | pos, plus
// the histogram of every radix digit the sort will use (onesweep's upfront histogram), accumulated per CTA in
// shared memory with warp-aggregated (ballot-matched) increments and flushed with one global atomic per bin.
// ------------------------------------------------------------------------------------------------------------
template <int THREADS, int RB>
__global__ void __launch_bounds__(THREADS) extract_1to1_kernel(const Rec* __restrict__ rec, u64 n, KeyLayout L,
                                                                u32 npass, u64* __restrict__ keys,
                                                                u32* __restrict__ hist /* [npass][1<<RB] */,
                                                                u64 pos_base) {
  constexpr int RADIX = 1 << RB;
  extern __shared__ __align__(128) unsigned char smem[];
  __shared__ u64 bars[EX_STAGES];
  u32* sh = reinterpret_cast<u32*>(smem + (size_t)EX_STAGES * EX_CHUNK);  // [warps][npass][RADIX]
  const u32 nsh = npass * RADIX * (THREADS / 32);
  for (u32 i = threadIdx.x; i < nsh; i += THREADS) sh[i] = 0;
  u32* wsh = sh + (threadIdx.x >> 5) * npass * RADIX;  // per-warp private sub-histograms: plain smem atomics
  BulkRing<EX_STAGES> ring(smem, bars, EX_CHUNK);
  ring.start(rec, n * 32);  // (contains __syncthreads)
  for (u64 j = 0; ring.next(j); j++) {
    const Rec* R = reinterpret_cast<const Rec*>(ring.wait(j));
    const u64 c0 = ring.chunk_index(j) * EX_RECS;
    const u32 nr = ring.chunk_bytes(j) / 32;
#pragma unroll
    for (int h = 0; h < EX_RECS / THREADS; h++) {
      const u32 t = h * THREADS + threadIdx.x;
      if (t >= nr) continue;
      const Rec& x = R[t];
      const u64 key = (key_hi_of(L, x.space, x.block, x.interval, x.addr >> L.log2G) << L.pos_bits) | (pos_base + c0 + t);
      __stcs(keys + c0 + t, key);
      for (u32 p = 0; p < npass; p++) atomicAdd(&wsh[p * RADIX + ((key >> (L.pos_bits + p * RB)) & (RADIX - 1))], 1u);
    }
    ring.release(j);
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS) {
    u32 v = 0;
    for (int w = 0; w < THREADS / 32; w++) v += sh[w * npass * RADIX + i];
    if (v) atomicAdd(&hist[i], v);
  }
}

void launch_extract_1to1(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, u64* keys, u32* hist, u64 pos_base,
                         int, cudaStream_t st) {
  static int grids[9] = {0};
  const size_t sm = (size_t)EX_STAGES * EX_CHUNK + (size_t)npass * 8 * RADIX * 4;  // ring + npass x 8 warps hist
  if (!grids[npass])
    grids[npass] = ring_grid((const void*)extract_1to1_kernel<256, RADIX_BITS>, 256, sm,
                             (size_t)EX_STAGES * EX_CHUNK + (size_t)8 * 8 * RADIX * 4);
  const int grid = grids[npass];
  const u64 chunks = (n * 32 + EX_CHUNK - 1) / EX_CHUNK;
  extract_1to1_kernel<256, RADIX_BITS><<<(unsigned)std::min<u64>(chunks, (u64)grid), 256, sm, st>>>(rec, n, L, npass,
                                                                                                   keys, hist, pos_base);
}

// ------------------------------------------------------------------------------------------------------------
// multi-granule path: entries per record = granules it covers (reading R1: byte ranges compared at granule G).
// count -> exclusive scan (offsets) -> expand.  Entry order = record order, then ascending granule.
// ------------------------------------------------------------------------------------------------------------
__global__ void entry_count_kernel(const Rec* __restrict__ rec, u64 n, u32 log2G, u32* __restrict__ cnt) {
  u64 k = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= n) return;
  Rec r = load_rec(rec + k);
  u64 glo = r.addr >> log2G, ghi = (r.addr + (u64)(r.size - 1)) >> log2G;
  cnt[k] = (u32)(ghi - glo + 1);
}

template <int THREADS, int RB>
__global__ void __launch_bounds__(THREADS) extract_multi_kernel(const Rec* __restrict__ rec, u64 n, KeyLayout L,
                                                                 u32 npass, const u32* __restrict__ off,
                                                                 u64* __restrict__ keys, u32* __restrict__ hist,
                                                                 u64 pos_base) {
  constexpr int RADIX = 1 << RB;
  extern __shared__ u32 sh[];
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS) sh[i] = 0;
  __syncthreads();
  const u64 stride = (u64)gridDim.x * THREADS;
  for (u64 k = (u64)blockIdx.x * THREADS + threadIdx.x; k < n; k += stride) {
    Rec r = load_rec(rec + k);
    u64 glo = r.addr >> L.log2G, ghi = (r.addr + (u64)(r.size - 1)) >> L.log2G;
    u64 o = off[k];
    for (u64 g = glo; g <= ghi; g++, o++) {
      u64 key = (key_hi_of(L, r.space, r.block, r.interval, g) << L.pos_bits) | (pos_base + k);
      keys[o] = key;
      for (u32 p = 0; p < npass; p++) atomicAdd(&sh[p * RADIX + ((key >> (L.pos_bits + p * RB)) & (RADIX - 1))], 1u);
    }
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS)
    if (sh[i]) atomicAdd(&hist[i], sh[i]);
}

void launch_entry_count(const Rec* rec, u64 n, u32 log2G, u32* cnt, cudaStream_t st) {
  entry_count_kernel<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(rec, n, log2G, cnt);
}

void launch_extract_multi(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, const u32* off, u64* keys,
                          u32* hist, u64 pos_base, int grid, cudaStream_t st) {
  size_t smem = (size_t)npass * (1 << RADIX_BITS) * sizeof(u32);
  extract_multi_kernel<256, RADIX_BITS><<<grid, 256, smem, st>>>(rec, n, L, npass, off, keys, hist, pos_base);
}

}  // namespace sesa
