// k_extract.cu — record validation + extents and key extraction with upfront digit
// histograms (row a2).  Both are HBM-streaming passes over the 32-byte records: one 32-byte sector per record,
// read with two 16-byte vector loads, grid sized to a multiple of the 148 SMs.
#include "kernels.cuh"

namespace sesa {

// ------------------------------------------------------------------------------------------------------------
// extents: per record check validity (include/sesa.h: space <= 1, rw <= 2, size >= 1, addr + size - 1 does not
// wrap — the bounds P:73 and the memory sorts of Fig. 3), and reduce per space: min/max granule,
// block, interval; count entries (granules) and multi-granule records; detect (block, interval) order.
// ------------------------------------------------------------------------------------------------------------
template <int THREADS>
__global__ void __launch_bounds__(THREADS) extents_kernel(const Rec* __restrict__ rec, u64 n, u32 log2G,
                                                          Summary* __restrict__ out) {
  u64 bad = ~0ull, ent = 0, multi = 0, cnt[2] = {0, 0};
  u64 gmin[2] = {~0ull, ~0ull}, gmax[2] = {0, 0};
  u32 bmin[2] = {~0u, ~0u}, bmax[2] = {0, 0}, imin[2] = {~0u, ~0u}, imax[2] = {0, 0};
  u32 unsorted = 0;
  const u64 stride = (u64)gridDim.x * THREADS;
  for (u64 k = (u64)blockIdx.x * THREADS + threadIdx.x; k < n; k += stride) {
    Rec r = load_rec(rec + k);
    bool ok = r.space <= 1 && r.rw <= 2 && r.size >= 1 && r.addr <= ~0ull - (u64)(r.size - 1);
    if (!ok) {
      bad = bad < k ? bad : k;
      continue;
    }
    u64 glo = r.addr >> log2G, ghi = (r.addr + (u64)(r.size - 1)) >> log2G;
    ent += ghi - glo + 1;
    multi += ghi != glo;
    int s = r.space;
    cnt[s]++;
    gmin[s] = min(gmin[s], glo);
    gmax[s] = max(gmax[s], ghi);
    bmin[s] = min(bmin[s], r.block);
    bmax[s] = max(bmax[s], r.block);
    imin[s] = min(imin[s], r.interval);
    imax[s] = max(imax[s], r.interval);
    if (k > 0) {
      const uint4* q = reinterpret_cast<const uint4*>(rec + k - 1) + 1;  // (block, thread, interval, ...)
      uint4 p = __ldg(q);
      if (r.block < p.x || (r.block == p.x && r.interval < p.z)) unsorted = 1;
    }
  }
  // block reduction through warp shuffles then one atomic per field per CTA
  __shared__ u64 s64[THREADS / 32][9];
  __shared__ u32 s32[THREADS / 32][9];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    bad = min(bad, __shfl_xor_sync(~0u, bad, o));
    ent += __shfl_xor_sync(~0u, ent, o);
    multi += __shfl_xor_sync(~0u, multi, o);
#pragma unroll
    for (int s = 0; s < 2; s++) {
      cnt[s] += __shfl_xor_sync(~0u, cnt[s], o);
      gmin[s] = min(gmin[s], __shfl_xor_sync(~0u, gmin[s], o));
      gmax[s] = max(gmax[s], __shfl_xor_sync(~0u, gmax[s], o));
      bmin[s] = min(bmin[s], __shfl_xor_sync(~0u, bmin[s], o));
      bmax[s] = max(bmax[s], __shfl_xor_sync(~0u, bmax[s], o));
      imin[s] = min(imin[s], __shfl_xor_sync(~0u, imin[s], o));
      imax[s] = max(imax[s], __shfl_xor_sync(~0u, imax[s], o));
    }
    unsorted |= __shfl_xor_sync(~0u, unsorted, o);
  }
  if (lane == 0) {
    s64[warp][0] = bad; s64[warp][1] = ent; s64[warp][2] = multi;
    s64[warp][3] = cnt[0]; s64[warp][4] = cnt[1];
    s64[warp][5] = gmin[0]; s64[warp][6] = gmin[1]; s64[warp][7] = gmax[0]; s64[warp][8] = gmax[1];
    s32[warp][0] = bmin[0]; s32[warp][1] = bmin[1]; s32[warp][2] = bmax[0]; s32[warp][3] = bmax[1];
    s32[warp][4] = imin[0]; s32[warp][5] = imin[1]; s32[warp][6] = imax[0]; s32[warp][7] = imax[1];
    s32[warp][8] = unsorted;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (int w = 1; w < THREADS / 32; w++) {
      s64[0][0] = min(s64[0][0], s64[w][0]);
      s64[0][1] += s64[w][1]; s64[0][2] += s64[w][2]; s64[0][3] += s64[w][3]; s64[0][4] += s64[w][4];
      s64[0][5] = min(s64[0][5], s64[w][5]); s64[0][6] = min(s64[0][6], s64[w][6]);
      s64[0][7] = max(s64[0][7], s64[w][7]); s64[0][8] = max(s64[0][8], s64[w][8]);
      for (int q = 0; q < 8; q += 2) {
        bool isMin = q == 0 || q == 4;
        s32[0][q] = isMin ? min(s32[0][q], s32[w][q]) : max(s32[0][q], s32[w][q]);
        s32[0][q + 1] = isMin ? min(s32[0][q + 1], s32[w][q + 1]) : max(s32[0][q + 1], s32[w][q + 1]);
      }
      s32[0][8] |= s32[w][8];
    }
    if (s64[0][0] != ~0ull) atomicMin(&out->bad_index, (unsigned long long)s64[0][0]);
    if (s64[0][1]) atomicAdd(&out->entries, (unsigned long long)s64[0][1]);
    if (s64[0][2]) atomicAdd(&out->multi, (unsigned long long)s64[0][2]);
    for (int s = 0; s < 2; s++) {
      if (!s64[0][3 + s]) continue;
      atomicAdd(&out->count[s], (unsigned long long)s64[0][3 + s]);
      atomicMin(&out->gmin[s], (unsigned long long)s64[0][5 + s]);
      atomicMax(&out->gmax[s], (unsigned long long)s64[0][7 + s]);
      atomicMin(&out->bmin[s], s32[0][0 + s]);
      atomicMax(&out->bmax[s], s32[0][2 + s]);
      atomicMin(&out->imin[s], s32[0][4 + s]);
      atomicMax(&out->imax[s], s32[0][6 + s]);
    }
    if (s32[0][8]) atomicOr(&out->unsorted, 1u);
  }
}

void launch_extents(const Rec* rec, u64 n, u32 log2G, Summary* d_sum, int grid, cudaStream_t st) {
  extents_kernel<256><<<grid, 256, 0, st>>>(rec, n, log2G, d_sum);
}

// ------------------------------------------------------------------------------------------------------------
// key extraction, 1 entry per record (every record within one granule): key = key_hi << pos_bits | pos, plus
// the histogram of every radix digit the sort will use (onesweep's upfront histogram), accumulated per CTA in
// shared memory with warp-aggregated (match_any) increments and flushed with one global atomic per bin.
// ------------------------------------------------------------------------------------------------------------
template <int THREADS, int RB>
__global__ void __launch_bounds__(THREADS) extract_1to1_kernel(const Rec* __restrict__ rec, u64 n, KeyLayout L,
                                                                u32 npass, u64* __restrict__ keys,
                                                                u32* __restrict__ hist /* [npass][1<<RB] */) {
  constexpr int RADIX = 1 << RB;
  extern __shared__ u32 sh[];  // [npass][RADIX]
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS) sh[i] = 0;
  __syncthreads();
  const u64 stride = (u64)gridDim.x * THREADS;
  const u64 nround = (n + stride - 1) / stride;
  for (u64 it = 0; it < nround; it++) {
    u64 k = it * stride + (u64)blockIdx.x * THREADS + threadIdx.x;
    bool valid = k < n;
    u64 key = 0;
    if (valid) {
      Rec r = load_rec(rec + k);
      u64 g = r.addr >> L.log2G;
      key = (key_hi_of(L, r.space, r.block, r.interval, g) << L.pos_bits) | k;
      keys[k] = key;
    }
    for (u32 p = 0; p < npass; p++) {
      u32 d = valid ? (u32)((key >> (L.pos_bits + p * RB)) & (RADIX - 1)) : RADIX;
      unsigned peers = __match_any_sync(~0u, d);
      if (valid && (threadIdx.x & 31) == 31 - __clz(peers)) atomicAdd(&sh[p * RADIX + d], __popc(peers));
    }
  }
  __syncthreads();
  for (u32 i = threadIdx.x; i < npass * RADIX; i += THREADS)
    if (sh[i]) atomicAdd(&hist[i], sh[i]);
}

void launch_extract_1to1(const Rec* rec, u64 n, const KeyLayout& L, u32 npass, u64* keys, u32* hist, int grid,
                         cudaStream_t st) {
  size_t smem = (size_t)npass * (1 << RADIX_BITS) * sizeof(u32);
  extract_1to1_kernel<256, RADIX_BITS><<<grid, 256, smem, st>>>(rec, n, L, npass, keys, hist);
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
                                                                 u64* __restrict__ keys, u32* __restrict__ hist) {
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
      u64 key = (key_hi_of(L, r.space, r.block, r.interval, g) << L.pos_bits) | k;
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
                          u32* hist, int grid, cudaStream_t st) {
  size_t smem = (size_t)npass * (1 << RADIX_BITS) * sizeof(u32);
  extract_multi_kernel<256, RADIX_BITS><<<grid, 256, smem, st>>>(rec, n, L, npass, off, keys, hist);
}

}  // namespace sesa
