// k_bucket.cu — the bucket path of the sort (SURVEY §8a rows a4 + a6: sort, then compaction to the locations
// touched at least twice), for large single-space traces whose granules are spread evenly (C5).
//
// A location touched once cannot race (P:43 needs two accesses), and on such traces almost every location is:
// C5 keeps 2e5 of its 1e9 entries.  The full LSD sort (4 passes over 16-byte key traffic) followed by a
// compaction spends its time ordering entries that are then thrown away.  The bucket path sorts only by the two
// HIGH key digits (key_hi bits [HYB_LO, HYB_LO + 16): the fused extract pass + one onesweep pass), which brings
// the entries of every chunk of 2^HYB_CHUNK consecutive granules together, and then resolves each chunk inside
// one CTA:
//   sweep 1  stream the chunk's keys; set a bit per granule in a shared-memory bitmap (atomicOr returns the old
//            word: a bit already set marks the granule "touched >= 2 times" in a second bitmap)
//   sweep 2  stream the keys again (an L2 hit: chunks are ~250 KB) and keep those at marked granules, in order
//   sort     the survivors by their full 64-bit key (granule, then record position) — a bitonic sort in shared
//            memory, or, beyond its capacity (2048), a stable two-pass radix sort of the chunk's range in global
//            memory
// Output: the chunk's survivors, sorted, at the chunk's own offset of the other key buffer, plus a count; a scan
// of the counts and a gather concatenate them — exactly the array the full sort + compaction produce.
//
// Exact for any input (the bitmap covers the chunk's whole granule span); fast when chunks are of similar size,
// which the host checks on a sample of the granules before choosing this path (sesa_api.cu).
#include <algorithm>

#include "kernels.cuh"

namespace sesa {

// Measured on C5 (bucket kernels per 1e9 keys): chunks of 2^15 granules with 8 keys in flight per thread and the
// next round's loads issued before the current round is processed: 2.28 ms; 4 in flight 2.37 (2.51 without the
// prefetch); chunks of 2^14: 2.39; 2^16: 3.21; sweep 2 from 16-bit granule offsets kept in shared memory instead
// of re-reading the keys (an L2 hit): 3.35 (the smem footprint halves the CTAs per SM).
constexpr int BK_THREADS = 256, BK_WORDS = (1 << HYB_CHUNK) / 32, BK_CAPC = 2048, BK_U = 8;
constexpr size_t BK_DSMEM = (size_t)BK_CAPC * 8;  // dynamic: the survivors

// ---- chunk boundaries: bounds[c] = first position whose key is >= c << (HYB_CHUNK + pos_bits) (warp per c) ----
__global__ void bucket_bounds_kernel(const u64* __restrict__ keys, u32 m, u32 nchunks, u32 shift,
                                     u32* __restrict__ bounds) {
  const u32 c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (c > nchunks) return;
  if (c == nchunks) {
    if (lane == 0) bounds[c] = m;
    return;
  }
  const u64 target = (u64)c << shift;  // lower bound of keys >= target
  u32 lo = 0, hi = m;                  // answer in [lo, hi]
  while (hi - lo > 32) {
    // 32 probes split [lo, hi) into 33 parts; lane l probes the end of part l
    const u64 span = hi - lo;
    const u32 p = lo + (u32)(span * (u64)(lane + 1) / 33);
    const bool below = keys[p] < target;
    const unsigned b = __ballot_sync(~0u, below);
    // probes are ascending: the below-set is a prefix
    const int nb = __popc(b);
    const u32 nlo = nb ? lo + (u32)(span * (u64)nb / 33) + 1 : lo;
    const u32 nhi = nb < 32 ? lo + (u32)(span * (u64)(nb + 1) / 33) : hi;
    lo = nlo, hi = nhi;
  }
  const u32 p = lo + lane;
  const bool below = p < hi && keys[p] < target;
  const unsigned b = __ballot_sync(~0u, below);
  if (lane == 0) bounds[c] = lo + __popc(b);
}

// ---- per-chunk bitmap filter + sort of the survivors ---------------------------------------------------------
struct BucketArgs {
  const u64* keys;    // sorted by key_hi >> HYB_LO
  u64* stage;         // other key buffer: chunk c's survivors go to [bounds[c], bounds[c] + cnt[c])
  u64* spare;         // = keys (dead after the chunk's sweeps): ping-pong space of the global fallback sort
  const u32* bounds;  // [nchunks + 1]
  u32* cnt;           // [nchunks]
  u32* ctr;           // [0]: chunk counter, [1]: overflow count
  u32* over;          // overflow chunk list
  u32 nchunks, pos_bits;
};

__device__ __forceinline__ void bitonic_smem(u64* a, u32 k, u32 kp) {
  // pad [k, kp) with ~0 (sorts last), then the classic bitonic network over kp (power of two) elements
  for (u32 i = k + threadIdx.x; i < kp; i += BK_THREADS) a[i] = ~0ull;
  __syncthreads();
  for (u32 size = 2; size <= kp; size <<= 1) {
    for (u32 stride = size >> 1; stride > 0; stride >>= 1) {
      for (u32 t = threadIdx.x; t < kp / 2; t += BK_THREADS) {
        const u32 lo = 2 * t - (t & (stride - 1)), hi = lo + stride;
        const bool up = (lo & size) == 0;
        const u64 x = a[lo], y = a[hi];
        if ((x > y) == up) a[lo] = y, a[hi] = x;
      }
      __syncthreads();
    }
  }
}

__global__ void __launch_bounds__(BK_THREADS) bucket_local_kernel(BucketArgs A) {
  __shared__ u32 seen[BK_WORDS], dup[BK_WORDS];
  extern __shared__ __align__(16) unsigned char bk_dyn[];
  u64* cand = reinterpret_cast<u64*>(bk_dyn);  // [BK_CAPC] survivors
  __shared__ u32 s_chunk, s_w[BK_THREADS / 32 + 1];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const u32 gmask = (1u << HYB_CHUNK) - 1u;
  const unsigned lt = lanemask_lt();
  while (true) {
    if (tid == 0) s_chunk = atomicAdd(&A.ctr[0], 1u);
    for (int i = tid; i < BK_WORDS; i += BK_THREADS) seen[i] = 0, dup[i] = 0;
    __syncthreads();
    const u32 c = s_chunk;
    if (c >= A.nchunks) return;
    const u32 s = A.bounds[c], e = A.bounds[c + 1];
    // sweep 1: the chunk's keys (BK_U in flight per thread, the next round's loads issued before this round is
    // processed; kept in L2 for sweep 2): granule bitmap, a second touch marks the granule
    u64 k[BK_U];
    auto load = [&](u64* dst, u32 b0) {
#pragma unroll
      for (int u = 0; u < BK_U; u++) {
        const u32 i = b0 + u * BK_THREADS + tid;
        dst[u] = i < e ? __ldcg(A.keys + i) : 0ull;
      }
    };
    load(k, s);
    for (u32 b0 = s; b0 < e; b0 += BK_THREADS * BK_U) {
      u64 kn[BK_U];
      load(kn, b0 + BK_THREADS * BK_U);  // next round in flight while this one is processed
#pragma unroll
      for (int u = 0; u < BK_U; u++) {
        const u32 i = b0 + u * BK_THREADS + tid;
        if (i >= e) continue;
        const u32 g = (u32)(k[u] >> A.pos_bits) & gmask, bit = 1u << (g & 31);
        if (atomicOr(&seen[g >> 5], bit) & bit) atomicOr(&dup[g >> 5], bit);
      }
#pragma unroll
      for (int u = 0; u < BK_U; u++) k[u] = kn[u];
    }
    __syncthreads();
    // sweep 2: the survivors (in element order, which need not be position order); their full keys are read back
    u32 k_total = 0;  // survivors so far (uniform)
    for (u32 b0 = s; b0 < e; b0 += BK_THREADS * BK_U) {
      bool keep[BK_U];
      bool any = false;
#pragma unroll
      for (int u = 0; u < BK_U; u++) {
        const u32 i = b0 + u * BK_THREADS + tid;
        u32 g = 0;
        if (i < e) g = (u32)(__ldcs(A.keys + i) >> A.pos_bits) & gmask;
        keep[u] = i < e && ((dup[g >> 5] >> (g & 31)) & 1u);
        any |= keep[u];
      }
      if (!__syncthreads_or(any)) continue;  // (C5: almost every round)
#pragma unroll
      for (int u = 0; u < BK_U; u++) {
        const unsigned bal = __ballot_sync(~0u, keep[u]);
        if (lane == 0) s_w[warp] = __popc(bal);
        __syncthreads();
        u32 before = 0, row = 0;
        for (int w = 0; w < BK_THREADS / 32; w++) {
          const u32 x = s_w[w];
          before += w < warp ? x : 0u;
          row += x;
        }
        if (keep[u]) {
          const u32 i = b0 + u * BK_THREADS + tid;
          const u64 key = __ldcg(A.keys + i);
          const u32 j = k_total + before + __popc(bal & lt);
          if (j < BK_CAPC) cand[j] = key;
          A.stage[s + j] = key;  // (also staged: the overflow path reads the survivors from here)
        }
        k_total += row;
        __syncthreads();
      }
    }
    if (tid == 0) A.cnt[c] = k_total;
    if (k_total > BK_CAPC) {  // too many survivors for shared memory: sorted later in global memory
      if (tid == 0) A.over[atomicAdd(&A.ctr[1], 1u)] = c;
      __syncthreads();
      continue;
    }
    if (k_total > 1) {
      u32 kp = 2;
      while (kp < k_total) kp <<= 1;
      bitonic_smem(cand, k_total, kp);
      for (u32 j = tid; j < k_total; j += BK_THREADS) A.stage[s + j] = cand[j];
    }
    __syncthreads();
  }
}

// ---- overflow chunks: stable LSD radix sort of the survivors by (key_hi bits [0, HYB_CHUNK), position) in global
// memory, one CTA per chunk: 8-bit passes over the position bits, then two passes of 8 / 7 bits over key_hi,
// ping-ponging between the staging range and the chunk's dead range of the sorted keys.  (The partition passes
// before are unstable and the fused extents pass writes its regions in window order, so the survivors of a chunk
// arrive in no particular position order.)
__global__ void __launch_bounds__(BK_THREADS) bucket_overflow_kernel(BucketArgs A) {
  __shared__ u32 hist[RADIX], run[RADIX], wc[BK_THREADS / 32][RADIX];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned lt = lanemask_lt();
  for (u32 o = blockIdx.x; o < A.ctr[1]; o += gridDim.x) {
  const u32 c = A.over[o];
  const u32 s = A.bounds[c], k = A.cnt[c];
  u64* src = A.stage + s;
  u64* dst = A.spare + s;
  const u32 npos = (A.pos_bits + RADIX_BITS - 1) / RADIX_BITS;
  for (u32 pass = 0; pass < npos + 2; pass++) {
    u32 sh, dmask;
    if (pass < npos) {  // position digits
      sh = pass * RADIX_BITS;
      dmask = (1u << min((u32)RADIX_BITS, A.pos_bits - sh)) - 1u;
    } else {            // key_hi bits [0, 8), [8, HYB_CHUNK)
      sh = A.pos_bits + (pass - npos) * RADIX_BITS;
      dmask = pass == npos ? RADIX - 1 : (1u << (HYB_CHUNK - RADIX_BITS)) - 1u;
    }
    for (int i = tid; i < RADIX; i += BK_THREADS) hist[i] = 0;
    __syncthreads();
    for (u32 i = tid; i < k; i += BK_THREADS) atomicAdd(&hist[(u32)(src[i] >> sh) & dmask], 1u);
    __syncthreads();
    if (tid == 0) {
      u32 acc = 0;
      for (int d = 0; d < RADIX; d++) run[d] = acc, acc += hist[d];
    }
    __syncthreads();
    // stable scatter, one row of BK_THREADS keys at a time: rank = warps before (per digit) + lanes before
    for (u32 r0 = 0; r0 < k; r0 += BK_THREADS) {
      const u32 i = r0 + tid;
      const bool valid = i < k;
      const u64 key = valid ? src[i] : 0ull;
      const u32 d = valid ? (u32)(key >> sh) & dmask : (u32)RADIX;
      const unsigned peers = peers_of<RADIX_BITS + 1>(d);
      for (int q = tid; q < (BK_THREADS / 32) * RADIX; q += BK_THREADS) (&wc[0][0])[q] = 0;
      __syncthreads();
      if (valid && lane == 31 - __clz(peers)) wc[warp][d] = __popc(peers);
      __syncthreads();
      u32 off = 0;
      if (valid) {
        for (int w = 0; w < warp; w++) off += wc[w][d];
        dst[run[d] + off + __popc(peers & lt)] = key;
      }
      __syncthreads();
      if (tid < RADIX) {
        u32 t = 0;
        for (int w = 0; w < BK_THREADS / 32; w++) t += wc[w][tid];
        run[tid] += t;
      }
      __syncthreads();
    }
    u64* t = src;
    src = dst;
    dst = t;
  }
  // an odd number of passes leaves the result in the dead range: back to the staging range
  if ((npos + 2) & 1u) {
    __syncthreads();
    for (u32 i = tid; i < k; i += BK_THREADS) dst[i] = src[i];
  }
  __syncthreads();
  }
}

// ---- concatenate the chunks' survivors: out[off[c] + j] = stage[bounds[c] + j] (warp per chunk) --------------
__global__ void bucket_gather_kernel(const u64* __restrict__ stage, const u32* __restrict__ bounds,
                                     const u32* __restrict__ cnt, const u32* __restrict__ off, u32 nchunks,
                                     u64* __restrict__ out) {
  const u32 c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (c >= nchunks) return;
  const u32 k = cnt[c], s = bounds[c], o = off[c];
  for (u32 j = lane; j < k; j += 32) out[o + j] = stage[s + j];
}

__global__ void bucket_total_kernel(const u32* off, const u32* cnt, u32 n, u32* total) {
  *total = off[n - 1] + cnt[n - 1];
}

// ---- sample of the chunk sizes: histogram of the chunks of every stride-th granule, and the maximum --------------
// (warp-aggregated: lanes of one chunk add once — a hot chunk, C3's bins, would otherwise serialise the atomics)
__global__ void bucket_sample_kernel(const u32* __restrict__ gran, u32 n, u32 stride, u32 gmin_lo, u32 nchunks,
                                     u32* __restrict__ hist) {
  const u64 step = (u64)gridDim.x * blockDim.x * stride;
  for (u64 i0 = (u64)(blockIdx.x * blockDim.x + (threadIdx.x & ~31u)) * stride; i0 < n; i0 += step) {
    const u64 i = i0 + (u64)(threadIdx.x & 31) * stride;
    const u32 c = i < n ? (gran[i] - gmin_lo) >> HYB_CHUNK : ~0u;
    const unsigned peers = __match_any_sync(~0u, c);
    if (c < nchunks && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&hist[c], (u32)__popc(peers));
  }
}

// the same from a key array: chunk = key >> shift
__global__ void bucket_sample_keys_kernel(const u64* __restrict__ keys, u32 m, u32 stride, u32 shift, u32 nchunks,
                                          u32* __restrict__ hist) {
  const u64 step = (u64)gridDim.x * blockDim.x * stride;
  for (u64 i0 = (u64)(blockIdx.x * blockDim.x + (threadIdx.x & ~31u)) * stride; i0 < m; i0 += step) {
    const u64 i = i0 + (u64)(threadIdx.x & 31) * stride;
    const u32 c = i < m ? (u32)min(keys[i] >> shift, (u64)~0u) : ~0u;
    const unsigned peers = __match_any_sync(~0u, c);
    if (c < nchunks && (threadIdx.x & 31) == __ffs(peers) - 1) atomicAdd(&hist[c], (u32)__popc(peers));
  }
}

__global__ void bucket_sample_max_kernel(const u32* __restrict__ hist, u32 nchunks, u32* __restrict__ out) {
  u32 mx = 0;
  for (u32 c = blockIdx.x * blockDim.x + threadIdx.x; c < nchunks; c += gridDim.x * blockDim.x) mx = max(mx, hist[c]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = max(mx, __shfl_xor_sync(~0u, mx, o));
  if ((threadIdx.x & 31) == 0) atomicMax(out, mx);
}

u32 bucket_sample_keys_max(const u64* keys, u32 m, u32 shift, u32 nchunks, void* temp, cudaStream_t st, u32* h_max,
                           u32* samples, u32 want) {
  u32* hist = reinterpret_cast<u32*>(temp);
  u32* mx = hist + nchunks;
  const u32 stride = std::max<u32>(1, m / want);
  *samples = (m + stride - 1) / stride;
  cudaMemsetAsync(temp, 0, ((size_t)nchunks + 1) * 4, st);
  const u32 grid = (u32)std::min<u64>(((u64)*samples + 255) / 256, (u64)dev_sm_count() * 8);
  bucket_sample_keys_kernel<<<grid, 256, 0, st>>>(keys, m, stride, shift, nchunks, hist);
  bucket_sample_max_kernel<<<std::min<u32>((nchunks + 255) / 256, 1024u), 256, 0, st>>>(hist, nchunks, mx);
  cudaMemcpyAsync(h_max, mx, 4, cudaMemcpyDeviceToHost, st);
  return 2;
}

size_t bucket_temp_bytes(u32 nchunks) {
  // bounds [nchunks + 1], cnt, off, over [nchunks], ctr[2] + total, sample histogram, scan temp
  return ((size_t)nchunks * 5 + 64) * 4 + scan_u32_temp_bytes(nchunks) + 512;
}

u32 bucket_sample_max(const u32* gran, u32 n, u32 gmin_lo, u32 nchunks, void* temp, cudaStream_t st, u32* h_max,
                      u32* samples, u32 want) {
  u32* hist = reinterpret_cast<u32*>(temp);
  u32* mx = hist + nchunks;
  const u32 stride = std::max<u32>(1, n / want);
  *samples = (n + stride - 1) / stride;
  cudaMemsetAsync(temp, 0, ((size_t)nchunks + 1) * 4, st);
  const u32 grid = (u32)std::min<u64>(((u64)*samples + 255) / 256, (u64)dev_sm_count() * 8);
  bucket_sample_kernel<<<grid, 256, 0, st>>>(gran, n, stride, gmin_lo, nchunks, hist);
  bucket_sample_max_kernel<<<std::min<u32>((nchunks + 255) / 256, 1024u), 256, 0, st>>>(hist, nchunks, mx);
  cudaMemcpyAsync(h_max, mx, 4, cudaMemcpyDeviceToHost, st);
  return 2;
}

// keys: sorted by key_hi >> HYB_LO (m entries); stage: the other key buffer (m); temp: bucket_temp_bytes(nchunks).
// Writes the compacted, fully sorted keys of the locations touched >= 2 times to `keys` and their count to *total
// (device).  Returns the number of kernels launched.
u32 launch_bucket_compact(u64* keys, u64* stage, u32 m, u32 pos_bits, u32 nchunks, void* temp, u32* total,
                          cudaStream_t st) {
  u32* bounds = reinterpret_cast<u32*>(temp);
  u32* cnt = bounds + nchunks + 1;
  u32* off = cnt + nchunks;
  u32* over = off + nchunks;
  u32* ctr = over + nchunks;  // [0] chunk counter, [1] overflow count
  void* stemp = reinterpret_cast<void*>((reinterpret_cast<uintptr_t>(ctr + 64) + 255) & ~(uintptr_t)255);
  cudaMemsetAsync(ctr, 0, 8, st);
  bucket_bounds_kernel<<<(unsigned)(((u64)(nchunks + 1) * 32 + 255) / 256), 256, 0, st>>>(keys, m, nchunks,
                                                                                          HYB_CHUNK + pos_bits, bounds);
  BucketArgs A;
  A.keys = keys;
  A.stage = stage;
  A.spare = keys;
  A.bounds = bounds;
  A.cnt = cnt;
  A.ctr = ctr;
  A.over = over;
  A.nchunks = nchunks;
  A.pos_bits = pos_bits;
  const int per = blocks_per_sm((const void*)bucket_local_kernel, BK_THREADS, BK_DSMEM);
  const u32 grid = std::min<u32>(nchunks, (u32)(dev_sm_count() * per));
  bucket_local_kernel<<<grid, BK_THREADS, BK_DSMEM, st>>>(A);
  // overflow chunks (rare on this path; their count is on the device): a small grid walks the list
  bucket_overflow_kernel<<<dev_sm_count(), BK_THREADS, 0, st>>>(A);
  launch_scan_exclusive_u32(cnt, off, nchunks, stemp, st);
  bucket_gather_kernel<<<(unsigned)(((u64)nchunks * 32 + 255) / 256), 256, 0, st>>>(stage, bounds, cnt, off, nchunks,
                                                                                    keys);
  bucket_total_kernel<<<1, 1, 0, st>>>(off, cnt, nchunks, total);
  return 6;
}

}  // namespace sesa
