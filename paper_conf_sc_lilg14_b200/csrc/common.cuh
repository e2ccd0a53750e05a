// common.cuh — shared device definitions of the sm_100a race-check pipeline (no oracle code here).
//
// Pipeline: extents (validate + key layout) -> key extract (+ digit histograms) -> onesweep LSD
// radix sort of 64-bit keys -> segmented conflict tiles (+ cross-tile carries) -> race sort -> race list.
//
// Sort key of one entry (a (record, granule) pair), DESIGN.md §4:
//   key = key_hi << pos_bits | pos          pos = record position (already ascending: LSD keeps it stable)
//   key_hi (shared) = [space] | (block - bminS) | (interval - iminS) | (granule - gminS)
//   key_hi (global) = [space] | (granule - gminG) [| (block - bminG) | (interval - iminG)  if input unsorted]
// so that one location λ ("same address", "address overlapping") is one contiguous run of
// sorted keys, runs appear in the canonical output order (space, block, interval, addr), and within a global
// run the entries of one (block, interval) — a "sub-run" — are contiguous.
#pragma once
#include <cstdint>
#include <cstdlib>
#include <cuda_runtime.h>

typedef uint64_t u64;
typedef uint32_t u32;
typedef uint16_t u16;
typedef uint8_t u8;

namespace sesa {

enum { SP_SHARED = 0, SP_GLOBAL = 1 };
enum { RW_READ = 0, RW_WRITE = 1, RW_ATOMIC = 2 };
enum { KIND_RW = 1, KIND_WW = 2, KIND_WWB = 3 };  // KIND_WWB: benign W/W (reported with flags bit 0)
static constexpr u32 NOBI = 0xFFFFFFFFu;

// Device-side view of one 32-byte access record (layout of sesa_access, include/sesa.h).
struct __align__(16) Rec {
  u64 addr, vh;
  u32 block, thread, interval;
  u16 size;
  u8 space, rw;
};
static_assert(sizeof(Rec) == 32, "record layout");

__device__ __forceinline__ Rec load_rec(const Rec* __restrict__ p) {
  // two 16-byte vector loads of one 32-byte sector
  const uint4* q = reinterpret_cast<const uint4*>(p);
  uint4 a = __ldg(q), b = __ldg(q + 1);
  Rec r;
  r.addr = (u64)a.x | ((u64)a.y << 32);
  r.vh = (u64)a.z | ((u64)a.w << 32);
  r.block = b.x;
  r.thread = b.y;
  r.interval = b.z;
  r.size = (u16)(b.w & 0xFFFF);
  r.space = (u8)((b.w >> 16) & 0xFF);
  r.rw = (u8)(b.w >> 24);
  return r;
}

struct KeyLayout {
  u32 log2G;
  u32 pos_bits, sort_bits;
  u32 both, single_space, space_shift;
  u64 gminS;
  u32 bminS, iminS, gbS, ibS, bbS;
  u64 gminG;
  u32 bminG, iminG, gbG, ibG, bbG, lowG;
  // wbit = 1 (sort + compaction path): the key carries one more bit below the position, set when the entry's
  // record writes (plain WRITE or ATOMIC): key = key_hi << (pos_bits + 1) | pos << 1 | w.  The order inside a
  // location run is still by position; compaction uses the bit to drop read-only runs (no race: P:43 needs a
  // write) and strips it, so every later stage sees the plain layout.
  u32 wbit;
};

__device__ __forceinline__ u64 lowmask(u32 b) { return b >= 64 ? ~0ull : ((1ull << b) - 1ull); }

__device__ __forceinline__ u64 key_hi_of(const KeyLayout& L, u32 space, u32 b, u32 i, u64 g) {
  u64 h;
  if (space == SP_SHARED) {
    h = ((u64)(b - L.bminS) << (L.ibS + L.gbS)) | ((u64)(i - L.iminS) << L.gbS) | (g - L.gminS);
  } else {
    h = (g - L.gminG) << L.lowG;
    if (L.lowG) h |= ((u64)(b - L.bminG) << L.ibG) | (u64)(i - L.iminG);
  }
  if (L.both) h |= (u64)space << L.space_shift;
  return h;
}

__device__ __forceinline__ u32 space_of_hi(const KeyLayout& L, u64 hi) {
  return L.both ? (u32)((hi >> L.space_shift) & 1ull) : L.single_space;
}

// location-run key: entries with equal group keys are at the same location λ
__device__ __forceinline__ u64 group_of_hi(const KeyLayout& L, u64 hi) {
  return space_of_hi(L, hi) == SP_GLOBAL ? (hi & ~lowmask(L.lowG)) : hi;
}

// same location run?  (sorted keys a, b; the run key drops the position bits and, for an unsorted-input global
// layout, the (block, interval) bits; different spaces differ in the space bit, which no mask clears)
__device__ __forceinline__ bool same_group(const KeyLayout& L, u64 a, u64 b) {
  const bool glob = L.both ? ((a >> (L.space_shift + L.pos_bits)) & 1ull) != 0 : L.single_space == SP_GLOBAL;
  return ((a ^ b) >> (L.pos_bits + (glob ? L.lowG : 0u))) == 0;
}

__device__ __forceinline__ u64 granule_of_hi(const KeyLayout& L, u64 hi) {
  if (space_of_hi(L, hi) == SP_SHARED) return (hi & lowmask(L.gbS)) + L.gminS;
  return ((hi >> L.lowG) & lowmask(L.gbG)) + L.gminG;
}

// Lanes holding the same digit (stable peers) without __match_any_sync: MATCH runs on the slow ADU pipe on
// sm_100 (ncu: 65-96% ADU busy), ballots run on the ALU pipe.  NB = digit bits to compare.
template <int NB>
__device__ __forceinline__ unsigned peers_of(u32 d) {
  unsigned p = ~0u;
#pragma unroll
  for (int b = 0; b < NB; b++) {
    const bool bit = (d >> b) & 1u;
    const unsigned m = __ballot_sync(~0u, bit);
    p &= bit ? m : ~m;
  }
  return p;
}

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm volatile("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}

// Counter-based value hash of flow accesses (include/sesa.h): splitmix64 finaliser of x + golden gamma.
__host__ __device__ __forceinline__ u64 sesa_mix(u64 x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}

// block-wide exclusive sum over THREADS values (one per thread)
template <int THREADS>
__device__ __forceinline__ u32 block_excl_sum(u32 v, u32* scratch /* [THREADS/32 + 1] */) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  u32 x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    u32 y = __shfl_up_sync(~0u, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) scratch[warp] = x;
  __syncthreads();
  if (threadIdx.x == 0) {
    u32 acc = 0;
    for (int w = 0; w < THREADS / 32; w++) {
      u32 c = scratch[w];
      scratch[w] = acc;
      acc += c;
    }
  }
  __syncthreads();
  return scratch[warp] + x - v;
}

// ---- TMA bulk copies (cp.async.bulk, 1-D: no tensor map) completing on an mbarrier -------------------------
__device__ __forceinline__ u32 smem_u32(const void* p) { return (u32)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(u64* bar, u32 count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() { asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
__device__ __forceinline__ void mbar_expect_tx(u64* bar, u32 bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
// bytes must be a multiple of 16, both addresses 16-byte aligned
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, u32 bytes, u64* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void mbar_wait(u64* bar, u32 parity) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n}" ::"r"(
          smem_u32(bar)),
      "r"(parity)
      : "memory");
}

// ---- TMA streaming ring: a persistent CTA walks chunks c = blockIdx.x + j*gridDim.x, keeping STAGES chunks in
// flight with cp.async.bulk (bytes in flight do not cost registers).  Usage:
//   BulkRing<S> ring(smem_bufs, bars, chunk_bytes);  ring.start(src, nbytes_total)   (all threads)
//   for (j = 0; ring.next(j); j++) { const char* data = ring.wait(j); ...; ring.release(j); }
template <int STAGES>
struct BulkRing {
  unsigned char* buf;  // [STAGES][chunk]
  u64* bar;            // [STAGES]
  u32 chunk;           // bytes per chunk (multiple of 16)
  const unsigned char* src;
  u64 total;           // bytes
  u64 nchunks;
  __device__ __forceinline__ BulkRing(unsigned char* b, u64* br, u32 ch) : buf(b), bar(br), chunk(ch) {}
  __device__ __forceinline__ void issue(u64 j) {  // thread 0: chunk #j of this CTA into slot j % STAGES
    const u64 c = blockIdx.x + j * gridDim.x;
    if (c >= nchunks) return;
    const u64 off = c * chunk;
    const u32 bytes = (u32)((min((u64)chunk, total - off) + 15) & ~15ull);
    const int slot = (int)(j % STAGES);
    mbar_expect_tx(&bar[slot], bytes);
    bulk_g2s(buf + (size_t)slot * chunk, src + off, bytes, &bar[slot]);
  }
  __device__ __forceinline__ void start(const void* s, u64 nbytes) {
    src = reinterpret_cast<const unsigned char*>(s);
    total = nbytes;
    nchunks = (nbytes + chunk - 1) / chunk;
    if (threadIdx.x == 0) {
      for (int i = 0; i < STAGES; i++) mbar_init(&bar[i], 1);
      fence_mbar_init();
      for (int i = 0; i < STAGES; i++) issue(i);
    }
    __syncthreads();
  }
  __device__ __forceinline__ bool next(u64 j) const { return blockIdx.x + j * gridDim.x < nchunks; }
  __device__ __forceinline__ u64 chunk_index(u64 j) const { return blockIdx.x + j * gridDim.x; }
  __device__ __forceinline__ u32 chunk_bytes(u64 j) const {
    return (u32)min((u64)chunk, total - chunk_index(j) * chunk);
  }
  __device__ __forceinline__ const unsigned char* wait(u64 j) {
    const int slot = (int)(j % STAGES);
    mbar_wait(&bar[slot], (u32)((j / STAGES) & 1));
    return buf + (size_t)slot * chunk;
  }
  __device__ __forceinline__ void release(u64 j) {  // all threads: slot j % STAGES may be refilled
    __syncthreads();
    if (threadIdx.x == 0) issue(j + STAGES);
  }
};

// ---- decoupled look-back (Merrill & Garland) for one scalar per tile, done by one whole warp ------------------
// Status word: bits 63..62 = 1 (tile aggregate) | 2 (inclusive prefix), low 62 bits = value; 0 = not yet
// published.  The warp inspects 32 predecessors per step (one per lane) instead of walking them one by one.
// All 32 lanes of the calling warp must call it; returns the exclusive prefix of `tile`.
__device__ __forceinline__ u64 warp_lookback(u64* lb, u32 tile, u64 agg, unsigned long long* dbg = nullptr) {
  const int lane = threadIdx.x & 31;
  volatile u64* v = lb;
  if (lane == 0) v[tile] = ((tile == 0 ? 2ull : 1ull) << 62) | agg;
  if (tile == 0) return 0;
  u64 excl = 0;
  long long base = (long long)tile - 1;
  while (true) {
    const long long p = base - lane;
    u64 w = 2ull << 62;  // "prefix 0" before tile 0
    if (p >= 0) {
      int spins = 0;
      while (true) {
        w = v[p];
        spins++;
        if ((w >> 62) != 0) break;
        __nanosleep(spins < 4 ? 32 : 128);  // back off: spinning warps otherwise flood L2
      }
      if (dbg) atomicAdd(&dbg[1], (unsigned long long)spins);
    }
    if (dbg && lane == 0) atomicAdd(&dbg[0], 1ull);
    const unsigned pre = __ballot_sync(~0u, (w >> 62) == 2);
    const int first = pre ? __ffs(pre) - 1 : 31;  // nearest predecessor holding an inclusive prefix
    u64 x = lane <= first ? (w & ((1ull << 62) - 1)) : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(~0u, x, o);
    excl += x;
    if (pre) break;
    base -= 32;
  }
  if (lane == 0) v[tile] = (2ull << 62) | (excl + agg);
  return excl;
}

// ---- device summary written by the extents pass ------------------------------------------------------------
struct Summary {
  unsigned long long bad_index;  // lowest invalid record index (~0 = none)
  unsigned long long entries;    // sum of granules per record
  unsigned long long multi;      // records spanning > 1 granule
  unsigned long long count[2];   // records per space
  unsigned long long gmin[2], gmax[2];
  unsigned int bmin[2], bmax[2], imin[2], imax[2];
  unsigned int unsorted;         // some record's (block, interval) < its predecessor's
  unsigned int pad;
  unsigned long long oob_count;  // valid records outside every registered region of their space (NEXT-1)
  unsigned long long oob_first;  // lowest such record index (~0 = none)
  // with tile histograms (fused-pass candidates): histograms of the raw granule bytes 1..3, (g >> 8b) & 255 —
  // the later sort digits once gmin is aligned down to a multiple of 2^(8 (npass - 1)) (sesa_api.cu); row 3:
  // (g >> (HYB_LO + 8)) & 255, the second global digit of the bucket path (k_bucket.cu)
  unsigned int bhist[4][256];
};

// bucket path (k_bucket.cu): the two global sort digits are key bits [HYB_LO, HYB_LO + 16); the bits below are
// resolved per chunk of 2^HYB_CHUNK granules by a shared-memory bitmap and a shared-memory sort of the survivors
constexpr unsigned HYB_LO = 14;
constexpr unsigned HYB_CHUNK = 15;  // >= HYB_LO: a chunk = 2^15 granules (4 KB bitmaps; ~30 K C5 keys)

// one registered memory region (include/sesa.h sesa_region), bytes [base, end)
struct Region {
  u64 base, end;
};
constexpr int MAX_REGIONS = 1024;

// ---- kernel launchers (implemented in the .cu files) -------------------------------------------------------
struct Launch {
  cudaStream_t stream;
};

}  // namespace sesa
