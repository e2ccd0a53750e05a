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
#include <cuda_runtime.h>

typedef uint64_t u64;
typedef uint32_t u32;
typedef uint16_t u16;
typedef uint8_t u8;

namespace sesa {

enum { SP_SHARED = 0, SP_GLOBAL = 1 };
enum { RW_READ = 0, RW_WRITE = 1, RW_ATOMIC = 2 };
enum { KIND_RW = 1, KIND_WW = 2 };
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

__device__ __forceinline__ u64 granule_of_hi(const KeyLayout& L, u64 hi) {
  if (space_of_hi(L, hi) == SP_SHARED) return (hi & lowmask(L.gbS)) + L.gminS;
  return ((hi >> L.lowG) & lowmask(L.gbG)) + L.gminG;
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

// ---- decoupled look-back (Merrill & Garland) for one scalar per tile, done by one whole warp ------------------
// Status word: bits 63..62 = 1 (tile aggregate) | 2 (inclusive prefix), low 62 bits = value; 0 = not yet
// published.  The warp inspects 32 predecessors per step (one per lane) instead of walking them one by one.
// All 32 lanes of the calling warp must call it; returns the exclusive prefix of `tile`.
__device__ __forceinline__ u64 warp_lookback(u64* lb, u32 tile, u64 agg) {
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
      do {
        w = v[p];
      } while ((w >> 62) == 0);
    }
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
};

// ---- kernel launchers (implemented in the .cu files) -------------------------------------------------------
struct Launch {
  cudaStream_t stream;
};

}  // namespace sesa
