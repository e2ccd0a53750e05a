// k_expand.cu — parametric-flow expansion.
//
// The paper models one parametric thread per flow and instantiates its race history at two symbolic thread
// ids ("we can obtain the race history of another thread tj by simply replacing every occurrence of i with j",
// P:163-169 §IV-A; conditional accesses `c(i) ? access`; flow conditions on tid).  Here every
// descriptor is instantiated at EVERY thread of every block of its flow.  Output order = the canonical
// sequential schedule: block, interval, thread, descriptor (program order), k.  One GPU thread per
// (block, interval, thread) cell: count -> exclusive scan -> write.
#include "kernels.cuh"

namespace sesa {

struct FlowDev {  // == sesa_flow (104 bytes)
  u64 base;
  long long bstride, tstride, istride;
  u64 value_seed;
  u32 block_lo, block_hi, nthreads, interval;
  u32 pmask, pval, pmod, prem, plo, phi;
  u32 fkind, fc, fm, count;
  u16 size;
  u8 space, rw;
  u32 flags;
};
static_assert(sizeof(FlowDev) == 104, "flow layout");

__device__ __forceinline__ bool flow_active(const FlowDev& f, u32 b, u32 t) {
  return b >= f.block_lo && b < f.block_hi && t < f.nthreads && (t & f.pmask) == f.pval &&
         (f.pmod == 0 || t % f.pmod == f.prem) && t >= f.plo && t < f.phi;
}

__device__ __forceinline__ u64 flow_f(const FlowDev& f, u32 t) {
  switch (f.fkind) {
    case 0: return t;
    case 1: return ((u64)t + f.fc) % f.fm;
    case 2: return (u64)(t ^ f.fc);
    case 3: return (u64)(t >> f.fc);
    default: return (u64)(t >> f.fc) * f.fm + (u64)(t & ((1u << f.fc) - 1u));
  }
}

// cell = ((b - bmin) * niv + q) * tmax + t; descriptors of interval slot q: idx[ivoff[q] .. ivoff[q+1])
__global__ void flow_count_kernel(const FlowDev* __restrict__ fl, const u32* __restrict__ ivoff,
                                  const u32* __restrict__ idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                                  u32* __restrict__ cnt) {
  const u64 c = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= ncell) return;
  const u32 t = (u32)(c % tmax);
  const u64 bq = c / tmax;
  const u32 q = (u32)(bq % niv), b = bmin + (u32)(bq / niv);
  u32 s = 0;
  for (u32 k = ivoff[q]; k < ivoff[q + 1]; k++) {
    const FlowDev& f = fl[idx[k]];
    if (flow_active(f, b, t)) s += f.count;
  }
  cnt[c] = s;
}

__global__ void flow_write_kernel(const FlowDev* __restrict__ fl, const u32* __restrict__ ivoff,
                                  const u32* __restrict__ idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                                  const u32* __restrict__ off, Rec* __restrict__ out) {
  const u64 c = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= ncell) return;
  const u32 t = (u32)(c % tmax);
  const u64 bq = c / tmax;
  const u32 q = (u32)(bq % niv), b = bmin + (u32)(bq / niv);
  u64 o = off[c];
  for (u32 k = ivoff[q]; k < ivoff[q + 1]; k++) {
    const FlowDev& f = fl[idx[k]];
    if (!flow_active(f, b, t)) continue;
    const u64 a0 = f.base + (u64)f.bstride * b + (u64)f.tstride * flow_f(f, t);
    for (u32 i = 0; i < f.count; i++, o++) {
      Rec r;
      r.addr = a0 + (u64)f.istride * i;
      r.vh = f.rw != RW_WRITE ? 0ull
             : (f.flags & 1u) ? f.value_seed
                              : sesa_mix(sesa_mix(sesa_mix(f.value_seed ^ (u64)b) ^ (u64)t) ^ (u64)i);
      r.block = b;
      r.thread = t;
      r.interval = f.interval;
      r.size = f.size;
      r.space = f.space;
      r.rw = f.rw;
      uint4* p = reinterpret_cast<uint4*>(out + o);
      p[0] = make_uint4((u32)r.addr, (u32)(r.addr >> 32), (u32)r.vh, (u32)(r.vh >> 32));
      p[1] = make_uint4(r.block, r.thread, r.interval, (u32)r.size | ((u32)r.space << 16) | ((u32)r.rw << 24));
    }
  }
}

void launch_flow_count2(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                        u32* cnt, cudaStream_t st) {
  if (!ncell) return;
  flow_count_kernel<<<(unsigned)((ncell + 255) / 256), 256, 0, st>>>(reinterpret_cast<const FlowDev*>(flows), ivoff,
                                                                    idx, niv, bmin, ncell, tmax, cnt);
}

void launch_flow_write2(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                        const u32* off, Rec* out, cudaStream_t st) {
  if (!ncell) return;
  flow_write_kernel<<<(unsigned)((ncell + 255) / 256), 256, 0, st>>>(reinterpret_cast<const FlowDev*>(flows), ivoff,
                                                                    idx, niv, bmin, ncell, tmax, off, out);
}


// ------------------------------------------------------------------------------------------------------------
// Descriptor-level check.  The paper decides races between two flows by instantiating their
// accesses at two symbolic threads t1 != t2 and asking whether an address can coincide.
// Here, per pair of descriptors, interval arithmetic on the address functions decides "no location in common /
// no race possible" without instantiating any thread:
//   * the granule range of a descriptor: base + bstride*[block_lo, block_hi) + tstride*f([0, nthreads))
//     + istride*[0, count) (+ size - 1), signed strides, f's range per kind — a superset of its instances;
//   * a pair can race only if both share a space, not both read, not both atomic, their granule ranges meet,
//     and (shared memory) same interval + a common block, or (global) same interval + a common block, or two
//     different blocks possible (blocks are unordered);
//   * a plain-write descriptor is race-free with ITSELF when its instances never share a granule: the address
//     is a mixed-radix number in its digits (thread [two digits for a 2-D tile], block in global memory, k) —
//     each coefficient clears the reach of the smaller ones by a granule (flow_range_kernel).
// Descriptors left in some undecided pair are instantiated (only those), with the canonical index every record
// has in the FULL expansion, so the witnesses equal those of expand-then-check.
struct FlowRange {
  u64 glo, ghi;  // granule range (conservative)
  u32 ok;        // 1 = range computed without overflow
  u32 self_free; // 1 = this descriptor's instances never share a granule (see above)
};

__device__ __forceinline__ void term_range(long long stride, u64 lo, u64 hi, long long* mn, long long* mx) {
  const long long a = stride * (long long)lo, b = stride * (long long)hi;
  *mn = a < b ? a : b;
  *mx = a < b ? b : a;
}

__device__ __forceinline__ void f_range(const FlowDev& f, u64* lo, u64* hi, bool* inj) {
  const u64 tmax = f.nthreads ? f.nthreads - 1 : 0;
  switch (f.fkind) {
    case 0: *lo = 0, *hi = tmax, *inj = true; break;
    case 1: *lo = 0, *hi = f.fm - 1, *inj = f.nthreads <= f.fm; break;
    case 2: {  // t ^ c < 2^bits(max(tmax, c))
      u64 m = tmax | f.fc, p = 1;
      while (p <= m) p <<= 1;
      *lo = 0, *hi = p - 1, *inj = true;
      break;
    }
    case 3: *lo = 0, *hi = tmax >> f.fc, *inj = f.fc == 0; break;
    default:
      *lo = 0, *hi = (tmax >> f.fc) * f.fm + ((1ull << f.fc) - 1ull), *inj = f.fm >= (1ull << f.fc);
  }
}

__global__ void flow_range_kernel(const FlowDev* __restrict__ fl, u32 nf, u32 log2G, FlowRange* __restrict__ out) {
  const u32 d = blockIdx.x * blockDim.x + threadIdx.x;
  if (d >= nf) return;
  const FlowDev f = fl[d];
  FlowRange r;
  r.ok = 0, r.self_free = 0, r.glo = 0, r.ghi = ~0ull;
  if (f.block_lo >= f.block_hi || f.nthreads == 0 || f.count == 0) {  // no instances at all
    r.ok = 1, r.self_free = 1, r.glo = 1, r.ghi = 0;
    out[d] = r;
    return;
  }
  u64 flo, fhi;
  bool inj;
  f_range(f, &flo, &fhi, &inj);
  // magnitudes small enough for signed 64-bit products (else: conservative full range)
  const bool small = llabs(f.bstride) < (1ll << 40) && llabs(f.tstride) < (1ll << 40) && llabs(f.istride) < (1ll << 40) &&
                     f.block_hi < (1u << 23) && fhi < (1ull << 23) && f.count < (1u << 23);
  if (small) {
    long long bmn, bmx, tmn, tmx, kmn, kmx;
    term_range(f.bstride, f.block_lo, f.block_hi - 1, &bmn, &bmx);
    term_range(f.tstride, flo, fhi, &tmn, &tmx);
    term_range(f.istride, 0, f.count - 1, &kmn, &kmx);
    const __int128 lo = (__int128)f.base + bmn + tmn + kmn, hi = (__int128)f.base + bmx + tmx + kmx + (f.size - 1);
    if (lo >= 0 && hi < ((__int128)1 << 64)) r.glo = (u64)lo >> log2G, r.ghi = (u64)hi >> log2G, r.ok = 1;
    // self-disjointness: the instance address is a sum of "digits" coef_i * x_i, x_i in [0, range_i) (the thread
    // part split in two for ROW2D; the block digit only in global memory with several blocks; k).  Sorted by
    // |coef|, two different instances differ by at least coef_{i+1} - sum_{j<=i} |coef_j| (range_j - 1) at their
    // highest differing digit: every such gap must reach `need` (1 granule when base, strides are multiples of G
    // and size <= G; else size + G - 1 bytes).  modadd / xor are injective single digits of their value range.
    const u64 G = 1ull << log2G;
    const bool aligned = (f.base % G) == 0 && f.size <= G && (f.bstride % (long long)G) == 0 &&
                         (f.tstride % (long long)G) == 0 && (f.istride % (long long)G) == 0;
    const u64 unit = aligned ? G : 1, need = aligned ? 1 : (u64)f.size + G - 1;
    u64 cf[4], rg[4];
    int nd = 0;
    bool injective = inj;
    const u64 ts = (u64)llabs(f.tstride) / unit;
    if (f.fkind == 4) {  // ROW2D: (t >> fc) * fm + (t & (2^fc - 1))
      cf[nd] = ts, rg[nd++] = min((u64)f.nthreads, (u64)(1ull << f.fc));
      cf[nd] = ts * f.fm, rg[nd++] = ((u64)(f.nthreads - 1) >> f.fc) + 1;
      injective = true;  // the mixed-radix test below decides
    } else {
      cf[nd] = ts, rg[nd++] = fhi - flo + 1;
    }
    if (f.space == SP_GLOBAL && f.block_hi - f.block_lo > 1)
      cf[nd] = (u64)llabs(f.bstride) / unit, rg[nd++] = f.block_hi - f.block_lo;
    if (f.count > 1) cf[nd] = (u64)llabs(f.istride) / unit, rg[nd++] = f.count;
    for (int i = 0; i < nd; i++)  // sort digits by coefficient
      for (int j = i + 1; j < nd; j++)
        if (cf[j] < cf[i]) {
          const u64 a = cf[i], b2 = rg[i];
          cf[i] = cf[j], rg[i] = rg[j], cf[j] = a, rg[j] = b2;
        }
    u64 reach = 0;  // sum of |coef| (range - 1) of the lower digits
    bool sep = injective;
    for (int i = 0; i < nd && sep; i++) {
      if (rg[i] <= 1) continue;
      sep = cf[i] >= reach + need;
      reach += cf[i] * (rg[i] - 1);
    }
    r.self_free = sep ? 1u : 0u;
  }
  out[d] = r;
}

// keep[d] = 1 if d is in an undecided pair (d1 <= d2; one thread per pair of a tile of the (nf x nf) triangle)
__global__ void flow_pair_kernel(const FlowDev* __restrict__ fl, const FlowRange* __restrict__ rg, u32 nf,
                                 u32* __restrict__ keep) {
  const u32 d1 = blockIdx.y * 16 + threadIdx.y, d2 = blockIdx.x * 16 + threadIdx.x;
  if (d1 >= nf || d2 >= nf || d2 < d1) return;
  const FlowDev a = fl[d1], b = fl[d2];
  const FlowRange ra = rg[d1], rb = rg[d2];
  if (a.block_lo >= a.block_hi || b.block_lo >= b.block_hi || a.count == 0 || b.count == 0 || a.nthreads == 0 ||
      b.nthreads == 0)
    return;
  if (a.space != b.space) return;
  if (a.rw == RW_READ && b.rw == RW_READ) return;      // (2)
  if (a.rw == RW_ATOMIC && b.rw == RW_ATOMIC) return;  // (3)
  if (d1 == d2) {
    if (a.rw != RW_WRITE || rg[d1].self_free) return;  // a read or atomic descriptor alone never races
  } else if (ra.ok && rb.ok && (ra.ghi < rb.glo || rb.ghi < ra.glo)) {
    return;  // no granule in common
  }
  const bool common_block = a.block_lo < b.block_hi && b.block_lo < a.block_hi;
  const bool same_iv = a.interval == b.interval;
  bool may;
  if (a.space == SP_SHARED) {
    may = same_iv && common_block;  // shared memory is per block and per interval
  } else {
    const bool one_block = a.block_hi - a.block_lo == 1 && b.block_hi - b.block_lo == 1 && a.block_lo == b.block_lo;
    may = (same_iv && common_block) || !one_block;  // different blocks are never ordered
  }
  if (!may) return;
  keep[d1] = 1;
  keep[d2] = 1;
}

// per cell: count of ALL instances (canonical index space) and of the kept descriptors' instances
__global__ void flow_count_sel_kernel(const FlowDev* __restrict__ fl, const u32* __restrict__ ivoff,
                                      const u32* __restrict__ idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                                      const u32* __restrict__ keep, u32* __restrict__ cnt_all,
                                      u32* __restrict__ cnt_kept) {
  const u64 c = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= ncell) return;
  const u32 t = (u32)(c % tmax);
  const u64 bq = c / tmax;
  const u32 q = (u32)(bq % niv), b = bmin + (u32)(bq / niv);
  u32 sa = 0, sk = 0;
  for (u32 k = ivoff[q]; k < ivoff[q + 1]; k++) {
    const FlowDev& f = fl[idx[k]];
    if (!flow_active(f, b, t)) continue;
    sa += f.count;
    if (keep[idx[k]]) sk += f.count;
  }
  cnt_all[c] = sa;
  cnt_kept[c] = sk;
}

__global__ void flow_write_sel_kernel(const FlowDev* __restrict__ fl, const u32* __restrict__ ivoff,
                                      const u32* __restrict__ idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                                      const u32* __restrict__ keep, const u32* __restrict__ off_all,
                                      const u32* __restrict__ off_kept, Rec* __restrict__ out,
                                      u32* __restrict__ orig) {
  const u64 c = (u64)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= ncell) return;
  const u32 t = (u32)(c % tmax);
  const u64 bq = c / tmax;
  const u32 q = (u32)(bq % niv), b = bmin + (u32)(bq / niv);
  u32 oa = off_all[c], ok = off_kept[c];
  for (u32 k = ivoff[q]; k < ivoff[q + 1]; k++) {
    const FlowDev& f = fl[idx[k]];
    if (!flow_active(f, b, t)) continue;
    if (!keep[idx[k]]) {
      oa += f.count;
      continue;
    }
    const u64 a0 = f.base + (u64)f.bstride * b + (u64)f.tstride * flow_f(f, t);
    for (u32 i = 0; i < f.count; i++, oa++, ok++) {
      const u64 addr = a0 + (u64)f.istride * i;
      const u64 vh = f.rw != RW_WRITE ? 0ull
                     : (f.flags & 1u) ? f.value_seed
                                      : sesa_mix(sesa_mix(sesa_mix(f.value_seed ^ (u64)b) ^ (u64)t) ^ (u64)i);
      uint4* p = reinterpret_cast<uint4*>(out + ok);
      p[0] = make_uint4((u32)addr, (u32)(addr >> 32), (u32)vh, (u32)(vh >> 32));
      p[1] = make_uint4(b, t, f.interval, (u32)f.size | ((u32)f.space << 16) | ((u32)f.rw << 24));
      orig[ok] = oa;
    }
  }
}

// race witnesses: checked-record positions -> canonical indices of the full expansion (a monotone map, so the
// lexicographic minimum and the canonical order are kept)
__global__ void race_remap_kernel(RaceOut* __restrict__ r, u32 nr, const u32* __restrict__ orig) {
  const u32 i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= nr) return;
  r[i].first = orig[r[i].first];
  r[i].second = orig[r[i].second];
}

void launch_flow_ranges(const void* flows, u32 nf, u32 log2G, void* ranges, u32* keep, cudaStream_t st) {
  if (!nf) return;
  flow_range_kernel<<<(nf + 127) / 128, 128, 0, st>>>(reinterpret_cast<const FlowDev*>(flows), nf, log2G,
                                                      reinterpret_cast<FlowRange*>(ranges));
  cudaMemsetAsync(keep, 0, (size_t)nf * 4, st);
  const dim3 grid((nf + 15) / 16, (nf + 15) / 16), blk(16, 16);
  flow_pair_kernel<<<grid, blk, 0, st>>>(reinterpret_cast<const FlowDev*>(flows),
                                         reinterpret_cast<const FlowRange*>(ranges), nf, keep);
}
size_t flow_range_bytes(u32 nf) { return (size_t)nf * sizeof(FlowRange); }

void launch_flow_count_sel(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                           const u32* keep, u32* cnt_all, u32* cnt_kept, cudaStream_t st) {
  if (!ncell) return;
  flow_count_sel_kernel<<<(unsigned)((ncell + 255) / 256), 256, 0, st>>>(
      reinterpret_cast<const FlowDev*>(flows), ivoff, idx, niv, bmin, ncell, tmax, keep, cnt_all, cnt_kept);
}

void launch_flow_write_sel(const void* flows, const u32* ivoff, const u32* idx, u32 niv, u32 bmin, u64 ncell, u32 tmax,
                           const u32* keep, const u32* off_all, const u32* off_kept, Rec* out, u32* orig,
                           cudaStream_t st) {
  if (!ncell) return;
  flow_write_sel_kernel<<<(unsigned)((ncell + 255) / 256), 256, 0, st>>>(
      reinterpret_cast<const FlowDev*>(flows), ivoff, idx, niv, bmin, ncell, tmax, keep, off_all, off_kept, out, orig);
}

void launch_race_remap(RaceOut* races, u32 nr, const u32* orig, cudaStream_t st) {
  if (nr) race_remap_kernel<<<(nr + 255) / 256, 256, 0, st>>>(races, nr, orig);
}

}  // namespace sesa
