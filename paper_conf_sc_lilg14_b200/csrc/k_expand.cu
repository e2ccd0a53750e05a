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

}  // namespace sesa
