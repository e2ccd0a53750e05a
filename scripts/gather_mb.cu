// microbenchmark: random 32-byte record gathers (the conflict kernels' access pattern) — DRAM bytes per gather
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t mix(uint64_t x) { x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33; return x; }
template <int V>
__global__ void gather(const uint4* __restrict__ rec, uint64_t nrec, uint64_t ng, uint32_t* out) {
  uint32_t acc = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < ng; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = mix(i) % nrec;
    const uint4* p = rec + 2 * r;
    uint32_t w[8];
    if (V == 0) {
      asm volatile("ld.global.cg.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];" : "=r"(w[0]),"=r"(w[1]),"=r"(w[2]),"=r"(w[3]),"=r"(w[4]),"=r"(w[5]),"=r"(w[6]),"=r"(w[7]) : "l"(p));
    } else if (V == 1) {
      asm volatile("ld.global.cg.L2::64B.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];" : "=r"(w[0]),"=r"(w[1]),"=r"(w[2]),"=r"(w[3]),"=r"(w[4]),"=r"(w[5]),"=r"(w[6]),"=r"(w[7]) : "l"(p));
    } else if (V == 2) {
      uint4 a = __ldg(p), b = __ldg(p + 1);
      w[0]=a.x;w[1]=a.y;w[2]=a.z;w[3]=a.w;w[4]=b.x;w[5]=b.y;w[6]=b.z;w[7]=b.w;
    } else {
      uint4 a = __ldcg(p);  // 16 bytes only
      w[0]=a.x;w[1]=a.y;w[2]=a.z;w[3]=a.w;w[4]=w[5]=w[6]=w[7]=0;
    }
    acc ^= w[0] ^ w[3] ^ w[4] ^ w[7];
  }
  if (acc == 0x12345678u) out[0] = acc;
}
int main() {
  const uint64_t nrec = 392000000ull, ng = 266000000ull;
  uint4* rec; uint32_t* out;
  cudaMalloc(&rec, nrec * 32); cudaMalloc(&out, 4);
  cudaMemset(rec, 1, nrec * 32);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int v = 0; v < 4; v++) {
    for (int rep = 0; rep < 3; rep++) {
      cudaEventRecord(e0);
      if (v == 0) gather<0><<<148 * 8, 256>>>(rec, nrec, ng, out);
      if (v == 1) gather<1><<<148 * 8, 256>>>(rec, nrec, ng, out);
      if (v == 2) gather<2><<<148 * 8, 256>>>(rec, nrec, ng, out);
      if (v == 3) gather<3><<<148 * 8, 256>>>(rec, nrec, ng, out);
      cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1);
      if (rep == 2) printf("variant %d: %.3f ms, %.2f Ggather/s, %.1f GB/s at 32 B\n", v, ms, ng / ms / 1e6, ng * 32.0 / ms / 1e6);
    }
  }
  return 0;
}
