// probe: where a 2-D TMA box {4 x u64, 256 rows} lands in shared memory with a swizzle (32B: rows stay 32 bytes apart, halves swapped when offset bit 7 is set; 128B: each row padded to 128 bytes).  nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/p scripts/tma_swz_probe.cu
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cstdio>
#include <cstdint>
#include <cstring>
__device__ __forceinline__ uint32_t su(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void k(const __grid_constant__ CUtensorMap m, uint64_t* out, int words) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint64_t bar;
  for (int i = threadIdx.x; i < words; i += blockDim.x) ((uint64_t*)sm)[i] = 0xEEEEEEEEEEEEEEEEull;
  __syncthreads();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su(&bar)), "r"(8192));
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];"
                 ::"r"(su(sm)), "l"((uint64_t)&m), "r"(0), "r"(0), "r"(su(&bar)) : "memory");
    asm volatile("{\n .reg .pred p;\n W: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra W;\n}" ::"r"(su(&bar)));
  }
  __syncthreads();
  for (int i = threadIdx.x; i < words; i += blockDim.x) out[i] = ((uint64_t*)sm)[i];
}
int main() {
  const int rows = 512;
  uint64_t* h = new uint64_t[rows * 4];
  for (int r = 0; r < rows; r++) for (int c = 0; c < 4; c++) h[r * 4 + c] = ((uint64_t)r << 8) | c;  // row, u64 index
  uint64_t *d, *o; cudaMalloc(&d, rows * 32); cudaMalloc(&o, 65536);
  cudaMemcpy(d, h, rows * 32, cudaMemcpyHostToDevice);
  void* fn; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  auto enc = (PFN_cuTensorMapEncodeTiled_v12000)fn;
  CUtensorMap m; memset(&m, 0, sizeof m);
  cuuint64_t dims[2] = {4, (cuuint64_t)rows}; cuuint64_t str[1] = {32}; cuuint32_t box[2] = {4, 256}, es[2] = {1, 1};
  CUresult r = enc(&m, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                   CU_TENSOR_MAP_SWIZZLE_32B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode %d\n", (int)r);
  const int words = 65536 / 8;
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536);
  k<<<1, 256, 65536>>>(m, o, words);
  printf("launch %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  uint64_t* ho = new uint64_t[words]; cudaMemcpy(ho, o, 65536, cudaMemcpyDeviceToHost);
  // first 16 rows' locations: for each u64 slot in the first 2 KB print (row, idx)
  for (int w = 0; w < 64; w++) { uint64_t v = ho[w]; if (v == 0xEEEEEEEEEEEEEEEEull) printf("[%3d] --   ", w); else printf("[%3d] r%llu.%llu ", w, (unsigned long long)(v >> 8), (unsigned long long)(v & 255)); if (w % 8 == 7) printf("\n"); }
  int last = 0; for (int w = 0; w < words; w++) if (ho[w] != 0xEEEEEEEEEEEEEEEEull) last = w;
  printf("last written u64 slot %d (bytes %d)\n", last, (last + 1) * 8);
  return 0;
}
