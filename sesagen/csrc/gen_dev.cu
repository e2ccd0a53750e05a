// gen_dev.cu — CUDA build of the C3-C5 generators (bench inputs, written straight into HBM).  Same formulas as
// gen_host.c (gen_common.h); offsets between per-thread record groups come from the caller (torch cumsum).
#include <cuda_runtime.h>

#include "gen_common.h"

__global__ void k_c5(c5cfg c, uint64_t lo, uint64_t hi, grec* out) {
  for (uint64_t i = lo + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < hi; i += (uint64_t)gridDim.x * blockDim.x)
    c5_record(&c, i, &out[i - lo]);
}

__global__ void k_c3_count(c3cfg c, uint32_t* cnt) {
  const uint64_t T = (uint64_t)c.blocks * c.threads;
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g < T) cnt[g] = c3_count(&c, g);
}

__global__ void k_c3_write(c3cfg c, const uint64_t* cdf, const uint64_t* off, grec* out) {
  const uint64_t T = (uint64_t)c.blocks * c.threads;
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g < T) c3_write(&c, cdf, g, out + off[g]);
}

__global__ void k_c4_degree(c4cfg c, const uint64_t* dcdf, uint32_t* deg) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v < (1ull << c.log2n)) deg[v] = c4_degree(&c, dcdf, v);
}

__global__ void k_c4_count(c4cfg c, const uint64_t* dcdf, const uint64_t* rows, uint32_t* cnt) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v < (1ull << c.log2n)) cnt[v] = c4_count(&c, dcdf, v, rows[v]);
}

__global__ void k_c4_write(c4cfg c, const uint64_t* dcdf, const uint64_t* rows, const uint64_t* off, grec* out) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v < (1ull << c.log2n)) c4_write(&c, dcdf, v, rows[v], out + off[v]);
}

static unsigned blocks_for(uint64_t n) { return (unsigned)((n + 255) / 256); }

extern "C" {
int gen_c5_dev(const c5cfg* c, uint64_t lo, uint64_t hi, void* out, void* stream) {
  const uint64_t n = hi - lo;
  unsigned g = blocks_for(n);
  if (g > 148 * 32) g = 148 * 32;
  if (n) k_c5<<<g, 256, 0, (cudaStream_t)stream>>>(*c, lo, hi, (grec*)out);
  return (int)cudaGetLastError();
}
int gen_c3_count_dev(const c3cfg* c, uint32_t* cnt, void* stream) {
  const uint64_t T = (uint64_t)c->blocks * c->threads;
  k_c3_count<<<blocks_for(T), 256, 0, (cudaStream_t)stream>>>(*c, cnt);
  return (int)cudaGetLastError();
}
int gen_c3_write_dev(const c3cfg* c, const uint64_t* cdf, const uint64_t* off, void* out, void* stream) {
  const uint64_t T = (uint64_t)c->blocks * c->threads;
  k_c3_write<<<blocks_for(T), 256, 0, (cudaStream_t)stream>>>(*c, cdf, off, (grec*)out);
  return (int)cudaGetLastError();
}
int gen_c4_degree_dev(const c4cfg* c, const uint64_t* dcdf, uint32_t* deg, void* stream) {
  k_c4_degree<<<blocks_for(1ull << c->log2n), 256, 0, (cudaStream_t)stream>>>(*c, dcdf, deg);
  return (int)cudaGetLastError();
}
int gen_c4_count_dev(const c4cfg* c, const uint64_t* dcdf, const uint64_t* rows, uint32_t* cnt, void* stream) {
  k_c4_count<<<blocks_for(1ull << c->log2n), 256, 0, (cudaStream_t)stream>>>(*c, dcdf, rows, cnt);
  return (int)cudaGetLastError();
}
int gen_c4_write_dev(const c4cfg* c, const uint64_t* dcdf, const uint64_t* rows, const uint64_t* off, void* out,
                     void* stream) {
  k_c4_write<<<blocks_for(1ull << c->log2n), 256, 0, (cudaStream_t)stream>>>(*c, dcdf, rows, off, (grec*)out);
  return (int)cudaGetLastError();
}
}
