// Test helper (tests/test_gpu_philox.py, SURVEY.md §4 pin P2): cuRAND's own Philox4x32-10, compiled by the
// test with nvcc. curand_philox_blocks: curand_Philox4x32_10(ctr, key) per element; curand_stream_blocks:
// curand_init(seed, subsequence w, offset 4t) then curand4() — the walk RNG's blk(w, t, 0) (reading R3).
#include <curand_kernel.h>
#include <cstdint>

__global__ void k_blocks(const uint4* ctr, const uint2* key, uint4* out, uint64_t n) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = curand_Philox4x32_10(ctr[i], key[i]);
}

__global__ void k_stream(unsigned long long seed, const unsigned long long* w, const uint32_t* t, uint4* out, uint64_t n) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  curandStatePhilox4_32_10_t st;
  curand_init(seed, w[i], 4ull * t[i], &st);
  out[i] = curand4(&st);
}

extern "C" int curand_philox_blocks(const uint32_t* ctr, const uint32_t* key, uint32_t* out, uint64_t n) {
  uint4 *dc, *dout;
  uint2* dk;
  cudaMalloc(&dc, n * 16);
  cudaMalloc(&dk, n * 8);
  cudaMalloc(&dout, n * 16);
  cudaMemcpy(dc, ctr, n * 16, cudaMemcpyHostToDevice);
  cudaMemcpy(dk, key, n * 8, cudaMemcpyHostToDevice);
  k_blocks<<<(unsigned)((n + 255) / 256), 256>>>(dc, dk, dout, n);
  const cudaError_t e = cudaMemcpy(out, dout, n * 16, cudaMemcpyDeviceToHost);
  cudaFree(dc);
  cudaFree(dk);
  cudaFree(dout);
  return (int)e;
}

extern "C" int curand_stream_blocks(unsigned long long seed, const unsigned long long* w, const uint32_t* t, uint32_t* out,
                                    uint64_t n) {
  unsigned long long* dw;
  uint32_t* dt;
  uint4* dout;
  cudaMalloc(&dw, n * 8);
  cudaMalloc(&dt, n * 4);
  cudaMalloc(&dout, n * 16);
  cudaMemcpy(dw, w, n * 8, cudaMemcpyHostToDevice);
  cudaMemcpy(dt, t, n * 4, cudaMemcpyHostToDevice);
  k_stream<<<(unsigned)((n + 255) / 256), 256>>>(seed, dw, dt, dout, n);
  const cudaError_t e = cudaMemcpy(out, dout, n * 16, cudaMemcpyDeviceToHost);
  cudaFree(dw);
  cudaFree(dt);
  cudaFree(dout);
  return (int)e;
}
