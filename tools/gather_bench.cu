// gather_bench.cu — measured roofline for random gathers on this B200.
// Each thread issues `iters` rounds of U independent random loads of `width` bytes (aligned) from
// a buffer of `bytes`, optionally as a dependent chain (the next address depends on the loaded
// value, like a walk step). Reports loads/s and useful GB/s; pair with ncu dram__bytes_read.sum to
// get the DRAM bytes actually moved per load (the DRAM access atom).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/gather_bench tools/gather_bench.cu
//   tools/gather_bench <bytes> <width 4|8|16|32|64> <U 1|2|4|8|16|32> <dependent 0|1> [iters] [blocks_per_sm] [mode]
// mode (width 16): 0 plain __ldg, 1 L2::64B, 3 L2 evict_first + L2::64B (the walk kernel's gather)
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#include <stdint.h>

__device__ __forceinline__ uint64_t mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

__device__ int g_mode;  // load flavour for 4-byte gathers (see ld4)

__device__ __forceinline__ uint32_t ld4(const uint32_t* p, int mode) {
  uint32_t v;
  switch (mode) {
    case 1: asm volatile("ld.global.nc.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    case 2: asm volatile("ld.global.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    case 3: {
      uint64_t pol;
      asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
      asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
      break;
    }
    case 4: asm volatile("ld.global.cs.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    case 5: asm volatile("ld.global.cg.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    case 6: asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    case 7: asm volatile("ld.global.nc.L1::no_allocate.L2::64B.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    case 8: asm volatile("ld.global.nc.L2::128B.u32 %0, [%1];" : "=r"(v) : "l"(p)); break;
    default: v = __ldg(p);
  }
  return v;
}

template <int WIDTH, int U, bool DEP>
__global__ void __launch_bounds__(256) k_gather(const uint4* __restrict__ buf, uint64_t slots, int iters,
                                                 unsigned long long* sink) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint64_t h[U];
#pragma unroll
  for (int u = 0; u < U; ++u) h[u] = mix(tid * 0x9E3779B97F4A7C15ULL + u + 1);
  uint32_t acc = 0;
  for (int i = 0; i < iters; ++i) {
    uint32_t got[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      // slot of WIDTH bytes: a mask for power-of-two slot counts, else a multiply-high reduction
      const uint64_t s = (slots & (slots - 1)) ? __umul64hi(h[u], slots) : (h[u] & (slots - 1));
      const char* p = (const char*)buf + s * WIDTH;
      uint32_t v;
      if (WIDTH == 4) v = ld4((const uint32_t*)p, g_mode);
      else if (WIDTH == 8) { uint2 t = __ldg((const uint2*)p); v = t.x ^ t.y; }
      else if (WIDTH == 16) {
        uint4 t;
        if (g_mode == 3) {  // the walk kernel's neighbour gather: L2 evict_first + 64-B fill
          uint64_t pol;
          asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
          asm volatile("ld.global.nc.L2::cache_hint.L2::64B.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
                       : "=r"(t.x), "=r"(t.y), "=r"(t.z), "=r"(t.w) : "l"(p), "l"(pol));
        } else if (g_mode == 1) {
          asm volatile("ld.global.nc.L2::64B.v4.u32 {%0, %1, %2, %3}, [%4];"
                       : "=r"(t.x), "=r"(t.y), "=r"(t.z), "=r"(t.w) : "l"(p));
        } else {
          t = __ldg((const uint4*)p);
        }
        v = t.x ^ t.y ^ t.z ^ t.w;
      }
      else {
        v = 0;
#pragma unroll
        for (int q = 0; q < WIDTH / 16; ++q) { uint4 t = __ldg((const uint4*)p + q); v ^= t.x ^ t.w; }
      }
      got[u] = v;
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      acc += got[u];
      // cheap next address (one IMAD + shift-xor): the benchmark must be bound by the gathers
      h[u] = DEP ? (h[u] * 0x9E3779B97F4A7C15ULL + got[u]) ^ (h[u] >> 29)
                 : (h[u] * 0x9E3779B97F4A7C15ULL + 0x632BE59BD9B4E019ULL) ^ (h[u] >> 29);
    }
  }
  if (acc == 0x12345678u) atomicAdd(sink, 1ull);
}

template <int WIDTH, int U, bool DEP>
float run(const uint4* buf, uint64_t bytes, int iters, int grid, unsigned long long* sink) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  k_gather<WIDTH, U, DEP><<<grid, 256>>>(buf, bytes / WIDTH, 2, sink);  // warm
  cudaEventRecord(a);
  k_gather<WIDTH, U, DEP><<<grid, 256>>>(buf, bytes / WIDTH, iters, sink);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  return ms;
}

template <int WIDTH>
float dispatch_u(int U, bool dep, const uint4* buf, uint64_t bytes, int iters, int grid, unsigned long long* s) {
  switch (U * 2 + (dep ? 1 : 0)) {
    case 2: return run<WIDTH, 1, false>(buf, bytes, iters, grid, s);
    case 3: return run<WIDTH, 1, true>(buf, bytes, iters, grid, s);
    case 4: return run<WIDTH, 2, false>(buf, bytes, iters, grid, s);
    case 5: return run<WIDTH, 2, true>(buf, bytes, iters, grid, s);
    case 8: return run<WIDTH, 4, false>(buf, bytes, iters, grid, s);
    case 9: return run<WIDTH, 4, true>(buf, bytes, iters, grid, s);
    case 32: return run<WIDTH, 16, false>(buf, bytes, iters, grid, s);
    case 64: return run<WIDTH, 32, false>(buf, bytes, iters, grid, s);
    default: return run<WIDTH, 8, false>(buf, bytes, iters, grid, s);
  }
}

int main(int argc, char** argv) {
  uint64_t bytes = argc > 1 ? strtoull(argv[1], 0, 10) : (16ull << 30);
  if (bytes % 64) { printf("bytes must be a multiple of 64\n"); return 1; }
  int width = argc > 2 ? atoi(argv[2]) : 4;
  int U = argc > 3 ? atoi(argv[3]) : 4;
  int dep = argc > 4 ? atoi(argv[4]) : 0;
  int iters = argc > 5 ? atoi(argv[5]) : 64;
  int bps = argc > 6 ? atoi(argv[6]) : 8;
  int mode = argc > 7 ? atoi(argv[7]) : 0;
  cudaMemcpyToSymbol(g_mode, &mode, sizeof(int));
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  uint4* buf = nullptr;
  unsigned long long* sink = nullptr;
  if (cudaMalloc(&buf, bytes) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  cudaMemset(buf, 1, bytes);
  cudaMalloc(&sink, 8);
  int grid = sms * bps;
  float ms = 0;
  switch (width) {
    case 4: ms = dispatch_u<4>(U, dep, buf, bytes, iters, grid, sink); break;
    case 8: ms = dispatch_u<8>(U, dep, buf, bytes, iters, grid, sink); break;
    case 16: ms = dispatch_u<16>(U, dep, buf, bytes, iters, grid, sink); break;
    case 32: ms = dispatch_u<32>(U, dep, buf, bytes, iters, grid, sink); break;
    default: ms = dispatch_u<64>(U, dep, buf, bytes, iters, grid, sink); break;
  }
  double loads = (double)grid * 256 * iters * U;
  printf("{\"mode\": %d, \"bytes\": %llu, \"width\": %d, \"U\": %d, \"dependent\": %d, \"blocks_per_sm\": %d, \"ms\": %.3f, "
         "\"gloads_per_s\": %.3f, \"useful_gbs\": %.1f, \"sector_gbs\": %.1f}\n",
         mode, (unsigned long long)bytes, width, U, dep, bps, ms, loads / ms / 1e6, loads * width / ms / 1e6,
         loads * (width < 32 ? 32 : width) / ms / 1e6);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) printf("err %s\n", cudaGetErrorString(e));
  return 0;
}
