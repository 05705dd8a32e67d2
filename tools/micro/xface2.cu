// Microbenchmark (tuning aid, not product code): DRAM bytes fetched per scattered
// 4-byte load on B200 for different load flavours (x-face pattern: 512x512 floats
// at pitch 2056 B / 1,056,784 B).  Run under ncu for dram__bytes_read.sum.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int L = 514;
template <int MODE>
__device__ __forceinline__ float ld(const float* p) {
  float v;
  if (MODE == 0) asm volatile("ld.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 1) asm volatile("ld.global.cs.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 2) asm volatile("ld.global.nc.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 3) asm volatile("ld.global.cg.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 4) asm volatile("ld.global.L1::no_allocate.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 5) asm volatile("ld.global.L2::64B.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 6) asm volatile("ld.volatile.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
  if (MODE == 7) asm volatile("ld.relaxed.gpu.global.f32 %0, [%1];" : "=f"(v) : "l"(p));
  return v;
}
template <int MODE>
__global__ void xface(const float* A, float* out) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= 512 * 512) return;
  int z = t >> 9, y = t & 511;
  out[t] = ld<MODE>(A + ((size_t)(z + 1) * L + (y + 1)) * L + 1);
}

int main(int argc, char** argv) {
  float* A;
  float* out;
  uint8_t* flush;
  size_t nA = (size_t)L * L * L;
  cudaMalloc(&A, nA * 4);
  cudaMalloc(&out, 1 << 20);
  cudaMalloc(&flush, 512 << 20);
  cudaMemset(A, 1, nA * 4);
  if (argc > 1) {
    cudaDeviceSetLimit(cudaLimitMaxL2FetchGranularity, atoi(argv[1]));
    size_t v;
    cudaDeviceGetLimit(&v, cudaLimitMaxL2FetchGranularity);
    printf("MaxL2FetchGranularity = %zu\n", v);
  }
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char* nm, auto fn) {
    float best = 1e9;
    for (int rep = 0; rep < 13; rep++) {
      cudaMemset(flush, rep, 512 << 20);
      cudaEventRecord(a);
      fn();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep >= 3) best = ms < best ? ms : best;
    }
    printf("%-28s best %.2f us\n", nm, best * 1e3);
  };
  run("ld.global", [&] { xface<0><<<1024, 256>>>(A, out); });
  run("ld.global.cs", [&] { xface<1><<<1024, 256>>>(A, out); });
  run("ld.global.nc", [&] { xface<2><<<1024, 256>>>(A, out); });
  run("ld.global.cg", [&] { xface<3><<<1024, 256>>>(A, out); });
  run("ld.global.L1::no_allocate", [&] { xface<4><<<1024, 256>>>(A, out); });
  run("ld.global.L2::64B", [&] { xface<5><<<1024, 256>>>(A, out); });
  run("ld.volatile.global", [&] { xface<6><<<1024, 256>>>(A, out); });
  run("ld.relaxed.gpu.global", [&] { xface<7><<<1024, 256>>>(A, out); });
  return 0;
}
