// Microbenchmark (tuning aid, not product code): floor of the C4 x-face gather
// (512 x 512 floats at pitch 2056 B in y and 1,056,784 B in z) on B200, vs an
// empty kernel and a contiguous 1 MiB copy, all event-timed after an L2 flush.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int L = 514;
__global__ void empty_k() {}
__global__ void copy_k(const uint4* a, uint4* b, int n) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) b[i] = a[i];
}
// thread per EPT consecutive (y) elements; output coalesced
template <int EPT>
__global__ void xface_k(const float* A, float* out) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;  // group of EPT outputs
  int e0 = t * EPT;
  if (e0 >= 512 * 512) return;
  float v[EPT];
#pragma unroll
  for (int k = 0; k < EPT; k++) {
    int e = e0 + k, z = e >> 9, y = e & 511;
    v[k] = __ldcs(A + ((size_t)(z + 1) * L + (y + 1)) * L + 1);
  }
#pragma unroll
  for (int k = 0; k < EPT; k++) out[e0 + k] = v[k];
}
// transposed assignment: consecutive threads take consecutive z (different 1 MB planes)
__global__ void xface_zmajor(const float* A, float* out) {
  int t = blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= 512 * 512) return;
  int z = t & 511, y = t >> 9;
  out[z * 512 + y] = __ldcs(A + ((size_t)(z + 1) * L + (y + 1)) * L + 1);
}

int main() {
  float* A;
  float* out;
  uint8_t* flush;
  size_t nA = (size_t)L * L * L;
  cudaMalloc(&A, nA * 4);
  cudaMalloc(&out, 1 << 20);
  cudaMalloc(&flush, 512 << 20);
  cudaMemset(A, 1, nA * 4);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  auto run = [&](const char* nm, auto fn) {
    float best = 1e9, sum = 0;
    for (int rep = 0; rep < 23; rep++) {
      cudaMemset(flush, rep, 512 << 20);
      cudaEventRecord(a);
      fn();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      if (rep >= 3) { best = ms < best ? ms : best; sum += ms; }
    }
    printf("%-34s best %.2f us  mean %.2f us  (%.0f GB/s R+W of 1 MiB payload at best)\n", nm, best * 1e3,
           sum / 20 * 1e3, 2.0 * (1 << 20) / (best * 1e-3) / 1e9);
  };
  run("empty kernel", [&] { empty_k<<<1, 32>>>(); });
  run("contiguous copy 1 MiB", [&] { copy_k<<<256, 256>>>((const uint4*)A, (uint4*)out, 65536); });
  run("x-face 1 elem/thread", [&] { xface_k<1><<<1024, 256>>>(A, out); });
  run("x-face 4 elem/thread", [&] { xface_k<4><<<256, 256>>>(A, out); });
  run("x-face 8 elem/thread", [&] { xface_k<8><<<128, 256>>>(A, out); });
  run("x-face 16 elem/thread", [&] { xface_k<16><<<64, 256>>>(A, out); });
  run("x-face z-major", [&] { xface_zmajor<<<1024, 256>>>(A, out); });
  return 0;
}
