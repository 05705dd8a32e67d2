// Microbenchmark (tuning aid, not product code): cost of partial-sector writes on
// B200 HBM3e.  Scatter 56-byte records (bytes 0..3 and 8..63 of 64-byte slots,
// the C5 particle layout) vs writing the whole 64-byte slot, for a sorted
// Bernoulli(1/2) subset of slots, and the dense (every slot) case.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <random>
#include <cuda_runtime.h>

__global__ void scatter(const uint4* __restrict__ pk, const int64_t* __restrict__ idx, int64_t n, uint8_t* dst,
                        int mode) {
  // thread t handles chunk t of the record stream: record r = t/4, chunk c = t%4
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (; t < n * 4; t += stride) {
    int64_t r = t >> 2;
    int c = (int)(t & 3);
    uint4 v = __ldcs(pk + t);  // (payload layout irrelevant for the timing)
    uint8_t* d = dst + idx[r] * 64 + 16 * c;
    if (mode == 0 || c != 0) {
      __stcs(reinterpret_cast<uint4*>(d), v);
    } else if (mode == 1) {  // bytes 0..3 and 8..15
      *reinterpret_cast<uint32_t*>(d) = v.x;
      *reinterpret_cast<uint2*>(d + 8) = make_uint2(v.z, v.w);
    }
  }
}

__global__ void gather(const uint8_t* src, const int64_t* __restrict__ idx, int64_t n, uint4* pk) {
  int64_t t = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (; t < n * 4; t += stride) {
    int64_t r = t >> 2;
    int c = (int)(t & 3);
    __stcs(pk + t, __ldcs(reinterpret_cast<const uint4*>(src + idx[r] * 64 + 16 * c)));
  }
}

int main() {
  const int64_t n = (1ll << 30) / 64;  // records selected
  for (int dense = 0; dense < 2; dense++) {
    std::vector<int64_t> h(n);
    std::mt19937_64 g(1234);
    int64_t k = 0;
    for (int64_t i = 0; k < n; i++)
      if (dense || (g() & 1)) h[k++] = i;
    const int64_t slots = h[n - 1] + 1;
    int64_t* idx;
    uint8_t* dst;
    uint4* pk;
    uint8_t* flush;
    cudaMalloc(&idx, n * 8);
    cudaMalloc(&dst, slots * 64);
    cudaMalloc(&pk, n * 64);
    cudaMalloc(&flush, 512 << 20);
    cudaMemcpy(idx, h.data(), n * 8, cudaMemcpyHostToDevice);
    cudaMemset(dst, 0, slots * 64);
    cudaMemset(pk, 1, n * 64);
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    for (int mode = 0; mode < 4; mode++) {
      float best = 1e9;
      for (int rep = 0; rep < 5; rep++) {
        cudaMemset(flush, rep, 512 << 20);
        cudaEventRecord(a);
        if (mode < 3) scatter<<<148 * 8, 256>>>(pk, idx, n, dst, mode);
        else gather<<<148 * 8, 256>>>(dst, idx, n, pk);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        best = ms < best ? ms : best;
      }
      const char* nm[] = {"scatter full 64B", "scatter 60B (gap 4..7)", "scatter 48B (chunk0 skipped)", "gather 64B"};
      printf("%s records=%lld %-30s %.1f us  (%.0f GB/s of 2x64B/record)\n", dense ? "dense " : "bern.5", (long long)n,
             nm[mode], best * 1e3, 2.0 * 64 * n / (best * 1e-3) / 1e9);
    }
    cudaFree(idx); cudaFree(dst); cudaFree(pk); cudaFree(flush);
  }
  return 0;
}
