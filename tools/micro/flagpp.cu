// Microbenchmark (tuning aid, not product code): flag round trip between two CTAs
// on one GPU (the loopback ring's signalling), and a 2-CTA piece pipeline: CTA 0
// writes a piece of P bytes with 512 threads, barrier, publishes a flag; CTA 1
// waits, reads the piece, barrier, acks.  Variants: release/acquire at .sys and
// .gpu scope, and a fence.acq_rel.sys + relaxed store.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o flagpp flagpp.cu
#include <cuda_runtime.h>

#include <cstdint>
#include <cstdio>

template <int SC>
__device__ __forceinline__ uint64_t ldacq(const uint64_t* p) {
  uint64_t v;
  if (SC == 0) asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  else asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
template <int SC>
__device__ __forceinline__ void strel(uint64_t* p, uint64_t v) {
  if (SC == 0) asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else if (SC == 1) asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  else {
    asm volatile("fence.acq_rel.sys;" ::: "memory");
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
  }
}

// mode 0: flag ping-pong only; mode 1: piece pipeline with `depth` slots
template <int SC>
__global__ void __launch_bounds__(512, 1) pp(uint64_t* flags, uint4* ring, uint4* src, uint4* dst, int rounds,
                                             int piece16, int depth, int mode, unsigned long long* out) {
  uint64_t* ready = flags;
  uint64_t* ack = flags + 64;
  __shared__ int stop;
  const uint64_t t0 = clock64();
  for (int r = 0; r < rounds; r++) {
    const int slot = r % depth;
    if (blockIdx.x == 0) {  // sender
      if (threadIdx.x == 0 && r >= depth)
        while (ldacq<SC>(ack + slot) < (uint64_t)(r - depth + 1)) {
        }
      __syncthreads();
      if (mode) {
        uint4* d = ring + (size_t)slot * piece16;
        const uint4* s = src + (size_t)r * piece16;
        for (int i = threadIdx.x; i < piece16; i += blockDim.x) __stcs(d + i, __ldcs(s + i));
      }
      __syncthreads();
      if (threadIdx.x == 0) strel<SC>(ready + slot, (uint64_t)(r + 1));
    } else {  // receiver
      if (threadIdx.x == 0)
        while (ldacq<SC>(ready + slot) < (uint64_t)(r + 1)) {
        }
      __syncthreads();
      if (mode) {
        const uint4* s = ring + (size_t)slot * piece16;
        uint4* d = dst + (size_t)r * piece16;
        for (int i = threadIdx.x; i < piece16; i += blockDim.x) __stcs(d + i, __ldcg(s + i));
      }
      __syncthreads();
      if (threadIdx.x == 0) strel<SC>(ack + slot, (uint64_t)(r + 1));
    }
  }
  if (threadIdx.x == 0) out[blockIdx.x] = clock64() - t0;
  (void)stop;
}

int main() {
  uint64_t* flags;
  uint4 *ring, *src, *dst;
  unsigned long long* out;
  const int rounds = 2000;
  cudaMalloc(&flags, 4096);
  cudaMalloc(&ring, 64 << 20);
  cudaMalloc(&src, (size_t)512 << 20);
  cudaMalloc(&dst, (size_t)512 << 20);
  cudaMalloc(&out, 64);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const char* sn[] = {"rel/acq.sys", "rel/acq.gpu", "fence.sys+relaxed"};
  for (int sc = 0; sc < 3; sc++) {
    for (int mode = 0; mode < 2; mode++) {
      for (int piece : {32 << 10, 128 << 10}) {
        for (int depth : {1, 4}) {
          if (mode == 0 && (piece != (32 << 10) || depth != 1)) continue;
          const int n = mode ? std::min(rounds, (int)(((size_t)512 << 20) / piece)) : rounds;
          cudaMemset(flags, 0, 4096);
          cudaEventRecord(a);
          auto k = sc == 0 ? pp<0> : sc == 1 ? pp<1> : pp<2>;
          k<<<2, 512>>>(flags, ring, src, dst, n, piece / 16, depth, mode, out);
          cudaEventRecord(b);
          cudaEventSynchronize(b);
          float ms;
          cudaEventElapsedTime(&ms, a, b);
          if (cudaGetLastError() != cudaSuccess) { printf("error\n"); return 1; }
          printf("%-18s mode=%s piece=%6dK depth=%d: %.2f us per round, %.1f GB/s\n", sn[sc],
                 mode ? "pipe" : "flag", piece >> 10, depth, ms * 1e3 / n, mode ? (double)piece * n / (ms * 1e6) : 0.0);
        }
      }
    }
  }
  return 0;
}
