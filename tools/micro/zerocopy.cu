// Microbenchmark (tuning aid, not product code): zero-copy traffic over the host link
// from SM loads/stores vs TMA bulk copies, against cudaMemcpyAsync, pinned host memory.
//   read:  host (pinned, mapped) -> device      write: device -> host
//   both:  a kernel that reads host and writes host at once (the pack_host traffic)
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int U>
__global__ void __launch_bounds__(256) vcopy(const uint4* __restrict__ a, uint4* __restrict__ b, int64_t n) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t st = (int64_t)gridDim.x * blockDim.x;
  for (; i + (U - 1) * st < n; i += U * st) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; u++) v[u] = __ldcs(a + i + u * st);
#pragma unroll
    for (int u = 0; u < U; u++) __stcs(b + i + u * st, v[u]);
  }
  for (; i < n; i += st) b[i] = a[i];
}

// one warp per CTA, lane 0 drives NB stages of CH bytes: bulk load -> bulk store
template <int NB>
__global__ void __launch_bounds__(32) tcopy(const uint8_t* a, uint8_t* b, int64_t nbytes, int CH) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ uint64_t mb[NB];
  const int64_t nch = nbytes / CH;
  if (threadIdx.x == 0) {
    for (int s = 0; s < NB; s++) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(mb + s)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncwarp();
  if (threadIdx.x != 0) return;
  const int64_t c0 = blockIdx.x, cs = gridDim.x;
  int k = 0;
  for (int64_t c = c0; c < nch && k < NB; c += cs, k++) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(mb + k)), "r"(CH));
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     sa(sm + (size_t)k * CH)), "l"(a + c * CH), "r"(CH), "r"(sa(mb + k)) : "memory");
  }
  int it = 0;
  for (int64_t c = c0; c < nch; c += cs, it++) {
    const int s = it % NB;
    const uint32_t par = (it / NB) & 1;
    asm volatile("{\n.reg .pred p;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W;\n}\n" ::"r"(
                     sa(mb + s)), "r"(par) : "memory");
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(b + c * CH), "r"(sa(sm + (size_t)s * CH)),
                 "r"(CH) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    const int64_t cn = c + (int64_t)NB * cs;
    if (cn < nch) {
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(mb + s)), "r"(CH));
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       sa(sm + (size_t)s * CH)), "l"(a + cn * CH), "r"(CH), "r"(sa(mb + s)) : "memory");
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main() {
  const int64_t n = 64ll << 20;
  uint8_t *h1, *h2, *d1, *d2, *hd1, *hd2;
  cudaHostAlloc(&h1, n, cudaHostAllocMapped);
  cudaHostAlloc(&h2, n, cudaHostAllocMapped);
  cudaHostGetDevicePointer((void**)&hd1, h1, 0);
  cudaHostGetDevicePointer((void**)&hd2, h2, 0);
  cudaMalloc(&d1, n);
  cudaMalloc(&d2, n);
  for (int64_t i = 0; i < n; i += 4096) h1[i] = (uint8_t)i;
  cudaMemset(d1, 1, n);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaStream_t s1, s2;
  cudaStreamCreate(&s1);
  cudaStreamCreate(&s2);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto run = [&](const char* nm, double bytes, auto fn) {
    float best = 1e9;
    for (int r = 0; r < 6; r++) {
      cudaDeviceSynchronize();
      cudaEventRecord(e0);
      fn();
      cudaEventRecord(e1);
      cudaDeviceSynchronize();
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (r) best = ms < best ? ms : best;
    }
    cudaError_t er = cudaGetLastError();
    printf("%-52s %9.1f us  %6.1f GB/s  %s\n", nm, best * 1e3, bytes / (best * 1e-3) / 1e9,
           er == cudaSuccess ? "" : cudaGetErrorString(er));
  };
  const int64_t nv = n / 16;
  cudaFuncSetAttribute(tcopy<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
  run("memcpy H2D", n, [&] { cudaMemcpyAsync(d1, h1, n, cudaMemcpyHostToDevice, 0); });
  run("memcpy D2H", n, [&] { cudaMemcpyAsync(h2, d1, n, cudaMemcpyDeviceToHost, 0); });
  run("memcpy H2D || D2H (bytes = both)", 2.0 * n, [&] {
    cudaEventRecord(e0, s1);
    cudaMemcpyAsync(d1, h1, n, cudaMemcpyHostToDevice, s1);
    cudaMemcpyAsync(h2, d2, n, cudaMemcpyDeviceToHost, s2);
    cudaStreamSynchronize(s1);
    cudaStreamSynchronize(s2);
  });
  for (int occ : {2, 8}) {
    char nm[96];
    snprintf(nm, 96, "LDG read host->dev U=8 grid=%d/SM", occ);
    run(nm, n, [&] { vcopy<8><<<sms * occ, 256>>>((const uint4*)hd1, (uint4*)d1, nv); });
    snprintf(nm, 96, "STG write dev->host U=8 grid=%d/SM", occ);
    run(nm, n, [&] { vcopy<8><<<sms * occ, 256>>>((const uint4*)d1, (uint4*)hd2, nv); });
    snprintf(nm, 96, "LDG/STG host->host U=8 grid=%d/SM (bytes = both)", occ);
    run(nm, 2.0 * n, [&] { vcopy<8><<<sms * occ, 256>>>((const uint4*)hd1, (uint4*)hd2, nv); });
  }
  for (int CH : {4096, 16384}) {
    for (int per : {1, 4}) {
      char nm[96];
      const size_t smem = 4 * (size_t)CH;
      snprintf(nm, 96, "TMA read host->dev CH=%d ctas=%d/SM", CH, per);
      run(nm, n, [&] { tcopy<4><<<sms * per, 32, smem>>>(hd1, d1, n, CH); });
      snprintf(nm, 96, "TMA write dev->host CH=%d ctas=%d/SM", CH, per);
      run(nm, n, [&] { tcopy<4><<<sms * per, 32, smem>>>(d1, hd2, n, CH); });
      snprintf(nm, 96, "TMA host->host CH=%d ctas=%d/SM (bytes = both)", CH, per);
      run(nm, 2.0 * n, [&] { tcopy<4><<<sms * per, 32, smem>>>(hd1, hd2, n, CH); });
    }
  }
  return 0;
}
