// Microbenchmark (tuning aid, not product code): how fast can a 64 MiB device copy
// run right after an L2 flush (the bench regime) -- register-staged vector copies
// with U 16-byte loads in flight per thread vs a TMA bulk pipeline (cp.async.bulk
// global->shared with mbarrier completion, then shared->global bulk stores).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

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

// read-only stream (sum of words; result stored only to defeat dead-code elimination)
template <int U>
__global__ void __launch_bounds__(256) vread(const uint4* __restrict__ a, uint4* __restrict__ b, int64_t n) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t st = (int64_t)gridDim.x * blockDim.x;
  unsigned acc = 0;
  for (; i + (U - 1) * st < n; i += U * st) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; u++) v[u] = __ldcs(a + i + u * st);
#pragma unroll
    for (int u = 0; u < U; u++) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  if (acc == 0x12345678u) b[0] = make_uint4(acc, 0, 0, 0);
}
// software-pipelined copy: the loads of iteration k+1 are issued before the stores of k
template <int U>
__global__ void __launch_bounds__(256) vcopy_pipe(const uint4* __restrict__ a, uint4* __restrict__ b, int64_t n) {
  int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int64_t st = (int64_t)gridDim.x * blockDim.x;
  uint4 v[U], w[U];
  if (i + (U - 1) * st >= n) { for (; i < n; i += st) b[i] = a[i]; return; }
#pragma unroll
  for (int u = 0; u < U; u++) v[u] = __ldcs(a + i + u * st);
  for (;;) {
    const int64_t j = i + U * st;
    const bool more = j + (U - 1) * st < n;
    if (more) {
#pragma unroll
      for (int u = 0; u < U; u++) w[u] = __ldcs(a + j + u * st);
    }
#pragma unroll
    for (int u = 0; u < U; u++) __stcs(b + i + u * st, v[u]);
    i = j;
    if (!more) break;
#pragma unroll
    for (int u = 0; u < U; u++) v[u] = w[u];
  }
  for (; i < n; i += st) b[i] = a[i];
}
__global__ void empty_k() {}

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
// each CTA: NB stages of CH bytes; thread 0 issues bulk loads, waits, issues bulk stores
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
  int64_t c0 = blockIdx.x;
  const int64_t cs = gridDim.x;
  // prologue
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
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // stage s free again
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(mb + s)), "r"(CH));
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       sa(sm + (size_t)s * CH)), "l"(a + cn * CH), "r"(CH), "r"(sa(mb + s)) : "memory");
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main() {
  const int64_t n = 64ll << 20;
  uint8_t *a, *b, *fl;
  int* rd;
  cudaMalloc(&a, n);
  cudaMalloc(&b, n);
  cudaMalloc(&fl, 512 << 20);
  cudaMalloc(&rd, 512 << 20);
  cudaMemset(a, 1, n);
  cudaMemset(rd, 0, 512 << 20);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  auto run = [&](const char* nm, auto fn) {
    float best = 1e9;
    for (int r = 0; r < 13; r++) {
      cudaMemset(fl, r, 512 << 20);
      cudaMemcpy(fl, rd, 4, cudaMemcpyDeviceToDevice);
      cudaEventRecord(e0);
      fn();
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      if (r >= 3) best = ms < best ? ms : best;
    }
    cudaError_t er = cudaGetLastError();
    printf("%-40s %8.2f us  %7.0f GB/s (R+W)  %s\n", nm, best * 1e3, 2.0 * n / (best * 1e-3) / 1e9,
           er == cudaSuccess ? "" : cudaGetErrorString(er));
  };
  const int64_t nv = n / 16;
  run("empty kernel", [&] { empty_k<<<sms, 256>>>(); });
  run("cudaMemcpyAsync D2D 64 MiB", [&] { cudaMemcpyAsync(b, a, n, cudaMemcpyDeviceToDevice); });
  for (int occ : {4, 8}) {
    char nm[64];
    snprintf(nm, 64, "vread U=8 grid=%d/SM (GB/s = 2x read)", occ);
    run(nm, [&] { vread<8><<<sms * occ, 256>>>((const uint4*)a, (uint4*)b, nv); });
    snprintf(nm, 64, "vcopy_pipe U=4 grid=%d/SM", occ);
    run(nm, [&] { vcopy_pipe<4><<<sms * occ, 256>>>((const uint4*)a, (uint4*)b, nv); });
    snprintf(nm, 64, "vcopy_pipe U=8 grid=%d/SM", occ);
    run(nm, [&] { vcopy_pipe<8><<<sms * occ, 256>>>((const uint4*)a, (uint4*)b, nv); });
  }
  for (int occ : {4, 8}) {
    char nm[64];
    snprintf(nm, 64, "vcopy U=4 grid=%d/SM", occ);
    run(nm, [&] { vcopy<4><<<sms * occ, 256>>>((const uint4*)a, (uint4*)b, nv); });
    snprintf(nm, 64, "vcopy U=8 grid=%d/SM", occ);
    run(nm, [&] { vcopy<8><<<sms * occ, 256>>>((const uint4*)a, (uint4*)b, nv); });
    snprintf(nm, 64, "vcopy U=16 grid=%d/SM", occ);
    run(nm, [&] { vcopy<16><<<sms * occ, 256>>>((const uint4*)a, (uint4*)b, nv); });
  }
  for (int CH : {8192, 16384, 32768}) {
    for (int per : {1, 2, 4}) {
      const int NB = 4;
      size_t smem = (size_t)NB * CH;
      if (smem > 200 * 1024) continue;
      cudaFuncSetAttribute(tcopy<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, 220 * 1024);
      char nm[64];
      snprintf(nm, 64, "tma bulk CH=%d NB=4 ctas=%d/SM", CH, per);
      run(nm, [&] { tcopy<4><<<sms * per, 32, smem>>>(a, b, n, CH); });
    }
  }
  cudaMemset(b, 0, n);
  tcopy<4><<<sms, 32, 4 * 16384>>>(a, b, n, 16384);
  cudaDeviceSynchronize();
  uint8_t h[4];
  cudaMemcpy(h, b + n - 4, 4, cudaMemcpyDeviceToHost);
  printf("check %d\n", h[0]);
  return 0;
}
