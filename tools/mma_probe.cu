// mma_probe.cu — microbenchmark: tcgen05.mma.cta_group::1.kind::f16 issue rate vs N (SS mode, operands
// resident in shared memory, no loads).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
//   -I paper_conf_sigmod_nakandalak20_b200/csrc -o tools/mma_probe tools/mma_probe.cu
// Prints cycles per MMA (M = 128, K = 16) for N = 64 / 128 / 256, one CTA and all SMs.
#include <cstdio>

#include "ptx.cuh"

using namespace vista;

template <int N>
__global__ void __launch_bounds__(128, 1) probe(int iters, unsigned long long* out, int ashift, int alt = 1) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t base = (smem_u32(smem) + 1023u) & ~1023u;
  // A: 128 x 64 bf16 starting ashift 128-byte rows into a 256-row buffer (halo-style row-shifted operand),
  // B: N x 64 bf16 (zeros are fine)
  const uint32_t sA = base + ashift * 128, sB = base + 256 * 128;
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < (256 + N) * 128 / 16; i += blockDim.x) sts128(base + i * 16, make_uint4(0, 0, 0, 0));
  fence_proxy_async_smem();
  if (warp == 0) tmem_alloc(&slot, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = slot;
  if (threadIdx.x == 0) {
    constexpr uint32_t idesc = umma_idesc_bf16(128, N);
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int k = 0; k < 4; ++k)
        tc_mma_bf16(tmem + (alt ? (i & 1) * N : 0), umma_desc_k_sw128(sA + k * 32), umma_desc_k_sw128(sB + k * 32), idesc,
                    1u);
    }
    tc_commit(&bar);
    mbar_wait(&bar, 0);
    const long long t1 = clock64();
    if (blockIdx.x == 0) out[0] = (unsigned long long)(t1 - t0);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, 512);
}

// commit latency / throughput: (a) commit then wait on the same barrier, repeated; (b) MMA + commit + wait
__global__ void __launch_bounds__(128, 1) commit_probe(int iters, int with_mma, unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t base = (smem_u32(smem) + 1023u) & ~1023u;
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < (128 + 64) * 128 / 16; i += blockDim.x) sts128(base + i * 16, make_uint4(0, 0, 0, 0));
  fence_proxy_async_smem();
  if (warp == 0) tmem_alloc(&slot, 512);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = slot;
  if (threadIdx.x == 0) {
    constexpr uint32_t idesc = umma_idesc_bf16(128, 64);
    const long long t0 = clock64();
    if (with_mma < 2) {
      for (int i = 0; i < iters; ++i) {
        if (with_mma)
          tc_mma_bf16(tmem, umma_desc_k_sw128(base), umma_desc_k_sw128(base + 16384), idesc, 1u);
        tc_commit(&bar);
        mbar_wait(&bar, i & 1);
      }
    } else {  // back-to-back commits without waiting (2: commits only, 3: 8 MMAs + 1 commit per iteration)
      for (int i = 0; i < iters; ++i) {
        if (with_mma == 3)
          for (int k = 0; k < 8; ++k)
            tc_mma_bf16(tmem, umma_desc_k_sw128(base), umma_desc_k_sw128(base + 16384), idesc, 1u);
        tc_commit(&bar);
      }
      mbar_wait(&bar, (iters - 1) & 1);
    }
    const long long t1 = clock64();
    if (blockIdx.x == 0) out[0] = (unsigned long long)(t1 - t0);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) tmem_dealloc(tmem, 512);
}

template <int N>
void run(int grid, int ashift = 0, int alt = 1) {
  unsigned long long* d;
  cudaMalloc(&d, 8);
  const int iters = 20000;
  const int smem = (256 + N) * 128 + 2048;
  cudaFuncSetAttribute(probe<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  probe<N><<<grid, 128, smem>>>(100, d, ashift, alt);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  probe<N><<<grid, 128, smem>>>(iters, d, ashift, alt);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  unsigned long long cyc = 0;
  cudaMemcpy(&cyc, d, 8, cudaMemcpyDeviceToHost);
  const double mmas = 4.0 * iters;
  const double tflops = 2.0 * 128 * N * 16 * mmas * grid / (ms * 1e-3) / 1e12;
  printf("N=%3d grid=%3d ashift=%3d alt=%d: %.1f cycles/MMA (block 0), %.3f ms, %.0f TFLOP/s  err=%s\n", N, grid, ashift, alt, cyc / mmas, ms,
         tflops, cudaGetErrorString(cudaGetLastError()));
  cudaFree(d);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  {
    unsigned long long* d;
    cudaMalloc(&d, 8);
    cudaFuncSetAttribute(commit_probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    const char* what[4] = {"commit+wait round trip", "MMA+commit+wait round trip", "back-to-back commit",
                           "8 MMA (N=64) + commit, no wait"};
    for (int m = 0; m < 4; ++m) {
      commit_probe<<<1, 128, 64 * 1024>>>(1000, m, d);
      cudaDeviceSynchronize();
      unsigned long long cyc = 0;
      cudaMemcpy(&cyc, d, 8, cudaMemcpyDeviceToHost);
      printf("%s: %.0f cycles per iteration\n", what[m], cyc / 1000.0);
    }
  }
  for (int g : {1, sms}) {
    run<64>(g);
    run<128>(g);
    run<256>(g);
  }
  // row-shifted A operands (A_HALO): does a start that is not a multiple of 8 rows cost smem bandwidth?
  // one accumulator for every MMA (a conv tile's whole K loop) vs alternating two
  for (int g : {1, sms}) {
    run<64>(g, 0, 0);
    run<128>(g, 0, 0);
    run<256>(g, 0, 0);
  }
  for (int sh : {1, 59}) {
    run<64>(1, sh);
    run<128>(1, sh);
    run<256>(1, sh);
  }
  return 0;
}
