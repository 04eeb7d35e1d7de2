// mma_probe.cu — microbenchmark: tcgen05.mma.cta_group::1.kind::f16 issue rate vs N (SS mode, operands
// resident in shared memory, no loads).  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
//   -I paper_conf_sigmod_nakandalak20_b200/csrc -o tools/mma_probe tools/mma_probe.cu
// Prints cycles per MMA (M = 128, K = 16) for N = 64 / 128 / 256, one CTA and all SMs.
#include <cstdio>

#include "ptx.cuh"

using namespace vista;

template <int N>
__global__ void __launch_bounds__(128, 1) probe(int iters, unsigned long long* out, int ashift, int alt = 1, int rnd = 0) {
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
  for (int i = threadIdx.x; i < (256 + N) * 128 / 16; i += blockDim.x) {
    uint4 v = make_uint4(0, 0, 0, 0);
    if (rnd) {  // random bf16 values in [-2, 2): a hash of the index
      uint32_t h[4];
      for (int k = 0; k < 4; ++k) {
        uint32_t x = (uint32_t)(i * 4 + k) * 2654435761u + 12345u;
        x ^= x >> 13;
        x *= 0x5bd1e995u;
        x ^= x >> 15;
        h[k] = (x & 0x807F807Fu) | 0x3F803F80u;  // sign, mantissa random; exponent ~ 1
      }
      v = make_uint4(h[0], h[1], h[2], h[3]);
    }
    sts128(base + i * 16, v);
  }
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

// distinct operands per MMA (as in a real K loop): A walks 8 k-blocks of 128 x 64 (128 KB), B 8 k-blocks of
// N x 64; every MMA reads smem it has not read in the previous 31 MMAs
template <int N>
__global__ void __launch_bounds__(128, 1) probe_stream(int iters, unsigned long long* out, int halo) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t base = (smem_u32(smem) + 1023u) & ~1023u;
  const uint32_t sA = base, sB = base + 8 * 16384;
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    mbar_init(&bar, 1);
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < (8 * 16384 + 8 * N * 128) / 16; i += blockDim.x) {
    uint32_t x = (uint32_t)i * 2654435761u + 777u;
    x ^= x >> 13;
    x *= 0x5bd1e995u;
    sts128(base + i * 16, make_uint4((x & 0x807F807Fu) | 0x3F803F80u, (x * 3u & 0x807F807Fu) | 0x3F803F80u,
                                     (x * 5u & 0x807F807Fu) | 0x3F803F80u, (x * 7u & 0x807F807Fu) | 0x3F803F80u));
  }
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
      for (int kb = 0; kb < 8; ++kb)
#pragma unroll
        for (int k = 0; k < 4; ++k)
          tc_mma_bf16(tmem,
                      umma_desc_k_sw128(halo ? sA + (37 + (kb / 3) * 58 + kb % 3) * 128 + k * 32
                                             : sA + kb * 16384 + k * 32),
                      umma_desc_k_sw128(sB + kb * N * 128 + k * 32), idesc, 1u);
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

template <int N>
void run_stream(int grid, int halo = 0) {
  unsigned long long* d;
  cudaMalloc(&d, 8);
  const int iters = 2000;
  const int smem = 8 * 16384 + 8 * N * 128 + 2048;
  cudaFuncSetAttribute(probe_stream<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  probe_stream<N><<<grid, 128, smem>>>(10, d, halo);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  probe_stream<N><<<grid, 128, smem>>>(iters, d, halo);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  unsigned long long cyc = 0;
  cudaMemcpy(&cyc, d, 8, cudaMemcpyDeviceToHost);
  const double mmas = 32.0 * iters;
  printf("stream N=%3d grid=%3d halo=%d: %.1f cycles/MMA, %.0f TFLOP/s  err=%s\n", N, grid, halo, cyc / mmas,
         2.0 * 128 * N * 16 * mmas * grid / (ms * 1e-3) / 1e12, cudaGetErrorString(cudaGetLastError()));
  cudaFree(d);
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
void run(int grid, int ashift = 0, int alt = 1, int rnd = 0) {
  unsigned long long* d;
  cudaMalloc(&d, 8);
  const int iters = 20000;
  const int smem = (256 + N) * 128 + 2048;
  cudaFuncSetAttribute(probe<N>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  probe<N><<<grid, 128, smem>>>(100, d, ashift, alt, rnd);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  cudaEventRecord(a);
  probe<N><<<grid, 128, smem>>>(iters, d, ashift, alt, rnd);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms = 0;
  cudaEventElapsedTime(&ms, a, b);
  unsigned long long cyc = 0;
  cudaMemcpy(&cyc, d, 8, cudaMemcpyDeviceToHost);
  const double mmas = 4.0 * iters;
  const double tflops = 2.0 * 128 * N * 16 * mmas * grid / (ms * 1e-3) / 1e12;
  printf("N=%3d grid=%3d ashift=%3d alt=%d rnd=%d: %.1f cycles/MMA (block 0), %.3f ms, %.0f TFLOP/s  err=%s\n", N, grid, ashift, alt, rnd, cyc / mmas, ms,
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
  for (int g : {1, sms}) {
    run_stream<64>(g);
    run_stream<64>(g, 1);  // A = row-shifted windows of one buffer (the halo 3x3 taps)
  }
  // random operand values (zeros above): data-dependent MMA throughput / power
  for (int g : {1, sms}) {
    run<64>(g, 0, 0, 1);
    run<128>(g, 0, 0, 1);
    run<256>(g, 0, 0, 1);
  }
  for (int sh : {1, 59}) {
    run<64>(1, sh);
    run<128>(1, sh);
    run<256>(1, sh);
  }
  return 0;
}
