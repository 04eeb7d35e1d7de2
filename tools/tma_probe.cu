// tma_probe.cu — microbenchmark: TMA load throughput per SM for the operand layouts of the conv kernels.
//   plain2d : 2-D tiled box {64 bf16, 128 rows}, 128B swizzle (1x1 conv / FC A operand)
//   rowview : 4-D overlapping row view {64, 128 pixels (32 B stride), 1, 1} (ResNet conv1 s2d A operand)
//   rowview4: the same 16 KB as four 32-pixel boxes
// Each CTA (one per SM) keeps `depth` loads in flight into a ring of 16 KB slots; prints GB/s.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -I paper_conf_sigmod_nakandalak20_b200/csrc
//        -o tools/tma_probe tools/tma_probe.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>

#include <cstdio>
#include <vector>

#include "ptx.cuh"

using namespace vista;

__global__ void __launch_bounds__(32, 1)
    tma_kernel(const __grid_constant__ CUtensorMap m, int mode, int iters, int depth, int rows_total) {
  extern __shared__ __align__(1024) uint8_t smem[];
  const uint32_t base = (smem_u32(smem) + 1023u) & ~1023u;
  __shared__ uint64_t bar[16];
  if (threadIdx.x != 0) return;
  for (int i = 0; i < depth; ++i) mbar_init(&bar[i], 1);
  fence_mbar_init();
  for (int i = 0; i < iters; ++i) {
    const int slot = i % depth;
    if (i >= depth) mbar_wait(&bar[slot], ((i / depth) - 1) & 1);
    mbar_arrive_expect_tx(&bar[slot], 16384);
    const int r = (blockIdx.x * 7919 + i * 13) % rows_total;
    const uint32_t dst = base + slot * 16384;
    if (mode == 0) {
      tma_load_2d(dst, &m, 0, (r * 128) % (rows_total * 128 - 128), &bar[slot]);
    } else if (mode == 1) {
      tma_load_4d(dst, &m, 0, 0, r % 117, (r / 117) % 64, &bar[slot]);
    } else {
      for (int k = 0; k < 4; ++k) tma_load_4d(dst + k * 4096, &m, 0, k * 32, r % 117, (r / 117) % 64, &bar[slot]);
    }
  }
  for (int i = iters - depth; i < iters; ++i)
    if (i >= 0) mbar_wait(&bar[i % depth], (i / depth) & 1);
}

int main() {
  PFN_cuTensorMapEncodeTiled_v12000 enc = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  // 64 images of the space-to-depth input [64, 117, 117, 16] bf16 (56 MB) and a [rows, 64] matrix
  const int N = 64, H = 117, W = 117, C = 16;
  void* x = nullptr;
  cudaMalloc(&x, (size_t)N * H * W * C * 2);
  cudaMemset(x, 0, (size_t)N * H * W * C * 2);
  CUtensorMap m2, m4, m4s;
  {
    cuuint64_t dims[2] = {64, (cuuint64_t)N * H * W * C / 64};
    cuuint64_t str[1] = {128};
    cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
    enc(&m2, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, x, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  }
  for (int variant = 0; variant < 2; ++variant) {
    cuuint64_t dims[4] = {64, 114, (cuuint64_t)H, (cuuint64_t)N};
    cuuint64_t str[3] = {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, (cuuint64_t)H * W * C * 2};
    cuuint32_t box[4] = {64, variant == 0 ? 128u : 32u, 1, 1}, es[4] = {1, 1, 1, 1};
    CUresult rc = enc(variant == 0 ? &m4 : &m4s, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, x, dims, str, box, es,
                      CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                      CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    if (rc != CUDA_SUCCESS) printf("encode rowview variant %d failed: %d\n", variant, (int)rc);
  }
  const int smem = 8 * 16384 + 2048;
  cudaFuncSetAttribute(tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  const char* names[3] = {"plain2d", "rowview", "rowview4"};
  for (int mode = 0; mode < 3; ++mode)
    for (int depth : {1, 2, 4, 8}) {
      const int iters = 2000;
      const CUtensorMap& m = mode == 0 ? m2 : (mode == 1 ? m4 : m4s);
      const int rows_total = mode == 0 ? N * H * W * C / 64 / 128 : N * H;
      tma_kernel<<<sms, 32, smem>>>(m, mode, 50, depth, rows_total);
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a);
      tma_kernel<<<sms, 32, smem>>>(m, mode, iters, depth, rows_total);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms = 0;
      cudaEventElapsedTime(&ms, a, b);
      const double bytes = 16384.0 * iters * sms;
      printf("%-9s depth %d: %8.1f GB/s total, %6.2f us per 16 KB load per SM  (%s)\n", names[mode], depth,
             bytes / (ms * 1e-3) / 1e9, ms * 1e3 / iters * depth, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
