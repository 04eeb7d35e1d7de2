// conv_tc.cu — implicit-GEMM convolution / fully-connected layer on the sm_100a
// 5th-generation tensor cores (tcgen05.mma, fp32 accumulators in TMEM), with a fused
// epilogue: per-channel scale/shift (BN in inference form or bias, reading R12),
// residual add (ResNet unit), ReLU, RNE to bf16.
//
// This is S1 of SURVEY.md §8a: partial CNN inference f^_{i -> j} (Def 3.7,
// PAPER.md:138-141) is a chain of these TensorOps.  GEMM view per group g:
//   D[m, n] = sum_k A[m, k] * B[n, k],  m = output pixel (n_img, ho, wo),
//   n = output channel, k = (r*S + s)*Cg_in + c.
// Tile 128 x BN x 64; A (the implicit im2col of the NHWC activation) is gathered by
// 128 producer threads with 16-byte cp.async into the 128B-swizzled K-major layout,
// B (weights [Cout][Kp]) arrives by TMA with the same swizzle; one elected thread
// issues tcgen05.mma into TMEM; the 4 producer warps then drain TMEM (tcgen05.ld)
// through the epilogue.  mbarriers pipeline STAGES k-blocks.
#include <cudaTypedefs.h>

#include <cstring>
#include <mutex>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

struct ConvParams {
  const bf16* x;
  bf16* y;
  const bf16* res;
  const float* scale;
  const float* shift;
  int H, W, Cin, Ho, Wo, Cout, R, S, stride, pad, Cg_in, Cg_out, K, nkb, M, relu;
};

constexpr int BM = 128, BK = 64;
constexpr int kProducerThreads = 128;
constexpr int kThreads = kProducerThreads + 32;  // + 1 MMA warp
constexpr int kLag = 2;                           // cp.async groups in flight before arriving

template <int BN, int STAGES>
struct ConvSmem {
  static constexpr int kABytes = BM * BK * 2;  // 16 KB
  static constexpr int kBBytes = BN * BK * 2;
  static constexpr int kBarOff = STAGES * (kABytes + kBBytes);
  static constexpr int kBytes = kBarOff + (2 * STAGES + 1) * 8 + 16 + 1024;  // + alignment slack
};

template <int BN, int STAGES, bool kFast>
__global__ void __launch_bounds__(kThreads, 1)
    conv_tc_kernel(const __grid_constant__ CUtensorMap tmap_w, const ConvParams p) {
  using L = ConvSmem<BN, STAGES>;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t sA = base, sB = base + STAGES * L::kABytes;
  uint64_t* full = reinterpret_cast<uint64_t*>(gbase + L::kBarOff);
  uint64_t* empty = full + STAGES;
  uint64_t* tmem_full = empty + STAGES;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tmem_full + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int m0 = blockIdx.x * BM;
  const int n0 = blockIdx.y * BN;  // within the group
  const int g = blockIdx.z;

  if (threadIdx.x == 0) {
    for (int i = 0; i < STAGES; ++i) {
      mbar_init(&full[i], kProducerThreads + 1);
      mbar_init(&empty[i], 1);
    }
    mbar_init(tmem_full, 1);
    fence_mbar_init();
    tma_prefetch(&tmap_w);
  }
  if (warp == 4) tmem_alloc(tmem_slot, BN);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp < 4) {
    // ================= A producers (one output row each) + B TMA (thread 0) =================
    const int t = threadIdx.x;
    const int m = m0 + t;
    const bool mvalid = m < p.M;
    int nimg = 0, ho = 0, wo = 0;
    if (mvalid) {
      const int hw = p.Ho * p.Wo;
      nimg = m / hw;
      const int rem = m - nimg * hw;
      ho = rem / p.Wo;
      wo = rem - ho * p.Wo;
    }
    const bf16* xb = p.x + (size_t)nimg * p.H * p.W * p.Cin + (size_t)g * p.Cg_in;
    const int hi0 = ho * p.stride - p.pad, wi0 = wo * p.stride - p.pad;
    const uint32_t arow = (uint32_t)t * 128u;
    const uint32_t sw = (uint32_t)(t & 7);
    const int CC = p.Cg_in >> 3;  // 16-byte chunks per filter tap
    int fr = 0, fs = 0, fc = 0;   // fast-path filter position
    for (int kb = 0; kb < p.nkb; ++kb) {
      const int stage = kb % STAGES;
      if (kb >= STAGES) mbar_wait(&empty[stage], ((kb / STAGES) - 1) & 1);
      if (t == 0) {
        mbar_arrive_expect_tx(&full[stage], L::kBBytes);
        tma_load_2d(sB + stage * L::kBBytes, &tmap_w, kb * BK, g * p.Cg_out + n0, &full[stage]);
      }
      const uint32_t dst = sA + stage * L::kABytes + arow;
      if constexpr (kFast) {
        const int hi = hi0 + fr, wi = wi0 + fs;
        const bool ok = mvalid && hi >= 0 && hi < p.H && wi >= 0 && wi < p.W;
        const bf16* src = ok ? xb + ((size_t)hi * p.W + wi) * p.Cin + fc : p.x;
        const uint32_t nb = ok ? 16u : 0u;
#pragma unroll
        for (int j = 0; j < 8; ++j) cp_async_16(dst + (((uint32_t)j ^ sw) << 4), src + (ok ? j * 8 : 0), nb);
        fc += BK;
        if (fc == p.Cg_in) {
          fc = 0;
          if (++fs == p.S) {
            fs = 0;
            ++fr;
          }
        }
      } else {
#pragma unroll
        for (int j = 0; j < 8; ++j) {
          const int kc = kb * 8 + j;
          bool ok = mvalid && kc * 8 < p.K;
          const bf16* src = p.x;
          if (ok) {
            const int rs = kc / CC;
            const int cc = kc - rs * CC;
            const int r = rs / p.S;
            const int s = rs - r * p.S;
            const int hi = hi0 + r, wi = wi0 + s;
            ok = hi >= 0 && hi < p.H && wi >= 0 && wi < p.W;
            if (ok) src = xb + ((size_t)hi * p.W + wi) * p.Cin + cc * 8;
          }
          cp_async_16(dst + (((uint32_t)j ^ sw) << 4), src, ok ? 16u : 0u);
        }
      }
      cp_async_commit();
      if (kb >= kLag) {
        cp_async_wait<kLag>();
        fence_proxy_async_smem();
        mbar_arrive(&full[(kb - kLag) % STAGES]);
      }
    }
    cp_async_wait<0>();
    fence_proxy_async_smem();
    for (int kb = (p.nkb > kLag ? p.nkb - kLag : 0); kb < p.nkb; ++kb) mbar_arrive(&full[kb % STAGES]);

    // ================= epilogue: TMEM -> registers -> scale/shift/res/ReLU -> bf16 =================
    mbar_wait(tmem_full, 0);
    tc_fence_after();
    const int row = warp * 32 + lane;
    const int mo = m0 + row;
    const uint32_t taddr = tmem_base + ((uint32_t)(warp * 32) << 16);
#pragma unroll 1
    for (int cb = 0; cb < BN / 32; ++cb) {
      const int n = n0 + cb * 32;
      if (n >= p.Cg_out) break;  // warp-uniform
      uint32_t v[32];
      tmem_ld_32x32b_x32(taddr + cb * 32, v);
      tc_wait_ld();
      if (mo < p.M) {
        const int ng = g * p.Cg_out + n;
        const size_t off = (size_t)mo * p.Cout + ng;
        const int nvalid = p.Cg_out - n;  // >= 8, multiple of 8
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          if (q * 8 < nvalid) {
            const float4 sc0 = __ldg(reinterpret_cast<const float4*>(p.scale + ng + q * 8));
            const float4 sc1 = __ldg(reinterpret_cast<const float4*>(p.scale + ng + q * 8 + 4));
            const float4 sh0 = __ldg(reinterpret_cast<const float4*>(p.shift + ng + q * 8));
            const float4 sh1 = __ldg(reinterpret_cast<const float4*>(p.shift + ng + q * 8 + 4));
            float f[8];
            const float scv[8] = {sc0.x, sc0.y, sc0.z, sc0.w, sc1.x, sc1.y, sc1.z, sc1.w};
            const float shv[8] = {sh0.x, sh0.y, sh0.z, sh0.w, sh1.x, sh1.y, sh1.z, sh1.w};
#pragma unroll
            for (int j = 0; j < 8; ++j) f[j] = fmaf(__uint_as_float(v[q * 8 + j]), scv[j], shv[j]);
            if (p.res) {
              const uint4 rv = __ldg(reinterpret_cast<const uint4*>(p.res + off + q * 8));
              const uint32_t rr[4] = {rv.x, rv.y, rv.z, rv.w};
#pragma unroll
              for (int j = 0; j < 4; ++j) {
                const float2 a = unpack_bf16x2(rr[j]);
                f[2 * j] += a.x;
                f[2 * j + 1] += a.y;
              }
            }
            if (p.relu) {
#pragma unroll
              for (int j = 0; j < 8; ++j) f[j] = fmaxf(f[j], 0.0f);
            }
            uint4 o;
            o.x = pack_bf16x2(f[0], f[1]);
            o.y = pack_bf16x2(f[2], f[3]);
            o.z = pack_bf16x2(f[4], f[5]);
            o.w = pack_bf16x2(f[6], f[7]);
            *reinterpret_cast<uint4*>(p.y + off + q * 8) = o;
          }
        }
      }
    }
  } else if (lane == 0) {
    // ================= MMA issuer (single thread) =================
    constexpr uint32_t idesc = umma_idesc_bf16(BM, BN);
    for (int kb = 0; kb < p.nkb; ++kb) {
      const int stage = kb % STAGES;
      mbar_wait(&full[stage], (kb / STAGES) & 1);
      tc_fence_after();
      const uint32_t a0 = sA + stage * L::kABytes, b0 = sB + stage * L::kBBytes;
#pragma unroll
      for (int k = 0; k < BK / 16; ++k)
        tc_mma_bf16(tmem_base, umma_desc_k_sw128(a0 + k * 32), umma_desc_k_sw128(b0 + k * 32), idesc,
                    (kb | k) != 0 ? 1u : 0u);
      tc_commit(&empty[stage]);
    }
    tc_commit(tmem_full);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 4) tmem_dealloc(tmem_base, BN);
}

// ------------------------------------------------------------------------------------------
static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  });
  if (!fn) fail(5, "cuTensorMapEncodeTiled unavailable (driver too old or no GPU)");
  return fn;
}

static int pick_bn(int Cg_out) {
  if (Cg_out % 256 == 0) return 256;
  if (Cg_out % 128 == 0) return 128;
  if (Cg_out % 64 == 0) return 64;
  return 128;
}

void conv_layer_init(ConvLayer& L, const std::vector<uint16_t>& w, int Cin_real, const std::vector<float>& scale,
                     const std::vector<float>& shift) {
  if (L.Cin % L.groups || L.Cout % L.groups) fail(1, "conv: channels not divisible by groups");
  L.Cg_in = L.Cin / L.groups;
  L.Cg_out = L.Cout / L.groups;
  if (L.Cg_in % 8 || L.Cg_out % 8) fail(1, "conv: per-group channels must be multiples of 8");
  const int cg_real = Cin_real / L.groups;
  L.K = L.R * L.S * L.Cg_in;
  L.Kp = (L.K + BK - 1) / BK * BK;
  L.BN = pick_bn(L.Cg_out);
  // repack OHWI [Cout][R][S][cg_real] -> [Cout][Kp] with channel padding cg_real -> Cg_in and K padding
  std::vector<uint16_t> packed((size_t)L.Cout * L.Kp, 0);
  for (int o = 0; o < L.Cout; ++o)
    for (int r = 0; r < L.R; ++r)
      for (int s = 0; s < L.S; ++s)
        for (int c = 0; c < cg_real; ++c)
          packed[(size_t)o * L.Kp + (size_t)(r * L.S + s) * L.Cg_in + c] =
              w[(((size_t)o * L.R + r) * L.S + s) * cg_real + c];
  VCHECK(cudaMalloc(&L.w, packed.size() * 2));
  VCHECK(cudaMemcpy(L.w, packed.data(), packed.size() * 2, cudaMemcpyHostToDevice));
  VCHECK(cudaMalloc(&L.scale, L.Cout * sizeof(float)));
  VCHECK(cudaMalloc(&L.shift, L.Cout * sizeof(float)));
  VCHECK(cudaMemcpy(L.scale, scale.data(), L.Cout * sizeof(float), cudaMemcpyHostToDevice));
  VCHECK(cudaMemcpy(L.shift, shift.data(), L.Cout * sizeof(float), cudaMemcpyHostToDevice));
  cuuint64_t dims[2] = {(cuuint64_t)L.Kp, (cuuint64_t)L.Cout};
  cuuint64_t strides[1] = {(cuuint64_t)L.Kp * 2};
  cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)L.BN};
  cuuint32_t estr[2] = {1, 1};
  CUresult rc = get_encode()(&L.tmap_w, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, L.w, dims, strides, box, estr,
                             CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (rc != CUDA_SUCCESS) fail(5, "cuTensorMapEncodeTiled failed for conv weights");
}

void conv_layer_free(ConvLayer& L) {
  if (L.w) cudaFree(L.w);
  if (L.scale) cudaFree(L.scale);
  if (L.shift) cudaFree(L.shift);
  L.w = nullptr;
  L.scale = L.shift = nullptr;
}

template <int BN, int STAGES, bool kFast>
static void launch_t(const ConvLayer& L, const ConvParams& p, cudaStream_t st) {
  auto kern = conv_tc_kernel<BN, STAGES, kFast>;
  constexpr int smem = ConvSmem<BN, STAGES>::kBytes;
  static bool attr_set = false;  // per instantiation
  if (!attr_set) {
    VCHECK(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, smem));
    attr_set = true;
  }
  dim3 grid((p.M + BM - 1) / BM, (L.Cg_out + BN - 1) / BN, L.groups);
  kern<<<grid, kThreads, smem, st>>>(L.tmap_w, p);
  LAUNCHED();
}

void conv_forward(const ConvLayer& L, const bf16* x, int N, int H, int W, const bf16* res, bf16* y,
                  cudaStream_t st) {
  ConvParams p;
  p.x = x;
  p.y = y;
  p.res = res;
  p.scale = L.scale;
  p.shift = L.shift;
  p.H = H;
  p.W = W;
  p.Cin = L.Cin;
  p.Ho = conv_out_dim(H, L.R, L.stride, L.pad);
  p.Wo = conv_out_dim(W, L.S, L.stride, L.pad);
  p.Cout = L.Cout;
  p.R = L.R;
  p.S = L.S;
  p.stride = L.stride;
  p.pad = L.pad;
  p.Cg_in = L.Cg_in;
  p.Cg_out = L.Cg_out;
  p.K = L.K;
  p.nkb = L.Kp / BK;
  const int64_t M = (int64_t)N * p.Ho * p.Wo;
  if (M <= 0) return;
  if (M > INT32_MAX - BM) fail(1, "conv: M too large for one launch");
  p.M = (int)M;
  p.relu = L.relu ? 1 : 0;
  const bool fast = (L.Cg_in % BK) == 0;
  const double flops = 2.0 * (double)M * L.Cout * L.K;
  const double bytes = 2.0 * ((double)N * H * W * L.Cin + (double)M * L.Cout * (res ? 2 : 1) + (double)L.Cout * L.Kp);
  prof_begin(st);
  if (L.BN == 256) {
    if (fast) launch_t<256, 4, true>(L, p, st); else launch_t<256, 4, false>(L, p, st);
  } else if (L.BN == 128) {
    if (fast) launch_t<128, 4, true>(L, p, st); else launch_t<128, 4, false>(L, p, st);
  } else {
    if (fast) launch_t<64, 4, true>(L, p, st); else launch_t<64, 4, false>(L, p, st);
  }
  prof_end(st, 0, flops, bytes);
}

}  // namespace vista
