// conv_f32.cu — the fp32 check mode of S1 (reading R23 in DESIGN.md): fp32
// storage and fp32 SIMT FFMA accumulation for every conv / FC layer.  TF32 tensor cores are not
// accurate enough for the 1e-4 check tolerance (measured 1.7e-4..2.4e-4 normwise),
// so this path deliberately stays on the CUDA cores; it is a verification mode, not the product path.
//
// Implicit GEMM per group g: D[m, n] = sum_k A[m, k] B[n, k], m = output pixel, n = output channel,
// k = (r*S + s)*Cg_in + c; tile 128 x 64 x 16 in shared memory, 256 threads x (8 x 4) outputs.
#include "internal.h"

namespace vista {

constexpr int FBM = 128, FBN = 64, FBK = 16;

struct ConvF32Params {
  const float* x;
  float* y;
  const float* res;
  const float* w;  // [Cout][K]
  const float* scale;
  const float* shift;
  int H, W, Cin, Ho, Wo, Cout, R, S, stride, pad, Cg_in, Cg_out, K, M, relu;
};

__global__ void __launch_bounds__(256) conv_f32_kernel(const ConvF32Params p) {
  __shared__ float As[FBK][FBM + 4];
  __shared__ float Bs[FBK][FBN + 4];
  const int tid = threadIdx.x;
  const int m0 = blockIdx.x * FBM, n0 = blockIdx.y * FBN, g = blockIdx.z;
  const int tm = (tid / 16) * 8, tn = (tid % 16) * 4;  // this thread's 8 x 4 outputs
  float acc[8][4];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[i][j] = 0.f;
  const int hw = p.Ho * p.Wo;
  for (int k0 = 0; k0 < p.K; k0 += FBK) {
    // A tile: 128 rows x 16 k (2048 elements, 8 per thread), implicit im2col with zero padding
    for (int e = tid; e < FBM * FBK; e += 256) {
      const int mm = e / FBK, kk = e % FBK;
      const int m = m0 + mm, k = k0 + kk;
      float v = 0.f;
      if (m < p.M && k < p.K) {
        const int nimg = m / hw, rem = m - nimg * hw;
        const int ho = rem / p.Wo, wo = rem - ho * p.Wo;
        const int rs = k / p.Cg_in, c = k - rs * p.Cg_in;
        const int r = rs / p.S, s = rs - r * p.S;
        const int hi = ho * p.stride - p.pad + r, wi = wo * p.stride - p.pad + s;
        if (hi >= 0 && hi < p.H && wi >= 0 && wi < p.W)
          v = p.x[(((size_t)nimg * p.H + hi) * p.W + wi) * p.Cin + (size_t)g * p.Cg_in + c];
      }
      As[kk][mm] = v;
    }
    for (int e = tid; e < FBN * FBK; e += 256) {
      const int nn = e / FBK, kk = e % FBK;
      const int n = n0 + nn, k = k0 + kk;
      Bs[kk][nn] = (n < p.Cg_out && k < p.K) ? p.w[(size_t)(g * p.Cg_out + n) * p.K + k] : 0.f;
    }
    __syncthreads();
#pragma unroll
    for (int kk = 0; kk < FBK; ++kk) {
      float a[8], b[4];
#pragma unroll
      for (int i = 0; i < 8; ++i) a[i] = As[kk][tm + i];
#pragma unroll
      for (int j = 0; j < 4; ++j) b[j] = Bs[kk][tn + j];
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int m = m0 + tm + i;
    if (m >= p.M) continue;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      const int n = n0 + tn + j;
      if (n >= p.Cg_out) continue;
      const int ng = g * p.Cg_out + n;
      const size_t o = (size_t)m * p.Cout + ng;
      float v = fmaf(acc[i][j], p.scale[ng], p.shift[ng]);
      if (p.res) v += p.res[o];
      if (p.relu) v = fmaxf(v, 0.f);
      p.y[o] = v;
    }
  }
}

void conv_layer_init_f32(ConvLayerF32& L, const std::vector<float>& w, int Cin_real, const std::vector<float>& scale,
                         const std::vector<float>& shift) {
  if (L.Cin % L.groups || L.Cout % L.groups) fail(1, "conv(f32): channels not divisible by groups");
  L.Cg_in = L.Cin / L.groups;
  L.Cg_out = L.Cout / L.groups;
  const int cg_real = Cin_real / L.groups;
  L.K = L.R * L.S * L.Cg_in;
  std::vector<float> packed((size_t)L.Cout * L.K, 0.f);
  for (int o = 0; o < L.Cout; ++o)
    for (int r = 0; r < L.R; ++r)
      for (int s = 0; s < L.S; ++s)
        for (int c = 0; c < cg_real; ++c)
          packed[(size_t)o * L.K + (size_t)(r * L.S + s) * L.Cg_in + c] =
              w[(((size_t)o * L.R + r) * L.S + s) * cg_real + c];
  VCHECK(cudaMalloc(&L.w, packed.size() * 4));
  VCHECK(cudaMemcpy(L.w, packed.data(), packed.size() * 4, cudaMemcpyHostToDevice));
  VCHECK(cudaMalloc(&L.scale, L.Cout * 4));
  VCHECK(cudaMalloc(&L.shift, L.Cout * 4));
  VCHECK(cudaMemcpy(L.scale, scale.data(), L.Cout * 4, cudaMemcpyHostToDevice));
  VCHECK(cudaMemcpy(L.shift, shift.data(), L.Cout * 4, cudaMemcpyHostToDevice));
}

void conv_layer_free_f32(ConvLayerF32& L) {
  if (L.w) cudaFree(L.w);
  if (L.scale) cudaFree(L.scale);
  if (L.shift) cudaFree(L.shift);
  L.w = L.scale = L.shift = nullptr;
}

void conv_forward_f32(const ConvLayerF32& L, const float* x, int N, int H, int W, const float* res, float* y,
                      cudaStream_t st) {
  ConvF32Params p;
  p.x = x;
  p.y = y;
  p.res = res;
  p.w = L.w;
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
  const int64_t M = (int64_t)N * p.Ho * p.Wo;
  if (M <= 0) return;
  if (M > INT32_MAX - FBM) fail(1, "conv(f32): M too large");
  p.M = (int)M;
  p.relu = L.relu ? 1 : 0;
  dim3 grid((p.M + FBM - 1) / FBM, (L.Cg_out + FBN - 1) / FBN, L.groups);
  prof_begin(st);
  conv_f32_kernel<<<grid, 256, 0, st>>>(p);
  LAUNCHED();
  prof_end(st, 0, 2.0 * (double)M * L.Cout * L.R * L.S * L.Cg_in, 0);
}

}  // namespace vista
