// simt_ops.cu — the memory-bound TensorOps of the path (S0 ingest, pools, LRN) and the
// tap g_l (S2).  All NHWC, 8 channels per thread (16-byte bf16 / 32-byte fp32 vectors), grids
// sized in multiples of the SM count by a grid-stride loop.  Templated on the element type:
// bf16 (the product) and fp32 (the check mode, reading R23).
#include "internal.h"
#include "ptx.cuh"

namespace vista {

static int grid_for(int64_t work, int threads) {
  const int64_t blocks = (work + threads - 1) / threads;
  const int64_t cap = (int64_t)num_sms() * 16;
  return (int)(blocks < cap ? (blocks > 0 ? blocks : 1) : cap);
}

__device__ __forceinline__ void ld8(const bf16* p, float (&f)[8]) {
  const uint4 v = *reinterpret_cast<const uint4*>(p);
  const uint32_t u[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const float2 a = unpack_bf16x2(u[j]);
    f[2 * j] = a.x;
    f[2 * j + 1] = a.y;
  }
}
__device__ __forceinline__ void ld8(const float* p, float (&f)[8]) {
  const float4 a = reinterpret_cast<const float4*>(p)[0], b = reinterpret_cast<const float4*>(p)[1];
  f[0] = a.x; f[1] = a.y; f[2] = a.z; f[3] = a.w; f[4] = b.x; f[5] = b.y; f[6] = b.z; f[7] = b.w;
}
__device__ __forceinline__ void st8(bf16* p, const float (&f)[8]) {  // RNE
  uint4 v;
  v.x = pack_bf16x2(f[0], f[1]);
  v.y = pack_bf16x2(f[2], f[3]);
  v.z = pack_bf16x2(f[4], f[5]);
  v.w = pack_bf16x2(f[6], f[7]);
  *reinterpret_cast<uint4*>(p) = v;
}
__device__ __forceinline__ void st8(float* p, const float (&f)[8]) {
  reinterpret_cast<float4*>(p)[0] = make_float4(f[0], f[1], f[2], f[3]);
  reinterpret_cast<float4*>(p)[1] = make_float4(f[4], f[5], f[6], f[7]);
}
__device__ __forceinline__ float ld1(const bf16* p) { return __bfloat162float(*p); }
__device__ __forceinline__ float ld1(const float* p) { return *p; }

// ---- S0: uint8 NHWC3 -> NHWC8, x = (p - 128) / 128 (reading R10; exact in bf16) ----
template <typename T>
__global__ void ingest_kernel(const uint8_t* __restrict__ px, int64_t npix, T* __restrict__ y) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < npix; i += (int64_t)gridDim.x * blockDim.x) {
    const uint8_t* q = px + i * 3;
    float f[8] = {0, 0, 0, 0, 0, 0, 0, 0};
#pragma unroll
    for (int c = 0; c < 3; ++c) f[c] = ((float)q[c] - 128.0f) * (1.0f / 128.0f);
    st8(y + i * 8, f);
  }
}
template <typename T>
static void ingest_t(const uint8_t* px, int64_t n, T* y, cudaStream_t st) {
  const int64_t npix = n * 227 * 227;
  prof_begin(st);
  ingest_kernel<T><<<grid_for(npix, 256), 256, 0, st>>>(px, npix, y);
  LAUNCHED();
  prof_end(st, 2, 0, (double)npix * (3 + 8 * sizeof(T)));
}
void launch_ingest(const uint8_t* px, int64_t n, bf16* y, cudaStream_t st) { ingest_t(px, n, y, st); }
void launch_ingest_f32(const uint8_t* px, int64_t n, float* y, cudaStream_t st) { ingest_t(px, n, y, st); }

// ---- S0 for ResNet conv1: uint8 NHWC3 -> zero-padded 2x2 space-to-depth [n, 117, 117, 16] ----
// channel c' = (dy*2 + dx)*3 + ch (c' >= 12 zero) of position (h2, w2) holds (p - 128)/128 of pixel
// (2*h2 + dy - 3, 2*w2 + dx - 3), 0 outside the image (the conv's zero padding of 3).
// 2-D grid: x over the 117 x 117 positions of an image (32-bit index math; the grid-stride loop over a
// flat int64 index spent most of its instructions in 64-bit divisions), y over images
template <typename T>
__global__ void ingest_s2d_kernel(const uint8_t* __restrict__ px, int64_t n, T* __restrict__ y) {
  const int p = blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= 117 * 117) return;
  const int h2 = p / 117, w2 = p - h2 * 117;
  for (int64_t img = blockIdx.y; img < n; img += gridDim.y) {
    const uint8_t* src = px + img * (227 * 227 * 3);
    float f[16];
#pragma unroll
    for (int c = 0; c < 16; ++c) f[c] = 0.f;
#pragma unroll
    for (int d = 0; d < 4; ++d) {
      const int h = 2 * h2 + (d >> 1) - 3, w = 2 * w2 + (d & 1) - 3;
      if (h >= 0 && h < 227 && w >= 0 && w < 227) {
        const uint8_t* q = src + (h * 227 + w) * 3;
#pragma unroll
        for (int c = 0; c < 3; ++c) f[d * 3 + c] = ((float)q[c] - 128.0f) * (1.0f / 128.0f);
      }
    }
    float lo[8], hi[8];
#pragma unroll
    for (int c = 0; c < 8; ++c) {
      lo[c] = f[c];
      hi[c] = f[8 + c];
    }
    T* o = y + (img * (117 * 117) + p) * 16;
    st8(o, lo);
    st8(o + 8, hi);
  }
}
template <typename T>
static void ingest_s2d_t(const uint8_t* px, int64_t n, T* y, cudaStream_t st) {
  const int64_t total = n * 117 * 117;
  prof_begin(st);
  const dim3 grid((117 * 117 + 255) / 256, (unsigned)(n < 65535 ? (n > 0 ? n : 1) : 65535));
  ingest_s2d_kernel<T><<<grid, 256, 0, st>>>(px, n, y);
  LAUNCHED();
  prof_end(st, 2, 0, (double)n * 227 * 227 * 3 + (double)total * 16 * sizeof(T));
}
void launch_ingest_s2d(const uint8_t* px, int64_t n, bf16* y, cudaStream_t st) { ingest_s2d_t(px, n, y, st); }
void launch_ingest_s2d_f32(const uint8_t* px, int64_t n, float* y, cudaStream_t st) { ingest_s2d_t(px, n, y, st); }

// ---- unpadded max pool (k, s) ----
template <typename T>
__global__ void maxpool_kernel(const T* __restrict__ x, int N, int H, int W, int C, int k, int s, int Ho, int Wo,
                               T* __restrict__ y) {
  const int C8 = C >> 3;
  const int64_t total = (int64_t)N * Ho * Wo * C8;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c8 = (int)(i % C8);
    int64_t pix = i / C8;
    const int wo = (int)(pix % Wo);
    pix /= Wo;
    const int ho = (int)(pix % Ho);
    const int n = (int)(pix / Ho);
    float m[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) m[j] = -INFINITY;
    for (int r = 0; r < k; ++r) {
      const int hi = ho * s + r;
      if (hi >= H) break;
      for (int q = 0; q < k; ++q) {
        const int wi = wo * s + q;
        if (wi >= W) break;
        float f[8];
        ld8(x + (((size_t)n * H + hi) * W + wi) * C + c8 * 8, f);
#pragma unroll
        for (int j = 0; j < 8; ++j) m[j] = fmaxf(m[j], f[j]);
      }
    }
    st8(y + (((size_t)n * Ho + ho) * Wo + wo) * C + c8 * 8, m);
  }
}
template <typename T>
static void maxpool_t(const T* x, int N, int H, int W, int C, int k, int s, T* y, cudaStream_t st) {
  const int Ho = (H - k) / s + 1, Wo = (W - k) / s + 1;
  const int64_t total = (int64_t)N * Ho * Wo * (C / 8);
  prof_begin(st);
  maxpool_kernel<T><<<grid_for(total, 256), 256, 0, st>>>(x, N, H, W, C, k, s, Ho, Wo, y);
  LAUNCHED();
  prof_end(st, 2, 0, (double)sizeof(T) * ((double)N * H * W * C + (double)N * Ho * Wo * C));
}
void launch_maxpool(const bf16* x, int N, int H, int W, int C, int k, int s, bf16* y, cudaStream_t st) {
  maxpool_t(x, N, H, W, C, k, s, y, st);
}
void launch_maxpool_f32(const float* x, int N, int H, int W, int C, int k, int s, float* y, cudaStream_t st) {
  maxpool_t(x, N, H, W, C, k, s, y, st);
}

// ---- AlexNet LRN (reading R3): y_c = x_c / (1 + 2e-5 sum_{|c'-c|<=2} x_c'^2)^0.75 ----
template <typename T>
__global__ void lrn_kernel(const T* __restrict__ x, int64_t npix, int C, T* __restrict__ y) {
  const int C8 = C >> 3;
  const int64_t total = npix * C8;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c8 = (int)(i % C8);
    const int64_t pix = i / C8;
    const T* xp = x + pix * C;
    float w[12];  // channels c8*8-2 .. c8*8+9
#pragma unroll
    for (int j = 0; j < 12; ++j) {
      const int c = c8 * 8 - 2 + j;
      w[j] = (c >= 0 && c < C) ? ld1(xp + c) : 0.0f;
    }
    float o[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      float ss = 0.0f;
#pragma unroll
      for (int d = 0; d < 5; ++d) ss = fmaf(w[j + d], w[j + d], ss);
      o[j] = w[j + 2] * exp2f(-0.75f * log2f(fmaf(2e-5f, ss, 1.0f)));
    }
    st8(y + pix * C + c8 * 8, o);
  }
}
template <typename T>
static void lrn_t(const T* x, int N, int H, int W, int C, T* y, cudaStream_t st) {
  const int64_t npix = (int64_t)N * H * W;
  prof_begin(st);
  lrn_kernel<T><<<grid_for(npix * (C / 8), 256), 256, 0, st>>>(x, npix, C, y);
  LAUNCHED();
  prof_end(st, 2, 0, 2.0 * sizeof(T) * (double)npix * C);
}
void launch_lrn(const bf16* x, int N, int H, int W, int C, bf16* y, cudaStream_t st) { lrn_t(x, N, H, W, C, y, st); }
void launch_lrn_f32(const float* x, int N, int H, int W, int C, float* y, cudaStream_t st) {
  lrn_t(x, N, H, W, C, y, st);
}

// ---- global average pool [N,H,W,C] -> [N,C] ----
template <typename T>
__global__ void avgpool_kernel(const T* __restrict__ x, int N, int HW, int C, T* __restrict__ y) {
  const int C8 = C >> 3;
  const int64_t total = (int64_t)N * C8;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c8 = (int)(i % C8);
    const int64_t n = i / C8;
    float acc[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int p = 0; p < HW; ++p) {
      float f[8];
      ld8(x + ((size_t)n * HW + p) * C + c8 * 8, f);
#pragma unroll
      for (int j = 0; j < 8; ++j) acc[j] += f[j];
    }
    const float inv = 1.0f / (float)HW;
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[j] *= inv;
    st8(y + (size_t)n * C + c8 * 8, acc);
  }
}
template <typename T>
static void avgpool_t(const T* x, int N, int H, int W, int C, T* y, cudaStream_t st) {
  const int64_t total = (int64_t)N * (C / 8);
  prof_begin(st);
  avgpool_kernel<T><<<grid_for(total, 256), 256, 0, st>>>(x, N, H * W, C, y);
  LAUNCHED();
  prof_end(st, 2, 0, (double)sizeof(T) * ((double)N * H * W * C + (double)N * C));
}
void launch_avgpool(const bf16* x, int N, int H, int W, int C, bf16* y, cudaStream_t st) {
  avgpool_t(x, N, H, W, C, y, st);
}
void launch_avgpool_f32(const float* x, int N, int H, int W, int C, float* y, cudaStream_t st) {
  avgpool_t(x, N, H, W, C, y, st);
}

// ---- S2 tap g_l (PAPER.md:369 fn 4, Def 3.5; reading R7/R8): 2x2 grid max, NHWC flatten ----
// F[n][(2i + j) C + c] = max_{h in R_i, w in R_j} A[n, h, w, c], R_0 = [0, ceil(H/2)), R_1 = [ceil(H/2), H).
// Max is exact, so F is bit-identical to a max over the stored activation.
template <typename T>
__global__ void tap_kernel(const T* __restrict__ A, int64_t N, int H, int W, int C, T* __restrict__ F) {
  const int C8 = C >> 3;
  const int h2 = (H + 1) >> 1, w2 = (W + 1) >> 1;
  const int64_t total = N * 4 * C8;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c8 = (int)(i % C8);
    const int64_t t = i / C8;
    const int q = (int)(t & 3);
    const int64_t n = t >> 2;
    const int qi = q >> 1, qj = q & 1;
    const int hb = qi ? h2 : 0, he = qi ? H : h2;
    const int wb = qj ? w2 : 0, we = qj ? W : w2;
    float m[8];
#pragma unroll
    for (int j = 0; j < 8; ++j) m[j] = -INFINITY;
    for (int h = hb; h < he; ++h)
      for (int w = wb; w < we; ++w) {
        float f[8];
        ld8(A + (((size_t)n * H + h) * W + w) * C + c8 * 8, f);
#pragma unroll
        for (int j = 0; j < 8; ++j) m[j] = fmaxf(m[j], f[j]);
      }
    st8(F + (size_t)n * 4 * C + (size_t)q * C + c8 * 8, m);
  }
}
// bf16 form: max on packed bf16x2 (exact), four independent 16-byte loads in flight per thread
__device__ __forceinline__ uint4 bmax4(uint4 a, uint4 b) {
  uint4 o;
  const __nv_bfloat162* pa = reinterpret_cast<const __nv_bfloat162*>(&a);
  const __nv_bfloat162* pb = reinterpret_cast<const __nv_bfloat162*>(&b);
  __nv_bfloat162* po = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
  for (int j = 0; j < 4; ++j) po[j] = __hmax2(pa[j], pb[j]);
  return o;
}
__global__ void tap_bf16_kernel(const bf16* __restrict__ A, int64_t N, int H, int W, int C, bf16* __restrict__ F) {
  const int C8 = C >> 3;
  const int h2 = (H + 1) >> 1, w2 = (W + 1) >> 1;
  const int64_t total = N * 4 * C8;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int c8 = (int)(i % C8);
    const int64_t t = i / C8;
    const int q = (int)(t & 3);
    const int64_t n = t >> 2;
    const int qi = q >> 1, qj = q & 1;
    const int hb = qi ? h2 : 0, he = qi ? H : h2;
    const int wb = qj ? w2 : 0, we = qj ? W : w2;
    const uint4 ninf = make_uint4(0xFF80FF80u, 0xFF80FF80u, 0xFF80FF80u, 0xFF80FF80u);
    uint4 m0 = ninf, m1 = ninf;
    for (int h = hb; h < he; ++h) {
      const uint4* row = reinterpret_cast<const uint4*>(A + (((size_t)n * H + h) * W) * C + c8 * 8);
      int w = wb;
      for (; w + 4 <= we; w += 4) {
        const uint4 a = __ldcs(row + (size_t)w * C8), b = __ldcs(row + (size_t)(w + 1) * C8);
        const uint4 c = __ldcs(row + (size_t)(w + 2) * C8), d = __ldcs(row + (size_t)(w + 3) * C8);
        m0 = bmax4(m0, bmax4(a, b));
        m1 = bmax4(m1, bmax4(c, d));
      }
      for (; w < we; ++w) m0 = bmax4(m0, __ldcs(row + (size_t)w * C8));
    }
    *reinterpret_cast<uint4*>(F + (size_t)n * 4 * C + (size_t)q * C + c8 * 8) = bmax4(m0, m1);
  }
}
template <typename T>
static void tap_t(const T* A, int64_t N, int H, int W, int C, T* F, cudaStream_t st) {
  const int64_t total = N * 4 * (C / 8);
  prof_begin(st);
  if constexpr (sizeof(T) == 2) tap_bf16_kernel<<<grid_for(total, 256), 256, 0, st>>>(A, N, H, W, C, F);
  else tap_kernel<T><<<grid_for(total, 256), 256, 0, st>>>(A, N, H, W, C, F);
  LAUNCHED();
  prof_end(st, 1, 0, (double)sizeof(T) * ((double)N * H * W * C + (double)N * 4 * C));
}
void launch_tap(const bf16* A, int64_t N, int H, int W, int C, bf16* F, cudaStream_t st) {
  tap_t(A, N, H, W, C, F, st);
}
void launch_tap_f32(const float* A, int64_t N, int H, int W, int C, float* F, cudaStream_t st) {
  tap_t(A, N, H, W, C, F, st);
}

// finalize of the fused tap (conv_tc.cu): fp32 maxima -> bf16, 8 values per thread (exact)
__global__ void tap_finalize_kernel(const unsigned int* __restrict__ in, int64_t n8, bf16* __restrict__ F) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n8; i += (int64_t)gridDim.x * blockDim.x) {
    const uint4 a = reinterpret_cast<const uint4*>(in)[2 * i], b = reinterpret_cast<const uint4*>(in)[2 * i + 1];
    const float f[8] = {__uint_as_float(a.x), __uint_as_float(a.y), __uint_as_float(a.z), __uint_as_float(a.w),
                        __uint_as_float(b.x), __uint_as_float(b.y), __uint_as_float(b.z), __uint_as_float(b.w)};
    st8(F + i * 8, f);
  }
}
void launch_tap_finalize(const unsigned int* tapf, int64_t count, bf16* F, cudaStream_t st) {
  const int64_t n8 = count / 8;
  prof_begin(st);
  tap_finalize_kernel<<<grid_for(n8, 256), 256, 0, st>>>(tapf, n8, F);
  LAUNCHED();
  prof_end(st, 1, 0, (double)count * 6);
}

}  // namespace vista
