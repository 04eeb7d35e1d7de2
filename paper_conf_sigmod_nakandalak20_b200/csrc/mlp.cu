// mlp.cu — second downstream model M: the 3-layer MLP of PAPER.md:383 ("a 3-layer MLP (each
// hidden layer has 1024 units) for 10 iterations using distributed TF/Horovod"), SURVEY.md §8f #4,
// trained data-parallel on the multimodal rows MM_l (Eq. (4)) of one layer.
//
// Reading R30: inputs z-scored with the train statistics (O6 step 2), h1 = ReLU(W1 x + b1), h2 = ReLU(W2 h1 + b2), z = w3 . h2 + b3, mean
// logistic loss over the train rows, T full-batch gradient-descent steps of size lr (full batch like
// the LR reading R17, so the model does not depend on the number of GPUs), predict 1 iff z >= 0.
//
// Every dense contraction runs on the tcgen05 GEMM (gemm_tn in conv_tc.cu, bf16 operands, fp32 TMEM
// accumulation); K-major operands of the weight-gradient GEMMs are built by a tiled transpose that
// also applies the ReLU mask and produces the bias-gradient column sums:
//   forward   H1 = ReLU(X W1^T + b1)            gemm  M = n, N = h,  K = ld
//             H2 = ReLU(H1 W2^T + b2)           gemm  M = n, N = h,  K = h
//   head      z, dz = (sigmoid(z) - y) / n, loss, dH2 = dz w3^T . [H2 > 0], grad w3 = H2^T dz  (one warp per row)
//   backward  dW2 = dH2^T H1                    gemm  M = h, N = h,  K = n  (operands transposed)
//             dH1 = (dH2 W2) . [H1 > 0]         gemm  M = n, N = h,  K = h  (B = W2^T copy) + mask
//             dW1 = dH1^T X                     gemm  M = h, N = Kp, K = n  (X^T built once)
//   update    fp32 master weights -= lr * grad; bf16 operand copies refreshed
// Data parallel (Horovod analogue): each rank's gradient sums over its rows are summed
// across ranks by one fp32 allreduce per step (NCCL over NVLink), the loss and counts in fp64.
#include <cmath>
#include <cstring>

#include "internal.h"

namespace vista {

namespace {

constexpr int kMlpCls = 7;  // vista_profile class "mlp"
constexpr int kTT = 64;     // transpose tile

// out[c][r] = in[r][c] * (mask == null || mask[r][c] > 0) for r < rows, c < cols; optional column sums
// of the (bf16) outputs per 64-row tile: part[tile_r][c]  (fixed-order reduction later)
__global__ void __launch_bounds__(256) transpose_mask_kernel(const bf16* __restrict__ in, int64_t ld_in,
                                                             const bf16* __restrict__ mask, int64_t ld_mask,
                                                             int64_t rows, int cols, bf16* __restrict__ out,
                                                             int64_t ld_out, float* __restrict__ part) {
  __shared__ float tile[kTT][kTT + 1];
  const int64_t r0 = (int64_t)blockIdx.y * kTT;
  const int c0 = blockIdx.x * kTT;
  const int tx = threadIdx.x & 63, ty = threadIdx.x >> 6;  // 64 x 4
  for (int i = ty; i < kTT; i += 4) {
    const int64_t r = r0 + i;
    const int c = c0 + tx;
    float v = 0.f;
    if (r < rows && c < cols) {
      v = __bfloat162float(in[r * ld_in + c]);
      if (mask && !(__bfloat162float(mask[r * ld_mask + c]) > 0.f)) v = 0.f;
    }
    tile[i][tx] = v;
  }
  __syncthreads();
  if (part && ty == 0 && c0 + tx < cols) {
    float s = 0.f;
    for (int i = 0; i < kTT; ++i) s += tile[i][tx];
    part[(int64_t)blockIdx.y * cols + c0 + tx] = s;
  }
  for (int i = ty; i < kTT; i += 4) {
    const int c = c0 + i;
    const int64_t r = r0 + tx;
    if (c < cols && r < rows) out[(int64_t)c * ld_out + r] = __float2bfloat16_rn(tile[tx][i]);
  }
}

// per row j of X^T (= column j of the train rows): sum_p (x - c_j) for c == null, else sum_p (x - c_j)^2,
// in fp64, fixed order (one CTA per row).  Two passes give the O6 step-2 statistics exactly as the oracle.
__global__ void __launch_bounds__(256) xt_row_moment_kernel(const bf16* __restrict__ XT, int64_t ld_xt, int64_t n,
                                                            const double* __restrict__ c, double* __restrict__ out) {
  __shared__ double sh[256];
  const int64_t j = blockIdx.x;
  const double cj = c ? c[j] : 0.0;
  double s = 0.0;
  for (int64_t p = threadIdx.x; p < n; p += blockDim.x) {
    const double v = (double)__bfloat162float(XT[j * ld_xt + p]) - cj;
    s += c ? v * v : v;
  }
  sh[threadIdx.x] = s;
  __syncthreads();
  for (int o = 128; o > 0; o >>= 1) {
    if (threadIdx.x < o) sh[threadIdx.x] += sh[threadIdx.x + o];
    __syncthreads();
  }
  if (threadIdx.x == 0) out[j] = sh[0];
}

// The z-scoring is folded into the first layer (the rows of MM stay exact bf16; rounding x~ to bf16
// broke the cancellation of the centred gradient, measured 5 % gradient error in emulation):
//   W1 x~ + b1 = W1' x + b1',  W1' = W1 diag(inv),  b1' = b1 - W1' mu
//   dL/dW1 = dH1^T X~ = (dH1^T X - gb1 mu^T) diag(inv)      (gb1 = dH1^T 1)
// W1b = bf16(W1m[i][j] * inv[j]) is the GEMM operand; b1' uses the same rounded W1b.
__global__ void w1_update_kernel(float* __restrict__ W1m, const float* __restrict__ G1raw, const float* __restrict__ gb1,
                                 const float* __restrict__ mu, const float* __restrict__ inv, int h, int Kp, float lr,
                                 float* __restrict__ G1, bf16* __restrict__ W1b) {
  const int64_t total = (int64_t)h * Kp;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int o = (int)(i / Kp), j = (int)(i - (int64_t)o * Kp);
    float w = W1m[i];
    if (G1raw) {
      const float g = (G1raw[i] - mu[j] * gb1[o]) * inv[j];
      if (G1) G1[i] = g;
      w -= lr * g;
      W1m[i] = w;
    }
    W1b[i] = __float2bfloat16_rn(w * inv[j]);
  }
}
// b1'[o] = b1[o] - sum_j W1b[o][j] mu[j]   (one warp per row, fixed order)
__global__ void b1_fold_kernel(const bf16* __restrict__ W1b, const float* __restrict__ mu, const float* __restrict__ b1,
                               int h, int Kp, float* __restrict__ b1p) {
  const int o = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5), lane = threadIdx.x & 31;
  if (o >= h) return;
  float s = 0.f;
  for (int j = lane; j < Kp; j += 32) s = fmaf(__bfloat162float(W1b[(int64_t)o * Kp + j]), mu[j], s);
#pragma unroll
  for (int k = 16; k > 0; k >>= 1) s += __shfl_xor_sync(0xffffffffu, s, k);
  if (lane == 0) b1p[o] = b1[o] - s;
}

// fixed-order sum of partials [nb][n] -> out[j] (fp64 accumulation, fp32 result) * scale
__global__ void colsum_reduce_kernel(const float* __restrict__ part, int nb, int n, float* __restrict__ out) {
  const int j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j >= n) return;
  double s = 0.0;
  for (int b = 0; b < nb; ++b) s += part[(int64_t)b * n + j];
  out[j] = (float)s;
}

// head (H = 1024 = 32 lanes x 32 columns): one warp per row of H2.
//   z = H2 . w3 + b3 (fp32), dz = (sigmoid(z) - y) * inv_n, loss_p = softplus(z) - y z,
//   dH2[p, j] = bf16(dz * w3[j] * [H2 > 0]); per-block partials of sum_p H2[p, j] dz_p (grad w3),
//   sum_p dz_p (grad b3) and sum_p loss_p (fp64).
template <int H>
__global__ void __launch_bounds__(256) mlp_head_kernel(const bf16* __restrict__ H2, const float* __restrict__ w3,
                                                       const float* __restrict__ b3, const uint8_t* __restrict__ y,
                                                       int64_t rows, int rows_per_block, float inv_n,
                                                       bf16* __restrict__ dH2, float* __restrict__ gw3_part,
                                                       double* __restrict__ scal_part /* [nb][2]: loss, dz */) {
  static_assert(H == 1024, "head kernel is specialised for 1024 hidden units");
  constexpr int PER = H / 32;  // 32 columns per lane: 4 x 8 (16-byte chunks at lane*8 + 256*q)
  __shared__ float sg[8][H];
  __shared__ double sl[8][2];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float w[PER], acc[PER];
#pragma unroll
  for (int q = 0; q < 4; ++q)
#pragma unroll
    for (int e = 0; e < 8; ++e) {
      w[q * 8 + e] = w3[q * 256 + lane * 8 + e];
      acc[q * 8 + e] = 0.f;
    }
  const float bb = *b3;
  double lsum = 0.0, dsum = 0.0;
  const int64_t r_begin = (int64_t)blockIdx.x * rows_per_block;
  const int64_t r_end = min(rows, r_begin + rows_per_block);
  for (int64_t r = r_begin + warp; r < r_end; r += 8) {
    const uint4* src = reinterpret_cast<const uint4*>(H2 + r * H);
    float hv[PER];
    float z = 0.f;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint4 u = src[q * 32 + lane];
      const uint32_t uu[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&uu[e]));
        hv[q * 8 + 2 * e] = f.x;
        hv[q * 8 + 2 * e + 1] = f.y;
      }
    }
#pragma unroll
    for (int j = 0; j < PER; ++j) z = fmaf(hv[j], w[j], z);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) z += __shfl_xor_sync(0xffffffffu, z, o);
    z += bb;
    const float yy = (float)y[r];
    const float sig = 1.f / (1.f + __expf(-z));
    const float dz = (sig - yy) * inv_n;
    if (lane == 0) {
      const double zd = z;
      lsum += (zd > 0 ? zd + log1p(exp(-zd)) : log1p(exp(zd))) - (double)yy * zd;
      dsum += dz;
    }
    uint4* dst = reinterpret_cast<uint4*>(dH2 + r * H);
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint32_t o[4];
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int j = q * 8 + 2 * e;
        const float a = hv[j] > 0.f ? dz * w[j] : 0.f;
        const float b = hv[j + 1] > 0.f ? dz * w[j + 1] : 0.f;
        const __nv_bfloat162 v = __floats2bfloat162_rn(a, b);
        o[e] = *reinterpret_cast<const uint32_t*>(&v);
      }
      dst[q * 32 + lane] = make_uint4(o[0], o[1], o[2], o[3]);
    }
#pragma unroll
    for (int j = 0; j < PER; ++j) acc[j] = fmaf(hv[j], dz, acc[j]);
  }
#pragma unroll
  for (int q = 0; q < 4; ++q)
#pragma unroll
    for (int e = 0; e < 8; ++e) sg[warp][q * 256 + lane * 8 + e] = acc[q * 8 + e];
  if (lane == 0) {
    sl[warp][0] = lsum;
    sl[warp][1] = dsum;
  }
  __syncthreads();
  for (int j = threadIdx.x; j < H; j += blockDim.x) {
    float s = 0.f;
#pragma unroll
    for (int k = 0; k < 8; ++k) s += sg[k][j];
    gw3_part[(int64_t)blockIdx.x * H + j] = s;
  }
  if (threadIdx.x == 0) {
    double a = 0, b = 0;
    for (int k = 0; k < 8; ++k) {
      a += sl[k][0];
      b += sl[k][1];
    }
    scal_part[2 * blockIdx.x] = a;
    scal_part[2 * blockIdx.x + 1] = b;
  }
}

// predictions on rows [0, rows): counts per block [nb][6] = train_ok, tp, fp, tn, fn, (unused); rows < n_train are train
template <int H>
__global__ void __launch_bounds__(256) mlp_eval_kernel(const bf16* __restrict__ H2, const float* __restrict__ w3,
                                                       const float* __restrict__ b3, const uint8_t* __restrict__ y,
                                                       int64_t rows, int64_t n_train, int rows_per_block,
                                                       double* __restrict__ cnt_part) {
  __shared__ double sc[8][5];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  float w[H / 32];
#pragma unroll
  for (int q = 0; q < 4; ++q)
#pragma unroll
    for (int e = 0; e < 8; ++e) w[q * 8 + e] = w3[q * 256 + lane * 8 + e];
  double c[5] = {0, 0, 0, 0, 0};
  const int64_t r_begin = (int64_t)blockIdx.x * rows_per_block;
  const int64_t r_end = min(rows, r_begin + rows_per_block);
  for (int64_t r = r_begin + warp; r < r_end; r += 8) {
    const uint4* src = reinterpret_cast<const uint4*>(H2 + r * H);
    float z = 0.f;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const uint4 u = src[q * 32 + lane];
      const uint32_t uu[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const float2 f = __bfloat1622float2(*reinterpret_cast<const __nv_bfloat162*>(&uu[e]));
        z = fmaf(f.x, w[q * 8 + 2 * e], z);
        z = fmaf(f.y, w[q * 8 + 2 * e + 1], z);
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) z += __shfl_xor_sync(0xffffffffu, z, o);
    z += *b3;
    if (lane == 0) {
      const bool pred = z >= 0.f, yy = y[r] != 0;
      if (r < n_train) {
        c[0] += pred == yy;
      } else {
        c[1] += pred && yy;
        c[2] += pred && !yy;
        c[3] += !pred && !yy;
        c[4] += !pred && yy;
      }
    }
  }
  if (lane == 0)
    for (int k = 0; k < 5; ++k) sc[warp][k] = c[k];
  __syncthreads();
  if (threadIdx.x < 5) {
    double s = 0;
    for (int k = 0; k < 8; ++k) s += sc[k][threadIdx.x];
    cnt_part[blockIdx.x * 5 + threadIdx.x] = s;
  }
}

// W -= lr * G (fp32 master), Wb = bf16(W)
__global__ void sgd_update_kernel(float* __restrict__ W, const float* __restrict__ G, int64_t n, float lr,
                                  bf16* __restrict__ Wb) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const float v = W[i] - lr * G[i];
    W[i] = v;
    if (Wb) Wb[i] = __float2bfloat16_rn(v);
  }
}

__global__ void f32_to_bf16_kernel(const float* __restrict__ a, int64_t n, bf16* __restrict__ b) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    b[i] = __float2bfloat16_rn(a[i]);
}

__global__ void fill_f32_kernel(float* p, int64_t n, float v) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

// stream-ordered scratch, released on the same stream
struct Dev {
  void* p = nullptr;
  cudaStream_t s = nullptr;
  void* alloc(size_t bytes, cudaStream_t st) {
    s = st;
    VCHECK(cudaMallocAsync(&p, bytes ? bytes : 16, st));
    return p;
  }
  ~Dev() {
    if (p) cudaFreeAsync(p, s);
  }
};

void transpose(const bf16* in, int64_t ld_in, const bf16* mask, int64_t ld_mask, int64_t rows, int cols, bf16* out,
               int64_t ld_out, float* part, cudaStream_t st) {
  if (rows <= 0) return;
  dim3 grid((cols + kTT - 1) / kTT, (unsigned)((rows + kTT - 1) / kTT));
  prof_begin(st);
  transpose_mask_kernel<<<grid, 256, 0, st>>>(in, ld_in, mask, ld_mask, rows, cols, out, ld_out, part);
  LAUNCHED();
  prof_end(st, kMlpCls, 0, 4.0 * rows * cols + (mask ? 2.0 * rows * cols : 0), "mlp transpose");
}

void colsum(const float* part, int nb, int n, float* out, cudaStream_t st) {
  prof_begin(st);
  colsum_reduce_kernel<<<(n + 255) / 256, 256, 0, st>>>(part, nb, n, out);
  LAUNCHED();
  prof_end(st, kMlpCls, 0, 4.0 * nb * n, "mlp colsum");
}

}  // namespace

MLPResult mlp_train(const bf16* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                    const std::vector<int>& real_cols, const float* W1p_0, const float* W2_0, const float* w3_0,
                    int h, int iters, double lr, bool want_weights, allreduce_fn ar64, allreduce_f32_fn ar32,
                    void* ar_user, cudaStream_t st) {
  if (h != 1024) fail(1, "mlp: the head kernel is specialised for 1024 hidden units");
  if (ld % 8) fail(1, "mlp: ld must be a multiple of 8");
  const int d = (int)real_cols.size();
  if (!W1p_0 || !W2_0 || !w3_0) fail(1, "mlp: initial weights missing");
  MLPResult res;
  const int Kp = (ld + 63) / 64 * 64;
  const int64_t n = n_train, np = std::max<int64_t>((n + 63) / 64 * 64, 64);
  // global train rows (mean over the union of all ranks' train rows)
  double n_glob = (double)n;
  {
    Dev t;
    double* dn = (double*)t.alloc(8, st);
    VCHECK(cudaMemcpyAsync(dn, &n_glob, 8, cudaMemcpyHostToDevice, st));
    if (ar64) ar64(dn, 1, st, ar_user);
    VCHECK(cudaMemcpyAsync(&n_glob, dn, 8, cudaMemcpyDeviceToHost, st));
    VCHECK(cudaStreamSynchronize(st));
  }
  if (n_glob <= 0) fail(1, "mlp: no train rows");
  const float inv_n = (float)(1.0 / n_glob);
  // ---- device state ----
  const int64_t nW1 = (int64_t)h * Kp, nW2 = (int64_t)h * h;
  const int64_t nG = nW1 + nW2 + 3 * (int64_t)h + 8;  // [G1 | G2 | g3 | gb1 | gb2 | gb3]
  Dev mstat, mmu, minv, mb1p;
  Dev mW1m, mW1b, mW2m, mW2b, mW2T, mw3, mb1, mb2, mb3, mG, mones, mzeros, mXT, mH1, mH2, mdH2, mdH1p, mH1T,
      mdH2T, mdH1T, mpart, mscal, mcnt;
  float* W1m = (float*)mW1m.alloc(nW1 * 4, st);
  bf16* W1b = (bf16*)mW1b.alloc(nW1 * 2, st);
  float* W2m = (float*)mW2m.alloc(nW2 * 4, st);
  bf16* W2b = (bf16*)mW2b.alloc(nW2 * 2, st);
  bf16* W2T = (bf16*)mW2T.alloc(nW2 * 2, st);
  float* w3 = (float*)mw3.alloc(h * 4, st);
  float* b1 = (float*)mb1.alloc(h * 4, st);
  float* b2 = (float*)mb2.alloc(h * 4, st);
  float* b3 = (float*)mb3.alloc(16, st);
  float* G = (float*)mG.alloc(nG * 4, st);
  float *G1 = G, *G2 = G + nW1, *g3 = G2 + nW2, *gb1 = g3 + h, *gb2 = gb1 + h, *gb3 = gb2 + h;
  const int nmax = std::max(Kp, h);
  float* ones = (float*)mones.alloc(nmax * 4, st);
  float* zeros = (float*)mzeros.alloc(nmax * 4, st);
  bf16* XT = (bf16*)mXT.alloc((size_t)Kp * np * 2, st);
  const int64_t nr = std::max<int64_t>(n_rows, 1);
  bf16* H1 = (bf16*)mH1.alloc((size_t)nr * h * 2, st);
  bf16* H2 = (bf16*)mH2.alloc((size_t)nr * h * 2, st);
  bf16* dH2 = (bf16*)mdH2.alloc((size_t)std::max<int64_t>(n, 1) * h * 2, st);
  bf16* dH1p = (bf16*)mdH1p.alloc((size_t)std::max<int64_t>(n, 1) * h * 2, st);
  bf16* H1T = (bf16*)mH1T.alloc((size_t)h * np * 2, st);
  bf16* dH2T = (bf16*)mdH2T.alloc((size_t)h * np * 2, st);
  bf16* dH1T = (bf16*)mdH1T.alloc((size_t)h * np * 2, st);
  const int nbt = (int)((n + kTT - 1) / kTT);  // transpose row tiles
  const int head_blocks = (int)std::max<int64_t>(1, std::min<int64_t>(2 * num_sms(), (n + 63) / 64));
  const int rows_per_block = (int)((n + head_blocks - 1) / head_blocks);
  float* part = (float*)mpart.alloc((size_t)std::max(nbt, head_blocks) * h * 4, st);
  double* scal = (double*)mscal.alloc((size_t)head_blocks * 2 * 8, st);
  const int eval_blocks = (int)std::max<int64_t>(1, std::min<int64_t>(2 * num_sms(), (n_rows + 63) / 64));
  double* cnt = (double*)mcnt.alloc((size_t)eval_blocks * 5 * 8 + 64, st);
  VCHECK(cudaMemsetAsync(XT, 0, (size_t)Kp * np * 2, st));
  VCHECK(cudaMemsetAsync(H1T, 0, (size_t)h * np * 2, st));
  VCHECK(cudaMemsetAsync(dH2T, 0, (size_t)h * np * 2, st));
  VCHECK(cudaMemsetAsync(dH1T, 0, (size_t)h * np * 2, st));
  VCHECK(cudaMemsetAsync(G, 0, nG * 4, st));
  fill_f32_kernel<<<64, 256, 0, st>>>(ones, nmax, 1.f);
  LAUNCHED();
  VCHECK(cudaMemsetAsync(zeros, 0, nmax * 4, st));
  // initial weights (W1 already in the padded column layout of MM; columns outside real_cols are 0)
  VCHECK(cudaMemcpyAsync(W1m, W1p_0, nW1 * 4, cudaMemcpyDeviceToDevice, st));
  VCHECK(cudaMemcpyAsync(W2m, W2_0, nW2 * 4, cudaMemcpyDeviceToDevice, st));
  VCHECK(cudaMemcpyAsync(w3, w3_0, h * 4, cudaMemcpyDeviceToDevice, st));
  VCHECK(cudaMemsetAsync(b1, 0, h * 4, st));
  VCHECK(cudaMemsetAsync(b2, 0, h * 4, st));
  VCHECK(cudaMemsetAsync(b3, 0, 16, st));
  f32_to_bf16_kernel<<<num_sms(), 256, 0, st>>>(W2m, nW2, W2b);
  LAUNCHED();
  transpose(W2b, h, nullptr, 0, h, h, W2T, h, nullptr, st);
  const float flr = (float)lr;
  // X^T of the train rows (K-major B operand of dW1 = dH1^T X), once
  transpose(MM, ld, nullptr, 0, n, ld, XT, np, nullptr, st);
  // z-scoring (O6 step 2 statistics over the union of all ranks' train rows): mu, then the centred second
  // moment; inv_j = 0 for sigma_j <= 1e-12 (and for the zero padding columns of MM)
  float* fmu = (float*)mmu.alloc((size_t)Kp * 4, st);
  float* finv = (float*)minv.alloc((size_t)Kp * 4, st);
  float* b1p = (float*)mb1p.alloc((size_t)h * 4, st);
  {
    double* stat = (double*)mstat.alloc((size_t)2 * ld * 8, st);
    std::vector<double> hs1(ld), hmu(ld);
    prof_begin(st);
    xt_row_moment_kernel<<<ld, 256, 0, st>>>(XT, np, n, nullptr, stat);
    LAUNCHED();
    if (ar64) ar64(stat, ld, st, ar_user);
    VCHECK(cudaMemcpyAsync(hs1.data(), stat, (size_t)ld * 8, cudaMemcpyDeviceToHost, st));
    VCHECK(cudaStreamSynchronize(st));
    for (int j = 0; j < ld; ++j) hmu[j] = hs1[j] / n_glob;
    VCHECK(cudaMemcpyAsync(stat, hmu.data(), (size_t)ld * 8, cudaMemcpyHostToDevice, st));
    xt_row_moment_kernel<<<ld, 256, 0, st>>>(XT, np, n, stat, stat + ld);
    LAUNCHED();
    if (ar64) ar64(stat + ld, ld, st, ar_user);
    VCHECK(cudaMemcpyAsync(hs1.data(), stat + ld, (size_t)ld * 8, cudaMemcpyDeviceToHost, st));
    VCHECK(cudaStreamSynchronize(st));
    std::vector<float> hmuf(Kp, 0.f), hinv(Kp, 0.f);
    for (int j = 0; j < ld; ++j) {
      const double sig = std::sqrt(hs1[j] / n_glob);
      hmuf[j] = (float)hmu[j];
      hinv[j] = sig > 1e-12 ? (float)(1.0 / sig) : 0.f;
    }
    VCHECK(cudaMemcpyAsync(fmu, hmuf.data(), (size_t)Kp * 4, cudaMemcpyHostToDevice, st));
    VCHECK(cudaMemcpyAsync(finv, hinv.data(), (size_t)Kp * 4, cudaMemcpyHostToDevice, st));
    prof_end(st, kMlpCls, 0, 2.0 * 2 * n * ld, "mlp stats");
    VCHECK(cudaStreamSynchronize(st));  // host staging vectors die at scope end
  }
  // first-layer operand W1' = bf16(W1 diag(inv)) and its folded bias
  auto fold_w1 = [&](const float* G1raw, float* G1out) {
    prof_begin(st);
    w1_update_kernel<<<2 * num_sms(), 256, 0, st>>>(W1m, G1raw, gb1, fmu, finv, h, Kp, flr, G1out, W1b);
    LAUNCHED();
    b1_fold_kernel<<<(h + 7) / 8, 256, 0, st>>>(W1b, fmu, b1, h, Kp, b1p);
    LAUNCHED();
    prof_end(st, kMlpCls, 0, (G1raw ? 14.0 : 6.0) * nW1, "mlp w1 update/fold");
  };
  std::vector<double> hs(2 * head_blocks);
  fold_w1(nullptr, nullptr);
  for (int t = 0; t < iters; ++t) {
    // forward
    gemm_tn(MM, n, ld, ld, W1b, h, Kp, ones, b1p, true, H1, false, st, kMlpCls);
    gemm_tn(H1, n, h, h, W2b, h, h, ones, b2, true, H2, false, st, kMlpCls);
    // head: dz, dH2, grad w3 / b3 partials, loss
    if (n > 0) {
      prof_begin(st);
      mlp_head_kernel<1024><<<head_blocks, 256, 0, st>>>(H2, w3, b3, y, n, rows_per_block, inv_n, dH2, part, scal);
      LAUNCHED();
      prof_end(st, kMlpCls, 2.0 * n * h, 4.0 * n * h, "mlp head");
      colsum(part, head_blocks, h, g3, st);
    }
    // backward
    if (n > 0) {
      transpose(dH2, h, nullptr, 0, n, h, dH2T, np, part, st);  // + grad b2 partials
      colsum(part, nbt, h, gb2, st);
      transpose(H1, h, nullptr, 0, n, h, H1T, np, nullptr, st);
      gemm_tn(dH2T, h, (int)n, (int)np, H1T, h, (int)np, ones, zeros, false, G2, true, st, kMlpCls);  // dW2
      gemm_tn(dH2, n, h, h, W2T, h, h, ones, zeros, false, dH1p, false, st, kMlpCls);                  // dH2 W2
      transpose(dH1p, h, H1, h, n, h, dH1T, np, part, st);  // . [H1 > 0], + grad b1 partials
      colsum(part, nbt, h, gb1, st);
      gemm_tn(dH1T, h, (int)n, (int)np, XT, Kp, (int)np, ones, zeros, false, G1, true, st, kMlpCls);  // dW1
    } else {
      // a rank without train rows still takes part in every collective, with a zero contribution (G was
      // allreduced in place last step, so it must be cleared, not left holding the global sums)
      VCHECK(cudaMemsetAsync(G, 0, nG * 4, st));
    }
    // loss and grad b3 (fp64, fixed order), then the allreduces across ranks
    VCHECK(cudaMemcpyAsync(hs.data(), scal, 2 * head_blocks * 8, cudaMemcpyDeviceToHost, st));
    VCHECK(cudaStreamSynchronize(st));
    double lsum = 0, dsum = 0;
    for (int b = 0; b < head_blocks && n > 0; ++b) {
      lsum += hs[2 * b];
      dsum += hs[2 * b + 1];
    }
    const float gb3v = (float)dsum;
    VCHECK(cudaMemcpyAsync(gb3, &gb3v, 4, cudaMemcpyHostToDevice, st));
    if (ar32) ar32(G, nG, st, ar_user);
    if (ar64) {
      Dev t1;
      double* dl = (double*)t1.alloc(8, st);
      VCHECK(cudaMemcpyAsync(dl, &lsum, 8, cudaMemcpyHostToDevice, st));
      ar64(dl, 1, st, ar_user);
      VCHECK(cudaMemcpyAsync(&lsum, dl, 8, cudaMemcpyDeviceToHost, st));
    }
    VCHECK(cudaStreamSynchronize(st));
    res.loss.push_back(lsum / n_glob);
    // update (the gradients are already means: dz carries 1 / n)
    prof_begin(st);
    sgd_update_kernel<<<num_sms(), 256, 0, st>>>(W2m, G2, nW2, flr, W2b);
    LAUNCHED();
    sgd_update_kernel<<<4, 256, 0, st>>>(w3, g3, h, flr, nullptr);
    LAUNCHED();
    sgd_update_kernel<<<4, 256, 0, st>>>(b1, gb1, h, flr, nullptr);
    LAUNCHED();
    sgd_update_kernel<<<4, 256, 0, st>>>(b2, gb2, h, flr, nullptr);
    LAUNCHED();
    sgd_update_kernel<<<1, 32, 0, st>>>(b3, gb3, 1, flr, nullptr);
    LAUNCHED();
    prof_end(st, kMlpCls, 0, 10.0 * nW2, "mlp update");
    fold_w1(G1, nullptr);  // G1 holds dH1^T X (raw rows): centred and scaled inside
    transpose(W2b, h, nullptr, 0, h, h, W2T, h, nullptr, st);
  }
  // ---- evaluation with the final weights on every row: train accuracy and test confusion counts ----
  gemm_tn(MM, n_rows, ld, ld, W1b, h, Kp, ones, b1p, true, H1, false, st, kMlpCls);
  gemm_tn(H1, n_rows, h, h, W2b, h, h, ones, b2, true, H2, false, st, kMlpCls);
  VCHECK(cudaMemsetAsync(cnt, 0, (size_t)eval_blocks * 5 * 8, st));
  if (n_rows > 0) {
    const int rpb = (int)((n_rows + eval_blocks - 1) / eval_blocks);
    mlp_eval_kernel<1024><<<eval_blocks, 256, 0, st>>>(H2, w3, b3, y, n_rows, n_train, rpb, cnt);
    LAUNCHED();
  }
  std::vector<double> hc((size_t)eval_blocks * 5);
  VCHECK(cudaMemcpyAsync(hc.data(), cnt, hc.size() * 8, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaStreamSynchronize(st));
  double c5[5] = {0, 0, 0, 0, 0};
  for (int b = 0; b < eval_blocks; ++b)
    for (int k = 0; k < 5; ++k) c5[k] += hc[(size_t)b * 5 + k];
  double tot[7] = {c5[0], c5[1], c5[2], c5[3], c5[4], (double)n_train, (double)(n_rows - n_train)};
  if (ar64) {
    Dev t2;
    double* dc = (double*)t2.alloc(7 * 8, st);
    VCHECK(cudaMemcpyAsync(dc, tot, 7 * 8, cudaMemcpyHostToDevice, st));
    ar64(dc, 7, st, ar_user);
    VCHECK(cudaMemcpyAsync(tot, dc, 7 * 8, cudaMemcpyDeviceToHost, st));
    VCHECK(cudaStreamSynchronize(st));
  }
  res.train_ok = (int64_t)tot[0];
  res.tp = (int64_t)tot[1];
  res.fp = (int64_t)tot[2];
  res.tn = (int64_t)tot[3];
  res.fn = (int64_t)tot[4];
  res.n_train = (int64_t)tot[5];
  res.n_test = (int64_t)tot[6];
  if (!want_weights) return res;
  // ---- final weights to the host (real columns of W1) ----
  std::vector<float> w1p((size_t)nW1);
  res.W2.resize(nW2);
  res.w3.resize(h);
  res.b1.resize(h);
  res.b2.resize(h);
  VCHECK(cudaMemcpyAsync(w1p.data(), W1m, nW1 * 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaMemcpyAsync(res.W2.data(), W2m, nW2 * 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaMemcpyAsync(res.w3.data(), w3, h * 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaMemcpyAsync(res.b1.data(), b1, h * 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaMemcpyAsync(res.b2.data(), b2, h * 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaMemcpyAsync(&res.b3, b3, 4, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaStreamSynchronize(st));
  res.W1.resize((size_t)h * d);
  for (int o = 0; o < h; ++o)
    for (int j = 0; j < d; ++j) res.W1[(size_t)o * d + j] = w1p[(size_t)o * Kp + real_cols[j]];
  return res;
}

}  // namespace vista
