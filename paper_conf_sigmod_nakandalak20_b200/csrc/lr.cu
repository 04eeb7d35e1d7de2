// lr.cu — S5 of SURVEY.md §8a: train M (logistic regression; elastic net
// alpha = 0.5, lambda = 0.01) on X'_l = [X, F_l] (Eq. (4)) by the
// full-batch proximal-gradient reading R17, step for step as O6:
//   stats (mu, sigma over train rows) -> K power iterations for lambda_max ->
//   T ISTA steps from w = 0, b = 0 -> evaluation (predict 1 iff z >= 0).
// Every pass is ONE read of MM_l (HBM-bound): each CTA owns a contiguous block of rows
// ("minibatch"), computes z_p = b + sum_j w^_j (x_pj - mu_j) per row with a block
// reduction, applies phi (identity for the power iteration, sigmoid residual for the
// gradient) and accumulates sum_p phi_p (x_pj - mu_j) per column in registers.  Per-CTA
// partials are reduced in a fixed order in fp64 (deterministic), then allreduced across
// ranks (fp64 NCCL) and applied by a one-block update kernel in fp64.
#include <cmath>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

constexpr int RG = 4;  // rows per block-reduction round

struct PassArgs {
  const bf16* MM;
  const uint8_t* y;
  int64_t r0, r1;       // row range [r0, r1) of this pass (train rows)
  int ld, chunks;       // ld elements per row, chunks = ld / 8
  const float* mu;      // [ld]
  const float* what;    // [ld]  inv_j * (w_j or v_j), 0 on excluded / pad columns
  const float* bhat;    // [1]
  float* partial;       // [gridDim.x][ld + 4] (16-byte aligned rows; ld + 2 used)
};

__device__ __forceinline__ float softplusf(float z) { return z > 0.f ? z + log1pf(__expf(-z)) : log1pf(__expf(z)); }

// MODE 0: sum x; MODE 1: sum (x - mu)^2; MODE 2: power pass (phi = z); MODE 3: gradient pass
template <int CH, int MODE>
__global__ void __launch_bounds__(1024) lr_pass_kernel(const PassArgs a) {
  __shared__ float red[2][RG][32];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarps = blockDim.x >> 5;
  const int64_t n = a.r1 - a.r0;
  const int64_t rb = a.r0 + n * blockIdx.x / gridDim.x, re = a.r0 + n * (blockIdx.x + 1) / gridDim.x;
  float mu[CH][8], wv[CH][8], acc[CH][8];
  bool act[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tid + c * blockDim.x;
    act[c] = ch < a.chunks;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      mu[c][j] = (MODE != 0 && act[c]) ? a.mu[ch * 8 + j] : 0.f;
      wv[c][j] = (MODE >= 2 && act[c]) ? a.what[ch * 8 + j] : 0.f;
      acc[c][j] = 0.f;
    }
  }
  const float bh = MODE >= 2 ? a.bhat[0] : 0.f;
  float sum_r = 0.f, sum_loss = 0.f;
  int buf = 0;
  for (int64_t r = rb; r < re; r += RG) {
    uint4 xv[RG][CH];
#pragma unroll
    for (int q = 0; q < RG; ++q)
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        const int ch = tid + c * blockDim.x;
        xv[q][c] = (act[c] && r + q < re)
                       ? __ldg(reinterpret_cast<const uint4*>(a.MM + (size_t)(r + q) * a.ld) + ch)
                       : make_uint4(0, 0, 0, 0);
      }
    if constexpr (MODE <= 1) {
#pragma unroll
      for (int q = 0; q < RG; ++q) {
        const float vq = r + q < re ? 1.f : 0.f;  // rows past the block's range must not add mu^2
#pragma unroll
        for (int c = 0; c < CH; ++c) {
          const uint32_t u[4] = {xv[q][c].x, xv[q][c].y, xv[q][c].z, xv[q][c].w};
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float2 f = unpack_bf16x2(u[j]);
            if (MODE == 0) {
              acc[c][2 * j] += f.x;
              acc[c][2 * j + 1] += f.y;
            } else {
              const float d0 = (f.x - mu[c][2 * j]) * vq, d1 = (f.y - mu[c][2 * j + 1]) * vq;
              acc[c][2 * j] = fmaf(d0, d0, acc[c][2 * j]);
              acc[c][2 * j + 1] = fmaf(d1, d1, acc[c][2 * j + 1]);
            }
          }
        }
      }
    } else {
      float dot[RG];
#pragma unroll
      for (int q = 0; q < RG; ++q) {
        float s = 0.f;
#pragma unroll
        for (int c = 0; c < CH; ++c) {
          const uint32_t u[4] = {xv[q][c].x, xv[q][c].y, xv[q][c].z, xv[q][c].w};
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float2 f = unpack_bf16x2(u[j]);
            s = fmaf(f.x - mu[c][2 * j], wv[c][2 * j], s);
            s = fmaf(f.y - mu[c][2 * j + 1], wv[c][2 * j + 1], s);
          }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        dot[q] = s;
      }
      if (lane == 0) {
#pragma unroll
        for (int q = 0; q < RG; ++q) red[buf][q][warp] = dot[q];
      }
      __syncthreads();
      float phi[RG];
#pragma unroll
      for (int q = 0; q < RG; ++q) {
        float z = bh;
        for (int w = 0; w < nwarps; ++w) z += red[buf][q][w];  // fixed order
        const bool valid = r + q < re;
        if (MODE == 2) {
          phi[q] = valid ? z : 0.f;
        } else {
          const float yv = valid ? (float)a.y[r + q] : 0.f;
          const float p = 1.f / (1.f + __expf(-z));
          phi[q] = valid ? p - yv : 0.f;
          if (valid) sum_loss += softplusf(z) - yv * z;
        }
        sum_r += phi[q];
      }
      buf ^= 1;
#pragma unroll
      for (int q = 0; q < RG; ++q)
#pragma unroll
        for (int c = 0; c < CH; ++c) {
          const uint32_t u[4] = {xv[q][c].x, xv[q][c].y, xv[q][c].z, xv[q][c].w};
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float2 f = unpack_bf16x2(u[j]);
            acc[c][2 * j] = fmaf(phi[q], f.x - mu[c][2 * j], acc[c][2 * j]);
            acc[c][2 * j + 1] = fmaf(phi[q], f.y - mu[c][2 * j + 1], acc[c][2 * j + 1]);
          }
        }
    }
  }
  float* out = a.partial + (size_t)blockIdx.x * (a.ld + 4);
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tid + c * blockDim.x;
    if (act[c]) {
      float4* o = reinterpret_cast<float4*>(out + ch * 8);
      o[0] = make_float4(acc[c][0], acc[c][1], acc[c][2], acc[c][3]);
      o[1] = make_float4(acc[c][4], acc[c][5], acc[c][6], acc[c][7]);
    }
  }
  if (tid == 0) {
    out[a.ld] = sum_r;        // identical in every thread (all threads saw every phi)
    out[a.ld + 1] = sum_loss;
  }
}

// G[j] = sum_cta partial[cta][j] in fp64, fixed order; ncols = ld + 2, row pitch ld + 4
__global__ void reduce_partials_kernel(const float* __restrict__ partial, int nct, int ncols, int pitch, double* G) {
  for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < ncols; j += gridDim.x * blockDim.x) {
    double s = 0.0;
    for (int c = 0; c < nct; ++c) s += (double)partial[(size_t)c * pitch + j];
    G[j] = s;
  }
}

struct LRState {  // device, fp64 master copies
  double n_train;   // global train rows
  double lambda_hat, eta;
  double b, vb;
  double loss;
};

__device__ double block_sum(double v, double* sh) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  __syncthreads();
  if (lane == 0) sh[warp] = v;
  __syncthreads();
  double t = 0.0;
  for (int w = 0; w < (int)(blockDim.x >> 5); ++w) t += sh[w];  // fixed order, all threads
  return t;
}

// stats finalize. step 0: mu = G / n (G[ld] holds n_train); step 1: sigma -> inv
__global__ void stats_finalize_kernel(const double* G, int ld, int step, const uint8_t* real, double* mu,
                                      float* mu_f, double* inv, LRState* st) {
  if (step == 0 && blockIdx.x == 0 && threadIdx.x == 0) st->n_train = G[ld];
  const double n = step == 0 ? G[ld] : st->n_train;
  for (int j = blockIdx.x * blockDim.x + threadIdx.x; j < ld; j += gridDim.x * blockDim.x) {
    if (step == 0) {
      mu[j] = G[j] / n;
      mu_f[j] = (float)mu[j];
    } else {
      const double sigma = sqrt(G[j] / n);
      inv[j] = (real[j] && sigma > 1e-12) ? 1.0 / sigma : 0.0;
    }
  }
}

// power iteration (O6 step 3).  init: v = 1/sqrt(d+1) on real columns and the bias.
// update: q_j = inv_j G_j / n, q_b = G_ld / n, lambda = ||q||, v = q / lambda.
// Both end by publishing w^ = inv * v (fp32) and b^ = v_b for the next pass.
__global__ void power_kernel(const double* G, int ld, int init, int d_real, const uint8_t* real, const double* inv,
                             double* v, float* what, float* bhat, LRState* st) {
  __shared__ double sh[32];
  const double n = st->n_train;
  if (init) {
    const double v0 = 1.0 / sqrt((double)(d_real + 1));
    for (int j = threadIdx.x; j < ld; j += blockDim.x) v[j] = real[j] ? v0 : 0.0;
    if (threadIdx.x == 0) st->vb = v0;
  } else {
    double ss = 0.0;
    for (int j = threadIdx.x; j < ld; j += blockDim.x) {
      const double q = inv[j] * G[j] / n;
      ss += q * q;
    }
    const double qb = G[ld] / n;
    const double lam = sqrt(block_sum(ss, sh) + qb * qb);
    for (int j = threadIdx.x; j < ld; j += blockDim.x) v[j] = lam > 0 ? inv[j] * G[j] / n / lam : 0.0;
    if (threadIdx.x == 0) {
      st->vb = lam > 0 ? qb / lam : 0.0;
      st->lambda_hat = lam;
    }
  }
  __syncthreads();
  for (int j = threadIdx.x; j < ld; j += blockDim.x) what[j] = (float)(inv[j] * v[j]);
  if (threadIdx.x == 0) bhat[0] = (float)st->vb;
}

// ISTA (O6 steps 4-5).  init: eta = 1 / (0.25 * 1.05 * lambda_hat + lambda (1 - alpha)), w = 0, b = 0.
// update: g_j = inv_j G_j / n + lambda (1 - alpha) w_j; w = soft(w - eta g, eta lambda alpha);
//         b -= eta G_ld / n; loss = G_{ld+1} / n (at the pre-update w).
__global__ void grad_kernel(const double* G, int ld, int init, double lambda, double alpha, const double* inv,
                            double* w, float* what, float* bhat, LRState* st, double* loss_out) {
  if (init) {
    for (int j = threadIdx.x; j < ld; j += blockDim.x) w[j] = 0.0;
    if (threadIdx.x == 0) {
      st->eta = 1.0 / (0.25 * 1.05 * st->lambda_hat + lambda * (1.0 - alpha));
      st->b = 0.0;
    }
  } else {
    const double n = st->n_train, eta = st->eta, thr = eta * lambda * alpha;
    for (int j = threadIdx.x; j < ld; j += blockDim.x) {
      const double g = inv[j] * G[j] / n + lambda * (1.0 - alpha) * w[j];
      const double vv = w[j] - eta * g;
      w[j] = (vv > 0 ? 1.0 : (vv < 0 ? -1.0 : 0.0)) * fmax(fabs(vv) - thr, 0.0);
    }
    if (threadIdx.x == 0) {
      *loss_out = G[ld + 1] / n;
      st->b -= eta * G[ld] / n;
    }
  }
  __syncthreads();
  for (int j = threadIdx.x; j < ld; j += blockDim.x) what[j] = (float)(inv[j] * w[j]);
  if (threadIdx.x == 0) bhat[0] = (float)st->b;
}

// eval (O6 step 6): counts[0] train correct, [1] tp, [2] fp, [3] tn, [4] fn (integers, exact)
template <int CH>
__global__ void __launch_bounds__(1024) lr_eval_kernel(const PassArgs a, int64_t n_train, unsigned long long* counts) {
  __shared__ float red[RG][32];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwarps = blockDim.x >> 5;
  const int64_t n = a.r1 - a.r0;
  const int64_t rb = a.r0 + n * blockIdx.x / gridDim.x, re = a.r0 + n * (blockIdx.x + 1) / gridDim.x;
  float mu[CH][8], wv[CH][8];
  bool act[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tid + c * blockDim.x;
    act[c] = ch < a.chunks;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      mu[c][j] = act[c] ? a.mu[ch * 8 + j] : 0.f;
      wv[c][j] = act[c] ? a.what[ch * 8 + j] : 0.f;
    }
  }
  const float bh = a.bhat[0];
  unsigned long long cnt[5] = {0, 0, 0, 0, 0};
  for (int64_t r = rb; r < re; r += RG) {
    float dot[RG];
#pragma unroll
    for (int q = 0; q < RG; ++q) {
      float s = 0.f;
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        const int ch = tid + c * blockDim.x;
        if (act[c] && r + q < re) {
          const uint4 xv = __ldg(reinterpret_cast<const uint4*>(a.MM + (size_t)(r + q) * a.ld) + ch);
          const uint32_t u[4] = {xv.x, xv.y, xv.z, xv.w};
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float2 f = unpack_bf16x2(u[j]);
            s = fmaf(f.x - mu[c][2 * j], wv[c][2 * j], s);
            s = fmaf(f.y - mu[c][2 * j + 1], wv[c][2 * j + 1], s);
          }
        }
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      dot[q] = s;
    }
    __syncthreads();
    if (lane == 0)
#pragma unroll
      for (int q = 0; q < RG; ++q) red[q][warp] = dot[q];
    __syncthreads();
    if (tid == 0) {
      for (int q = 0; q < RG && r + q < re; ++q) {
        float z = bh;
        for (int w = 0; w < nwarps; ++w) z += red[q][w];
        const int pred = z >= 0.f ? 1 : 0;
        const int yv = a.y[r + q];
        if (r + q < n_train) {
          cnt[0] += pred == yv;
        } else {
          cnt[pred && yv ? 1 : (pred ? 2 : (yv ? 4 : 3))] += 1;
        }
      }
    }
  }
  if (tid == 0)
    for (int k = 0; k < 5; ++k)
      if (cnt[k]) atomicAdd(&counts[k], cnt[k]);
}

// ------------------------------------------------------------------------------------------
template <int MODE>
static void run_pass(const PassArgs& a0, int threads, int grid, int ch, cudaStream_t st) {
  PassArgs a = a0;
  switch (ch) {
    case 1: lr_pass_kernel<1, MODE><<<grid, threads, 0, st>>>(a); break;
    case 2: lr_pass_kernel<2, MODE><<<grid, threads, 0, st>>>(a); break;
    case 4: lr_pass_kernel<4, MODE><<<grid, threads, 0, st>>>(a); break;
    default: fail(1, "lr: unsupported row width");
  }
  LAUNCHED();
}

LRResult lr_train(const bf16* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                  const uint8_t* real_host, int iters, int power_iters, double lambda, double alpha,
                  allreduce_fn allreduce, void* ar_user, cudaStream_t st) {
  LRResult res;
  if (ld % 8) fail(1, "lr: ld must be a multiple of 8");
  const int chunks = ld / 8;
  int ch = chunks <= 512 ? 1 : (chunks <= 2048 ? 2 : 4);
  int threads = ((chunks + ch - 1) / ch + 31) / 32 * 32;
  if (threads > 1024) fail(1, "lr: row too wide");
  const int per_sm = std::max(1, 2048 / threads);
  auto grid_for_rows = [&](int64_t rows) {
    int64_t g = (rows + 4 * RG - 1) / (4 * RG);
    const int64_t cap = (int64_t)num_sms() * per_sm;
    return (int)std::max<int64_t>(1, std::min(g, cap));
  };
  const int grid_tr = grid_for_rows(n_train);
  const int ncols = ld + 2;
  int d_real = 0;
  for (int j = 0; j < ld; ++j) d_real += real_host[j] ? 1 : 0;

  // scratch
  size_t off = 0;
  auto carve = [&](size_t bytes) { size_t o = off; off += (bytes + 255) & ~(size_t)255; return o; };
  const size_t o_part = carve((size_t)grid_tr * (ld + 4) * 4), o_G = carve(ncols * 8), o_mu = carve(ld * 8),
               o_muf = carve(ld * 4), o_inv = carve(ld * 8), o_v = carve(ld * 8), o_w = carve(ld * 8),
               o_what = carve(ld * 4), o_bhat = carve(16), o_st = carve(sizeof(LRState)),
               o_real = carve(ld), o_loss = carve((size_t)(iters + 1) * 8), o_cnt = carve(64);
  uint8_t* scr = nullptr;
  VCHECK(cudaMallocAsync(&scr, off, st));
  float* partial = reinterpret_cast<float*>(scr + o_part);
  double* G = reinterpret_cast<double*>(scr + o_G);
  double* mu = reinterpret_cast<double*>(scr + o_mu);
  float* mu_f = reinterpret_cast<float*>(scr + o_muf);
  double* inv = reinterpret_cast<double*>(scr + o_inv);
  double* v = reinterpret_cast<double*>(scr + o_v);
  double* w = reinterpret_cast<double*>(scr + o_w);
  float* what = reinterpret_cast<float*>(scr + o_what);
  float* bhat = reinterpret_cast<float*>(scr + o_bhat);
  LRState* dst = reinterpret_cast<LRState*>(scr + o_st);
  uint8_t* real = scr + o_real;
  double* loss = reinterpret_cast<double*>(scr + o_loss);
  unsigned long long* cnt = reinterpret_cast<unsigned long long*>(scr + o_cnt);
  VCHECK(cudaMemcpyAsync(real, real_host, ld, cudaMemcpyHostToDevice, st));
  VCHECK(cudaMemsetAsync(cnt, 0, 64, st));

  PassArgs a;
  a.MM = MM;
  a.y = y;
  a.r0 = 0;
  a.r1 = n_train;
  a.ld = ld;
  a.chunks = chunks;
  a.mu = mu_f;
  a.what = what;
  a.bhat = bhat;
  a.partial = partial;
  const double pass_bytes = (double)n_train * ld * 2;
  auto reduce = [&](double extra_n) {
    prof_begin(st);
    reduce_partials_kernel<<<(ncols + 255) / 256, 256, 0, st>>>(partial, grid_tr, ncols, ld + 4, G);
    LAUNCHED();
    prof_end(st, 6, 0, (double)grid_tr * ncols * 4);
    if (extra_n >= 0) {  // stats pass 1 carries the local train-row count in G[ld]
      VCHECK(cudaMemcpyAsync(G + ld, &extra_n, 8, cudaMemcpyHostToDevice, st));
    }
    if (allreduce) allreduce(G, ncols, st, ar_user);
  };
  const int ublk = 1024;
  // ---- O6 step 2: standardisation statistics (two passes: mean, then centred squares) ----
  prof_begin(st);
  run_pass<0>(a, threads, grid_tr, ch, st);
  prof_end(st, 5, 0, pass_bytes);
  reduce((double)n_train);
  stats_finalize_kernel<<<(ld + 255) / 256, 256, 0, st>>>(G, ld, 0, real, mu, mu_f, inv, dst);
  LAUNCHED();
  prof_begin(st);
  run_pass<1>(a, threads, grid_tr, ch, st);
  prof_end(st, 5, 0, pass_bytes);
  reduce(-1);
  stats_finalize_kernel<<<(ld + 255) / 256, 256, 0, st>>>(G, ld, 1, real, mu, mu_f, inv, dst);
  LAUNCHED();
  // ---- O6 step 3: K power iterations ----
  power_kernel<<<1, ublk, 0, st>>>(G, ld, 1, d_real, real, inv, v, what, bhat, dst);
  LAUNCHED();
  for (int k = 0; k < power_iters; ++k) {
    prof_begin(st);
    run_pass<2>(a, threads, grid_tr, ch, st);
    prof_end(st, 5, 0, pass_bytes);
    reduce(-1);
    power_kernel<<<1, ublk, 0, st>>>(G, ld, 0, d_real, real, inv, v, what, bhat, dst);
    LAUNCHED();
  }
  // ---- O6 steps 4-5: ISTA ----
  grad_kernel<<<1, ublk, 0, st>>>(G, ld, 1, lambda, alpha, inv, w, what, bhat, dst, loss);
  LAUNCHED();
  for (int t = 0; t < iters; ++t) {
    prof_begin(st);
    run_pass<3>(a, threads, grid_tr, ch, st);
    prof_end(st, 5, 0, pass_bytes);
    reduce(-1);
    grad_kernel<<<1, ublk, 0, st>>>(G, ld, 0, lambda, alpha, inv, w, what, bhat, dst, loss + t);
    LAUNCHED();
  }
  // ---- O6 step 6: eval over all local rows ----
  {
    PassArgs e = a;
    e.r0 = 0;
    e.r1 = n_rows;
    const int ge = grid_for_rows(n_rows);
    prof_begin(st);
    if (n_rows > 0) {
      switch (ch) {
        case 1: lr_eval_kernel<1><<<ge, threads, 0, st>>>(e, n_train, cnt); break;
        case 2: lr_eval_kernel<2><<<ge, threads, 0, st>>>(e, n_train, cnt); break;
        default: lr_eval_kernel<4><<<ge, threads, 0, st>>>(e, n_train, cnt); break;
      }
      LAUNCHED();
    }
    prof_end(st, 5, 0, (double)n_rows * ld * 2);
  }
  // counts -> fp64 for the allreduce (exact below 2^53)
  unsigned long long hc[5];
  VCHECK(cudaMemcpyAsync(hc, cnt, sizeof(hc), cudaMemcpyDeviceToHost, st));
  LRState hs;
  VCHECK(cudaMemcpyAsync(&hs, dst, sizeof(hs), cudaMemcpyDeviceToHost, st));
  res.w.resize(ld);
  VCHECK(cudaMemcpyAsync(res.w.data(), w, ld * 8, cudaMemcpyDeviceToHost, st));
  res.loss.resize(iters);
  if (iters) VCHECK(cudaMemcpyAsync(res.loss.data(), loss, iters * 8, cudaMemcpyDeviceToHost, st));
  VCHECK(cudaStreamSynchronize(st));
  double dc[6] = {(double)hc[0], (double)hc[1], (double)hc[2], (double)hc[3], (double)hc[4],
                  (double)(n_rows - n_train)};
  if (allreduce) {
    double* dd = reinterpret_cast<double*>(scr + o_G);  // reuse G
    VCHECK(cudaMemcpyAsync(dd, dc, sizeof(dc), cudaMemcpyHostToDevice, st));
    allreduce(dd, 6, st, ar_user);
    VCHECK(cudaMemcpyAsync(dc, dd, sizeof(dc), cudaMemcpyDeviceToHost, st));
    VCHECK(cudaStreamSynchronize(st));
  }
  VCHECK(cudaFreeAsync(scr, st));
  res.b = hs.b;
  res.lambda_hat = hs.lambda_hat;
  res.eta = hs.eta;
  res.n_train = (int64_t)hs.n_train;
  res.train_ok = (int64_t)dc[0];
  res.tp = (int64_t)dc[1];
  res.fp = (int64_t)dc[2];
  res.tn = (int64_t)dc[3];
  res.fn = (int64_t)dc[4];
  res.n_test = (int64_t)dc[5];
  return res;
}

}  // namespace vista
