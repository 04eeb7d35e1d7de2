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
#include <mutex>
#include <set>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

constexpr int kMaxRB = 16;     // rows per streamed block (upper bound)
constexpr int kStagesLR = 3;   // row blocks in flight per CTA
constexpr int kLRThreads = 576;  // 18 compute warps: 1041 chunks of a conv5_x row (ld 8328) = 2 per thread, no 3-chunk stragglers

struct PassArgs {
  const uint8_t* MM;   // row-major [rows][ld] elements of E (bf16, or fp32 in check mode)
  const uint8_t* y;
  int64_t r0, r1;       // row range [r0, r1) of this pass
  int64_t n_train;      // rows < n_train are train rows (eval mode)
  int ld, chunks;       // ld elements per row, chunks = ld * sizeof(E) / 16
  int rb;               // rows per streamed block
  const float* mu;      // [ld]
  const float* what;    // [ld]  inv_j * (w_j or v_j), 0 on excluded / pad columns
  const float* bhat;    // [1]
  float* partial;       // [gridDim.x][ld + 4] (16-byte aligned rows; ld + 2 used)
  unsigned long long* counts;  // eval: [5]
};

__device__ __forceinline__ float softplusf(float z) { return z > 0.f ? z + log1pf(__expf(-z)) : log1pf(__expf(z)); }

__device__ __forceinline__ void bulk_load(uint32_t dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}

// One pass over rows [r0, r1) of MM.  Rows are streamed into shared memory in blocks of
// rb contiguous rows by the bulk-copy engine (kStagesLR blocks in flight per CTA, one CTA per
// SM) issued by a dedicated producer warp, so HBM stays busy while the compute threads work.
// Compute thread t owns 16-byte column chunks t, t + nthr, ... of every row.
//   MODE 0: sum_p x_pj                          MODE 1: sum_p (x_pj - mu_j)^2
//   MODE 2: power pass  phi_p = z_p             MODE 3: gradient pass  phi_p = sigmoid(z_p) - y_p
//   MODE 4: evaluation (counts only)
// with z_p = b' + sum_j w^_j x_pj, b' = b^ - sum_j w^_j mu_j (the centred score, folded on the host
// side of the pass in fp64); modes 2/3 accumulate sum_p phi_p x_pj, sum_p phi_p and sum_p loss_p into
// this CTA's partial row (fixed row-block -> CTA map); the reduction subtracts mu_j sum_p phi_p.
// One named barrier per row block (the per-row dot products); stages are recycled through
// "empty" mbarriers, so compute warps never wait for the producer's refills.
template <typename E>
__device__ __forceinline__ void unpack16(uint4 v, float (&x)[16 / sizeof(E)]);
template <>
__device__ __forceinline__ void unpack16<bf16>(uint4 v, float (&x)[8]) {
  const uint32_t u[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    x[2 * j] = __uint_as_float(u[j] << 16);
    x[2 * j + 1] = __uint_as_float(u[j] & 0xffff0000u);
  }
}
template <>
__device__ __forceinline__ void unpack16<float>(uint4 v, float (&x)[4]) {
  x[0] = __uint_as_float(v.x);
  x[1] = __uint_as_float(v.y);
  x[2] = __uint_as_float(v.z);
  x[3] = __uint_as_float(v.w);
}

template <int CH, int MODE, typename E>
__global__ void __launch_bounds__(kLRThreads + 32, 1) lr_stream_kernel(const PassArgs a) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 127u) & ~127u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t row_bytes = (uint32_t)a.ld * (uint32_t)sizeof(E);
  const uint32_t stage_bytes = ((uint32_t)a.rb * row_bytes + 127u) & ~127u;
  float* red_all = reinterpret_cast<float*>(gbase + kStagesLR * stage_bytes);  // [kStagesLR][kMaxRB][32]
  uint64_t* full = reinterpret_cast<uint64_t*>(red_all + kStagesLR * kMaxRB * 32);  // [kStagesLR]
  uint64_t* empty = full + kStagesLR;                                               // [kStagesLR]

  const int nthr = (int)blockDim.x - 32;  // compute threads; the last warp is the producer
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwc = nthr >> 5;
  const int64_t nrows = a.r1 - a.r0;
  const int64_t nblk = (nrows + a.rb - 1) / a.rb;
  if (tid == 0) {
    for (int i = 0; i < kStagesLR; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], nthr);
    }
    fence_mbar_init();
  }
  __syncthreads();
  if (warp == nwc) {
    // ---- producer warp ----
    if (lane == 0) {
      int it = 0;
      for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x, ++it) {
        const int stage = it % kStagesLR;
        if (it >= kStagesLR) mbar_wait(&empty[stage], ((it / kStagesLR) - 1) & 1);
        const int64_t r = a.r0 + blk * a.rb;
        const int64_t nr = min((int64_t)a.rb, a.r1 - r);
        const uint32_t bytes = (uint32_t)nr * row_bytes;
        mbar_arrive_expect_tx(&full[stage], bytes);
        bulk_load(base + stage * stage_bytes, a.MM + (size_t)r * row_bytes, bytes, &full[stage]);
      }
    }
    return;
  }
  constexpr int EPC = 16 / (int)sizeof(E);  // elements per 16-byte chunk: 8 bf16 or 4 fp32
  float mu[CH][EPC], wv[CH][EPC], acc[CH][EPC];
  bool act[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tid + c * nthr;
    act[c] = ch < a.chunks;
#pragma unroll
    for (int j = 0; j < EPC; ++j) {
      mu[c][j] = (MODE == 1 && act[c]) ? a.mu[ch * EPC + j] : 0.f;
      wv[c][j] = (MODE >= 2 && act[c]) ? a.what[ch * EPC + j] : 0.f;
      acc[c][j] = 0.f;
    }
  }
  const float bh = MODE >= 2 ? a.bhat[0] : 0.f;
  float sum_r = 0.f, sum_loss = 0.f;  // warp 0, lane = row within the block
  unsigned long long cnt[5] = {0, 0, 0, 0, 0};
  int it = 0;
  for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x, ++it) {
    const int stage = it % kStagesLR;
    mbar_wait(&full[stage], (it / kStagesLR) & 1);
    const int64_t r = a.r0 + blk * a.rb;
    const int nr = (int)min((int64_t)a.rb, a.r1 - r);
    const uint32_t sbase = base + stage * stage_bytes;
    if constexpr (MODE <= 1) {
      for (int q = 0; q < nr; ++q) {
#pragma unroll
        for (int c = 0; c < CH; ++c) {
          if (c == CH - 1 && !act[c]) continue;
          float x[EPC];
          unpack16<E>(lds128(sbase + q * row_bytes + (uint32_t)(tid + c * nthr) * 16u), x);
#pragma unroll
          for (int j = 0; j < EPC; ++j) {
            if (MODE == 0) {
              acc[c][j] += x[j];
            } else {
              const float d = x[j] - mu[c][j];
              acc[c][j] = fmaf(d, d, acc[c][j]);
            }
          }
        }
      }
    } else {
      float* red = red_all + stage * (kMaxRB * 32);
      // four rows at a time: four independent FMA chains and shuffle trees
      for (int q0 = 0; q0 < nr; q0 += 4) {
        float sd[4] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll
        for (int qq = 0; qq < 4; ++qq) {
          if (q0 + qq < nr) {  // block-uniform
#pragma unroll
            for (int c = 0; c < CH; ++c) {
              if (c == CH - 1 && !act[c]) continue;  // chunks c < CH - 1 exist for every thread
              float x[EPC];
              unpack16<E>(lds128(sbase + (q0 + qq) * row_bytes + (uint32_t)(tid + c * nthr) * 16u), x);
#pragma unroll
              for (int j = 0; j < EPC; ++j) sd[qq] = fmaf(x[j], wv[c][j], sd[qq]);
            }
          }
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1)
#pragma unroll
          for (int qq = 0; qq < 4; ++qq) sd[qq] += __shfl_xor_sync(0xffffffffu, sd[qq], o);
        if (lane == 0)
#pragma unroll
          for (int qq = 0; qq < 4; ++qq)
            if (q0 + qq < nr) red[(q0 + qq) * 32 + warp] = sd[qq];
      }
      named_bar_sync(1, nthr);
      // every warp: lane q < nr forms z_q from the per-warp partials (fixed order) and phi_q
      float phi = 0.f;
      if (lane < nr) {
        float z = bh;
        for (int w = 0; w < nwc; ++w) z += red[lane * 32 + w];
        const int64_t row = r + lane;
        if (MODE == 2) {
          phi = z;
          if (warp == 0) sum_r += z;
        } else {
          const int yv = a.y[row];
          if (MODE == 3) {
            phi = 1.f / (1.f + __expf(-z)) - (float)yv;
            if (warp == 0) {
              sum_r += phi;
              sum_loss += softplusf(z) - (float)yv * z;
            }
          } else if (warp == 0) {  // MODE 4: predict 1 iff z >= 0
            const int pred = z >= 0.f ? 1 : 0;
            if (row < a.n_train) cnt[0] += pred == yv;
            else cnt[pred && yv ? 1 : (pred ? 2 : (yv ? 4 : 3))] += 1;
          }
        }
      }
      if (MODE == 2 || MODE == 3) {
        for (int q = 0; q < nr; ++q) {
          const float ph = __shfl_sync(0xffffffffu, phi, q);
#pragma unroll
          for (int c = 0; c < CH; ++c) {
            if (c == CH - 1 && !act[c]) continue;
            float x[EPC];
            unpack16<E>(lds128(sbase + q * row_bytes + (uint32_t)(tid + c * nthr) * 16u), x);
#pragma unroll
            for (int j = 0; j < EPC; ++j) acc[c][j] = fmaf(ph, x[j], acc[c][j]);
          }
        }
      }
    }
    mbar_arrive(&empty[stage]);  // this thread is done with the stage
  }
  if constexpr (MODE == 4) {
    if (warp == 0) {
#pragma unroll
      for (int k = 0; k < 5; ++k) {
        unsigned long long v = cnt[k];
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0 && v) atomicAdd(&a.counts[k], v);
      }
    }
    return;
  }
  float* out = a.partial + (size_t)blockIdx.x * (a.ld + 4);
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tid + c * nthr;
    if (act[c]) {
      float4* o = reinterpret_cast<float4*>(out + ch * EPC);
#pragma unroll
      for (int j = 0; j < EPC / 4; ++j)
        o[j] = make_float4(acc[c][4 * j], acc[c][4 * j + 1], acc[c][4 * j + 2], acc[c][4 * j + 3]);
    }
  }
  if (warp == 0) {  // fixed-order (lane) reduction of the per-row scalars
    for (int o = 16; o > 0; o >>= 1) {
      sum_r += __shfl_xor_sync(0xffffffffu, sum_r, o);
      sum_loss += __shfl_xor_sync(0xffffffffu, sum_loss, o);
    }
    if (lane == 0) {
      out[a.ld] = sum_r;
      out[a.ld + 1] = sum_loss;
    }
  }
}

// G[j] = sum_cta partial[cta][j] in fp64, fixed order (8 contiguous CTA ranges, one per warp, then
// the 8 range sums in order); ncols = ld + 2, row pitch ld + 4.  center (power / gradient passes):
// G[j] -= mu_j G[ld] for j < ld, turning sum_p phi_p x_pj into sum_p phi_p (x_pj - mu_j).
// One block per 32 columns; every block forms G[ld] with the same order, so all agree bit for bit.
__global__ void __launch_bounds__(256) reduce_partials_kernel(const float* __restrict__ partial, int nct, int ncols,
                                                              int pitch, const double* __restrict__ mu, int ld,
                                                              int center, double* G) {
  __shared__ double sh[8][33];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int c0 = (int)((int64_t)nct * warp / 8), c1 = (int)((int64_t)nct * (warp + 1) / 8);
  const int j = blockIdx.x * 32 + lane;
  double s = 0.0, t = 0.0;
  for (int c = c0; c < c1; ++c) {
    if (j < ncols) s += (double)partial[(size_t)c * pitch + j];
    if (center) t += (double)partial[(size_t)c * pitch + ld];
  }
  sh[warp][lane] = s;
  if (lane == 0) sh[warp][32] = t;
  __syncthreads();
  if (warp == 0 && j < ncols) {
    double g = 0.0, phisum = 0.0;
    for (int w = 0; w < 8; ++w) {
      g += sh[w][lane];
      phisum += sh[w][32];
    }
    if (center && j < ld) g -= mu[j] * phisum;
    G[j] = g;
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
// Both end by publishing w^ = inv * v (fp32) and b' = v_b - sum_j w^_j mu_j for the next pass.
__device__ void block_sum2(double& a, double& b, double* sh) {  // fixed order, result in every thread
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  for (int o = 16; o > 0; o >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, o);
    b += __shfl_xor_sync(0xffffffffu, b, o);
  }
  __syncthreads();
  if (lane == 0) {
    sh[warp] = a;
    sh[32 + warp] = b;
  }
  __syncthreads();
  a = b = 0.0;
  for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
    a += sh[w];
    b += sh[32 + w];
  }
}

__global__ void __launch_bounds__(1024) power_kernel(const double* G, int ld, int init, int d_real,
                                                     const uint8_t* real, const double* inv, const double* mu,
                                                     double* v, float* what, float* bhat, LRState* st) {
  __shared__ double sh[64];
  const double rn = 1.0 / st->n_train;
  double vb, scale;  // v_j = scale * (init ? real_j : inv_j G_j)
  if (init) {
    vb = 1.0 / sqrt((double)(d_real + 1));
    scale = vb;
  } else {
    double ss = 0.0, sm = 0.0;
    for (int j = threadIdx.x; j < ld; j += blockDim.x) {
      const double q = inv[j] * G[j] * rn;
      ss += q * q;
    }
    block_sum2(ss, sm, sh);
    const double qb = G[ld] * rn;
    const double lam = sqrt(ss + qb * qb);
    const double rl = lam > 0 ? 1.0 / lam : 0.0;
    vb = qb * rl;
    scale = rn * rl;
    if (threadIdx.x == 0) st->lambda_hat = lam;
  }
  double sm = 0.0, dummy = 0.0;
  for (int j = threadIdx.x; j < ld; j += blockDim.x) {
    const double vj = init ? (real[j] ? scale : 0.0) : scale * inv[j] * G[j];
    v[j] = vj;
    const double wj = inv[j] * vj;
    what[j] = (float)wj;
    sm += wj * mu[j];
  }
  block_sum2(sm, dummy, sh);
  if (threadIdx.x == 0) {
    st->vb = vb;
    bhat[0] = (float)(vb - sm);  // centred score folded into the bias
  }
}

// ISTA (O6 steps 4-5).  init: eta = 1 / (0.25 * 1.05 * lambda_hat + lambda (1 - alpha)), w = 0, b = 0.
// update: g_j = inv_j G_j / n + lambda (1 - alpha) w_j; w = soft(w - eta g, eta lambda alpha);
//         b -= eta G_ld / n; loss = G_{ld+1} / n (at the pre-update w).
__global__ void __launch_bounds__(1024) grad_kernel(const double* G, int ld, int init, double lambda, double alpha,
                                                    const double* inv, const double* mu, double* w, float* what,
                                                    float* bhat, LRState* st, double* loss_out) {
  __shared__ double sh[64];
  double b;
  if (init) {
    b = 0.0;
    if (threadIdx.x == 0) st->eta = 1.0 / (0.25 * 1.05 * st->lambda_hat + lambda * (1.0 - alpha));
  } else {
    const double rn = 1.0 / st->n_train;
    b = st->b - st->eta * G[ld] * rn;
    if (threadIdx.x == 0) *loss_out = G[ld + 1] * rn;
  }
  const double eta = init ? 0.0 : st->eta, thr = eta * lambda * alpha, l2 = lambda * (1.0 - alpha);
  const double rn = init ? 0.0 : 1.0 / st->n_train;
  double sm = 0.0, dummy = 0.0;
  for (int j = threadIdx.x; j < ld; j += blockDim.x) {
    double wj = 0.0;
    if (!init) {
      const double g = inv[j] * G[j] * rn + l2 * w[j];
      const double vv = w[j] - eta * g;
      wj = (vv > 0 ? 1.0 : (vv < 0 ? -1.0 : 0.0)) * fmax(fabs(vv) - thr, 0.0);
    }
    w[j] = wj;
    const double hj = inv[j] * wj;
    what[j] = (float)hj;
    sm += hj * mu[j];
  }
  block_sum2(sm, dummy, sh);
  __syncthreads();  // every thread has read st->b / st->eta
  if (threadIdx.x == 0) {
    st->b = b;
    bhat[0] = (float)(b - sm);  // centred score folded into the bias
  }
}

// ------------------------------------------------------------------------------------------
struct StreamCfg {
  int threads, ch, rb, grid;
  size_t smem;
};

template <int MODE, typename E>
static void run_pass(const PassArgs& a, const StreamCfg& c, cudaStream_t st) {
  auto go = [&](void (*kern)(PassArgs)) {
    ensure_smem_attr((const void*)kern, 227 * 1024);
    kern<<<c.grid, c.threads + 32, c.smem, st>>>(a);
  };
  switch (c.ch) {
    case 1: go(lr_stream_kernel<1, MODE, E>); break;
    case 2: go(lr_stream_kernel<2, MODE, E>); break;
    case 3: go(lr_stream_kernel<3, MODE, E>); break;
    case 4: go(lr_stream_kernel<4, MODE, E>); break;
    case 5: go(lr_stream_kernel<5, MODE, E>); break;
    case 6: go(lr_stream_kernel<6, MODE, E>); break;
    default: fail(1, "lr: unsupported row width");
  }
  LAUNCHED();
}

template <typename E>
static LRResult lr_train_impl(const E* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                              const uint8_t* real_host, int iters, int power_iters, double lambda, double alpha,
                              allreduce_fn allreduce, void* ar_user, cudaStream_t st) {
  LRResult res;
  constexpr int esz = (int)sizeof(E);
  if (ld % 8) fail(1, "lr: ld must be a multiple of 8");
  const int chunks = ld * esz / 16;
  // one CTA per SM streaming row blocks of ~64 KB through a 3-deep bulk-copy ring
  StreamCfg cfg;
  cfg.threads = std::min(kLRThreads, (chunks + 31) / 32 * 32);
  cfg.ch = (chunks + cfg.threads - 1) / cfg.threads;
  if (cfg.ch > 6) fail(1, "lr: row too wide");
  if (cfg.ch == 3 && chunks <= 2 * cfg.threads) cfg.ch = 2;
  cfg.rb = (int)std::max<int64_t>(1, std::min<int64_t>(kMaxRB, (200 * 1024 / kStagesLR) / ((int64_t)ld * esz)));
  const size_t stage_bytes = ((size_t)cfg.rb * ld * esz + 127) & ~(size_t)127;
  cfg.smem = kStagesLR * stage_bytes + kStagesLR * kMaxRB * 32 * 4 + 2 * kStagesLR * 8 + 128;
  if (cfg.smem > 227 * 1024) fail(1, "lr: row block does not fit in shared memory");
  auto grid_for_rows = [&](int64_t rows) {
    const int64_t blocks = (rows + cfg.rb - 1) / cfg.rb;
    return (int)std::max<int64_t>(1, std::min<int64_t>(blocks, num_sms()));
  };
  cfg.grid = grid_for_rows(n_train);
  const int grid_tr = cfg.grid;
  const int ncols = ld + 2;
  int d_real = 0;
  for (int j = 0; j < ld; ++j) d_real += real_host[j] ? 1 : 0;

  // scratch
  size_t off = 0;
  auto carve = [&](size_t bytes) { size_t o = off; off += (bytes + 255) & ~(size_t)255; return o; };
  const size_t o_part = carve((size_t)std::max(grid_tr, 1) * (ld + 4) * 4), o_G = carve(ncols * 8), o_mu = carve(ld * 8),
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
  a.MM = reinterpret_cast<const uint8_t*>(MM);
  a.y = y;
  a.r0 = 0;
  a.r1 = n_train;
  a.ld = ld;
  a.chunks = chunks;
  a.mu = mu_f;
  a.what = what;
  a.bhat = bhat;
  a.partial = partial;
  a.n_train = n_train;
  a.rb = cfg.rb;
  a.counts = nullptr;
  const double pass_bytes = (double)n_train * ld * esz;
  auto reduce = [&](double extra_n, int center) {
    prof_begin(st);
    reduce_partials_kernel<<<(ncols + 31) / 32, 256, 0, st>>>(partial, grid_tr, ncols, ld + 4, mu, ld, center, G);
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
  run_pass<0, E>(a, cfg, st);
  prof_end(st, 5, 0, pass_bytes);
  reduce((double)n_train, 0);
  stats_finalize_kernel<<<(ld + 255) / 256, 256, 0, st>>>(G, ld, 0, real, mu, mu_f, inv, dst);
  LAUNCHED();
  prof_begin(st);
  run_pass<1, E>(a, cfg, st);
  prof_end(st, 5, 0, pass_bytes);
  reduce(-1, 0);
  stats_finalize_kernel<<<(ld + 255) / 256, 256, 0, st>>>(G, ld, 1, real, mu, mu_f, inv, dst);
  LAUNCHED();
  // ---- O6 step 3: K power iterations ----
  power_kernel<<<1, ublk, 0, st>>>(G, ld, 1, d_real, real, inv, mu, v, what, bhat, dst);
  LAUNCHED();
  for (int k = 0; k < power_iters; ++k) {
    prof_begin(st);
    run_pass<2, E>(a, cfg, st);
    prof_end(st, 5, 0, pass_bytes);
    reduce(-1, 1);
    power_kernel<<<1, ublk, 0, st>>>(G, ld, 0, d_real, real, inv, mu, v, what, bhat, dst);
    LAUNCHED();
  }
  // ---- O6 steps 4-5: ISTA ----
  grad_kernel<<<1, ublk, 0, st>>>(G, ld, 1, lambda, alpha, inv, mu, w, what, bhat, dst, loss);
  LAUNCHED();
  for (int t = 0; t < iters; ++t) {
    prof_begin(st);
    run_pass<3, E>(a, cfg, st);
    prof_end(st, 5, 0, pass_bytes);
    reduce(-1, 1);
    grad_kernel<<<1, ublk, 0, st>>>(G, ld, 0, lambda, alpha, inv, mu, w, what, bhat, dst, loss + t);
    LAUNCHED();
  }
  // ---- O6 step 6: eval over all local rows ----
  {
    PassArgs e = a;
    e.r0 = 0;
    e.r1 = n_rows;
    e.counts = cnt;
    StreamCfg ce = cfg;
    ce.grid = grid_for_rows(n_rows);
    prof_begin(st);
    if (n_rows > 0) run_pass<4, E>(e, ce, st);
    prof_end(st, 5, 0, (double)n_rows * ld * esz);
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

LRResult lr_train(const bf16* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                  const uint8_t* real_host, int iters, int power_iters, double lambda, double alpha,
                  allreduce_fn allreduce, void* ar_user, cudaStream_t st) {
  return lr_train_impl<bf16>(MM, y, n_rows, n_train, ld, real_host, iters, power_iters, lambda, alpha, allreduce,
                             ar_user, st);
}

LRResult lr_train_f32(const float* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                      const uint8_t* real_host, int iters, int power_iters, double lambda, double alpha,
                      allreduce_fn allreduce, void* ar_user, cudaStream_t st) {
  return lr_train_impl<float>(MM, y, n_rows, n_train, ld, real_host, iters, power_iters, lambda, alpha, allreduce,
                              ar_user, st);
}

}  // namespace vista
