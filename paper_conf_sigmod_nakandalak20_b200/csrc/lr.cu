// lr.cu — S5 of SURVEY.md §8a: train M (logistic regression; elastic net
// alpha = 0.5, lambda = 0.01) on X'_l = [X, F_l] (Eq. (4)) by the
// full-batch proximal-gradient reading R17, step for step as O6:
//   stats (mu, sigma over train rows) -> K power iterations for lambda_max ->
//   T ISTA steps from w = 0, b = 0 -> evaluation (predict 1 iff z >= 0).
// Every pass is ONE read of MM_l (HBM-bound): each CTA owns a contiguous block of rows
// ("minibatch"), computes z_p = b + sum_j w^_j (x_pj - mu_j) per row with a block
// reduction, applies phi (identity for the power iteration, sigmoid residual for the
// gradient) and accumulates sum_p phi_p (x_pj - mu_j) per column in registers.  Per-CTA
// partials are reduced in a fixed order in fp64 (deterministic).  One rank (world == 1): the
// reduction and the fp64 update of the pass (mean / sigma, power step, ISTA step) run in the
// pass kernel's own tail, behind grid-wide barriers of the cooperative launch -- one launch per
// pass.  world > 1: partials -> reduce kernel -> fp64 allreduce (NCCL or the caller's hook) ->
// one-block update kernel.
#include <cmath>
#include <cstdlib>
#include <cstring>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

constexpr int kMaxRB = 16;     // rows per streamed block (upper bound)
constexpr int kStagesLR = 3;   // row blocks in flight per CTA
constexpr int kLRThreads = 576;  // 18 compute warps: 1041 chunks of a conv5_x row (ld 8328) = 2 per thread, no 3-chunk stragglers

struct LRState {  // device, fp64 master copies
  double n_train;   // global train rows
  double lambda_hat, eta;
  double b, vb;
  double loss;
};

// world == 1: the pass kernel reduces its partials and applies the O6 update itself (see fused_tail)
struct FusedArgs {
  int on;                 // 0: partials only (reduce / allreduce / update kernels follow)
  int ncols;              // ld + 2
  unsigned int* bar;      // [2] grid barrier: monotonic arrival count (zeroed once per lr_train)
  unsigned int sync_base; // arrivals before this pass (sum of grid syncs of earlier passes x grid)
  double* G;              // [ncols] reduced sums
  double* scal;           // [2 gridDim.x] per-CTA partial scalars (two reductions per pass at most)
  const uint8_t* real;    // [ld] real (non-padding) columns
  double *mu, *inv, *v, *w;
  float *mu_f, *what, *bhat;
  LRState* st;
  double* loss_out;       // MODE 3: loss of this iteration
  double lambda, alpha;
  int d_real;
  int init_next;          // MODE 1: initialise the power iteration; MODE 2: last power pass, initialise ISTA
};

struct PassArgs {
  const uint8_t* MM;   // row-major [rows][ld] elements of E (bf16, or fp32 in check mode)
  const uint8_t* y;
  int64_t r0, r1;       // row range [r0, r1) of this pass
  int64_t n_train;      // rows < n_train are train rows (eval mode)
  int ld, chunks;       // ld elements per row, chunks = ld * sizeof(E) / 16
  int rb;               // rows per streamed block
  int rev;              // 1: every CTA walks its row blocks last-to-first (passes alternate, so each pass starts on
                        //    the blocks the previous one read last -- still in L2)
  int alt;              // 1: directions alternate (the next pass runs with rev ^ 1)
  int pf_next;          // 1: the next pass reads the same rows -- the producer prefetches its first blocks into L2
  int dbg;              // VISTA_LR_DBG (measurement only, results wrong): 1 = dot kernel consumes blocks without computing
  const float* mu;      // [ld]
  const float* what;    // [ld]  inv_j * (w_j or v_j), 0 on excluded / pad columns
  const float* bhat;    // [1]
  float* partial;       // [gridDim.x][ld + 4] (16-byte aligned rows; ld + 2 used)
  float* zbuf;          // [r1] lr_dot_kernel MODE 3: per-row scores, the loss is summed after the row loop
  unsigned long long* counts;  // eval: [5]
  FusedArgs f;
};

template <int MODE>
__device__ void fused_tail(const PassArgs& a, uint8_t* scratch, int nthr);

// programmatic dependent launch (consecutive passes on one stream): a pass lets the next one launch as its CTAs
// exit; the next pass's producer streams rows (MM is not written by any pass) while its compute threads wait
// for the previous grid's results (w^, b', the reduced statistics)
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

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
  pdl_trigger();
  if (warp != nwc) pdl_wait();
  if (warp == nwc) {
    // ---- producer warp ----
    if (lane == 0) {
      int it = 0;
      const int64_t nb_cta = nblk > (int64_t)blockIdx.x ? (nblk - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
      for (int64_t bi = 0; bi < nb_cta; ++bi, ++it) {
        const int64_t blk = blockIdx.x + (a.rev ? nb_cta - 1 - bi : bi) * (int64_t)gridDim.x;
        const int stage = it % kStagesLR;
        if (it >= kStagesLR) mbar_wait(&empty[stage], ((it / kStagesLR) - 1) & 1);
        const int64_t r = a.r0 + blk * a.rb;
        const int64_t nr = min((int64_t)a.rb, a.r1 - r);
        const uint32_t bytes = (uint32_t)nr * row_bytes;
        mbar_arrive_expect_tx(&full[stage], bytes);
        bulk_load(base + stage * stage_bytes, a.MM + (size_t)r * row_bytes, bytes, &full[stage]);
        const int64_t pi = bi + kStagesLR;  // the block one ring-length ahead in this pass's order
        if (pi < nb_cta) {
          const int64_t pb = blockIdx.x + (a.rev ? nb_cta - 1 - pi : pi) * (int64_t)gridDim.x;
          const int64_t pr = a.r0 + pb * a.rb;
          prefetch_l2_range(a.MM + (size_t)pr * row_bytes, (uint32_t)min((int64_t)a.rb, a.r1 - pr) * row_bytes);
        }
      }
      // the next pass's first blocks into L2 while this pass drains and reduces (with alternating directions
      // they are the blocks just read: a no-op then)
      for (int64_t k = 0; a.pf_next && k < nb_cta && k < kStagesLR + 2; ++k) {
        const int64_t blk = blockIdx.x + ((a.rev ^ a.alt) ? nb_cta - 1 - k : k) * (int64_t)gridDim.x;
        const int64_t pr = a.r0 + blk * a.rb;
        prefetch_l2_range(a.MM + (size_t)pr * row_bytes, (uint32_t)min((int64_t)a.rb, a.r1 - pr) * row_bytes);
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
  const int64_t nb_cta = nblk > (int64_t)blockIdx.x ? (nblk - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  for (int64_t bi = 0; bi < nb_cta; ++bi, ++it) {
    const int64_t blk = blockIdx.x + (a.rev ? nb_cta - 1 - bi : bi) * (int64_t)gridDim.x;
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
  if (a.f.on) fused_tail<MODE>(a, gbase, nthr);
}

// ---- bf16 power / gradient / eval passes (MODE 2, 3, 4): the same schedule as lr_stream_kernel with
// an instruction-lean inner loop (ncu on the r1 kernel: 62 % issue-slot busy, FFMA 20 % of the
// instructions -- the pass was issue-bound, not HBM-bound):
//  * RB rows per block as a compile-time constant (4 / 8 / 16 by row width); a partial last block
//    computes garbage dot products for its missing rows and never uses them;
//  * every thread owns exactly CH 16-byte chunks: a chunk past the row end reads chunk 0 with w = 0
//    (no per-chunk branches), and its accumulator is never stored;
//  * bf16 pairs unpacked with one PRMT each, dot and accumulate on packed fp32 FMAs (FFMA2);
//  * the RB per-warp dot products reduced by a halving butterfly: RB - 1 + log2(32 / RB) shuffles
//    instead of 5 RB.
__device__ __forceinline__ float2 bf2_f2(uint32_t u) {  // exact: bf16 = the high half of an fp32
  return make_float2(__uint_as_float(__byte_perm(u, 0u, 0x1044u)), __uint_as_float(__byte_perm(u, 0u, 0x3244u)));
}
__device__ __forceinline__ float2 ffma2(float2 a, float2 b, float2 c) {  // (a.x b.x + c.x, a.y b.y + c.y), RN
  unsigned long long r;
  asm("fma.rn.f32x2 %0, %1, %2, %3;"
      : "=l"(r)
      : "l"(*reinterpret_cast<unsigned long long*>(&a)), "l"(*reinterpret_cast<unsigned long long*>(&b)),
        "l"(*reinterpret_cast<unsigned long long*>(&c)));
  return *reinterpret_cast<float2*>(&r);
}

// v[0..N) per lane -> after the call, lane l holds the warp sum of value (l >> (5 - log2 N)) in v[0]
// (valid in every lane; representative lanes: l % (32 / N) == 0).  Fixed order: deterministic.
template <int N>
__device__ __forceinline__ void butterfly(float (&v)[16], int lane) {
  int o = 16;
#pragma unroll
  for (int n = N; n > 1; n >>= 1, o >>= 1) {
    const bool up = (lane & o) != 0;
#pragma unroll
    for (int i = 0; i < n / 2; ++i) {
      const float send = up ? v[i] : v[i + n / 2];
      const float keep = up ? v[i + n / 2] : v[i];
      v[i] = keep + __shfl_xor_sync(0xffffffffu, send, o);
    }
  }
#pragma unroll
  for (; o > 0; o >>= 1) v[0] += __shfl_xor_sync(0xffffffffu, v[0], o);
}

template <int RB, int CH, int MODE>
__global__ void __launch_bounds__(kLRThreads + 32, 1) lr_dot_kernel(const PassArgs a) {
  static_assert(RB == 4 || RB == 8 || RB == 16, "rows per block");
  constexpr int LOGRB = RB == 4 ? 2 : (RB == 8 ? 3 : 4);
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 127u) & ~127u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t row_bytes = (uint32_t)a.ld * 2u;
  const uint32_t stage_bytes = ((uint32_t)RB * row_bytes + 127u) & ~127u;
  float* red_all = reinterpret_cast<float*>(gbase + kStagesLR * stage_bytes);  // [kStagesLR][kMaxRB][32]
  uint64_t* full = reinterpret_cast<uint64_t*>(red_all + kStagesLR * kMaxRB * 32);
  uint64_t* empty = full + kStagesLR;
  const int nthr = (int)blockDim.x - 32;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, nwc = nthr >> 5;
  const int64_t nrows = a.r1 - a.r0;
  const int64_t nblk = (nrows + RB - 1) / RB;
  if (tid == 0) {
    for (int i = 0; i < kStagesLR; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], nthr);
    }
    fence_mbar_init();
  }
  __syncthreads();
  pdl_trigger();
  if (warp != nwc) pdl_wait();
  if (warp == nwc) {  // producer warp: bulk copies of RB-row blocks into the ring
    if (lane == 0) {
      int it = 0;
      const int64_t nb_cta = nblk > (int64_t)blockIdx.x ? (nblk - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
      for (int64_t bi = 0; bi < nb_cta; ++bi, ++it) {
        const int64_t blk = blockIdx.x + (a.rev ? nb_cta - 1 - bi : bi) * (int64_t)gridDim.x;
        const int stage = it % kStagesLR;
        if (it >= kStagesLR) mbar_wait(&empty[stage], ((it / kStagesLR) - 1) & 1);
        const int64_t r = a.r0 + blk * RB;
        const uint32_t bytes = (uint32_t)min((int64_t)RB, a.r1 - r) * row_bytes;
        mbar_arrive_expect_tx(&full[stage], bytes);
        bulk_load(base + stage * stage_bytes, a.MM + (size_t)r * row_bytes, bytes, &full[stage]);
        // the block one ring-length ahead goes to L2 now: more bytes in flight than the ring holds
        const int64_t pi = bi + kStagesLR;  // the block one ring-length ahead in this pass's order
        if (pi < nb_cta) {
          const int64_t pb = blockIdx.x + (a.rev ? nb_cta - 1 - pi : pi) * (int64_t)gridDim.x;
          const int64_t pr = a.r0 + pb * RB;
          prefetch_l2_range(a.MM + (size_t)pr * row_bytes, (uint32_t)min((int64_t)RB, a.r1 - pr) * row_bytes);
        }
      }
      // the next pass's first blocks into L2 while this pass drains and reduces (with alternating directions
      // they are the blocks just read: a no-op then)
      for (int64_t k = 0; a.pf_next && k < nb_cta && k < kStagesLR + 2; ++k) {
        const int64_t blk = blockIdx.x + ((a.rev ^ a.alt) ? nb_cta - 1 - k : k) * (int64_t)gridDim.x;
        const int64_t pr = a.r0 + blk * RB;
        prefetch_l2_range(a.MM + (size_t)pr * row_bytes, (uint32_t)min((int64_t)RB, a.r1 - pr) * row_bytes);
      }
    }
    return;
  }
  uint32_t coff[CH];
  float2 wv[CH][4], acc[CH][4];
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tid + c * nthr;
    const bool act = ch < a.chunks;
    coff[c] = act ? (uint32_t)ch * 16u : 0u;
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      wv[c][j] = act ? make_float2(a.what[ch * 8 + 2 * j], a.what[ch * 8 + 2 * j + 1]) : make_float2(0.f, 0.f);
      acc[c][j] = make_float2(0.f, 0.f);
    }
  }
  const float bh = a.bhat[0];
  float sum_r = 0.f, sum_loss = 0.f;
  unsigned long long cnt[5] = {0, 0, 0, 0, 0};
  int it = 0;
  const int64_t nb_cta = nblk > (int64_t)blockIdx.x ? (nblk - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  for (int64_t bi = 0; bi < nb_cta; ++bi, ++it) {
    const int64_t blk = blockIdx.x + (a.rev ? nb_cta - 1 - bi : bi) * (int64_t)gridDim.x;
    const int stage = it % kStagesLR;
    const int64_t r = a.r0 + blk * RB;
    const int nr = (int)min((int64_t)RB, a.r1 - r);
    // labels of the block's rows: loaded before the data wait so their latency leaves the per-block chain
    const int yv = (MODE != 2 && lane < nr) ? (int)a.y[r + lane] : 0;
    mbar_wait(&full[stage], (it / kStagesLR) & 1);
    if (a.dbg == 1) {
      mbar_arrive(&empty[stage]);
      continue;
    }
    const uint8_t* sb = gbase + stage * stage_bytes;
    float* red = red_all + stage * (kMaxRB * 32);
    float sd[16];
    if (a.dbg != 3) {
#pragma unroll
    for (int q = 0; q < RB; ++q) {
      float2 s2 = make_float2(0.f, 0.f);
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        const uint4 v = *reinterpret_cast<const uint4*>(sb + q * row_bytes + coff[c]);
        s2 = ffma2(bf2_f2(v.x), wv[c][0], s2);
        s2 = ffma2(bf2_f2(v.y), wv[c][1], s2);
        s2 = ffma2(bf2_f2(v.z), wv[c][2], s2);
        s2 = ffma2(bf2_f2(v.w), wv[c][3], s2);
      }
      sd[q] = s2.x + s2.y;
    }
    butterfly<RB>(sd, lane);
    if ((lane & ((32 >> LOGRB) - 1)) == 0) red[(lane >> (5 - LOGRB)) * 32 + warp] = sd[0];
    named_bar_sync(1, nthr);
    }
    // every warp: lane q < nr forms z_q from the per-warp partials (fixed order) and phi_q
    float phi = a.dbg == 3 ? 1.f : 0.f;
    if (lane < nr && a.dbg != 3) {
      float z = bh;
      const float* rq = red + lane * 32;
      for (int w = 0; w < nwc; ++w) z += rq[w];
      const int64_t row = r + lane;
      if (MODE == 2) {
        phi = z;
        if (warp == 0) sum_r += z;
      } else {
        if (MODE == 3) {
          phi = 1.f / (1.f + __expf(-z)) - (float)yv;
          if (warp == 0) {
            sum_r += phi;
            a.zbuf[row] = z;  // loss after the row loop (softplus off the per-block chain)
          }
        } else if (warp == 0) {  // MODE 4: predict 1 iff z >= 0
          const int pred = z >= 0.f ? 1 : 0;
          if (row < a.n_train) cnt[0] += pred == yv;
          else cnt[pred && yv ? 1 : (pred ? 2 : (yv ? 4 : 3))] += 1;
        }
      }
    }
    if (MODE != 4 && a.dbg != 2) {
#pragma unroll
      for (int q = 0; q < RB; ++q) {
        if (q < nr) {  // block-uniform
          const float ph = __shfl_sync(0xffffffffu, phi, q);
          const float2 p2 = make_float2(ph, ph);
#pragma unroll
          for (int c = 0; c < CH; ++c) {
            const uint4 v = *reinterpret_cast<const uint4*>(sb + q * row_bytes + coff[c]);
            acc[c][0] = ffma2(bf2_f2(v.x), p2, acc[c][0]);
            acc[c][1] = ffma2(bf2_f2(v.y), p2, acc[c][1]);
            acc[c][2] = ffma2(bf2_f2(v.z), p2, acc[c][2]);
            acc[c][3] = ffma2(bf2_f2(v.w), p2, acc[c][3]);
          }
        }
      }
    }
    mbar_arrive(&empty[stage]);
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
  } else {
    if constexpr (MODE == 3) {
      // sum_p softplus(z_p) - y_p z_p over this CTA's rows (scores stored by warp 0), fixed order: thread-strided
      // partial sums, warp shuffles, then the warps in order
      __threadfence_block();
      named_bar_sync(1, nthr);
      float l = 0.f;
      for (int64_t i = tid; i < nb_cta * RB; i += nthr) {
        const int64_t row = a.r0 + (blockIdx.x + (i / RB) * (int64_t)gridDim.x) * RB + (i % RB);
        if (row < a.r1) {
          const float z = a.zbuf[row];
          l += softplusf(z) - (float)a.y[row] * z;
        }
      }
      for (int o = 16; o > 0; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o);
      if (lane == 0) red_all[warp] = l;
      named_bar_sync(1, nthr);
      sum_loss = 0.f;
      for (int w = 0; w < nwc; ++w) sum_loss += red_all[w];
    }
    float* out = a.partial + (size_t)blockIdx.x * (a.ld + 4);
#pragma unroll
    for (int c = 0; c < CH; ++c) {
      const int ch = tid + c * nthr;
      if (ch < a.chunks) {
        float4* o = reinterpret_cast<float4*>(out + ch * 8);
        o[0] = make_float4(acc[c][0].x, acc[c][0].y, acc[c][1].x, acc[c][1].y);
        o[1] = make_float4(acc[c][2].x, acc[c][2].y, acc[c][3].x, acc[c][3].y);
      }
    }
    if (warp == 0) {
      for (int o = 16; o > 0; o >>= 1) sum_r += __shfl_xor_sync(0xffffffffu, sum_r, o);
      if (lane == 0) {
        out[a.ld] = sum_r;
        out[a.ld + 1] = sum_loss;  // MODE 3: the CTA total above; MODE 2: 0
      }
    }
    if (a.f.on) fused_tail<MODE>(a, gbase, nthr);
  }
}

// ---- two-group variant of lr_dot_kernel (power / gradient / eval passes of wide rows) ----
// ncu on lr_dot_kernel<4, 2, 2> (conv5_x layer, 16k rows): 39 % issue-slot busy, 0.88 eligible warps per
// scheduler, a quarter of the stall samples at the per-block CTA barrier -- every compute warp walks the
// same serial chain per row block (dots -> butterfly -> barrier -> z -> phi -> accumulate) in lockstep.
// Here the compute warps form two independent groups of kGW warps; group g consumes the row blocks
// it % 2 == g of this CTA (two rows per block, kStages2 blocks in flight), syncing only its own warps
// (named barrier 1 + 2g), so one group's chain overlaps the other's.  Each thread owns CH 16-byte column
// chunks (tg, tg + 32 kGW, ...) in BOTH groups with separate accumulators; at the end group 1's sums are
// added to group 0's in a fixed order (deterministic).
constexpr int kGW = 9;         // warps per consumer group
constexpr int kStages2 = 5;    // two-row blocks in flight per CTA
template <int CH, int MODE>
__global__ void __launch_bounds__(2 * kGW * 32 + 32, 1) lr_dot2_kernel(const PassArgs a) {
  constexpr int RB = 2, NG = kGW * 32;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 127u) & ~127u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t row_bytes = (uint32_t)a.ld * 2u;
  const uint32_t stage_bytes = ((uint32_t)RB * row_bytes + 127u) & ~127u;
  float* red_all = reinterpret_cast<float*>(gbase + kStages2 * stage_bytes);  // [kStages2][RB][16]
  uint64_t* full = reinterpret_cast<uint64_t*>(red_all + kStages2 * RB * 16);
  uint64_t* empty = full + kStages2;
  // w^ in shared memory (fp32, 8 zeros past the end for inactive chunks): keeps CH = 4 free of spills
  float* wsm = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(empty + kStages2) + 16);
  const int nthr = 2 * NG;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int grp = warp / kGW, gw = warp - grp * kGW, tg = tid - grp * NG;
  const int64_t nrows = a.r1 - a.r0;
  const int64_t nblk = (nrows + RB - 1) / RB;
  if (tid == 0) {
    for (int i = 0; i < kStages2; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], NG);
    }
    fence_mbar_init();
  }
  __syncthreads();
  pdl_trigger();
  if (warp != 2 * kGW) pdl_wait();
  if (warp == 2 * kGW) {  // producer warp
    if (lane == 0) {
      int it = 0;
      for (int64_t blk = blockIdx.x; blk < nblk; blk += gridDim.x, ++it) {
        const int stage = it % kStages2;
        if (it >= kStages2) mbar_wait(&empty[stage], ((it / kStages2) - 1) & 1);
        const int64_t r = a.r0 + blk * RB;
        const uint32_t bytes = (uint32_t)min((int64_t)RB, a.r1 - r) * row_bytes;
        mbar_arrive_expect_tx(&full[stage], bytes);
        bulk_load(base + stage * stage_bytes, a.MM + (size_t)r * row_bytes, bytes, &full[stage]);
        const int64_t pb = blk + (int64_t)kStages2 * gridDim.x;
        if (pb < nblk) {
          const int64_t pr = a.r0 + pb * RB;
          prefetch_l2_range(a.MM + (size_t)pr * row_bytes, (uint32_t)min((int64_t)RB, a.r1 - pr) * row_bytes);
        }
      }
    }
    return;
  }
  for (int i = tid; i < a.chunks * 8 + 8; i += nthr) wsm[i] = i < a.chunks * 8 ? a.what[i] : 0.f;
  named_bar_sync(2, nthr);
  uint32_t coff[CH], woff[CH];
  float2 acc[CH][4];
#pragma unroll
  for (int c = 0; c < CH; ++c) {
    const int ch = tg + c * NG;
    const bool act = ch < a.chunks;
    coff[c] = act ? (uint32_t)ch * 16u : 0u;
    woff[c] = act ? (uint32_t)ch * 8u : (uint32_t)a.chunks * 8u;
#pragma unroll
    for (int j = 0; j < 4; ++j) acc[c][j] = make_float2(0.f, 0.f);
  }
  const float bh = a.bhat[0];
  float sum_r = 0.f, sum_loss = 0.f;
  unsigned long long cnt[5] = {0, 0, 0, 0, 0};
  int it = grp;
  for (int64_t blk = blockIdx.x + (int64_t)grp * gridDim.x; blk < nblk; blk += 2 * (int64_t)gridDim.x, it += 2) {
    const int stage = it % kStages2;
    mbar_wait(&full[stage], (it / kStages2) & 1);
    const int64_t r = a.r0 + blk * RB;
    const int nr = (int)min((int64_t)RB, a.r1 - r);
    const uint8_t* sb = gbase + stage * stage_bytes;
    float* red = red_all + stage * (RB * 16);
    float sd[16];
#pragma unroll
    for (int q = 0; q < RB; ++q) {
      float2 s2 = make_float2(0.f, 0.f);
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        const uint4 v = *reinterpret_cast<const uint4*>(sb + q * row_bytes + coff[c]);
        const float4 w0 = *reinterpret_cast<const float4*>(wsm + woff[c]);
        const float4 w1 = *reinterpret_cast<const float4*>(wsm + woff[c] + 4);
        s2 = ffma2(bf2_f2(v.x), make_float2(w0.x, w0.y), s2);
        s2 = ffma2(bf2_f2(v.y), make_float2(w0.z, w0.w), s2);
        s2 = ffma2(bf2_f2(v.z), make_float2(w1.x, w1.y), s2);
        s2 = ffma2(bf2_f2(v.w), make_float2(w1.z, w1.w), s2);
      }
      sd[q] = s2.x + s2.y;
    }
    butterfly<RB>(sd, lane);
    if ((lane & 15) == 0) red[(lane >> 4) * 16 + gw] = sd[0];
    named_bar_sync(1 + 2 * grp, NG);
    float phi = 0.f;
    if (lane < nr) {
      float z = bh;
      const float* rq = red + lane * 16;
#pragma unroll
      for (int w = 0; w < kGW; ++w) z += rq[w];
      const int64_t row = r + lane;
      if (MODE == 2) {
        phi = z;
        if (gw == 0) sum_r += z;
      } else {
        const int yv = a.y[row];
        if (MODE == 3) {
          phi = 1.f / (1.f + __expf(-z)) - (float)yv;
          if (gw == 0) {
            sum_r += phi;
            sum_loss += softplusf(z) - (float)yv * z;
          }
        } else if (gw == 0) {  // MODE 4: predict 1 iff z >= 0
          const int pred = z >= 0.f ? 1 : 0;
          if (row < a.n_train) cnt[0] += pred == yv;
          else cnt[pred && yv ? 1 : (pred ? 2 : (yv ? 4 : 3))] += 1;
        }
      }
    }
    if (MODE != 4) {
#pragma unroll
      for (int q = 0; q < RB; ++q) {
        if (q < nr) {  // group-uniform
          const float ph = __shfl_sync(0xffffffffu, phi, q);
          const float2 p2 = make_float2(ph, ph);
#pragma unroll
          for (int c = 0; c < CH; ++c) {
            const uint4 v = *reinterpret_cast<const uint4*>(sb + q * row_bytes + coff[c]);
            acc[c][0] = ffma2(bf2_f2(v.x), p2, acc[c][0]);
            acc[c][1] = ffma2(bf2_f2(v.y), p2, acc[c][1]);
            acc[c][2] = ffma2(bf2_f2(v.z), p2, acc[c][2]);
            acc[c][3] = ffma2(bf2_f2(v.w), p2, acc[c][3]);
          }
        }
      }
    }
    mbar_arrive(&empty[stage]);
  }
  if constexpr (MODE == 4) {
    if (gw == 0) {
#pragma unroll
      for (int k = 0; k < 5; ++k) {
        unsigned long long v = cnt[k];
        for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (lane == 0 && v) atomicAdd(&a.counts[k], v);
      }
    }
    return;
  } else {
    // group 1 hands its sums to group 0 through the (drained) ring: [chunk][8] floats + 2 scalars
    named_bar_sync(2, nthr);  // both groups done with every stage
    float* xfer = reinterpret_cast<float*>(gbase);
    if (grp == 1) {
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        const int ch = tg + c * NG;
        if (ch < a.chunks) {
          float4* o = reinterpret_cast<float4*>(xfer + ch * 8);
          o[0] = make_float4(acc[c][0].x, acc[c][0].y, acc[c][1].x, acc[c][1].y);
          o[1] = make_float4(acc[c][2].x, acc[c][2].y, acc[c][3].x, acc[c][3].y);
        }
      }
      if (gw == 0) {
        for (int o = 16; o > 0; o >>= 1) {
          sum_r += __shfl_xor_sync(0xffffffffu, sum_r, o);
          sum_loss += __shfl_xor_sync(0xffffffffu, sum_loss, o);
        }
        if (lane == 0) {
          xfer[a.ld + 8] = sum_r;
          xfer[a.ld + 9] = sum_loss;
        }
      }
    }
    named_bar_sync(2, nthr);
    float* out = a.partial + (size_t)blockIdx.x * (a.ld + 4);
    if (grp == 0) {
#pragma unroll
      for (int c = 0; c < CH; ++c) {
        const int ch = tg + c * NG;
        if (ch < a.chunks) {
          const float4* o1 = reinterpret_cast<const float4*>(xfer + ch * 8);
          const float4 u0 = o1[0], u1 = o1[1];
          float4* o = reinterpret_cast<float4*>(out + ch * 8);
          o[0] = make_float4(acc[c][0].x + u0.x, acc[c][0].y + u0.y, acc[c][1].x + u0.z, acc[c][1].y + u0.w);
          o[1] = make_float4(acc[c][2].x + u1.x, acc[c][2].y + u1.y, acc[c][3].x + u1.z, acc[c][3].y + u1.w);
        }
      }
      if (gw == 0) {
        for (int o = 16; o > 0; o >>= 1) {
          sum_r += __shfl_xor_sync(0xffffffffu, sum_r, o);
          sum_loss += __shfl_xor_sync(0xffffffffu, sum_loss, o);
        }
        if (lane == 0) {
          out[a.ld] = sum_r + xfer[a.ld + 8];
          out[a.ld + 1] = sum_loss + xfer[a.ld + 9];
        }
      }
    }
    if (a.f.on) {
      named_bar_sync(2, nthr);  // the transfer area is read before the tail reuses the ring
      fused_tail<MODE>(a, gbase, nthr);
    }
  }
}

// ---- fused reduce + update (world == 1) ----
// Grid-wide barrier of the cooperative launch (all CTAs co-resident): compute threads only (the
// producer warp has exited), named barrier 2 inside the CTA, one arrival per CTA on a global counter.
__device__ __forceinline__ void grid_sync(unsigned int* bar, int nthr, unsigned int target) {
  // monotonic counter: every CTA adds one with a fire-and-forget release reduction (no round trip, no reset, so
  // 148 arrivals pipeline in the L2 instead of serialising as returning atomics) and waits for the k-th sync's
  // total, target = sync_base + k * gridDim.x
  named_bar_sync(2, nthr);
  if (threadIdx.x == 0) {
    __threadfence();
    asm volatile("red.release.gpu.global.add.u32 [%0], 1;" ::"l"(bar) : "memory");
    unsigned int v;
    while (true) {
      asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(bar) : "memory");
      if (v >= target) break;
      __nanosleep(32);
    }
  }
  named_bar_sync(2, nthr);
}

// out[i] = sum over the G CTAs' partial rows of column j0 + i, i < n, in fp64 and a fixed order (each
// warp sums a contiguous CTA range per 32-column tile, then the warp sums in warp order).  Every CTA
// calling it for the same column gets the same bits.  sh: >= nwc * 32 doubles of shared memory.
__device__ void reduce_cols(const float* partial, int pitch, int G, int j0, int n, int ld, double* out, double* out2,
                            double* sh, int nthr) {
  // virtual column i < n + 2: partial column j0 + i (i < n) -> out[i], or ld + i - n (the two scalar columns,
  // reduced redundantly by every CTA: identical bits) -> out2[i - n]; one sweep serves both
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwc = nthr >> 5;
  const int nv = n + 2;
  auto col = [&](int i) { return i < n ? j0 + i : ld + (i - n); };
  auto put = [&](int i, double v) {
    if (i < n) out[i] = v;
    else out2[i - n] = v;
  };
  if (G < 4 * nwc) {
    // few CTAs (small inputs): the CTA-range split would leave most warps idle and walk the columns 32 at
    // a time behind two barriers each (measured: ~30 us per pass for one CTA at ld 4104); instead each
    // lane sums whole columns over the G partial rows in CTA order, warps on different 32-column tiles
    for (int t = warp * 32; t < nv; t += nwc * 32) {
      if (t + lane < nv) {
        const float* pc = partial + col(t + lane);
        double s = 0.0;
        for (int c = 0; c < G; ++c) s += (double)__ldcg(pc + (size_t)c * pitch);
        put(t + lane, s);
      }
    }
    named_bar_sync(2, nthr);
    return;
  }
  const int c0 = (int)((int64_t)G * warp / nwc), c1 = (int)((int64_t)G * (warp + 1) / nwc);
  for (int t = 0; t < nv; t += 32) {
    double s = 0.0;
    if (t + lane < nv) {
      const float* pc = partial + col(t + lane);
      int c = c0;
      for (; c + 8 <= c1; c += 8) {  // eight independent L2 loads in flight, added in order
        float x[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) x[u] = __ldcg(pc + (size_t)(c + u) * pitch);
#pragma unroll
        for (int u = 0; u < 8; ++u) s += (double)x[u];
      }
      for (; c < c1; ++c) s += (double)__ldcg(pc + (size_t)c * pitch);
    }
    sh[warp * 32 + lane] = s;
    named_bar_sync(2, nthr);
    if (warp == 0 && t + lane < nv) {
      double g = 0.0;
      for (int w = 0; w < nwc; ++w) g += sh[w * 32 + lane];
      put(t + lane, g);
    }
    named_bar_sync(2, nthr);
  }
}

// fixed-order sum of one double per compute thread (result in every thread)
__device__ double cta_sum(double v, double* sh, int nthr) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwc = nthr >> 5;
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  if (lane == 0) sh[warp] = v;
  named_bar_sync(2, nthr);
  double t = 0.0;
  for (int w = 0; w < nwc; ++w) t += sh[w];
  named_bar_sync(2, nthr);
  return t;
}

// the same for two values at once (one pair of barriers)
__device__ void cta_sum2(double& a, double& b, double* sh, int nthr) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwc = nthr >> 5;
  for (int o = 16; o > 0; o >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, o);
    b += __shfl_xor_sync(0xffffffffu, b, o);
  }
  if (lane == 0) {
    sh[warp] = a;
    sh[32 + warp] = b;
  }
  named_bar_sync(2, nthr);
  double ta = 0.0, tb = 0.0;
  for (int w = 0; w < nwc; ++w) {
    ta += sh[w];
    tb += sh[32 + w];
  }
  named_bar_sync(2, nthr);
  a = ta;
  b = tb;
}

// fixed-order sum of the G per-CTA scalars (result in every thread of every CTA, same bits)
__device__ double grid_scalar_sum(const double* scal, double* sh, int nthr) {
  if ((threadIdx.x >> 5) == 0) {
    const int lane = threadIdx.x & 31;
    double s = 0.0;
    for (int c = lane; c < (int)gridDim.x; c += 32) s += __ldcg(scal + c);
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) sh[0] = s;
  }
  named_bar_sync(2, nthr);
  const double t = sh[0];
  named_bar_sync(2, nthr);
  return t;
}

// The O6 update of one pass, distributed over the CTAs of the pass: CTA b owns columns
// [b ncols / G, (b + 1) ncols / G) of the reduction and [b ld / G, (b + 1) ld / G) of the update.
//   MODE 0: mu = G / n                    MODE 1: inv = 1 / sigma (+ power-iteration start)
//   MODE 2: power step (lambda, v, w^)    MODE 3: ISTA step (w, b, loss)
// Same arithmetic as stats_finalize_kernel / power_kernel / grad_kernel (world > 1 path).
template <int MODE>
__device__ void fused_tail(const PassArgs& a, uint8_t* scratch, int nthr) {
  const FusedArgs& f = a.f;
  const int G = gridDim.x, b = blockIdx.x, ld = a.ld, pitch = ld + 4;
  double* sh = reinterpret_cast<double*>(scratch);  // [nwc * 32]
  double* gs = sh + 32 * 32;                        // this CTA's reduced columns
  double* g2 = gs + ((ld + G - 1) / G + 2);         // G[ld], G[ld + 1]
  __threadfence();
  grid_sync(f.bar, nthr, f.sync_base + G);  // every CTA's partial row is written
  const int u0 = (int)((int64_t)ld * b / G), u1 = (int)((int64_t)ld * (b + 1) / G);
  reduce_cols(a.partial, pitch, G, u0, u1 - u0, ld, gs, g2, sh, nthr);
  const double phisum = g2[0];
  LRState* st = f.st;
  if (MODE == 0) {
    const double n = (double)a.n_train;
    for (int j = u0 + threadIdx.x; j < u1; j += nthr) {
      const double m = gs[j - u0] / n;
      f.mu[j] = m;
      f.mu_f[j] = (float)m;
    }
    if (b == 0 && threadIdx.x == 0) st->n_train = n;
    return;
  }
  const double n = st->n_train, rn = 1.0 / n;
  if (MODE == 1) {
    const double vb = 1.0 / sqrt((double)(f.d_real + 1));
    double sm = 0.0;
    for (int j = u0 + threadIdx.x; j < u1; j += nthr) {
      const double sigma = sqrt(gs[j - u0] / n);
      const double iv = (f.real[j] && sigma > 1e-12) ? 1.0 / sigma : 0.0;
      f.inv[j] = iv;
      // power-iteration start (O6 step 3): v = 1 / sqrt(d + 1) on real columns and the bias
      const double vj = f.real[j] ? vb : 0.0;
      f.v[j] = vj;
      const double wj = iv * vj;
      f.what[j] = (float)wj;
      sm += wj * f.mu[j];
    }
    sm = cta_sum(sm, sh, nthr);
    if (threadIdx.x == 0) f.scal[b] = sm;
    __threadfence();
    grid_sync(f.bar, nthr, f.sync_base + 2 * G);
    const double tot = grid_scalar_sum(f.scal, sh, nthr);
    if (b == 0 && threadIdx.x == 0) {
      st->vb = vb;
      f.bhat[0] = (float)(vb - tot);
    }
    return;
  }
  if (MODE == 2) {
    // centre: G_j <- G_j - mu_j sum_p phi_p; q_j = inv_j G_j / n; lambda = ||(q, q_b)||.  With v = q / lambda:
    // w^_j = inv_j v_j and b' = v_b - sum_j w^_j mu_j = (q_b - sum_j inv_j q_j mu_j) / lambda, so one grid
    // reduction of (sum q_j^2, sum inv_j q_j mu_j) serves both
    double ss = 0.0, sq = 0.0;
    for (int j = u0 + threadIdx.x; j < u1; j += nthr) {
      const double g = gs[j - u0] - f.mu[j] * phisum;
      gs[j - u0] = g;
      const double q = f.inv[j] * g * rn;
      ss += q * q;
      sq += f.inv[j] * q * f.mu[j];
    }
    cta_sum2(ss, sq, sh, nthr);
    if (threadIdx.x == 0) {
      f.scal[b] = ss;
      f.scal[G + b] = sq;
    }
    __threadfence();
    grid_sync(f.bar, nthr, f.sync_base + 2 * G);
    const double qb = phisum * rn;
    const double lam = sqrt(grid_scalar_sum(f.scal, sh, nthr) + qb * qb);
    const double sqt = grid_scalar_sum(f.scal + G, sh, nthr);
    const double rl = lam > 0 ? 1.0 / lam : 0.0;
    if (f.init_next) {
      // last power pass: lambda_hat is final; start ISTA (O6 step 4): eta = 1 / L, w = 0, b = 0
      for (int j = u0 + threadIdx.x; j < u1; j += nthr) {
        f.w[j] = 0.0;
        f.what[j] = 0.f;
      }
      if (b == 0 && threadIdx.x == 0) {
        st->lambda_hat = lam;
        st->eta = 1.0 / (0.25 * 1.05 * lam + f.lambda * (1.0 - f.alpha));
        st->b = 0.0;
        f.bhat[0] = 0.f;
      }
      return;
    }
    const double scale = rn * rl;
    for (int j = u0 + threadIdx.x; j < u1; j += nthr) {
      const double vj = scale * f.inv[j] * gs[j - u0];
      f.v[j] = vj;
      f.what[j] = (float)(f.inv[j] * vj);
    }
    if (b == 0 && threadIdx.x == 0) {
      st->lambda_hat = lam;
      st->vb = qb * rl;
      f.bhat[0] = (float)((qb - sqt) * rl);
    }
    return;
  }
  // MODE 3: ISTA step (O6 step 5) at the pre-update w: loss, g, soft threshold; bias unregularised
  const double eta = st->eta, thr = eta * f.lambda * f.alpha, l2 = f.lambda * (1.0 - f.alpha);
  const double bnew = st->b - eta * phisum * rn;
  double sm = 0.0;
  for (int j = u0 + threadIdx.x; j < u1; j += nthr) {
    const double g = f.inv[j] * (gs[j - u0] - f.mu[j] * phisum) * rn + l2 * f.w[j];
    const double vv = f.w[j] - eta * g;
    const double wj = (vv > 0 ? 1.0 : (vv < 0 ? -1.0 : 0.0)) * fmax(fabs(vv) - thr, 0.0);
    f.w[j] = wj;
    const double hj = f.inv[j] * wj;
    f.what[j] = (float)hj;
    sm += hj * f.mu[j];
  }
  sm = cta_sum(sm, sh, nthr);
  if (threadIdx.x == 0) f.scal[b] = sm;
  __threadfence();
  grid_sync(f.bar, nthr, f.sync_base + 2 * G);  // every CTA has read st->b / st->eta
  const double tot = grid_scalar_sum(f.scal, sh, nthr);
  if (b == 0 && threadIdx.x == 0) {
    st->b = bnew;
    *f.loss_out = g2[1] * rn;
    f.bhat[0] = (float)(bnew - tot);
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
  int dot_rb = 0;       // bf16 power / gradient / eval passes on lr_dot_kernel<dot_rb, ch, MODE> (0: not used)
  size_t dot_smem = 0;
  int dot2_ch = 0;      // > 0: those passes on lr_dot2_kernel<dot2_ch, MODE> (two consumer groups)
  size_t dot2_smem = 0;
};

static void launch_pass(const void* kern, const PassArgs& a, int grid, int threads, size_t smem, bool coop,
                        cudaStream_t st) {
  ensure_smem_attr(kern, 227 * 1024);
  static const bool coop_ok = !(getenv("VISTA_LR_COOP") && getenv("VISTA_LR_COOP")[0] == '0');  // A/B only
  static const bool pdl_ok = !(getenv("VISTA_LR_PDL") && getenv("VISTA_LR_PDL")[0] == '0');  // A/B only
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  int na = 0;
  if (coop && coop_ok) {  // the fused tail's grid barriers need every CTA resident: cooperative launch guarantees it
    attr[na].id = cudaLaunchAttributeCooperative;
    attr[na++].val.cooperative = 1;
  }
  if (pdl_ok) {
    attr[na].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[na++].val.programmaticStreamSerializationAllowed = 1;
  }
  cfg.attrs = attr;
  cfg.numAttrs = na;
  void* args[] = {const_cast<PassArgs*>(&a)};
  VCHECK(cudaLaunchKernelExC(&cfg, kern, args));
  LAUNCHED();
}

template <int MODE, typename E>
static void run_pass(const PassArgs& a_in, const StreamCfg& c, cudaStream_t st) {
  // alternating block order (PassArgs::rev): a per-thread pass counter picks the direction (VISTA_LR_REV=0: off)
  PassArgs a = a_in;
  static thread_local unsigned pass_no = 0;
  a.alt = (c.dot2_ch > 0 || (getenv("VISTA_LR_REV") && getenv("VISTA_LR_REV")[0] == '0')) ? 0 : 1;
  a.rev = a.alt ? (int)(pass_no++ & 1u) : 0;
  const bool coop = a.f.on != 0;
  if constexpr (MODE >= 2 && sizeof(E) == 2) {
    if (c.dot2_ch > 0) {
      const void* k = nullptr;
      switch (c.dot2_ch) {
        case 1: k = (const void*)lr_dot2_kernel<1, MODE>; break;
        case 2: k = (const void*)lr_dot2_kernel<2, MODE>; break;
        case 3: k = (const void*)lr_dot2_kernel<3, MODE>; break;
        case 4: k = (const void*)lr_dot2_kernel<4, MODE>; break;
        default: fail(1, "lr: no two-group pass kernel for this row width");
      }
      launch_pass(k, a, c.grid, 2 * kGW * 32 + 32, c.dot2_smem, coop, st);
      return;
    }
    if (c.dot_rb > 0) {
    const void* k = nullptr;
#define VISTA_DOT(RB, CH) \
  if (c.dot_rb == RB && c.ch == CH) k = (const void*)lr_dot_kernel<RB, CH, MODE>;
    VISTA_DOT(4, 1) VISTA_DOT(4, 2) VISTA_DOT(4, 3) VISTA_DOT(8, 1) VISTA_DOT(8, 2) VISTA_DOT(8, 3)
    VISTA_DOT(16, 1) VISTA_DOT(16, 2) VISTA_DOT(16, 3)
#undef VISTA_DOT
    if (!k) fail(1, "lr: no pass kernel for this row width");
    launch_pass(k, a, c.grid, c.threads + 32, c.dot_smem, coop, st);
    return;
    }
  }
  const void* k = nullptr;
  switch (c.ch) {
    case 1: k = (const void*)lr_stream_kernel<1, MODE, E>; break;
    case 2: k = (const void*)lr_stream_kernel<2, MODE, E>; break;
    case 3: k = (const void*)lr_stream_kernel<3, MODE, E>; break;
    case 4: k = (const void*)lr_stream_kernel<4, MODE, E>; break;
    case 5: k = (const void*)lr_stream_kernel<5, MODE, E>; break;
    case 6: k = (const void*)lr_stream_kernel<6, MODE, E>; break;
    default: fail(1, "lr: unsupported row width");
  }
  launch_pass(k, a, c.grid, c.threads + 32, c.smem, coop, st);
}

size_t lr_async_bytes(int ld, int iters) { return 40 + sizeof(LRState) + (size_t)ld * 8 + (size_t)iters * 8; }

LRResult lr_collect(const LRAsync& a) {
  LRResult res;
  VCHECK(cudaEventSynchronize(a.done));
  const uint8_t* hb = static_cast<const uint8_t*>(a.pinned);
  unsigned long long hc[5];
  std::memcpy(hc, hb, 40);
  LRState hs;
  std::memcpy(&hs, hb + 40, sizeof(hs));
  res.w.resize(a.ld);
  std::memcpy(res.w.data(), hb + 40 + sizeof(LRState), (size_t)a.ld * 8);
  res.loss.resize(a.iters);
  if (a.iters) std::memcpy(res.loss.data(), hb + 40 + sizeof(LRState) + (size_t)a.ld * 8, (size_t)a.iters * 8);
  res.b = hs.b;
  res.lambda_hat = hs.lambda_hat;
  res.eta = hs.eta;
  res.n_train = (int64_t)hs.n_train;
  res.train_ok = (int64_t)hc[0];
  res.tp = (int64_t)hc[1];
  res.fp = (int64_t)hc[2];
  res.tn = (int64_t)hc[3];
  res.fn = (int64_t)hc[4];
  res.n_test = a.n_rows - a.n_train;
  return res;
}

template <typename E>
static LRResult lr_train_impl(const E* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                              const uint8_t* real_host, int iters, int power_iters, double lambda, double alpha,
                              allreduce_fn allreduce, void* ar_user, cudaStream_t st, LRAsync* async, int grid_cap) {
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
  const size_t tail_smem = kStagesLR * kMaxRB * 32 * 4 + 2 * kStagesLR * 8 + 128;  // red + barriers + align
  cfg.smem = kStagesLR * stage_bytes + tail_smem;
  if (cfg.smem > 227 * 1024) fail(1, "lr: row block does not fit in shared memory");
  const char* dot_env = getenv("VISTA_LR_DOT");  // A/B switch: 0 = the r1 kernel for every pass
  if (esz == 2 && cfg.ch <= 3 && !(dot_env && dot_env[0] == '0')) {  // bf16: the lean dot kernel, 4 / 8 / 16 rows per block
    for (int rb : {16, 8, 4}) {
      const size_t sb = ((size_t)rb * ld * 2 + 127) & ~(size_t)127;
      if (kStagesLR * sb + tail_smem <= 227 * 1024) {
        cfg.dot_rb = rb;
        cfg.dot_smem = kStagesLR * sb + tail_smem;
        break;
      }
    }
  }
  // the two-group kernel for rows of at least VISTA_LR_DOT2 columns (opt-in: measured neutral, 87-94 vs 91 us
  // per conv5_x power pass -- the per-block barrier chain is not what bounds the pass)
  const char* dot2_env = getenv("VISTA_LR_DOT2");
  if (cfg.dot_rb > 0 && dot2_env && atoi(dot2_env) > 0 && ld >= atoi(dot2_env)) {
    const int ch2 = (chunks + kGW * 32 - 1) / (kGW * 32);
    const size_t sb2 = ((size_t)2 * ld * 2 + 127) & ~(size_t)127;
    const size_t smem2 = kStages2 * sb2 + kStages2 * 2 * 16 * 4 + 2 * kStages2 * 8 + 16 + ((size_t)chunks * 8 + 8) * 4 + 128;
    if (ch2 <= 4 && smem2 <= 227 * 1024) {
      cfg.dot2_ch = ch2;
      cfg.dot2_smem = smem2;
    }
  }
  const int64_t pass_rb = cfg.dot2_ch > 0 ? 2 : (cfg.dot_rb > 0 ? std::min(cfg.rb, cfg.dot_rb) : cfg.rb);  // grid: blocks of the finer kernel
  // at least one CTA per 128 columns: the fused tail splits the ld columns over the CTAs, and a grid sized
  // by a handful of rows left one CTA walking all of them behind L2 latency (C1: 33 -> ~9 us per pass)
  auto grid_for_rows = [&](int64_t rows) {
    const int64_t blocks = std::max<int64_t>((rows + pass_rb - 1) / pass_rb, (ld + 127) / 128);
    return (int)std::max<int64_t>(1, std::min<int64_t>(blocks, grid_cap > 0 ? std::min(grid_cap, num_sms()) : num_sms()));
  };
  cfg.grid = grid_for_rows(n_train);
  const int grid_tr = cfg.grid;
  const int ncols = ld + 2;
  int d_real = 0;
  for (int j = 0; j < ld; ++j) d_real += real_host[j] ? 1 : 0;
  // world == 1: reduction + update in the pass kernels' tails (one launch per pass).  The tail keeps this
  // CTA's reduced columns and a [32][32] double scratch in the (drained) stage ring.
  size_t ring_min = kStagesLR * std::min(stage_bytes, cfg.dot_rb > 0
                                                          ? (((size_t)cfg.dot_rb * ld * 2 + 127) & ~(size_t)127)
                                                          : stage_bytes);
  if (cfg.dot2_ch > 0) ring_min = std::min(ring_min, (size_t)kStages2 * (((size_t)2 * ld * 2 + 127) & ~(size_t)127));
  const size_t tail_need = 32 * 32 * 8 + ((size_t)(ld + grid_tr - 1) / grid_tr + 4) * 8;
  const bool fused = !allreduce && power_iters >= 1 && n_train > 0 && tail_need <= ring_min &&
                     !(getenv("VISTA_LR_FUSED") && getenv("VISTA_LR_FUSED")[0] == '0');

  // scratch
  size_t off = 0;
  auto carve = [&](size_t bytes) { size_t o = off; off += (bytes + 255) & ~(size_t)255; return o; };
  const size_t o_part = carve((size_t)std::max(grid_tr, 1) * (ld + 4) * 4), o_G = carve(ncols * 8), o_mu = carve(ld * 8),
               o_muf = carve(ld * 4), o_inv = carve(ld * 8), o_v = carve(ld * 8), o_w = carve(ld * 8),
               o_what = carve(ld * 4), o_bhat = carve(16), o_st = carve(sizeof(LRState)),
               o_real = carve(ld), o_loss = carve((size_t)(iters + 1) * 8), o_cnt = carve(64),
               o_bar = carve(16), o_scal = carve((size_t)2 * std::max(grid_tr, 1) * 8),
               o_z = carve((size_t)std::max<int64_t>(n_train, 1) * 4);
  uint8_t* scr = nullptr;
  VCHECK(cudaMallocAsync(&scr, off, st));
  VCHECK(cudaMemsetAsync(scr, 0, off, st));  // every byte defined (LRState fields a path leaves unwritten)
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

  PassArgs a;
  std::memset(&a, 0, sizeof(a));
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
  a.zbuf = reinterpret_cast<float*>(scr + o_z);
  a.n_train = n_train;
  a.rb = cfg.rb;
  a.dbg = getenv("VISTA_LR_DBG") ? atoi(getenv("VISTA_LR_DBG")) : 0;
  a.pf_next = (getenv("VISTA_LR_PFN") && getenv("VISTA_LR_PFN")[0] == '0') ? 0 : 1;  // A/B switch
  a.counts = nullptr;
  a.f.on = fused ? 1 : 0;
  a.f.ncols = ncols;
  a.f.bar = reinterpret_cast<unsigned int*>(scr + o_bar);
  a.f.G = G;
  a.f.scal = reinterpret_cast<double*>(scr + o_scal);
  a.f.real = real;
  a.f.mu = mu;
  a.f.inv = inv;
  a.f.v = v;
  a.f.w = w;
  a.f.mu_f = mu_f;
  a.f.what = what;
  a.f.bhat = bhat;
  a.f.st = dst;
  a.f.lambda = lambda;
  a.f.alpha = alpha;
  a.f.d_real = d_real;
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
  unsigned int sync_cum = 0;  // grid-barrier arrivals so far (fused passes: 1 sync in MODE 0, 2 otherwise)
  a.f.sync_base = sync_cum;
  run_pass<0, E>(a, cfg, st);
  sync_cum += (unsigned)cfg.grid;
  prof_end(st, 5, 0, pass_bytes);
  if (!fused) {
    reduce((double)n_train, 0);
    stats_finalize_kernel<<<(ld + 255) / 256, 256, 0, st>>>(G, ld, 0, real, mu, mu_f, inv, dst);
    LAUNCHED();
  }
  prof_begin(st);
  a.f.sync_base = sync_cum;
  run_pass<1, E>(a, cfg, st);  // fused: + the power-iteration start
  sync_cum += 2u * (unsigned)cfg.grid;
  prof_end(st, 5, 0, pass_bytes);
  if (!fused) {
    reduce(-1, 0);
    stats_finalize_kernel<<<(ld + 255) / 256, 256, 0, st>>>(G, ld, 1, real, mu, mu_f, inv, dst);
    LAUNCHED();
    // ---- O6 step 3: K power iterations ----
    power_kernel<<<1, ublk, 0, st>>>(G, ld, 1, d_real, real, inv, mu, v, what, bhat, dst);
    LAUNCHED();
  }
  for (int k = 0; k < power_iters; ++k) {
    a.f.init_next = k == power_iters - 1 ? 1 : 0;  // fused: the last power pass also starts ISTA
    prof_begin(st);
    a.f.sync_base = sync_cum;
    run_pass<2, E>(a, cfg, st);
    sync_cum += 2u * (unsigned)cfg.grid;
    prof_end(st, 5, 0, pass_bytes);
    if (!fused) {
      reduce(-1, 1);
      power_kernel<<<1, ublk, 0, st>>>(G, ld, 0, d_real, real, inv, mu, v, what, bhat, dst);
      LAUNCHED();
    }
  }
  a.f.init_next = 0;
  // ---- O6 steps 4-5: ISTA ----
  if (!fused) {
    grad_kernel<<<1, ublk, 0, st>>>(G, ld, 1, lambda, alpha, inv, mu, w, what, bhat, dst, loss);
    LAUNCHED();
  }
  for (int t = 0; t < iters; ++t) {
    a.f.loss_out = loss + t;
    prof_begin(st);
    a.f.sync_base = sync_cum;
    run_pass<3, E>(a, cfg, st);
    sync_cum += 2u * (unsigned)cfg.grid;
    prof_end(st, 5, 0, pass_bytes);
    if (!fused) {
      reduce(-1, 1);
      grad_kernel<<<1, ublk, 0, st>>>(G, ld, 0, lambda, alpha, inv, mu, w, what, bhat, dst, loss + t);
      LAUNCHED();
    }
  }
  // ---- O6 step 6: eval over all local rows ----
  {
    PassArgs e = a;
    e.r0 = 0;
    e.r1 = n_rows;
    e.counts = cnt;
    e.f.on = 0;
    e.pf_next = 0;  // the last pass of this layer
    StreamCfg ce = cfg;
    ce.grid = grid_for_rows(n_rows);
    prof_begin(st);
    if (n_rows > 0) run_pass<4, E>(e, ce, st);
    prof_end(st, 5, 0, (double)n_rows * ld * esz);
  }
  if (async) {
    // asynchronous (world == 1, the Staged plan's LR(k) beside stage k+1): results to the caller's pinned
    // buffer, scratch freed in stream order, completion event; lr_collect assembles them
    if (allreduce) fail(1, "lr: asynchronous training is single-rank only");
    uint8_t* hb = static_cast<uint8_t*>(async->pinned);
    if (!hb || async->bytes < lr_async_bytes(ld, iters)) fail(1, "lr: pinned result buffer too small");
    VCHECK(cudaMemcpyAsync(hb, cnt, 5 * 8, cudaMemcpyDeviceToHost, st));
    VCHECK(cudaMemcpyAsync(hb + 40, dst, sizeof(LRState), cudaMemcpyDeviceToHost, st));
    VCHECK(cudaMemcpyAsync(hb + 40 + sizeof(LRState), w, (size_t)ld * 8, cudaMemcpyDeviceToHost, st));
    if (iters)
      VCHECK(cudaMemcpyAsync(hb + 40 + sizeof(LRState) + (size_t)ld * 8, loss, (size_t)iters * 8,
                             cudaMemcpyDeviceToHost, st));
    VCHECK(cudaFreeAsync(scr, st));
    if (!async->done) VCHECK(cudaEventCreateWithFlags(&async->done, cudaEventDisableTiming));
    VCHECK(cudaEventRecord(async->done, st));
    async->n_rows = n_rows;
    async->n_train = n_train;
    async->ld = ld;
    async->iters = iters;
    return res;
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
                  allreduce_fn allreduce, void* ar_user, cudaStream_t st, LRAsync* async, int grid_cap) {
  return lr_train_impl<bf16>(MM, y, n_rows, n_train, ld, real_host, iters, power_iters, lambda, alpha, allreduce,
                             ar_user, st, async, grid_cap);
}

LRResult lr_train_f32(const float* MM, const uint8_t* y, int64_t n_rows, int64_t n_train, int ld,
                      const uint8_t* real_host, int iters, int power_iters, double lambda, double alpha,
                      allreduce_fn allreduce, void* ar_user, cudaStream_t st) {
  return lr_train_impl<float>(MM, y, n_rows, n_train, ld, real_host, iters, power_iters, lambda, alpha, allreduce,
                              ar_user, st, nullptr, 0);
}

}  // namespace vista
