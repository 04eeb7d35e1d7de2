// conv3x3_rows.cu — 3x3 / stride 1 / pad 1 convolution with Cin = Cout = 64 (ResNet50 res2 units,
// 56 x 56) + BN + ReLU, issued input-row-major: part of S1 of SURVEY.md §8a (partial CNN inference
// f^_{i -> j}, Def 3.7).
//
// Why a separate kernel: with Cout = 64 the implicit GEMM has N = 64, and a 128 x 64 x 16 MMA reads
// 4 KB of A + 2 KB of B from shared memory for 32 tensor-cycles of work: the halo kernel (conv_tc.cu
// A_HALO) is bound by shared-memory operand reads, not by the tensor pipe.  Here an A tile is ONE padded
// input row of two images, and each MMA multiplies it by the weights of all three filter rows side by side
// (N = 192: [W(r=2) | W(r=1) | W(r=0)] for one filter column s), accumulating into the accumulators of the
// three output rows that input row feeds (ip - 2, ip - 1, ip) -- 10 KB of operands per 96 tensor-cycles.
//
// Geometry.  M row m = img * 64 + j of a tile (img in {0, 1}: images 2p, 2p + 1 of pair p); A row j holds
// padded input column j - 1 (TMA box {64 ch, 64 columns from -1, 1 row, 2 images}, out-of-bounds = 0 =
// the conv's zero padding), so output column w reads input column w - 1 + s = A row w + s: filter column s
// is a 128-byte row shift of the A descriptor.  Rows m with w >= W are discarded.  Padded input row ip
// (ip - 1 = image row, ip in [1, H]) feeds output row o = ip - r through filter row r.
// TMEM: 8 accumulators of 64 columns, output-row instance k of this CTA in slot k % 8; the N = 192 MMA of
// input row ip covers the slots of rows ip - 2 .. ip (split in two where the ring wraps, trimmed at band
// and image edges); slots are zeroed by the epilogue after draining, so every MMA accumulates.  Per output
// row the products are accumulated in the same order as the halo kernel's (filter row r, then s, then
// channel), so the two kernels agree bit for bit.
// Work item = (image pair, band of output rows): one band, or two bands of H / 2 rows (2 recomputed input rows
// per pair) when the finer items balance the persistent grid better.
//
// Warps: 0 = TMA producer (weights once, then input rows through a kSA-slot ring), 1 = TMEM allocator + MMA
// issuer (one elected lane), 2..9 = epilogue: two groups of four warps (one per TMEM lane quadrant) take
// alternate output rows; a thread owns one pixel (all 64 channels: two 32-column TMEM loads), applies BN
// scale / shift + ReLU, RNE to bf16 and stores the pixel's 128 contiguous bytes.
#include <cstring>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

namespace {

constexpr int kC = 64;                   // Cin = Cout
constexpr int kSlotsImg = 64;            // A rows per image (padded columns -1 .. 62)
constexpr int kSA = 6;                   // input-row ring slots
constexpr int kNAcc = 8;                 // TMEM accumulator ring (64 columns each)
constexpr int kRowBytes = 128 * 128;     // one A slot: 128 rows x 64 bf16, 128B-swizzled
constexpr int kWBlk = 64 * 128;          // one filter tap: 64 output channels x 64 bf16
constexpr int kOffB = 0, kOffA = kOffB + 9 * kWBlk, kOffSS = kOffA + kSA * kRowBytes + 1024,
              kOffBar = kOffSS + 2 * kC * 4;
constexpr int kSmem = kOffBar + (2 * kSA + 2 * kNAcc + 2) * 8 + 1024;
constexpr int kEpiWarp0 = 2, kThreads = (kEpiWarp0 + 8) * 32;

struct RowConvParams {
  bf16* y;  // [N, H, W, 64]
  const float* scale;
  const float* shift;
  int N, H, W, relu;
  int nbands, band_h;  // output rows [b * band_h, min(H, (b + 1) * band_h)) per band
  int n_items;         // ceil(N / 2) * nbands
};

__device__ __forceinline__ void item_rows(const RowConvParams& p, int item, int& pair, int& o_lo, int& o_hi) {
  pair = item / p.nbands;
  const int b = item - pair * p.nbands;
  o_lo = b * p.band_h;
  o_hi = min(p.H, o_lo + p.band_h) - 1;
}

__global__ void __launch_bounds__(kThreads, 1)
    conv3x3_rows_kernel(const __grid_constant__ CUtensorMap tmap_w, const __grid_constant__ CUtensorMap tmap_a,
                        const RowConvParams p) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t sB = base + kOffB, sA = base + kOffA;
  float* ss = reinterpret_cast<float*>(gbase + kOffSS);  // [scale 64 | shift 64]
  uint64_t* full = reinterpret_cast<uint64_t*>(gbase + kOffBar);
  uint64_t* empty = full + kSA;
  uint64_t* tfull = empty + kSA;
  uint64_t* tempty = tfull + kNAcc;
  uint64_t* bbar = tempty + kNAcc;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bbar + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kSA; ++i) {
      mbar_init(&full[i], 1);
      mbar_init(&empty[i], 1);
    }
    for (int i = 0; i < kNAcc; ++i) {
      mbar_init(&tfull[i], 1);
      mbar_init(&tempty[i], 4);  // the four warps of the group draining the slot
    }
    mbar_init(bbar, 1);
    fence_mbar_init();
    tma_prefetch(&tmap_w);
    tma_prefetch(&tmap_a);
  }
  if (threadIdx.x < 2 * kC) ss[threadIdx.x] = threadIdx.x < kC ? p.scale[threadIdx.x] : p.shift[threadIdx.x - kC];
  if (warp == 1) tmem_alloc(tmem_slot, kNAcc * kC);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (warp >= kEpiWarp0) {  // zero the accumulator ring before the first MMA (group g: columns [g * 256, +256))
    const int q = warp & 3, g = (warp - kEpiWarp0) >> 2;
    for (int c = 0; c < 8; ++c) tmem_zero_32x32b_x32(tmem_base + g * 256 + c * 32 + ((uint32_t)(q * 32) << 16));
    tc_wait_st();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();

  if (warp == 0) {
    // ======================= producer =======================
    if (lane == 0) {
      // weights: tap (r, s) -> block s * 3 + (2 - r), so that [W(2,s) | W(1,s) | W(0,s)] are 192 consecutive rows
      mbar_arrive_expect_tx(bbar, 9 * kWBlk);
      for (int r = 0; r < 3; ++r)
        for (int s = 0; s < 3; ++s) tma_load_2d(sB + (s * 3 + (2 - r)) * kWBlk, &tmap_w, (r * 3 + s) * 64, 0, bbar);
      uint32_t g = 0;
      for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
        int pair, o_lo, o_hi;
        item_rows(p, item, pair, o_lo, o_hi);
        const int ip0 = max(1, o_lo), ip1 = min(p.H, o_hi + 2);
        for (int ip = ip0; ip <= ip1; ++ip, ++g) {
          const int slot = g % kSA;
          if (g >= (uint32_t)kSA) mbar_wait(&empty[slot], ((g / kSA) - 1) & 1);
          mbar_arrive_expect_tx(&full[slot], kRowBytes);
          tma_load_4d(sA + slot * kRowBytes, &tmap_a, 0, -1, ip - 1, 2 * pair, &full[slot]);
        }
      }
    }
  } else if (warp == 1) {
    // ======================= MMA issuer =======================
    mbar_wait(bbar, 0);
    uint32_t g = 0, kbase = 0;  // input-row counter (ring), first output-row instance of the item
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      int pair, o_lo, o_hi;
      item_rows(p, item, pair, o_lo, o_hi);
      const int ip0 = max(1, o_lo), ip1 = min(p.H, o_hi + 2);
      int next_open = o_lo, next_done = o_lo;
      for (int ip = ip0; ip <= ip1; ++ip, ++g) {
        const int r_hi = min(2, ip - o_lo), r_lo = max(0, ip - o_hi);  // filter rows feeding rows of this band
        // rows ip - r_hi .. ip - r_lo; open the new ones (their slots drained and zeroed by the epilogue)
        for (; next_open <= ip - r_lo; ++next_open) {
          const uint32_t k = kbase + (uint32_t)(next_open - o_lo);
          if (k >= (uint32_t)kNAcc) mbar_wait(&tempty[k % kNAcc], ((k / kNAcc) - 1) & 1);
        }
        const uint32_t slot = g % kSA;
        mbar_wait(&full[slot], (g / kSA) & 1);
        tc_fence_after();
        const int cnt = r_hi - r_lo + 1, b0 = 2 - r_hi;  // weight blocks b0 .. b0 + cnt - 1
        const uint32_t s0 = (kbase + (uint32_t)(ip - r_hi - o_lo)) % kNAcc;
        const uint32_t n1 = (uint32_t)cnt < kNAcc - s0 ? (uint32_t)cnt : kNAcc - s0;
        // 32-bit descriptor halves (SW128 K-major): filter column s = an s-row shift of A (128 B = 8 units),
        // K step = 32 B = 2 units; B block (s, b) at (s * 3 + b) * 8 KB = 512 units per block
        const uint32_t a_lo = umma_desc_lo_sw128(sA + slot * kRowBytes);
        const uint32_t b_lo = umma_desc_lo_sw128(sB + b0 * kWBlk);
        const uint32_t t0 = tmem_base + s0 * kC;
        const uint32_t id1 = umma_idesc_bf16(128, 64 * n1);
        if ((uint32_t)cnt == n1) {  // the rows' slots are contiguous: one N = 64 * cnt MMA per K step
#pragma unroll
          for (int s = 0; s < 3; ++s)
#pragma unroll
            for (int kk = 0; kk < 4; ++kk)
              tc_mma_bf16_lo_warp(t0, a_lo + s * 8 + kk * 2, b_lo + s * 3 * (kWBlk >> 4) + kk * 2, id1, 1u);
        } else {  // the ring wraps: slots s0 .. 7, then 0 ..
          const uint32_t id2 = umma_idesc_bf16(128, 64 * ((uint32_t)cnt - n1));
          const uint32_t b2 = b_lo + n1 * (kWBlk >> 4);
#pragma unroll
          for (int s = 0; s < 3; ++s)
#pragma unroll
            for (int kk = 0; kk < 4; ++kk) {
              tc_mma_bf16_lo_warp(t0, a_lo + s * 8 + kk * 2, b_lo + s * 3 * (kWBlk >> 4) + kk * 2, id1, 1u);
              tc_mma_bf16_lo_warp(tmem_base, a_lo + s * 8 + kk * 2, b2 + s * 3 * (kWBlk >> 4) + kk * 2, id2, 1u);
            }
        }
        tc_commit_warp(&empty[slot]);  // input row ip feeds no later MMA
        // rows whose last input row was ip are complete
        for (; next_done <= o_hi && min(next_done + 2, p.H) <= ip; ++next_done)
          tc_commit_warp(&tfull[(kbase + (uint32_t)(next_done - o_lo)) % kNAcc]);
      }
      kbase += (uint32_t)(o_hi - o_lo + 1);
    }
  } else {
    // ======================= epilogue: BN + ReLU, one pixel (64 channels) per thread =======================
    const int q = warp & 3, grp = (warp - kEpiWarp0) >> 2;
    const int m = q * 32 + lane, img = m / kSlotsImg, w = m % kSlotsImg;
    const uint32_t tl = (uint32_t)(q * 32) << 16;
    uint32_t k = 0;
    for (int item = blockIdx.x; item < p.n_items; item += gridDim.x) {
      int pair, o_lo, o_hi;
      item_rows(p, item, pair, o_lo, o_hi);
      const int n = 2 * pair + img;
      for (int o = o_lo; o <= o_hi; ++o, ++k) {
        if ((int)(k & 1) != grp) continue;
        const uint32_t acc = k % kNAcc, ta = tmem_base + acc * kC + tl;
        uint32_t v0[32], v1[32];
        mbar_wait(&tfull[acc], (k / kNAcc) & 1);
        tc_fence_after();
        tmem_ld_32x32b_x32(ta, v0);
        tmem_ld_32x32b_x32(ta + 32, v1);
        tc_wait_ld_regs(v0);
        tc_wait_ld_regs(v1);
        tmem_zero_32x32b_x32(ta);
        tmem_zero_32x32b_x32(ta + 32);
        tc_wait_st();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
        if (w < p.W && n < p.N) {
          uint4* dst = reinterpret_cast<uint4*>(p.y + (((size_t)n * p.H + o) * p.W + w) * kC);
#pragma unroll
          for (int c = 0; c < 4; ++c) dst[c] = epi8(v0 + c * 8, ss + c * 8, ss + kC + c * 8, make_uint4(0, 0, 0, 0), false, p.relu);
#pragma unroll
          for (int c = 0; c < 4; ++c)
            dst[4 + c] = epi8(v1 + c * 8, ss + 32 + c * 8, ss + kC + 32 + c * 8, make_uint4(0, 0, 0, 0), false, p.relu);
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc(tmem_base, kNAcc * kC);
}

}  // namespace

bool rowconv3x3_supported(const ConvLayer& L, int H, int W) {
  return L.R == 3 && L.S == 3 && L.stride == 1 && L.pad == 1 && L.groups == 1 && L.Cin == kC && L.Cout == kC &&
         L.BN == kC && L.Kp == 9 * kC && W >= 1 && W <= kSlotsImg - 2 && H >= 1;
}

void rowconv3x3_forward(const ConvLayer& L, const bf16* x, int N, int H, int W, bf16* y, cudaStream_t st) {
  if (N <= 0) return;
  CUtensorMap ta;
  const uint64_t dims[4] = {(uint64_t)kC, (uint64_t)W, (uint64_t)H, (uint64_t)N};
  const uint64_t strides[3] = {(uint64_t)kC * 2, (uint64_t)W * kC * 2, (uint64_t)H * W * kC * 2};
  const uint32_t box[4] = {(uint32_t)kC, (uint32_t)kSlotsImg, 1, 2};
  if (!make_nd_tmap(&ta, x, 4, dims, strides, box)) fail(5, "conv3x3_rows: tensor map failed");
  RowConvParams p;
  p.y = y;
  p.scale = L.scale;
  p.shift = L.shift;
  p.N = N;
  p.H = H;
  p.W = W;
  p.relu = L.relu ? 1 : 0;
  // one band per image pair unless two bands balance the persistent grid better: a band boundary recomputes two
  // input rows (H / (H + 2) of the MMA work is useful), a partial last round of items idles CTAs
  const int pairs = (N + 1) / 2, sms = num_sms();
  auto eff = [&](int nb) {
    const int items = pairs * nb, rounds = (items + sms - 1) / sms;
    return (double)items / ((double)rounds * sms) * (nb == 1 ? 1.0 : (double)H / (H + 2));
  };
  p.nbands = (H >= 8 && eff(2) > eff(1)) ? 2 : 1;
  p.band_h = (H + p.nbands - 1) / p.nbands;
  p.n_items = pairs * p.nbands;
  ensure_smem_attr((const void*)conv3x3_rows_kernel, kSmem);
  const int grid = p.n_items < num_sms() ? p.n_items : num_sms();
  prof_begin(st);
  conv3x3_rows_kernel<<<grid, kThreads, kSmem, st>>>(L.tmap_w, ta, p);
  LAUNCHED();
  const double M = (double)N * H * W;
  const double flops = 2.0 * M * kC * L.K_alg;
  const double bytes = 2.0 * (M * kC * 2 + (double)kC * L.Kp);
  prof_end(st, 0, flops, bytes, prof_labels() ? "conv3x3 rows (res2, N = 192 input-row MMAs)" : nullptr);
}

}  // namespace vista
