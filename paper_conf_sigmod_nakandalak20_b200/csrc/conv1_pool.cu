// conv1_pool.cu — ResNet50 stem fused: conv1 (7x7/2 pad 3, BN, ReLU; run as 4x4/1 on the 2x2
// space-to-depth input, roster.h kS2dHW) followed by pool1 (3x3/2 max, unpadded; reading R4) in ONE
// persistent tcgen05 kernel.  SURVEY.md §8a S1; the 114x114x64 conv1 activation (1.66 MB per
// image) never reaches HBM: per image the kernel reads the 438 KB space-to-depth input once and
// writes the 401 KB pooled [56, 56, 64] output.
//
// Each CTA owns whole images.  Tile = one conv output row ho (114 pixels in a 128-row M tile);
// k-block r = filter row r reads input row ho + r through the overlapping TMA row view (the same
// operand layout as conv_tc.cu's A_ROWVIEW mode), so every input row is loaded ONCE into a ring of
// kSA shared-memory slots and reused by the four tiles that need it.  The 4 k-blocks of the
// 64 x 256 weight matrix stay resident in shared memory for the whole kernel.
// Epilogue (8 warps): TMEM -> BN scale/shift -> ReLU -> bf16 (RNE) conv row in shared memory; then
// each thread owns fixed (pooled column j, 8-channel chunk) items: horizontal 3-max over conv
// columns 2j..2j+2, and a running vertical max over conv rows 2i..2i+2 kept in registers; pooled
// row i is stored (coalesced 16-byte stores) when conv row 2i+2 arrives.  Max is exact on bf16
// values, so the result is bit-identical to conv_forward + launch_maxpool.
#include <cstring>

#include "internal.h"
#include "ptx.cuh"
#include "roster.h"

namespace vista {

namespace {

constexpr int kHo = 114;           // conv1 output rows / cols (227 + 6 - 7) / 2 + 1
constexpr int kHin = 117;          // space-to-depth input rows (kS2dHW)
constexpr int kPo = 56;            // pool1 output (114 - 3) / 2 + 1
constexpr int kCo = 64;            // conv1 channels
constexpr int kSA = 6;             // input-row ring slots (rows 24 ahead are prefetched into L2)
constexpr int kNAcc = 8;           // TMEM accumulators (64 columns each; the classic issue order uses 4)
// One A slot = one space-to-depth input row, K-major with 32-byte swizzle: row q = position q's 16 channels (32 B).
// K step k (s2d position offset k of a filter row) is the slot shifted by k rows, so each input position lands in
// shared memory once (4.2 KB per row; the 128B-swizzled overlapping row view wrote each position four times,
// 16 KB per row -- the stem is shared-memory bound).  VISTA_STEM_SW32=0 keeps the row view (A/B).
constexpr int kRowPos = 131;                               // 128 M rows + 3 shifts
constexpr int kRowBytes = 128 * 128;                       // slot stride (the row view's 16 KB; SW32 uses 4.2 KB of it)
constexpr int kRowTx32 = kRowPos * 32;
constexpr int kBBytes = 4 * 64 * 128;  // 4 k-blocks x 64 output channels x 64 bf16
constexpr int kCrowBytes = 128 * 128;  // conv row: 128 pixels x 64 channels bf16
constexpr int kCrowBufs = 4;           // staged conv rows (two rows per epilogue step, double-buffered)
constexpr int kEpiWarp0 = 2;        // warp 0: TMA producer, warp 1: MMA issuer, then EPW epilogue warps
constexpr int kItems = kPo * 8;    // (pooled column, 8-channel chunk) items per pooled row
constexpr int kOffB = 0, kOffA = kOffB + kBBytes, kOffCrow = kOffA + kSA * kRowBytes,
              kOffSS = kOffCrow + kCrowBufs * kCrowBytes, kOffBar = kOffSS + 2 * kCo * 4;
constexpr int kSmem = kOffBar + (2 * kSA + 2 * kNAcc + 2) * 8 + 1024;

struct PoolParams {
  const bf16* x;  // [N, 117, 117, 16] (L2 prefetch of rows ahead of the TMA ring)
  bf16* y;        // [N, 56, 56, 64]
  const float* scale;
  const float* shift;
  int N;
  // irow = 1 (default): input-row-major issue.  Input row i feeds output rows i-3..i through filter rows
  // 3..0, so ONE 128 x 256 x 16 MMA step per K slice (weights of the four filter rows side by side, W_3 first)
  // accumulates into four consecutive output-row accumulators of an 8-slot TMEM ring (split where the ring
  // wraps / at image edges); slots are zeroed by the epilogue after draining, so every MMA accumulates.
  // Versus the row-major order (16 N = 64 MMAs per output row, shared-memory operand bound at 48 cycles
  // each): half the shared-memory operand bytes and full-rate N >= 128 instructions.
  int irow;
  int sw32;  // 1: A slots in the 32B-swizzled one-position-per-row layout (see kRowPos)
};

__device__ __forceinline__ uint4 max4(uint4 a, uint4 b) {
  uint4 o;
  const __nv_bfloat162* pa = reinterpret_cast<const __nv_bfloat162*>(&a);
  const __nv_bfloat162* pb = reinterpret_cast<const __nv_bfloat162*>(&b);
  __nv_bfloat162* po = reinterpret_cast<__nv_bfloat162*>(&o);
#pragma unroll
  for (int j = 0; j < 4; ++j) po[j] = __hmax2(pa[j], pb[j]);
  return o;
}

// EPW epilogue warps (8 or 16): EPW / 4 warps per TMEM lane quadrant, each owning CPT = 256 / EPW of the 64
// channels.  16 (default): twice the warps to hide the per-row TMEM-load / pack / barrier latency chain that
// bounded the 8-warp epilogue (ncu: 2.5 active warps per scheduler, 0.36 issued per cycle, tensor pipe 60 %)
template <int EPW>
__global__ void __launch_bounds__((kEpiWarp0 + EPW) * 32, 1)
    conv1_pool_kernel(const __grid_constant__ CUtensorMap tmap_w, const __grid_constant__ CUtensorMap tmap_a,
                      const PoolParams p) {
  constexpr int kEpiWarps = EPW, kEpiThreads = EPW * 32, CPT = kCo / (EPW / 4);
  constexpr int NI = (kItems + kEpiThreads - 1) / kEpiThreads;  // pooling items per thread
  static_assert(CPT == 16 || CPT == 32, "16 or 32 channels per epilogue thread");
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t sB = base + kOffB, sA = base + kOffA, sC = base + kOffCrow;
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
      mbar_init(&tempty[i], kEpiWarps);
    }
    mbar_init(bbar, 1);
    fence_mbar_init();
    tma_prefetch(&tmap_w);
    tma_prefetch(&tmap_a);
  }
  if (threadIdx.x < 2 * kCo) ss[threadIdx.x] = threadIdx.x < kCo ? p.scale[threadIdx.x] : p.shift[threadIdx.x - kCo];
  if (warp == 1) tmem_alloc(tmem_slot, kNAcc * kCo);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  if (p.irow && warp >= kEpiWarp0) {  // zero the whole accumulator ring before the first MMA
    const int q = warp & 3, grp = (warp - kEpiWarp0) >> 2;
    for (int sl = 0; sl < kNAcc; ++sl) {
      const uint32_t ta = tmem_base + sl * kCo + grp * CPT + ((uint32_t)(q * 32) << 16);
      if constexpr (CPT == 32) tmem_zero_32x32b_x32(ta);
      else tmem_zero_32x32b_x16(ta);
    }
    tc_wait_st();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();

  if (warp == 0) {
    // ======================= producer: weights once, then every input row once =======================
    if (lane == 0) {
      mbar_arrive_expect_tx(bbar, kBBytes);
      for (int r = 0; r < 4; ++r) tma_load_2d(sB + (p.irow ? 3 - r : r) * 64 * 128, &tmap_w, r * 64, 0, bbar);
      // The TMA ring holds only ~4 rows of lookahead and a row is 3.7 KB of unique input, far too little
      // in flight to cover HBM latency: rows kPfAhead ahead are prefetched into L2 in 8-row groups.
      constexpr int kPfAhead = 24, kPfGroup = 8;
      constexpr uint32_t kRowIn = kHin * kS2dC * 2;  // bytes of one input row
      auto prefetch_rows = [&](int n, int i0) {     // rows [i0, i0 + kPfGroup) of this CTA's row sequence
        while (i0 >= kHin) {
          i0 -= kHin;
          n += gridDim.x;
        }
        if (n >= p.N) return;
        const int i1 = min(i0 + kPfGroup, kHin);
        prefetch_l2_range(p.x + ((size_t)n * kHin + i0) * kHin * kS2dC, (uint64_t)(i1 - i0) * kRowIn);
        if (i1 - i0 < kPfGroup) {  // continue into this CTA's next image
          const int n2 = n + gridDim.x;
          if (n2 < p.N) prefetch_l2_range(p.x + (size_t)n2 * kHin * kHin * kS2dC, (uint64_t)(kPfGroup - (i1 - i0)) * kRowIn);
        }
      };
      if (blockIdx.x < p.N)
        for (int i = 0; i < kPfAhead; i += kPfGroup) prefetch_rows(blockIdx.x, i);
      uint32_t g = 0;
      for (int n = blockIdx.x; n < p.N; n += gridDim.x) {
        for (int i = 0; i < kHin; ++i, ++g) {
          if (i % kPfGroup == 0) prefetch_rows(n, i + kPfAhead);
          const int slot = g % kSA;
          if (g >= (uint32_t)kSA) mbar_wait(&empty[slot], ((g / kSA) - 1) & 1);
          mbar_arrive_expect_tx(&full[slot], p.sw32 ? kRowTx32 : kRowBytes);
          tma_load_4d(sA + slot * kRowBytes, &tmap_a, 0, 0, i, n, &full[slot]);
        }
      }
    }
  } else if (warp == 1 && p.irow) {
    // ============ MMA issuer, input-row-major (see PoolParams::irow) ============
    mbar_wait(bbar, 0);
    uint32_t grow = 0, orow = 0;  // this CTA's running input-row / output-row counters
    for (int n = blockIdx.x; n < p.N; n += gridDim.x, orow += kHo) {
      for (int i = 0; i < kHin; ++i, ++grow) {
        if (i < kHo) {  // output row i opens here: its ring slot must have been drained and zeroed
          const uint32_t o = orow + i;
          if (o >= (uint32_t)kNAcc) mbar_wait(&tempty[o % kNAcc], ((o / kNAcc) - 1) & 1);
        }
        const uint32_t slot = grow % kSA;
        mbar_wait(&full[slot], (grow / kSA) & 1);
        tc_fence_after();
        const int r_hi = i < 3 ? i : 3, r_lo = i > kHo - 1 ? i - (kHo - 1) : 0;
        const int j_lo = 3 - r_hi, cnt = r_hi - r_lo + 1;  // weight groups j_lo .. j_lo + cnt - 1 (j = 3 - r)
        const uint32_t s0 = (orow + (uint32_t)(i - r_hi)) % kNAcc;  // slot of output row i - r_hi
        const uint32_t n1 = (uint32_t)cnt < kNAcc - s0 ? (uint32_t)cnt : kNAcc - s0;
        // 32-bit descriptor halves (SW128 K-major; K step = 32 B = 2 units, weight group = 8 KB = 512 units) and
        // separate straight / wrapped paths: the MMA warp's per-row issue chain, not the tensor pipe, bounded
        // the kernel (ncu: tensor pipe 70 %, the epilogue waiting on full accumulators)
        // K step k: A = the 32-byte K slice k of the row view (+2 units), or with sw32 the slot shifted by k
        // 32-byte rows (+2 units as well); B = the weights' 32-byte K slice k of the 128B-swizzled groups
        const uint64_t da = p.sw32 ? umma_desc_k_sw32(sA + slot * kRowBytes) : umma_desc_k_sw128(sA + slot * kRowBytes);
        const uint64_t db = umma_desc_k_sw128(sB + (uint32_t)j_lo * 64 * 128);
        const uint32_t t0 = tmem_base + s0 * kCo, id1 = umma_idesc_bf16(128, 64 * n1);
        if ((uint32_t)cnt == n1) {
#pragma unroll
          for (int k = 0; k < 4; ++k) tc_mma_bf16_warp(t0, da + 2 * k, db + 2 * k, id1, 1u);
        } else {
          const uint32_t id2 = umma_idesc_bf16(128, 64 * ((uint32_t)cnt - n1));
          const uint64_t db2 = db + n1 * 512u;
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            tc_mma_bf16_warp(t0, da + 2 * k, db + 2 * k, id1, 1u);
            tc_mma_bf16_warp(tmem_base, da + 2 * k, db2 + 2 * k, id2, 1u);
          }
        }
        tc_commit_warp(&empty[slot]);  // input row i feeds no later MMA
        if (i >= 3) tc_commit_warp(&tfull[(orow + i - 3) % kNAcc]);  // output row i - 3 is complete
      }
    }
  } else if (warp == 1) {
    // ======================= MMA issuer (whole warp, one elected lane issues) =======================
    {
      constexpr uint32_t idesc = umma_idesc_bf16(128, kCo);
      mbar_wait(bbar, 0);
      uint32_t gbase_row = 0, it = 0;
      for (int n = blockIdx.x; n < p.N; n += gridDim.x, gbase_row += kHin) {
        for (int ho = 0; ho < kHo; ++ho, ++it) {
          const uint32_t acc = it % kNAcc;
          if (it >= (uint32_t)kNAcc) mbar_wait(&tempty[acc], ((it / kNAcc) - 1) & 1);
          tc_fence_after();
          const uint32_t tacc = tmem_base + acc * kCo;
          // k-block r = filter row r = input row ho + r (manually unrolled: a rolled loop costs a YIELD and a
          // branch-resolution stall per iteration, measured as the MMA warp's dominant cost)
          auto kblock = [&](const uint32_t r) {
            const uint32_t row = gbase_row + ho + r;
            const uint32_t slot = row % kSA;
            // (TMA completion on the mbarrier orders the smem writes before the async-proxy MMA reads)
            mbar_wait(&full[slot], (row / kSA) & 1);
            const uint64_t da = p.sw32 ? umma_desc_k_sw32(sA + slot * kRowBytes) : umma_desc_k_sw128(sA + slot * kRowBytes);
            const uint64_t db = umma_desc_k_sw128(sB + r * 64 * 128);
            // +32 bytes along K = +2 in the descriptors' address fields
            tc_mma_bf16_warp(tacc, da, db, idesc, r != 0 ? 1u : 0u);
            tc_mma_bf16_warp(tacc, da + 2, db + 2, idesc, 1u);
            tc_mma_bf16_warp(tacc, da + 4, db + 4, idesc, 1u);
            tc_mma_bf16_warp(tacc, da + 6, db + 6, idesc, 1u);
          };
          kblock(0);
          kblock(1);
          kblock(2);
          kblock(3);
          tc_commit_warp(&tfull[acc]);
          // input row ho is not read by any later tile of this image
          tc_commit_warp(&empty[(gbase_row + ho) % kSA]);
          if (ho == kHo - 1)
            for (int r = 1; r < 4; ++r) tc_commit_warp(&empty[(gbase_row + ho + r) % kSA]);
        }
      }
    }
  } else {
    // ======================= epilogue: BN + ReLU + 3x3/2 max pool =======================
    const int et = threadIdx.x - kEpiWarp0 * 32;
    const int q = warp & 3;                    // TMEM lane quadrant
    const int grp = (warp - kEpiWarp0) >> 2;   // channel group (CPT channels)
    const int wo = q * 32 + lane;              // conv output column (M row of the tile)
    uint32_t it = 0;
    // Two conv rows per step, software-pipelined: the TMEM loads of rows ho, ho + 1 are issued before the
    // pooling of rows ho - 2, ho - 1 (staged in the other two of four conv-row buffers), so their latency and
    // the accumulator zeroing hide behind that work; one named barrier per two rows separates "staged" from
    // "pooled" (the per-row latency chain, not the arithmetic, bounded the one-row loop: ~0.8 us per row).
    for (int n = blockIdx.x; n < p.N; n += gridDim.x) {
      uint4 vb0[NI], vb1[NI];  // running vertical max of the open pooled rows (even / odd i), per item
#pragma unroll
      for (int u = 0; u < NI; ++u) vb0[u] = vb1[u] = make_uint4(0, 0, 0, 0);
      bf16* yimg = p.y + (size_t)n * kPo * kPo * kCo;
      // conv row ho (staged in buffer ho & 3) -> pooled rows: even ho closes i = ho/2 - 1 and opens i = ho/2;
      // odd ho extends (ho-1)/2
      auto pool_row = [&](const int ho) {
        const uint32_t cbase = sC + (ho & 3) * kCrowBytes;
#pragma unroll
        for (int u = 0; u < NI; ++u) {
          const int item = et + u * kEpiThreads;
          if (item >= kItems) continue;
          const int j = item >> 3, c = item & 7;
          const int w0 = 2 * j;
          const uint4 a = lds128(cbase + w0 * 128 + (((uint32_t)c ^ (uint32_t)(w0 & 7)) << 4));
          const uint4 b = lds128(cbase + (w0 + 1) * 128 + (((uint32_t)c ^ (uint32_t)((w0 + 1) & 7)) << 4));
          const uint4 d = lds128(cbase + (w0 + 2) * 128 + (((uint32_t)c ^ (uint32_t)((w0 + 2) & 7)) << 4));
          const uint4 h = max4(max4(a, b), d);
          if ((ho & 1) == 0) {
            const int io = ho >> 1;
            if (ho >= 2) {  // close pooled row io - 1 (conv rows ho - 2, ho - 1, ho)
              const uint4 o = max4((io & 1) ? vb0[u] : vb1[u], h);
              *reinterpret_cast<uint4*>(yimg + ((size_t)(io - 1) * kPo + j) * kCo + c * 8) = o;
            }
            if (io < kPo) {  // open pooled row io
              if (io & 1) vb1[u] = h;
              else vb0[u] = h;
            }
          } else {
            const int ie = (ho - 1) >> 1;  // middle row of pooled row ie
            if (ie < kPo) {
              if (ie & 1) vb1[u] = max4(vb1[u], h);
              else vb0[u] = max4(vb0[u], h);
            }
          }
        }
      };
      static_assert(kHo % 2 == 0, "two conv rows per step");
      for (int ho = 0; ho < kHo; ho += 2, it += 2) {
        const uint32_t acc0 = it % kNAcc, acc1 = (it + 1) % kNAcc;
        const uint32_t t0 = tmem_base + acc0 * kCo + grp * CPT + ((uint32_t)(q * 32) << 16);
        const uint32_t t1 = tmem_base + acc1 * kCo + grp * CPT + ((uint32_t)(q * 32) << 16);
        uint32_t v0[CPT], v1[CPT];
        mbar_wait(&tfull[acc0], (it / kNAcc) & 1);
        tc_fence_after();
        if constexpr (CPT == 32) tmem_ld_32x32b_x32(t0, v0);
        else tmem_ld_32x32b_x16(t0, v0);
        mbar_wait(&tfull[acc1], ((it + 1) / kNAcc) & 1);
        tc_fence_after();
        if constexpr (CPT == 32) tmem_ld_32x32b_x32(t1, v1);
        else tmem_ld_32x32b_x16(t1, v1);
        if (ho > 0) {  // overlaps the TMEM loads
          pool_row(ho - 2);
          pool_row(ho - 1);
        }
        if constexpr (CPT == 32) {
          tc_wait_ld_regs(v0);
          tc_wait_ld_regs(v1);
        } else {
          tc_wait_ld_regs16(v0);
          tc_wait_ld_regs16(v1);
        }
        if (p.irow) {  // input-row-major issue accumulates into zeroed slots
          if constexpr (CPT == 32) {
            tmem_zero_32x32b_x32(t0);
            tmem_zero_32x32b_x32(t1);
          } else {
            tmem_zero_32x32b_x16(t0);
            tmem_zero_32x32b_x16(t1);
          }
          tc_wait_st();
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&tempty[acc0]);
          mbar_arrive(&tempty[acc1]);
        }
        if (wo < kHo) {
#pragma unroll
          for (int c4 = 0; c4 < CPT / 8; ++c4) {  // 8 channels per 16-byte chunk
            const int ch0 = grp * CPT + c4 * 8;
            const uint32_t sw = (((uint32_t)(ch0 >> 3)) ^ (uint32_t)(wo & 7)) << 4;
            sts128(sC + (ho & 3) * kCrowBytes + wo * 128 + sw,
                   epi8(v0 + c4 * 8, ss + ch0, ss + kCo + ch0, make_uint4(0, 0, 0, 0), false, true));
            sts128(sC + ((ho + 1) & 3) * kCrowBytes + wo * 128 + sw,
                   epi8(v1 + c4 * 8, ss + ch0, ss + kCo + ch0, make_uint4(0, 0, 0, 0), false, true));
          }
        }
        named_bar_sync(1, kEpiThreads);
      }
      pool_row(kHo - 2);
      pool_row(kHo - 1);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) tmem_dealloc(tmem_base, kNAcc * kCo);
}

}  // namespace

bool conv1_pool_supported(const ConvLayer& L, int H, int W) {
  return L.rowview && L.Cin == kS2dC && L.Cout == kCo && L.R == 4 && L.S == 4 && L.BN == kCo && H == kHin &&
         W == kHin && L.relu;
}

void conv1_pool_forward(const ConvLayer& L, const bf16* x, int N, bf16* y, cudaStream_t st) {
  if (N <= 0) return;
  CUtensorMap ta;
  // overlapping row view {64 elements, q < 114, h, n}: element (k, q, h, n) = x[n, h, q + k / 16, k % 16]
  PoolParams p;
  p.sw32 = !(getenv("VISTA_STEM_SW32") && getenv("VISTA_STEM_SW32")[0] == '0');
  if (p.sw32) {  // {16 ch, kRowPos positions from 0 (>= 117 read zeros), 1 row, 1 image}, 32-byte swizzle
    const uint64_t dims[4] = {(uint64_t)kS2dC, (uint64_t)kHin, (uint64_t)kHin, (uint64_t)N};
    const uint64_t strides[3] = {(uint64_t)kS2dC * 2, (uint64_t)kHin * kS2dC * 2, (uint64_t)kHin * kHin * kS2dC * 2};
    const uint32_t box[4] = {(uint32_t)kS2dC, (uint32_t)kRowPos, 1, 1};
    if (!make_nd_tmap(&ta, x, 4, dims, strides, box, 32)) fail(5, "conv1_pool: input tensor map failed");
  } else if (!make_rowview_tmap(&ta, x, N, kHin, kHin, kS2dC, kHo)) {
    fail(5, "conv1_pool: row-view tensor map failed");
  }
  p.x = x;
  p.y = y;
  p.scale = L.scale;
  p.shift = L.shift;
  p.N = N;
  const char* e = getenv("VISTA_STEM_IROW");  // read per launch (A/B within one process)
  p.irow = (e && e[0] == '0') ? 0 : 1;
  const char* ew = getenv("VISTA_STEM_EPW");  // epilogue warps: 16 (default) or 8 (A/B)
  const bool w16 = !(ew && atoi(ew) == 8);
  const void* kern = w16 ? (const void*)conv1_pool_kernel<16> : (const void*)conv1_pool_kernel<8>;
  ensure_smem_attr(kern, kSmem);
  const int grid = N < num_sms() ? N : num_sms();
  prof_begin(st);
  if (w16) conv1_pool_kernel<16><<<grid, (kEpiWarp0 + 16) * 32, kSmem, st>>>(L.tmap_w, ta, p);
  else conv1_pool_kernel<8><<<grid, (kEpiWarp0 + 8) * 32, kSmem, st>>>(L.tmap_w, ta, p);
  LAUNCHED();
  const double flops = 2.0 * (double)N * kHo * kHo * kCo * L.K_alg;
  const double bytes = (double)N * (kHin * kHin * kS2dC * 2 + kPo * kPo * kCo * 2) + (double)kCo * L.Kp * 2;
  prof_end(st, 0, flops, bytes, prof_labels() ? "conv1+pool1 fused (s2d rowview)" : nullptr);
}

}  // namespace vista
