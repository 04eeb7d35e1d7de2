// conv_tc.cu — implicit-GEMM convolution / fully-connected layer on the sm_100a
// 5th-generation tensor cores (tcgen05.mma, fp32 accumulators in TMEM), with a fused
// epilogue: per-channel scale/shift (BN in inference form or bias, reading R12),
// residual add (ResNet unit), ReLU, RNE to bf16.
//
// This is S1 of SURVEY.md §8a: partial CNN inference f^_{i -> j} (Def 3.7,
// PAPER.md:138-141) is a chain of these TensorOps.  GEMM view per group g:
//   D[m, n] = sum_k A[m, k] * B[n, k],  m = output pixel (n_img, ho, wo),
//   n = output channel, k = (r*S + s)*Cg_in + c.
//
// Persistent, warp-specialised kernel, one CTA per SM, 128 x BN x 64 tiles:
//   warps 0-3  A producers: either one elected thread issuing TMA for a plain [M, C]
//              activation (1x1 stride-1 convs, FC layers), or 128 threads gathering the
//              implicit im2col rows with 16-byte cp.async (zero-fill = padding) into the
//              128B-swizzled K-major layout.  Thread 0 also issues the weight (B) TMA.
//   warp 4     TMEM allocator + single-thread tcgen05.mma issuer.
//   warps 5-8  epilogue: tcgen05.ld -> scale/shift (smem) + residual + ReLU -> bf16.
// TMEM holds two accumulators (2 x BN columns) so the epilogue of tile i overlaps the
// mainloop of tile i+1; an mbarrier ring of STAGES k-blocks feeds the tensor core.
#include <cudaTypedefs.h>

#include <cstdio>
#include <cstring>
#include <mutex>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

enum AMode {
  A_GATHER_FAST = 0,
  A_GATHER_GENERAL = 1,
  A_TMA = 2,
  A_GATHER_ROW = 3,
  A_IM2COL = 4,
  A_IM2COL_C8 = 5,
  A_ROWVIEW = 6,
  A_HALO = 7,
  A_CAT = 8
};
__host__ __device__ constexpr bool a_by_tma(int m) {
  return m == A_TMA || m == A_IM2COL || m == A_IM2COL_C8 || m == A_ROWVIEW || m == A_HALO || m == A_CAT;
}
// A_HALO (3x3 stride 1 pad 1, one N tile): the output is computed on the padded-width grid (Wp = W + 2
// positions per row, the last two discarded) so that output position p reads padded input position
// p + r*Wp + s for filter tap (r, s): ONE TMA box {64 ch, Wp, hrows, 1} per channel block and tile lands
// the zero-padded input rows (out-of-bounds fill = padding) and every tap's A operand is that buffer
// shifted by (r*Wp + s) rows -- nine times fewer A bytes through shared memory than im2col boxes.
__host__ __device__ constexpr int halo_half_bytes(int BN) { return BN == 64 ? 45056 : (BN == 128 ? 61440 : 0); }

struct ConvParams {
  const bf16* x;
  bf16* y;
  const bf16* res;
  const float* scale;
  const float* shift;
  int H, W, Cin, Ho, Wo, Cout, R, S, stride, pad, Cg_in, Cg_out, K, nkb, M, relu;
  int n_mt, n_nt, n_tiles;
  int Wp, hrows, hsz, mt_per_img, cblocks;  // A_HALO geometry (see above)
  // A_HALO: per k-block offset of the A operand inside the halo buffer, in 16-byte descriptor units:
  // ((r*Wp + s) * 128 + cb * hsz) >> 4 for kb = (r*3 + s) * cblocks + cb.  Precomputed so that the MMA
  // issue loop has no integer division (measured: the per-k-block division chain made the issue latency
  // ~340 cycles, longer than the 4 MMAs it feeds)
  int koff[36];
  // A_HALO (padded-grid tiles): first output position's column in the first halo row of a tile, indexed by
  // (M tile index mod mt_per_img) -- removes the MMA warp's per-tile integer divisions (measured ~650 cycles
  // per tile on res3 3x3); valid when mt_per_img <= 64
  short hofft[64];
  // A_CAT (unit-1 closing conv with the projection shortcut folded in, see conv_cat_forward): k-blocks
  // [0, nkb1) read the b activation through tmap_a, k-blocks [nkb1, nkb) read the unit input x through
  // tmap_r (plain 2-D map, or an im2col map when the projection is strided: cat_im2col = 1)
  int nkb1, cat_im2col;
  // mc = 1: launched as clusters of 2 CTAs; the pair walks "pair tiles" (two adjacent M tiles, one N tile:
  // rank r takes M tile 2 * pair_m + r) in lockstep, and each CTA TMA-loads half of every weight (B) k-block
  // and multicasts it to both, halving the per-SM L2 -> shared-memory weight traffic of streamed-B layers
  int mc;
  // cg2 = 1 (with mc = 1, A_HALO padded-grid tiles): the CTA pair runs ONE tcgen05.mma.cta_group::2 over
  // M = 256 (rank r's 128 rows in its own shared memory and TMEM); the pair tile is the same position in two
  // consecutive images (rank r: image 2j + r), so both halos sit at the same offsets; each CTA loads half of
  // every weight k-block (B's N rows split between the pair): per-SM operand reads 4 KB + BN/2 * 32 B per
  // MMA instead of 4 KB + BN * 32 B, and half the weight bytes written into each CTA's shared memory.
  // cg2 = 2 (A_IM2COL / A_TMA, BN = 256): the same pair MMA over the multicast pair tile (two adjacent M
  // tiles; both CTAs' A tiles sit in the same ring stage)
  int cg2;
  // amc = 1 (resident weights, A_TMA / stride-1 A_CAT, an even number of N tiles): CTA pairs (blockIdx 2i, 2i+1)
  // hold adjacent N tiles and walk the same M tiles; each loads half of every A k-block's rows and multicasts
  // it to both, halving the per-SM L2 -> shared-memory A bytes (A is re-read once per N tile)
  int amc;
  // apf > 0 (resident-weight A_TMA launches): the CTA holding N tile 0 prefetches into L2 the A rows of the M tile
  // it will reach apf tiles later (the 64 KB A of a K = 256 tile is one contiguous range; the TMA loads of the
  // CTAs sharing that M tile then hit L2 instead of waiting on HBM behind a 4-stage ring)
  int apf;
  int no_sthr;  // 1: TMA epilogue without the store thread (VISTA_STORE_THR=0, A/B)
  int segs;  // A_ROWVIEW: 128-pixel segments per output row (1 unless Wo > 128); A_HALO + hseg: segments
  // A_HALO row-segment tiles (hseg = 1, rows too wide for the padded-grid halo): tile = (image, output row,
  // segment of seg_w <= 126 columns); the halo is 3 input rows x (seg_w + 2) padded columns (Wp = seg_w + 2)
  int hseg, seg_w;
  // fused tap g_l (PAPER.md:369 fn 4): per-image 2x2-grid channel maxima of the (post-ReLU, >= 0)
  // output, accumulated as fp32 bit patterns with red.global.max.u32 into tapf[n][4][Cout]
  unsigned int* tapf;
  int out_f32;  // register epilogue writes fp32 (gemm_tn: weight gradients of the MLP head)
  unsigned long long* dbg_buf;  // (dbg & 8): per-CTA cycle counters of the MMA warp [grid][8]
  int dbg;      // VISTA_CONV_DBG bit mask (measurement experiments only; results wrong when set): 1 = halo loaded
                // once, 2 = epilogue only waits / releases the accumulator, 8 = MMA-warp cycle counters (halo)
};

constexpr int BM = 128, BK = 64;
constexpr int kEpiWarps = 8;   // two per TMEM lane quadrant, each owning half of the tile's columns
constexpr int kEpiThreads = kEpiWarps * 32;
constexpr int kThreads = 160 + kEpiThreads;  // 4 producer warps + 1 MMA warp + epilogue warps
constexpr int kEpiWarp0 = 5;
constexpr int kLag = 2;        // cp.async groups in flight before a stage is published

// Shared memory: [A stages][B stages][output staging: NB buffers of BN/64 sub-tiles of 128 x 64 bf16,
// 128B-swizzled (TMA epilogue only)][scale/shift][barriers]
// NB (TMA epilogue): staging buffers; a residual tile is prefetched NB - 1 tiles ahead into the buffer
// the tile's output is later staged in, so NB >= 3 hides the residual's HBM latency behind a whole tile.
// RKB > 0 (resident weights): the CTA's whole B slice (RKB >= nkb k-blocks of BN x 64) is loaded once and
// stays in shared memory; the launch makes the grid a multiple of the N-tile count so that every tile a CTA
// visits (tile += gridDim.x) has the same N tile.  Only A streams through the ring (A_HALO: no ring at
// all, and three halo buffers).  Measured motivation: the per-SM L2 -> smem ingest is bounded by the
// bytes in flight / L2 latency, and re-loading the weights per tile doubled (1x1) or tripled (halo 3x3,
// Cout = 64) the bytes each tile needs.
template <int BN, bool TMA_EPI, int NB, bool HALO = false, int RKB = 0, bool CG2 = false>
struct Cfg {
  static constexpr int kHB = HALO ? (RKB ? 3 : 2) : 0;  // halo buffers (A_HALO)
  static constexpr int kHaloBytes = kHB * halo_half_bytes(BN);
  static constexpr int kABytes = HALO ? 0 : BM * BK * 2;  // 16 KB per stage (A_HALO: A lives in the halo)
  static constexpr int kBBytes = (CG2 ? BN / 2 : BN) * BK * 2;  // CTA pair: this CTA's half of the N rows
  static constexpr int kResBytes = RKB * kBBytes;          // resident weights
  static constexpr int kStageBytes = kABytes + (RKB ? 0 : kBBytes);
  static constexpr int kOutBufs = TMA_EPI ? NB : 0;
  static constexpr int kOutBytes = kOutBufs * BM * BN * 2;
  // TMA epilogue: one scale/shift buffer (a named barrier separates tiles); register epilogue: two
  static constexpr int kSbufBytes = (TMA_EPI ? 1 : 2) * 2 * BN * 4;
  // register epilogue with BN <= 128: four TMEM accumulators, and the two epilogue warp groups take
  // alternate tiles (each group drains all BN columns of its tiles), so two tiles' epilogues overlap
  static constexpr bool kSplit = !TMA_EPI && BN <= 128;
  // BN = 64 register epilogue: each warp stages its 32 rows x 32 columns in smem and writes them back with
  // 4 rows per instruction (per-row 16-byte stores touched 32 lines per instruction: LSU-bound, measured)
  static constexpr bool kStaged = kSplit && BN == 64;
  static constexpr int kStgBytes = kStaged ? kEpiWarps * 32 * 64 : 0;
  static constexpr int kNBar = 28;  // tfull/tempty[4], rbar[4], hfull/hempty[3], wres[1], staged/sfree[4], slack
  static constexpr int kFixed = kHaloBytes + kResBytes + kOutBytes + kSbufBytes + kStgBytes + 1024 + 16 + kNBar * 8;
  static constexpr int kStagesFit = kStageBytes ? (227 * 1024 - kFixed) / (kStageBytes + 16) : 2;
  static constexpr int kStages = kStagesFit > 8 ? 8 : kStagesFit;
  static constexpr int kResOff = kStages * kStageBytes;
  static constexpr int kHaloOff = kResOff + kResBytes;
  static constexpr int kOutOff = kHaloOff + kHaloBytes;
  static constexpr int kSbufOff = kOutOff + kOutBytes;
  static constexpr int kStgOff = kSbufOff + kSbufBytes;
  static constexpr int kBarOff = kStgOff + kStgBytes;
  static constexpr int kBytes = kBarOff + (2 * kStages + kNBar) * 8 + 16 + 1024;  // + alignment slack
  static constexpr int kAcc = kSplit ? 4 : 2;
  static constexpr int kTmemCols = kAcc * BN;
  static_assert(kStages >= 2, "shared memory too small for two k-block stages");
  static_assert(kBytes <= 227 * 1024, "shared memory over the 227 KB per-CTA limit");
};

// tile -> (first row m0, N-tile index nt, group g); N-tiles of one M-tile are adjacent so
// the 148 CTAs working at any moment share A rows in L2
__device__ __forceinline__ void decode_tile(const ConvParams& p, int tile, int& m0, int& nt, int& g) {
  if (p.cg2 == 1) {  // halo pair tile (j, t) -> M tile t of image 2j + rank (rank 1 past the last image: phantom)
    const int j = tile / p.mt_per_img, t = tile - j * p.mt_per_img;
    m0 = ((2 * j + (int)(blockIdx.x & 1)) * p.mt_per_img + t) * BM;
    nt = 0;
    g = 0;
    return;
  }
  if (p.mc) {  // pair tile -> this CTA's M tile (an odd last M tile leaves rank 1 a phantom tile past M)
    const int pm = tile / p.n_nt;
    nt = tile - pm * p.n_nt;
    m0 = (pm * 2 + (int)(blockIdx.x & 1)) * BM;
    g = 0;
    return;
  }
  const int per_g = p.n_mt * p.n_nt;
  g = tile / per_g;
  const int rem = tile - g * per_g;
  const int mt = rem / p.n_nt;
  m0 = mt * BM;
  nt = rem - mt * p.n_nt;
}

__device__ __forceinline__ void epi_math(const uint32_t* v, const float* scv, const float* shv, bool has_res,
                                         uint4 r, bool relu, uint4& o) {
  o = epi8(v, scv, shv, r, has_res, relu);
}

__device__ __forceinline__ void epi_math_f32(const uint32_t* v, const float* scv, const float* shv, bool relu,
                                             float* out) {
  float f[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) f[j] = fmaf(__uint_as_float(v[j]), scv[j], shv[j]);
  if (relu) {
#pragma unroll
    for (int j = 0; j < 8; ++j) f[j] = fmaxf(f[j], 0.0f);
  }
  reinterpret_cast<float4*>(out)[0] = make_float4(f[0], f[1], f[2], f[3]);
  reinterpret_cast<float4*>(out)[1] = make_float4(f[4], f[5], f[6], f[7]);
}

template <int BN, int AMODE, bool TMA_EPI, int NB, int RKB, bool CG2 = false>
__global__ void __launch_bounds__(kThreads, 1)
    conv_tc_kernel(const __grid_constant__ CUtensorMap tmap_w, const __grid_constant__ CUtensorMap tmap_a,
                   const __grid_constant__ CUtensorMap tmap_y, const __grid_constant__ CUtensorMap tmap_r,
                   const ConvParams p) {
  using C = Cfg<BN, TMA_EPI, NB, AMODE == A_HALO, RKB, CG2>;
  static_assert(!CG2 || (AMODE == A_HALO ? !TMA_EPI : (AMODE == A_IM2COL || AMODE == A_TMA || AMODE == A_CAT)),
                "CTA-pair MMA: halo (register epilogue) / im2col / plain TMA / cat A");
  constexpr int S = C::kStages;
  constexpr bool BRES = RKB > 0;
  constexpr int HB = C::kHB > 0 ? C::kHB : 1;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  uint8_t* gbase = smem_raw + (base - raw);
  // ring stage i: A at sA + i * kABytes; B (streamed weights) at sB + i * kBBytes; resident weights at sR
  const uint32_t sA = base, sB = base + S * C::kABytes, sO = base + C::kOutOff, sR = base + C::kResOff;
  float* sbuf = reinterpret_cast<float*>(gbase + C::kSbufOff);  // [1 or 2][scale BN | shift BN]
  uint64_t* full = reinterpret_cast<uint64_t*>(gbase + C::kBarOff);
  uint64_t* empty = full + S;
  constexpr int NACC = C::kAcc;
  constexpr bool SPLIT = C::kSplit;
  uint64_t* tfull = empty + S;      // [NACC]
  uint64_t* tempty = tfull + NACC;  // [NACC]
  uint64_t* rbar = tempty + NACC;   // [NB <= 4] residual tile landed in staging buffer b (TMA epilogue)
  uint64_t* hfull = rbar + 4;    // [3] halo buffer landed (A_HALO)
  uint64_t* hempty = hfull + 3;  // [3] halo buffer consumed by the tile's MMAs (A_HALO)
  uint64_t* wres = hempty + 3;   // [1] resident weights landed (RKB > 0)
  uint64_t* staged = wres + 1;   // [NB] store thread: the epilogue has written staging buffer b
  uint64_t* sfree = staged + 4;  // [NB] store thread: buffer b's TMA store has read it (no residual)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(sfree + 4);
  // TMA epilogue with a dedicated store thread (thread 32, idle in these A modes): it issues the output stores,
  // waits for their shared-memory reads and refills the freed buffer with a later tile's residual, so the
  // epilogue warps never wait on store completion or on one another (no per-tile named barriers)
  constexpr bool kStoreThrMode = TMA_EPI && (AMODE == A_TMA || AMODE == A_CAT || AMODE == A_IM2COL ||
                                             AMODE == A_ROWVIEW || AMODE == A_IM2COL_C8);
  const bool sthr = kStoreThrMode && !p.tapf && !p.no_sthr;
  const uint32_t sH = base + C::kHaloOff;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // this CTA's first tile and the tile stride (pair tiles when multicasting weights)
  const int cta0 = p.mc ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int ncta = p.mc ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  const uint32_t crank = (p.mc || p.amc) ? (blockIdx.x & 1u) : 0u;
  // weight k-block kb of N rows [row0, row0 + BN) into ring stage `stage` (multicast: this CTA's half)
  auto load_b = [&](int stage, int kb, int row0) {
    if (p.mc)
      tma_load_2d_mc(sB + stage * C::kBBytes + crank * (BN / 2) * 128, &tmap_w, kb * BK, row0 + (int)crank * (BN / 2),
                     &full[stage], (uint16_t)3);
    else
      tma_load_2d(sB + stage * C::kBBytes, &tmap_w, kb * BK, row0, &full[stage]);
  };
  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&full[i], a_by_tma(AMODE) ? (CG2 ? 2 : 1) : 128 + 1);  // CTA pair: both CTAs arrive
      // multicast: both CTAs' MMAs must release the stage; CTA pair: the leader's one pair commit does
      mbar_init(&empty[i], (p.mc && !CG2) || p.amc ? 2 : 1);
    }
    for (int i = 0; i < NACC; ++i) {
      mbar_init(&tfull[i], 1);
      // CTA pair: the leader's MMA reuses an accumulator once BOTH CTAs' epilogues drained it
      mbar_init(&tempty[i], (SPLIT ? kEpiWarps / 2 : kEpiWarps) * (CG2 ? 2 : 1));
    }
    for (int i = 0; i < 4; ++i) mbar_init(&rbar[i], 1);
    for (int i = 0; i < 3; ++i) {
      mbar_init(&hfull[i], CG2 ? 2 : 1);
      mbar_init(&hempty[i], 1);
    }
    mbar_init(wres, CG2 ? 2 : 1);
    for (int i = 0; i < 4; ++i) {
      mbar_init(&staged[i], kEpiWarps);
      mbar_init(&sfree[i], 1);
    }
    fence_mbar_init();
    tma_prefetch(&tmap_w);
    if (a_by_tma(AMODE)) tma_prefetch(&tmap_a);
    if (TMA_EPI) tma_prefetch(&tmap_y);
  }
  if constexpr (CG2) cluster_sync_all();  // both CTAs of the pair enter the pair allocation together
  if (warp == 4) {
    if constexpr (CG2) tmem_alloc_cg2(tmem_slot, C::kTmemCols);
    else tmem_alloc(tmem_slot, C::kTmemCols);
  }
  tc_fence_before();
  __syncthreads();
  if (p.mc || p.amc) cluster_sync_all();  // the partner's barriers are initialised before any multicast reaches them
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp < 4) {
    // ======================= producers =======================
    if (sthr && threadIdx.x == 32) {
      // ---- store thread (TMA epilogue): stores of tile it from buffer it % NB, residual refills ----
      const bool has_res = p.res != nullptr;
      auto issue_res = [&](int t, uint32_t b) {
        int tm0, tnt, tg;
        decode_tile(p, t, tm0, tnt, tg);
        const int tn0 = tnt * BN, tng0 = tg * p.Cg_out + tn0;
        const int nsub = (min(BN, p.Cg_out - tn0) + 63) / 64;
        mbar_arrive_expect_tx(&rbar[b], nsub * BM * 128);
        for (int st = 0; st < nsub; ++st)
          tma_load_2d(sO + b * (uint32_t)(BM * BN * 2) + st * BM * 128, &tmap_r, tng0 + st * 64, tm0, &rbar[b]);
      };
      if (has_res)  // the first residual tiles (NB = 1: the first tile's)
        for (int j = 0; j < (NB > 1 ? NB - 1 : 1); ++j)
          if (cta0 + j * ncta < p.n_tiles) issue_res(cta0 + j * ncta, j);
      uint32_t it = 0;
      for (int tile = cta0; tile < p.n_tiles; tile += ncta, ++it) {
        const uint32_t b = NB > 1 ? it % NB : 0;
        mbar_wait(&staged[b], (it / NB) & 1);
        int m0, nt, g;
        decode_tile(p, tile, m0, nt, g);
        const int n0 = nt * BN, ng0 = g * p.Cg_out + n0;
        const int nsub = (min(BN, p.Cg_out - n0) + 63) / 64;
        const uint32_t sb = sO + b * (uint32_t)(BM * BN * 2);
        for (int st = 0; st < nsub; ++st) {
          if constexpr (AMODE == A_ROWVIEW)  // 3-D output map {C, Wo, rows}: q >= Wo clipped
            tma_store_3d(&tmap_y, ng0 + st * 64, (m0 / BM) % p.segs * BM, (m0 / BM) / p.segs, sb + st * BM * 128);
          else
            tma_store_2d(&tmap_y, ng0 + st * 64, m0, sb + st * BM * 128);
        }
        bulk_commit();
        if (NB == 1) {  // this tile's buffer, once its stores have read it, serves the next tile
          bulk_wait_read0();
          if (has_res) {
            if (tile + ncta < p.n_tiles) issue_res(tile + ncta, 0);
          } else {
            mbar_arrive(&sfree[0]);
          }
        } else {  // buffer (it + NB - 1) % NB held tile it - 1: refill it for tile it + NB - 1
          if (it >= 1) bulk_wait_read<1>();
          const uint32_t fb = (it + NB - 1) % NB;
          if (has_res) {
            if (tile + (NB - 1) * ncta < p.n_tiles) issue_res(tile + (NB - 1) * ncta, fb);
          } else if (it >= 1) {
            mbar_arrive(&sfree[fb]);
          }
        }
      }
      bulk_wait0();
    }
    if constexpr (BRES) {
      // resident weights: the B slice of this CTA's (fixed) N tile, once
      if (threadIdx.x == 0) {
        int m0, nt, g;
        decode_tile(p, cta0, m0, nt, g);
        if constexpr (CG2) {  // CTA pair: this CTA's half of the N rows, completing on the leader's barrier
          const uint32_t wl = mapa_u32(smem_u32(wres), 0);
          if (crank == 0) mbar_arrive_expect_tx(wres, 2 * p.nkb * C::kBBytes);
          for (int kb = 0; kb < p.nkb; ++kb)
            tma_load_2d_cg2(sR + kb * C::kBBytes, &tmap_w, kb * BK, nt * BN + (int)crank * (BN / 2), wl);
          if (crank != 0) mbar_arrive_cluster(wl);
        } else {
          mbar_arrive_expect_tx(wres, p.nkb * C::kBBytes);
          for (int kb = 0; kb < p.nkb; ++kb)
            tma_load_2d(sR + kb * C::kBBytes, &tmap_w, kb * BK, g * p.Cg_out + nt * BN, wres);
        }
      }
    }
    if constexpr (AMODE == A_TMA) {
      if (threadIdx.x == 0) {
        uint32_t gk = 0;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta) {
          int m0, nt, g;
          decode_tile(p, tile, m0, nt, g);
          const int n0 = nt * BN;
          if (BRES && p.apf > 0 && nt == 0) {
            const int tf = tile + p.apf * ncta;
            if (tf < p.n_tiles) {
              int mf, ntf, gf;
              decode_tile(p, tf, mf, ntf, gf);
              const int rows = min(BM, p.M - mf);
              prefetch_l2_range(p.x + (size_t)mf * p.Cin, (uint64_t)rows * p.Cin * 2);
            }
          }
          for (int kb = 0; kb < p.nkb; ++kb, ++gk) {
            const int stage = gk % S;
            if (gk >= (uint32_t)S) mbar_wait(&empty[stage], ((gk / S) - 1) & 1);
            if constexpr (CG2) {  // own A rows + own half of the B rows, completing on the leader's barrier
              const uint32_t fl = mapa_u32(smem_u32(&full[stage]), 0);
              if (crank == 0) mbar_arrive_expect_tx(&full[stage], 2 * C::kStageBytes);
              tma_load_2d_cg2(sA + stage * C::kABytes, &tmap_a, kb * BK, m0, fl);
              if constexpr (!BRES)
                tma_load_2d_cg2(sB + stage * C::kBBytes, &tmap_w, kb * BK, n0 + (int)crank * (BN / 2), fl);
              if (crank != 0) mbar_arrive_cluster(fl);
              continue;
            }
            mbar_arrive_expect_tx(&full[stage], C::kStageBytes);
            if (BRES && p.amc)  // this CTA's half of the A rows, multicast to the pair (same M tile)
              tma_load_2d_mc(sA + stage * C::kABytes + crank * (BM / 2) * 128, &tmap_a, kb * BK,
                             m0 + (int)crank * (BM / 2), &full[stage], (uint16_t)3);
            else
              tma_load_2d(sA + stage * C::kABytes, &tmap_a, g * p.Cg_in + kb * BK, m0, &full[stage]);
            if constexpr (!BRES) load_b(stage, kb, g * p.Cg_out + n0);
          }
        }
      }
    } else if constexpr (AMODE == A_CAT) {
      if (threadIdx.x == 0) {
        const int hw = p.Ho * p.Wo;
        uint32_t gk = 0;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta) {
          int m0, nt, g;
          decode_tile(p, tile, m0, nt, g);
          const int n0 = nt * BN;
          const int nimg = m0 / hw, rem = m0 - nimg * hw;
          const int ho = rem / p.Wo, wo = rem - ho * p.Wo;
          for (int kb = 0; kb < p.nkb; ++kb, ++gk) {
            const int stage = gk % S;
            if (gk >= (uint32_t)S) mbar_wait(&empty[stage], ((gk / S) - 1) & 1);
            if constexpr (CG2) {  // own A rows + own half of the B rows, completing on the leader's barrier
              const uint32_t fl = mapa_u32(smem_u32(&full[stage]), 0);
              if (crank == 0) mbar_arrive_expect_tx(&full[stage], 2 * C::kStageBytes);
              if (kb < p.nkb1)
                tma_load_2d_cg2(sA + stage * C::kABytes, &tmap_a, kb * BK, m0, fl);
              else if (p.cat_im2col)
                tma_load_im2col_4d_cg2(sA + stage * C::kABytes, &tmap_r, (kb - p.nkb1) * BK, wo * p.stride,
                                       ho * p.stride, nimg, 0, 0, fl);
              else
                tma_load_2d_cg2(sA + stage * C::kABytes, &tmap_r, (kb - p.nkb1) * BK, m0, fl);
              if constexpr (!BRES)
                tma_load_2d_cg2(sB + stage * C::kBBytes, &tmap_w, kb * BK, n0 + (int)crank * (BN / 2), fl);
              if (crank != 0) mbar_arrive_cluster(fl);
              continue;
            }
            mbar_arrive_expect_tx(&full[stage], C::kStageBytes);
            if (BRES && p.amc) {  // stride 1: this CTA's half of the A rows of either source, multicast
              const uint32_t dst = sA + stage * C::kABytes + crank * (BM / 2) * 128;
              const int mr = m0 + (int)crank * (BM / 2);
              if (kb < p.nkb1) tma_load_2d_mc(dst, &tmap_a, kb * BK, mr, &full[stage], (uint16_t)3);
              else tma_load_2d_mc(dst, &tmap_r, (kb - p.nkb1) * BK, mr, &full[stage], (uint16_t)3);
            } else if (kb < p.nkb1)
              tma_load_2d(sA + stage * C::kABytes, &tmap_a, kb * BK, m0, &full[stage]);
            else if (p.cat_im2col)
              tma_load_im2col_4d(sA + stage * C::kABytes, &tmap_r, (kb - p.nkb1) * BK, wo * p.stride, ho * p.stride,
                                 nimg, 0, 0, &full[stage]);
            else
              tma_load_2d(sA + stage * C::kABytes, &tmap_r, (kb - p.nkb1) * BK, m0, &full[stage]);
            if constexpr (!BRES) load_b(stage, kb, n0);
          }
        }
      }
    } else if constexpr (AMODE == A_HALO) {
      // thread 0: halo boxes (tile t + 2's halo as soon as tile t's MMAs release its buffer); thread 32 (warp 1):
      // the streamed weight stages.  One thread doing both put the next halo behind the current tile's weight
      // loads, which wait for ring stages the running MMAs free (measured: the halo wait became the bound)
      if (!BRES && threadIdx.x == 32) {
        constexpr int S2 = S / 2;  // two k-blocks per ring stage (S / 2 stages of 2 x BN x 64)
        uint32_t gk = 0;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta)
          for (int kb = 0; kb < p.nkb; kb += 2, ++gk) {
            const int stage = gk % S2;
            if (gk >= (uint32_t)S2) mbar_wait(&empty[stage], ((gk / S2) - 1) & 1);
            const int two = kb + 1 < p.nkb ? 2 : 1;
            if constexpr (CG2) {
              // CTA pair: this CTA's half of the N rows into its own stage; both halves complete on the leader's
              // barrier, which the leader arms for both
              const uint32_t fl = mapa_u32(smem_u32(&full[stage]), 0);
              if (crank == 0) mbar_arrive_expect_tx(&full[stage], 2 * two * C::kBBytes);
              for (int h = 0; h < two; ++h)
                tma_load_2d_cg2(sB + (2 * stage + h) * C::kBBytes, &tmap_w, (kb + h) * BK, (int)crank * (BN / 2), fl);
              if (crank != 0) mbar_arrive_cluster(fl);
              continue;
            }
            mbar_arrive_expect_tx(&full[stage], two * C::kBBytes);
            for (int h = 0; h < two; ++h) {
              if (p.mc)  // this CTA's half of the k-block rows, multicast to the pair
                tma_load_2d_mc(sB + (2 * stage + h) * C::kBBytes + crank * (BN / 2) * 128, &tmap_w, (kb + h) * BK,
                               (int)crank * (BN / 2), &full[stage], (uint16_t)3);
              else
                tma_load_2d(sB + (2 * stage + h) * C::kBBytes, &tmap_w, (kb + h) * BK, 0, &full[stage]);
            }
          }
      }
      if (threadIdx.x == 0) {
        uint32_t it = 0;
        const uint32_t box_bytes = (uint32_t)p.hrows * p.Wp * 128u;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta, ++it) {
          int m0, nt, g;
          decode_tile(p, tile, m0, nt, g);
          const int mt = m0 / BM;
          int nimg, prow0, col0 = -1;
          if (p.hseg) {  // (image, output row ho, segment): input rows ho - 1 .. ho + 1, columns from seg * seg_w - 1
            const int rowi = mt / p.segs;
            nimg = rowi / p.Ho;
            prow0 = rowi - nimg * p.Ho;
            col0 = (mt - rowi * p.segs) * p.seg_w - 1;
          } else {
            nimg = mt / p.mt_per_img;
            const int p0 = (mt - nimg * p.mt_per_img) * BM;
            prow0 = p0 / p.Wp;  // first padded input row (input row prow0 - 1)
          }
          const uint32_t hb = it % HB;
          if (it >= (uint32_t)HB) mbar_wait(&hempty[hb], ((it / HB) - 1) & 1);
          if constexpr (CG2) {  // own halo, completing on the leader's barrier (armed by the leader for both)
            const uint32_t hl = mapa_u32(smem_u32(&hfull[hb]), 0);
            if (crank == 0) mbar_arrive_expect_tx(&hfull[hb], 2 * box_bytes * p.cblocks);
            for (int cb = 0; cb < p.cblocks; ++cb)
              tma_load_4d_cg2(sH + hb * halo_half_bytes(BN) + cb * p.hsz, &tmap_a, cb * BK, col0, prow0 - 1, nimg, hl);
            if (crank != 0) mbar_arrive_cluster(hl);
            continue;
          }
          if ((p.dbg & 1) && it >= (uint32_t)HB) {
            mbar_arrive(&hfull[hb]);
          } else {
            mbar_arrive_expect_tx(&hfull[hb], box_bytes * p.cblocks);
            for (int cb = 0; cb < p.cblocks; ++cb)
              tma_load_4d(sH + hb * halo_half_bytes(BN) + cb * p.hsz, &tmap_a, cb * BK, col0, prow0 - 1, nimg,
                          &hfull[hb]);
          }
        }
      }
    } else if constexpr (AMODE == A_ROWVIEW) {
      // one tile = one output row (n, p) of Wo <= 128 pixels; k-block = filter row r: a 4-D tiled
      // TMA over an overlapping view {64 elements, q, h, n} (q stride = one input pixel) lands the
      // 128-byte windows of input row p + r for q = 0..127 (q >= Wo out of bounds -> zeros).
      if (threadIdx.x == 0) {
        uint32_t gk = 0;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta) {
          int m0, nt, g;
          decode_tile(p, tile, m0, nt, g);
          const int n0 = nt * BN;
          const int rs = m0 / BM;  // (output row n * Ho + p) * segs + segment
          const int rr = rs / p.segs, seg = rs - rr * p.segs;
          const int nimg = rr / p.Ho, ho = rr - nimg * p.Ho;
          for (int kb = 0; kb < p.nkb; ++kb, ++gk) {
            const int stage = gk % S;
            if (gk >= (uint32_t)S) mbar_wait(&empty[stage], ((gk / S) - 1) & 1);
            mbar_arrive_expect_tx(&full[stage], C::kStageBytes);
            tma_load_4d(sA + stage * C::kABytes, &tmap_a, 0, seg * BM, ho + kb, nimg, &full[stage]);
            if constexpr (!BRES) load_b(stage, kb, g * p.Cg_out + n0);
          }
        }
      }
    } else if constexpr (AMODE == A_IM2COL_C8) {
      // first layers (input padded to 8 channels): every filter tap is one 16-byte K-slice; eight TMA
      // im2col loads of 128 pixels x 8 channels fill a k-block laid out as 8 no-swizzle core-matrix
      // columns (LBO 2 KB).  Taps past R*S repeat a valid tap against zero weights.
      if (threadIdx.x == 0) {
        const int hw = p.Ho * p.Wo;
        const int RS = p.R * p.S;
        uint32_t gk = 0;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta) {
          int m0, nt, g;
          decode_tile(p, tile, m0, nt, g);
          const int n0 = nt * BN;
          const int nimg = m0 / hw, rem = m0 - nimg * hw;
          const int ho = rem / p.Wo, wo = rem - ho * p.Wo;
          const int w0 = wo * p.stride - p.pad, h0 = ho * p.stride - p.pad;
          for (int kb = 0; kb < p.nkb; ++kb, ++gk) {
            const int stage = gk % S;
            if (gk >= (uint32_t)S) mbar_wait(&empty[stage], ((gk / S) - 1) & 1);
            mbar_arrive_expect_tx(&full[stage], C::kABytes + C::kBBytes);
#pragma unroll 1
            for (int j = 0; j < 8; ++j) {
              int t = kb * 8 + j;
              if (t >= RS) t -= RS;
              const int r = t / p.S, s = t - (t / p.S) * p.S;
              tma_load_im2col_4d(sA + stage * C::kABytes + j * 2048, &tmap_a, 0, w0, h0, nimg, (uint16_t)s,
                                 (uint16_t)r, &full[stage]);
            }
            load_b(stage, kb, g * p.Cg_out + n0);
          }
        }
      }
    } else if constexpr (AMODE == A_IM2COL) {
      // one TMA per k-block gathers 128 output pixels x 64 channels of filter tap (r, s):
      // k-block kb -> (r, s, channel block) with k = (r*S + s)*Cg_in + c
      if (threadIdx.x == 0) {
        const int cblocks = p.Cg_in / BK;
        const int hw = p.Ho * p.Wo;
        uint32_t gk = 0;
        for (int tile = cta0; tile < p.n_tiles; tile += ncta) {
          int m0, nt, g;
          decode_tile(p, tile, m0, nt, g);
          const int n0 = nt * BN;
          const int nimg = m0 / hw, rem = m0 - nimg * hw;
          const int ho = rem / p.Wo, wo = rem - ho * p.Wo;
          const int w0 = wo * p.stride - p.pad, h0 = ho * p.stride - p.pad;
          int r = 0, s = 0, cb = 0;
          for (int kb = 0; kb < p.nkb; ++kb, ++gk) {
            const int stage = gk % S;
            if (gk >= (uint32_t)S) mbar_wait(&empty[stage], ((gk / S) - 1) & 1);
            if constexpr (CG2) {  // own A rows + own half of the B rows, completing on the leader's barrier
              const uint32_t fl = mapa_u32(smem_u32(&full[stage]), 0);
              if (crank == 0) mbar_arrive_expect_tx(&full[stage], 2 * (C::kABytes + C::kBBytes));
              tma_load_im2col_4d_cg2(sA + stage * C::kABytes, &tmap_a, cb * BK, w0, h0, nimg, (uint16_t)s, (uint16_t)r,
                                     fl);
              tma_load_2d_cg2(sB + stage * C::kBBytes, &tmap_w, kb * BK, n0 + (int)crank * (BN / 2), fl);
              if (crank != 0) mbar_arrive_cluster(fl);
            } else {
              mbar_arrive_expect_tx(&full[stage], C::kABytes + C::kBBytes);
              tma_load_im2col_4d(sA + stage * C::kABytes, &tmap_a, g * p.Cg_in + cb * BK, w0, h0, nimg, (uint16_t)s,
                                 (uint16_t)r, &full[stage]);
              load_b(stage, kb, g * p.Cg_out + n0);
            }
            if (++cb == cblocks) {
              cb = 0;
              if (++s == p.S) {
                s = 0;
                ++r;
              }
            }
          }
        }
      }
    } else {
      const int t = threadIdx.x;
      const uint32_t arow = (uint32_t)t * 128u;
      const uint32_t sw = (uint32_t)(t & 7);
      const int CC = p.Cg_in >> 3;
      const int hw = p.Ho * p.Wo;
      uint32_t gk = 0;
      for (int tile = cta0; tile < p.n_tiles; tile += ncta) {
        int m0, nt, g;
        decode_tile(p, tile, m0, nt, g);
        const int n0 = nt * BN;
        const int m = m0 + t;
        const bool mvalid = m < p.M;
        int nimg = 0, ho = 0, wo = 0;
        if (mvalid) {
          nimg = m / hw;
          const int rem = m - nimg * hw;
          ho = rem / p.Wo;
          wo = rem - ho * p.Wo;
        }
        const bf16* xb = p.x + (size_t)nimg * p.H * p.W * p.Cin + (size_t)g * p.Cg_in;
        const int hi0 = ho * p.stride - p.pad, wi0 = wo * p.stride - p.pad;
        int fr = 0, fs = 0, fc = 0;  // fast-path filter position
        for (int kb = 0; kb < p.nkb; ++kb, ++gk) {
          const int stage = gk % S;
          if (gk >= (uint32_t)S) mbar_wait(&empty[stage], ((gk / S) - 1) & 1);
          if (t == 0) {
            mbar_arrive_expect_tx(&full[stage], C::kBBytes);
            load_b(stage, kb, g * p.Cg_out + n0);
          }
          const uint32_t dst = sA + stage * C::kABytes + arow;
          if constexpr (AMODE == A_GATHER_FAST) {
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
          } else if constexpr (AMODE == A_GATHER_ROW) {
            // k-block = filter row r (= kb); the S*Cin <= 64 elements of one filter row are contiguous
            // in the NHWC input (Cin = 8 or 16); 16-byte chunk j = pixel (8j)/Cin, channels (8j)%Cin.
            const int hi = hi0 + kb;
            const bool rowok = mvalid && hi >= 0 && hi < p.H;
            const bf16* rowp = xb + (size_t)hi * p.W * p.Cin;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              const int pix = (j * 8) / p.Cin;
              const int wi = wi0 + pix;
              const bool ok = rowok && pix < p.S && wi >= 0 && wi < p.W;
              cp_async_16(dst + (((uint32_t)j ^ sw) << 4), ok ? rowp + (size_t)wi * p.Cin + ((j * 8) % p.Cin) : p.x,
                          ok ? 16u : 0u);
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
          if (gk >= (uint32_t)kLag) {
            cp_async_wait<kLag>();
            fence_proxy_async_smem();
            mbar_arrive(&full[(gk - kLag) % S]);
          }
        }
      }
      cp_async_wait<0>();
      fence_proxy_async_smem();
      for (uint32_t j = gk > (uint32_t)kLag ? gk - kLag : 0; j < gk; ++j) mbar_arrive(&full[j % S]);
    }
  } else if (warp == 4) {
    // ======================= MMA issuer (whole warp, one elected lane issues) =======================
    // (CTA pair: the leader issues for both; the peer's MMA warp only allocated the pair's TMEM)
    if (!CG2 || crank == 0) {
      constexpr uint32_t idesc = umma_idesc_bf16(CG2 ? 2 * BM : BM, BN);
      uint32_t gk = 0, it = 0;
      long long c_te = 0, c_dec = 0, c_hf = 0, c_iss = 0, tA = 0, tB = 0;
      const bool prof_mma = (p.dbg & 8) && lane == 0;
      if constexpr (BRES) mbar_wait(wres, 0);
      const long long t_start = prof_mma ? clock64() : 0;
      if constexpr (AMODE == A_HALO && BRES) {
        // Resident weights + halo (Cout = 64): tiles are issued in PAIRS, so the per-tile waits, tile
        // decode and commits sit between pairs, not between every 36 MMAs (measured: the tensor queue drains
        // during that gap; issue-bound at 2620 cycles per 1728-cycle tile).  The producer and the epilogue
        // still work per tile.
        for (int tile = cta0; tile < p.n_tiles; tile += 2 * ncta, it += 2) {
          const int tiles[2] = {tile, tile + ncta};
          const int nt2 = tiles[1] < p.n_tiles ? 2 : 1;
          uint32_t alo[2], accs[2], hbs[2];
          if (prof_mma) tA = clock64();
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            if (j < nt2) {
              const uint32_t itj = it + j;
              accs[j] = itj % NACC;
              hbs[j] = itj % HB;
              if (itj >= (uint32_t)NACC) mbar_wait(&tempty[accs[j]], ((itj / NACC) - 1) & 1);
              // one N tile: tile index = M-tile index; row-segment tiles start at halo column 0
              const int hoffj = p.hseg ? 0 : p.hofft[tiles[j] % p.mt_per_img];
              alo[j] = umma_desc_lo_sw128(sH + hbs[j] * halo_half_bytes(BN) + hoffj * 128);
            }
          }
          if (prof_mma) {
            tB = clock64();
            c_te += tB - tA;
            tA = tB;
          }
#pragma unroll
          for (int j = 0; j < 2; ++j)
            if (j < nt2) mbar_wait(&hfull[hbs[j]], ((it + j) / HB) & 1);
          tc_fence_after();
          if (prof_mma) {
            tB = clock64();
            c_hf += tB - tA;
            tA = tB;
          }
          const uint32_t blo = umma_desc_lo_sw128(sR);
#pragma unroll
          for (int j = 0; j < 2; ++j) {
            if (j < nt2) {
              const uint32_t tacc = tmem_base + accs[j] * BN;
#pragma unroll
              for (int kb = 0; kb < RKB; ++kb) {
                const uint32_t a = alo[j] + (uint32_t)p.koff[kb];
                const uint32_t b = blo + (uint32_t)(kb * (C::kBBytes >> 4));
                if constexpr (CG2) {  // pair MMA: both CTAs' halos (same position, two images), B halves
                  tc_mma_bf16_lo_warp_cg2(tacc, a, b, idesc, kb != 0 ? 1u : 0u);
                  tc_mma_bf16_lo_warp_cg2(tacc, a + 2, b + 2, idesc, 1u);
                  tc_mma_bf16_lo_warp_cg2(tacc, a + 4, b + 4, idesc, 1u);
                  tc_mma_bf16_lo_warp_cg2(tacc, a + 6, b + 6, idesc, 1u);
                } else {
                  tc_mma_bf16_lo_warp(tacc, a, b, idesc, kb != 0 ? 1u : 0u);
                  tc_mma_bf16_lo_warp(tacc, a + 2, b + 2, idesc, 1u);
                  tc_mma_bf16_lo_warp(tacc, a + 4, b + 4, idesc, 1u);
                  tc_mma_bf16_lo_warp(tacc, a + 6, b + 6, idesc, 1u);
                }
              }
              if constexpr (CG2) {
                tc_commit_cg2_warp(&tfull[accs[j]], (uint16_t)3);
                tc_commit_cg2_warp(&hempty[hbs[j]], (uint16_t)3);
              } else {
                tc_commit_warp(&tfull[accs[j]]);
                tc_commit_warp(&hempty[hbs[j]]);
              }
            }
          }
          if (prof_mma) c_iss += clock64() - tA;
        }
      }
      int hmod = 0, hstep = 0;  // A_HALO: tile index mod mt_per_img and its per-iteration step
      if constexpr (AMODE == A_HALO) {
        // (multicast pairs: M tile = 2 * pair tile + rank; CTA pair: pair tile = position, same for both)
        hmod = (p.mc && !CG2 ? 2 * cta0 + (int)crank : cta0) % p.mt_per_img;
        hstep = (p.mc && !CG2 ? 2 * ncta : ncta) % p.mt_per_img;
      }
      if constexpr (!(AMODE == A_HALO && BRES))
      for (int tile = cta0; tile < p.n_tiles; tile += ncta, ++it) {
        const uint32_t acc = it % NACC, use = it / NACC;
        if (prof_mma) tA = clock64();
        if (it >= (uint32_t)NACC) mbar_wait(&tempty[acc], (use - 1) & 1);
        if (prof_mma) {
          tB = clock64();
          c_te += tB - tA;
          tA = tB;
        }
        tc_fence_after();
        const uint32_t tacc = tmem_base + acc * BN;
        uint32_t hbase = 0;
        int hoff = 0;
        uint64_t dah = 0;  // A_HALO: descriptor of the tile's first output position in the halo buffer
        if constexpr (AMODE == A_HALO) {
          // one N tile: tile index = M tile index; (tile mod mt_per_img) advances by ncta mod mt_per_img
          if (!p.hseg) hoff = p.hofft[hmod];
          hmod += hstep;
          if (hmod >= p.mt_per_img) hmod -= p.mt_per_img;
          hbase = sH + (it % HB) * halo_half_bytes(BN);
          dah = umma_desc_k_sw128(hbase + hoff * 128);
          if (prof_mma) {
            tB = clock64();
            c_dec += tB - tA;
            tA = tB;
          }
          mbar_wait(&hfull[it % HB], (it / HB) & 1);
          if (prof_mma) {
            tB = clock64();
            c_hf += tB - tA;
            tA = tB;
          }
        }
        if constexpr (AMODE == A_HALO && !BRES) {
          // streamed weights: one ring wait and one commit per TWO k-blocks (8 MMAs), 32-bit descriptor
          // arithmetic -- measured (dbg 8 counters, res3 3x3): one wait + commit + 64-bit descriptors per
          // k-block made the issue loop ~350 cycles per 256 cycles of N = 128 MMAs
          constexpr int S2 = S / 2;
          const uint32_t alo = umma_desc_lo_sw128(hbase + hoff * 128);
          const uint32_t blo0 = umma_desc_lo_sw128(sB);
          for (int kb = 0; kb < p.nkb; kb += 2, ++gk) {
            const int stage = gk % S2;
            mbar_wait(&full[stage], (gk / S2) & 1);
            const uint32_t b = blo0 + (uint32_t)(2 * stage) * (uint32_t)(C::kBBytes >> 4);
            const uint32_t a = alo + (uint32_t)p.koff[kb];
            if constexpr (CG2) {  // one pair MMA per K step: M = 256 over both CTAs' halos
              tc_mma_bf16_lo_warp_cg2(tacc, a, b, idesc, kb != 0 ? 1u : 0u);
              tc_mma_bf16_lo_warp_cg2(tacc, a + 2, b + 2, idesc, 1u);
              tc_mma_bf16_lo_warp_cg2(tacc, a + 4, b + 4, idesc, 1u);
              tc_mma_bf16_lo_warp_cg2(tacc, a + 6, b + 6, idesc, 1u);
              if (kb + 1 < p.nkb) {
                const uint32_t a1 = alo + (uint32_t)p.koff[kb + 1];
                const uint32_t b1 = b + (uint32_t)(C::kBBytes >> 4);
                tc_mma_bf16_lo_warp_cg2(tacc, a1, b1, idesc, 1u);
                tc_mma_bf16_lo_warp_cg2(tacc, a1 + 2, b1 + 2, idesc, 1u);
                tc_mma_bf16_lo_warp_cg2(tacc, a1 + 4, b1 + 4, idesc, 1u);
                tc_mma_bf16_lo_warp_cg2(tacc, a1 + 6, b1 + 6, idesc, 1u);
              }
              tc_commit_cg2_warp(&empty[stage], (uint16_t)3);  // both CTAs' stages are free
              continue;
            }
            tc_mma_bf16_lo_warp(tacc, a, b, idesc, kb != 0 ? 1u : 0u);
            tc_mma_bf16_lo_warp(tacc, a + 2, b + 2, idesc, 1u);
            tc_mma_bf16_lo_warp(tacc, a + 4, b + 4, idesc, 1u);
            tc_mma_bf16_lo_warp(tacc, a + 6, b + 6, idesc, 1u);
            if (kb + 1 < p.nkb) {
              const uint32_t a1 = alo + (uint32_t)p.koff[kb + 1];
              const uint32_t b1 = b + (uint32_t)(C::kBBytes >> 4);
              tc_mma_bf16_lo_warp(tacc, a1, b1, idesc, 1u);
              tc_mma_bf16_lo_warp(tacc, a1 + 2, b1 + 2, idesc, 1u);
              tc_mma_bf16_lo_warp(tacc, a1 + 4, b1 + 4, idesc, 1u);
              tc_mma_bf16_lo_warp(tacc, a1 + 6, b1 + 6, idesc, 1u);
            }
            if (p.mc) tc_commit_mc_warp(&empty[stage], (uint16_t)3);
            else tc_commit_warp(&empty[stage]);
          }
          if constexpr (CG2) {  // both CTAs' accumulators full, both halos free
            tc_commit_cg2_warp(&tfull[acc], (uint16_t)3);
            tc_commit_cg2_warp(&hempty[it % HB], (uint16_t)3);
          } else {
            tc_commit_warp(&tfull[acc]);
            tc_commit_warp(&hempty[it % HB]);
          }
          continue;
        }
        auto kblock = [&](const int kb) {
          const int stage = gk % S;
          // (TMA completion / the producers' fence.proxy.async + arrive order the smem writes before the MMA)
          constexpr bool kRing = !(BRES && AMODE == A_HALO);  // halo + resident weights: no ring
          if constexpr (kRing) mbar_wait(&full[stage], (gk / S) & 1);
          const uint32_t a0 = sA + stage * C::kABytes;
          const uint32_t b0 = BRES ? sR + kb * C::kBBytes : sB + stage * C::kBBytes;
          if constexpr (AMODE == A_HALO) {
            // k-block kb = tap * cblocks + cb, tap = r * 3 + s: A = halo rows shifted by r * Wp + s
            // (a row-shifted start needs no descriptor base offset: the 128B swizzle follows the absolute
            // shared-memory address bits, exactly as the TMA wrote them; measured: base offset = shift % 8 fails)
            const uint64_t da = dah + (uint64_t)(uint32_t)p.koff[kb];
            const uint64_t db = umma_desc_k_sw128(b0);
            tc_mma_bf16_warp(tacc, da, db, idesc, kb != 0 ? 1u : 0u);
            tc_mma_bf16_warp(tacc, da + 2, db + 2, idesc, 1u);
            tc_mma_bf16_warp(tacc, da + 4, db + 4, idesc, 1u);
            tc_mma_bf16_warp(tacc, da + 6, db + 6, idesc, 1u);
          } else if constexpr (AMODE == A_IM2COL_C8) {
#pragma unroll
            for (int k = 0; k < BK / 16; ++k)
              tc_mma_bf16_warp(tacc, umma_desc_k_none(a0 + k * 4096, 2048, 128), umma_desc_k_sw128(b0 + k * 32),
                               idesc, (kb | k) != 0 ? 1u : 0u);
          } else if constexpr (CG2) {  // one pair MMA per K step over both CTAs' A tiles and B halves
            const uint32_t a = umma_desc_lo_sw128(a0), b = umma_desc_lo_sw128(b0);
            tc_mma_bf16_lo_warp_cg2(tacc, a, b, idesc, kb != 0 ? 1u : 0u);
            tc_mma_bf16_lo_warp_cg2(tacc, a + 2, b + 2, idesc, 1u);
            tc_mma_bf16_lo_warp_cg2(tacc, a + 4, b + 4, idesc, 1u);
            tc_mma_bf16_lo_warp_cg2(tacc, a + 6, b + 6, idesc, 1u);
          } else {
            const uint64_t da = umma_desc_k_sw128(a0), db = umma_desc_k_sw128(b0);
            // +32 bytes along K = +2 in the descriptors' address fields
            tc_mma_bf16_warp(tacc, da, db, idesc, kb != 0 ? 1u : 0u);
            tc_mma_bf16_warp(tacc, da + 2, db + 2, idesc, 1u);
            tc_mma_bf16_warp(tacc, da + 4, db + 4, idesc, 1u);
            tc_mma_bf16_warp(tacc, da + 6, db + 6, idesc, 1u);
          }
          if constexpr (kRing) {
            if constexpr (CG2) tc_commit_cg2_warp(&empty[stage], (uint16_t)3);  // both CTAs' stages are free
            else if (p.mc || p.amc) tc_commit_mc_warp(&empty[stage], (uint16_t)3);
            else tc_commit_warp(&empty[stage]);
          }
          ++gk;
        };
        {
          // unrolled by 4: a rolled loop costs a YIELD + branch-resolution stall per k-block (measured)
          int kb = 0;
          for (; kb + 4 <= p.nkb; kb += 4) {
            kblock(kb);
            kblock(kb + 1);
            kblock(kb + 2);
            kblock(kb + 3);
          }
          for (; kb < p.nkb; ++kb) kblock(kb);
        }
        if constexpr (CG2) tc_commit_cg2_warp(&tfull[acc], (uint16_t)3);  // both CTAs' accumulators
        else tc_commit_warp(&tfull[acc]);
        if constexpr (AMODE == A_HALO) tc_commit_warp(&hempty[it % HB]);  // halo free once these MMAs finish
      }
      if (prof_mma && p.dbg_buf) {
        unsigned long long* o = p.dbg_buf + blockIdx.x * 8;
        o[0] = clock64() - t_start;
        o[1] = c_te;
        o[2] = c_dec;
        o[3] = c_hf;
        o[4] = c_iss;
        o[5] = it;
      }
    }
  } else {
    // ================ epilogue (8 warps, one output row per lane) ================
    // SPLIT: warp group (warp - 5) / 4 takes every other tile and all of its columns; otherwise the two
    // warps of a TMEM lane quadrant split each tile's columns in halves.
    const int et = threadIdx.x - kEpiWarp0 * 32;
    const int q = warp & 3;  // TMEM lane quadrant this warp may access
    const int row = q * 32 + lane;
    const int grp = (warp - kEpiWarp0) >> 2;
    const int half = SPLIT ? 0 : grp;  // column half of the tile this warp owns
    const int gthreads = SPLIT ? kEpiThreads / 2 : kEpiThreads;
    const int gt = SPLIT ? (et & (kEpiThreads / 2 - 1)) : et;
    const int gbar = SPLIT ? 1 + grp : 1;
    const bool has_res = p.res != nullptr;
    int loaded0 = -1, loaded1 = -1;  // N offset whose scale / shift each smem buffer holds
    const int tstep = SPLIT ? 2 : 1;
    uint32_t it = SPLIT ? grp : 0;
    for (int tile = cta0 + (SPLIT ? grp * ncta : 0); tile < p.n_tiles;
         tile += tstep * ncta, it += tstep) {
      const uint32_t acc = it % NACC, use = it / NACC;
      int m0, nt, g;
      decode_tile(p, tile, m0, nt, g);
      const int n0 = nt * BN;
      const int ng0 = g * p.Cg_out + n0;
      const int nvalid_tile = min(BN, p.Cg_out - n0);
      const uint32_t ob = NB > 1 ? it % NB : 0;
      const uint32_t sOb = sO + ob * (uint32_t)(BM * BN * 2);
      // residual tile t -> staging buffer b (TMA, 64-column 128B-swizzled sub-tiles)
      auto issue_res = [&](int t, uint32_t b) {
        int tm0, tnt, tg;
        decode_tile(p, t, tm0, tnt, tg);
        const int tn0 = tnt * BN, tng0 = tg * p.Cg_out + tn0;
        const int nsub = (min(BN, p.Cg_out - tn0) + 63) / 64;
        mbar_arrive_expect_tx(&rbar[b], nsub * BM * 128);
        for (int st = 0; st < nsub; ++st)
          tma_load_2d(sO + b * (uint32_t)(BM * BN * 2) + st * BM * 128, &tmap_r, tng0 + st * 64, tm0, &rbar[b]);
      };
      if constexpr (TMA_EPI) {
        if (et == 0 && !sthr) {
          if (NB == 1) {
            bulk_wait_read0();  // the previous tile's stores no longer read the staging buffer
            if (has_res) issue_res(tile, 0);
          } else if (has_res) {
            if (NB == 2) {
              if (it == 0) issue_res(tile, 0);
              // prefetch the next tile's residual into the other buffer once its stores (tile it-1) read it
              const int next = tile + ncta;
              if (next < p.n_tiles) {
                bulk_wait_read0();
                issue_res(next, ob ^ 1);
              }
            } else if (it == 0) {
              // NB >= 3: the first NB - 1 residual tiles now; the rest at the end of each tile (below)
              for (int j = 0; j < NB - 1; ++j)
                if (tile + j * ncta < p.n_tiles) issue_res(tile + j * ncta, j);
            }
          } else {
            bulk_wait_read<NB - 1>();  // tile it-NB (same buffer) has been read by its stores
          }
        }
      }
      // this tile's scale / shift in smem: SPLIT one buffer per warp group, TMA epilogue one buffer, else
      // double-buffered by accumulator; reloaded only when the tile's N offset changes (resident-weight
      // launches and single-N-tile layers load it once)
      const int sb = SPLIT ? grp : (TMA_EPI ? 0 : (int)acc);
      float* ss = sbuf + sb * 2 * BN;
      const bool reload = (sb == 0 ? loaded0 : loaded1) != ng0;
      if (reload) {
        if (!TMA_EPI || sthr) named_bar_sync(gbar, gthreads);  // every warp of the group is done with the buffer
        for (int i = gt; i < 2 * BN; i += gthreads) {
          const int c = i < BN ? i : i - BN;
          ss[i] = c < nvalid_tile ? (i < BN ? p.scale[ng0 + c] : p.shift[ng0 + c]) : 0.f;
        }
        if (sb == 0) loaded0 = ng0;
        else loaded1 = ng0;
      }
      if ((TMA_EPI && !sthr) || reload) named_bar_sync(gbar, gthreads);
      int mo = m0 + row;
      bool rvalid = mo < p.M;
      if constexpr (AMODE == A_HALO) {  // padded-width position -> output pixel (columns >= Wo discarded)
        const int mt = m0 / BM;
        if (p.hseg) {
          const int rowi = mt / p.segs, seg = mt - rowi * p.segs;
          const int wo = seg * p.seg_w + row;
          mo = rowi * p.Wo + wo;
          rvalid = row < p.seg_w && wo < p.Wo && rowi < p.n_mt / p.segs;
        } else {
          const int nimg = mt / p.mt_per_img;
          const int pp = (mt - nimg * p.mt_per_img) * BM + row;
          const int ho = pp / p.Wp, wo = pp - ho * p.Wp;
          mo = (nimg * p.Ho + ho) * p.Wo + wo;
          rvalid = ho < p.Ho && wo < p.Wo && mo < p.M;  // (a multicast phantom tile lies past the last image)
        }
      }
      const size_t off = (size_t)(rvalid ? mo : 0) * p.Cout + ng0;
      constexpr int kChunks = SPLIT ? BN / 32 : BN / 64;  // 32-column chunks per warp
      const int cb0 = half * kChunks;
      uint4 rres[4] = {};
      if constexpr (TMA_EPI) {
        if (has_res) mbar_wait(&rbar[ob], (it / NB) & 1);
        else if (sthr && it >= (uint32_t)NB) mbar_wait(&sfree[ob], ((it / NB) - 1) & 1);  // its last store read it
      } else if (has_res && rvalid) {
#pragma unroll
        for (int j = 0; j < 4; ++j)
          rres[j] = (cb0 * 32 + j * 8 < nvalid_tile)
                        ? __ldg(reinterpret_cast<const uint4*>(p.res + off + cb0 * 32) + j)
                        : make_uint4(0, 0, 0, 0);
      }
      mbar_wait(&tfull[acc], use & 1);
      tc_fence_after();
      if ((p.dbg & 2) && !TMA_EPI) {
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          if constexpr (CG2) mbar_arrive_cluster(mapa_u32(smem_u32(&tempty[acc]), 0));  // the leader's barrier
          else mbar_arrive(&tempty[acc]);
        }
        continue;
      }
      const uint32_t taddr = tmem_base + acc * BN + ((uint32_t)(q * 32) << 16);
#pragma unroll 1
      for (int cb = cb0; cb < cb0 + kChunks; ++cb) {
        if (cb * 32 >= nvalid_tile) break;  // warp-uniform
        uint32_t v[32];
        tmem_ld_32x32b_x32(taddr + cb * 32, v);
        const float* scv = ss + cb * 32;
        const float* shv = ss + BN + cb * 32;
        if constexpr (TMA_EPI) {
          tc_wait_ld();
          const uint32_t sub = sOb + (cb >> 1) * BM * 128 + row * 128;
#pragma unroll
          for (int qq = 0; qq < 4; ++qq) {
            const uint32_t addr = sub + (((uint32_t)((cb & 1) * 4 + qq) ^ (uint32_t)(row & 7)) << 4);
            const uint4 r = has_res ? lds128(addr) : make_uint4(0, 0, 0, 0);
            uint4 o;
            epi_math(v + qq * 8, scv + qq * 8, shv + qq * 8, has_res, r, p.relu, o);
            sts128(addr, o);
          }
        } else {
          if constexpr (C::kStaged) {
            if (!has_res && !p.out_f32) {
              tc_wait_ld();
              const uint32_t stg = base + C::kStgOff + (uint32_t)(warp - kEpiWarp0) * 2048u;
#pragma unroll
              for (int qq = 0; qq < 4; ++qq) {
                uint4 o;
                epi_math(v + qq * 8, scv + qq * 8, shv + qq * 8, false, make_uint4(0, 0, 0, 0), p.relu, o);
                sts128(stg + lane * 64 + (((uint32_t)qq ^ (uint32_t)(lane & 3)) << 4), o);
              }
              __syncwarp();
              const int part = lane & 3;
#pragma unroll
              for (int i = 0; i < 4; ++i) {
                const int r = i * 8 + (lane >> 2);
                const int mo_r = __shfl_sync(0xffffffffu, mo, r);
                const int ok = __shfl_sync(0xffffffffu, rvalid ? 1 : 0, r);
                const uint4 val = lds128(stg + r * 64 + (((uint32_t)part ^ (uint32_t)(r & 3)) << 4));
                if (ok && cb * 32 + part * 8 < nvalid_tile)
                  *reinterpret_cast<uint4*>(p.y + (size_t)mo_r * p.Cout + ng0 + cb * 32 + part * 8) = val;
              }
              __syncwarp();  // the next chunk reuses the staging rows
              continue;
            }
          }
          uint4 cur[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) cur[j] = rres[j];
          if (has_res && rvalid && cb + 1 < cb0 + kChunks && (cb + 1) * 32 < nvalid_tile) {  // prefetch next chunk
#pragma unroll
            for (int j = 0; j < 4; ++j)
              rres[j] = ((cb + 1) * 32 + j * 8 < nvalid_tile)
                            ? __ldg(reinterpret_cast<const uint4*>(p.res + off + (cb + 1) * 32) + j)
                            : make_uint4(0, 0, 0, 0);
          }
          tc_wait_ld();
          if (rvalid) {
#pragma unroll
            for (int qq = 0; qq < 4; ++qq) {
              if (cb * 32 + qq * 8 < nvalid_tile) {
                if (p.out_f32) {
                  epi_math_f32(v + qq * 8, scv + qq * 8, shv + qq * 8, p.relu,
                               reinterpret_cast<float*>(p.y) + off + cb * 32 + qq * 8);
                } else {
                  uint4 o;
                  epi_math(v + qq * 8, scv + qq * 8, shv + qq * 8, has_res, cur[qq], p.relu, o);
                  *reinterpret_cast<uint4*>(p.y + off + cb * 32 + qq * 8) = o;
                }
              }
            }
          }
        }
      }
      // accumulator drained: the MMA warp may reuse it
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if constexpr (CG2) mbar_arrive_cluster(mapa_u32(smem_u32(&tempty[acc]), 0));  // the leader's barrier
        else mbar_arrive(&tempty[acc]);
      }
      if (TMA_EPI && sthr) {  // hand the staged tile to the store thread
        fence_proxy_async_smem();
        __syncwarp();
        if (lane == 0) mbar_arrive(&staged[ob]);
      } else if constexpr (TMA_EPI) {
        fence_proxy_async_smem();
        named_bar_sync(1, kEpiThreads);
        if (et == 0) {
          const int nsub = (nvalid_tile + 63) / 64;
          for (int st = 0; st < nsub; ++st) {
            if constexpr (AMODE == A_ROWVIEW)  // 3-D output map {C, Wo, rows}: q >= Wo clipped
              tma_store_3d(&tmap_y, ng0 + st * 64, (m0 / BM) % p.segs * BM, (m0 / BM) / p.segs, sOb + st * BM * 128);
            else
              tma_store_2d(&tmap_y, ng0 + st * 64, m0, sOb + st * BM * 128);
          }
          bulk_commit();
          if (NB >= 3 && has_res) {
            // buffer (it + NB - 1) % NB held tile it-1's output: once its stores have read it, prefetch
            // the residual of this CTA's tile it + NB - 1 there (latency hidden behind ~NB - 2 tiles)
            const int ahead = tile + (NB - 1) * ncta;
            if (ahead < p.n_tiles) {
              bulk_wait_read<1>();
              issue_res(ahead, (it + NB - 1) % NB);
            }
          }
        }
        if (p.tapf) {
          // Fused tap: scan the staged bf16 tile column-wise (kEpiThreads / BN threads per column split
          // the rows), keep one running max per (image, quadrant) met in this tile, and publish each
          // with one red.max.  Quadrants: R_0 = [0, ceil(H/2)), R_1 = [ceil(H/2), H) (reading R7).
          constexpr int kTpc = kEpiThreads / BN;  // threads per column
          const int col = et % BN, part = et / BN;
          if (col < nvalid_tile) {
            const int hw = p.Ho * p.Wo, h2 = (p.Ho + 1) >> 1, w2 = (p.Wo + 1) >> 1;
            const int r0 = part * (BM / kTpc), r1 = r0 + BM / kTpc;
            const int n_first = m0 / hw;
            float mx[16];
#pragma unroll
            for (int k = 0; k < 16; ++k) mx[k] = -1.f;
            int m = m0 + r0;
            int n = m / hw, rem = m - n * hw;
            int h = rem / p.Wo, w = rem - h * p.Wo;
            const uint32_t cbase = sOb + (col >> 6) * BM * 128 + (col & 7) * 2;
            const uint32_t cchunk = (uint32_t)((col & 63) >> 3);
            for (int r = r0; r < r1 && m < p.M; ++r, ++m) {
              const uint32_t a = cbase + r * 128 + ((cchunk ^ (uint32_t)(r & 7)) << 4);
              unsigned short bits;
              asm volatile("ld.shared.u16 %0, [%1];" : "=h"(bits) : "r"(a));
              const float v = __uint_as_float((uint32_t)bits << 16);
              const int k = (n - n_first) * 4 + (h >= h2 ? 2 : 0) + (w >= w2 ? 1 : 0);
#pragma unroll
              for (int kk = 0; kk < 16; ++kk)
                if (kk == k) mx[kk] = fmaxf(mx[kk], v);
              if (++w == p.Wo) {
                w = 0;
                if (++h == p.Ho) {
                  h = 0;
                  ++n;
                }
              }
            }
#pragma unroll
            for (int k = 0; k < 16; ++k)
              if (mx[k] >= 0.f)
                atomicMax(p.tapf + ((size_t)(n_first + (k >> 2)) * 4 + (k & 3)) * p.Cout + ng0 + col,
                          __float_as_uint(mx[k]));
          }
          named_bar_sync(1, kEpiThreads);  // the staging buffer may be refilled after this
        }
      }
    }
    if (TMA_EPI && !sthr && et == 0) bulk_wait0();
  }
  tc_fence_before();
  __syncthreads();
  if (p.mc || p.amc) cluster_sync_all();  // no multicast write or commit arrival may target an exited partner
  if (warp == 4) {
    if constexpr (CG2) tmem_dealloc_cg2(tmem_base, C::kTmemCols);
    else tmem_dealloc(tmem_base, C::kTmemCols);
  }
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

// 2-D bf16 tensor map [rows, cols] (cols contiguous), box {64, box_rows}, 128B swizzle
static void make_tmap(CUtensorMap* m, const void* ptr, uint64_t cols, uint64_t rows, uint32_t box_rows) {
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
  cuuint32_t box[2] = {(cuuint32_t)BK, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult rc = get_encode()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(ptr), dims, strides, box,
                             estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                             CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (rc != CUDA_SUCCESS) fail(5, "cuTensorMapEncodeTiled failed");
}

typedef CUresult (*encode_im2col_fn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                     const cuuint64_t*, const int*, const int*, cuuint32_t, cuuint32_t,
                                     const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                                     CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static encode_im2col_fn get_encode_im2col() {
  static encode_im2col_fn fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<encode_im2col_fn>(p);
  });
  if (!fn) fail(5, "cuTensorMapEncodeIm2col unavailable");
  return fn;
}

// im2col tensor map over an NHWC bf16 activation for a conv with filter R x S, stride, zero pad:
// the box is 128 output pixels (W fastest, then H, then N) x 64 channels, 128B-swizzled.
// Lower corner = -pad, upper corner = pad - (filter - 1) (output extent (W + 2 pad - S) / stride + 1).
static void make_tmap_im2col(CUtensorMap* m, const void* x, int N, int H, int W, int C, int R, int S, int stride,
                             int pad, int channels_per_pixel, bool swizzle128) {
  cuuint64_t dims[4] = {(cuuint64_t)C, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, (cuuint64_t)H * W * C * 2};
  int lower[2] = {-pad, -pad};
  int upper[2] = {pad - (S - 1), pad - (R - 1)};
  cuuint32_t estr[4] = {1, (cuuint32_t)stride, (cuuint32_t)stride, 1};
  CUresult rc = get_encode_im2col()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 4, const_cast<void*>(x), dims, strides,
                                    lower, upper, (cuuint32_t)channels_per_pixel, BM, estr,
                                    CU_TENSOR_MAP_INTERLEAVE_NONE,
                                    swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                                    CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                                    CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (rc != CUDA_SUCCESS) fail(5, "cuTensorMapEncodeIm2col failed");
  // same driver workaround as CUTLASS (cute copy_traits_sm90_im2col.hpp) for small tensors
  int drv = 0;
  cudaDriverGetVersion(&drv);
  if (drv <= 13010 && (uint64_t)N * H * W * C * 2 < 131072ull) reinterpret_cast<uint64_t*>(m)[1] &= ~(1ull << 21);
}

// VISTA_IM2COL=0 / VISTA_ROWVIEW=0 fall back to the cp.async gathers (A/B comparisons)
static const bool g_im2col_enabled = [] {
  const char* e = getenv("VISTA_IM2COL");
  return !(e && e[0] == '0');
}();
static const bool g_rowview_enabled = [] {
  const char* e = getenv("VISTA_ROWVIEW");
  return !(e && e[0] == '0');
}();
// VISTA_HALO=0 disables the halo mode (3x3 convs fall back to im2col boxes; A/B measurements)
static const bool g_hseg_enabled = [] {  // VISTA_HALO_SEG=0: wide rows fall back to im2col (A/B)
  const char* e = getenv("VISTA_HALO_SEG");
  return !(e && e[0] == '0');
}();
static const bool g_halo_enabled = [] {
  const char* e = getenv("VISTA_HALO");
  return !(e && e[0] == '0');
}();

// VISTA_CONV_DBG: measurement experiments (see ConvParams::dbg); never set in tests or the bench
static const int g_conv_dbg = [] {
  const char* e = getenv("VISTA_CONV_DBG");
  return e ? atoi(e) : 0;
}();
// weight multicast across CTA pairs for streamed-weight launches (ConvParams::mc); VISTA_MC=0 disables.
// Measured: 256-wide tiles gain (VGG conv3_x 1353 -> 1496, conv4_x 1454 -> 1598 TF/s, ResNet res5 3x3
// 1452 -> 1557); 64/128-wide im2col / TMA tiles lose (VGG conv1_2 437 -> 406, conv2_2 928 -> 841), so they
// stay unicast; the streamed-weight halo 3x3 (BN = 128), weight-ingest bound once its halo and weight
// producers were split, gains ~2 % (res3: 903 -> 923 TF/s, same run; VISTA_MC_HALO=0 disables).  Flags are read per launch
// (tests switch them within one process).
static bool env_flag(const char* name, bool dflt) {
  const char* e = getenv(name);
  return e && *e ? e[0] == '1' : dflt;
}
static bool use_mc(const ConvLayer& L, int amode, int rkb, const ConvParams& p) {
  return env_flag("VISTA_MC", true) && rkb == 0 && L.groups == 1 && p.n_mt >= 2 &&
         (L.BN == 256 || (L.BN == 128 && (amode == A_HALO || env_flag("VISTA_MC128", false)))) &&
         (amode == A_TMA || amode == A_IM2COL || amode == A_CAT || (amode == A_HALO && env_flag("VISTA_MC_HALO", true))) &&
         (int64_t)p.n_nt * ((p.n_mt + 1) / 2) >= num_sms() / 2;
}
// L2 prefetch distance of the resident-weight A_TMA launches in tiles (ConvParams::apf; VISTA_APF, 0 = off)
static const int g_apf = [] {
  const char* e = getenv("VISTA_APF");
  return e ? atoi(e) : 0;  // measured neutral with the store-thread epilogue: off by default
}();
// VISTA_WRES=0 disables the resident-weight launches (A/B measurements)
static const bool g_wres_enabled = [] {
  const char* e = getenv("VISTA_WRES");
  return !(e && e[0] == '0');
}();

// N-D bf16 tiled tensor map with 128B swizzle; returns the driver status (callers may fall back)
static CUresult encode_nd(CUtensorMap* m, const void* ptr, int rank, const cuuint64_t* dims,
                          const cuuint64_t* strides, const cuuint32_t* box) {
  cuuint32_t estr[5] = {1, 1, 1, 1, 1};
  return get_encode()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, (cuuint32_t)rank, const_cast<void*>(ptr), dims, strides,
                      box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
}

bool make_nd_tmap(CUtensorMap* m, const void* ptr, int rank, const uint64_t* dims, const uint64_t* strides,
                  const uint32_t* box, int swizzle_bytes) {
  cuuint64_t d[5], s[4];
  cuuint32_t b[5], estr[5] = {1, 1, 1, 1, 1};
  for (int i = 0; i < rank; ++i) {
    d[i] = dims[i];
    b[i] = box[i];
    if (i + 1 < rank) s[i] = strides[i];
  }
  return get_encode()(m, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, (cuuint32_t)rank, const_cast<void*>(ptr), d, s, b, estr,
                      CU_TENSOR_MAP_INTERLEAVE_NONE,
                      swizzle_bytes == 128 ? CU_TENSOR_MAP_SWIZZLE_128B
                                           : (swizzle_bytes == 32 ? CU_TENSOR_MAP_SWIZZLE_32B : CU_TENSOR_MAP_SWIZZLE_NONE),
                      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// [rows, cols] bf16 matrix, box {64, 128}, 128B swizzle (A operands / staged outputs of 128-row tiles)
bool make_plain_tmap(CUtensorMap* m, const void* ptr, int cols, int rows) {
  const cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows};
  const cuuint64_t strides[1] = {(cuuint64_t)cols * 2};
  const cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)BM};
  return encode_nd(m, ptr, 2, dims, strides, box) == CUDA_SUCCESS;
}

// overlapping 4-D row view of an NHWC input with C * S == 64 (A_ROWVIEW): element (k, q, h, n) =
// x[n, h, q + k / C, k % C] for q < Wo; box {64, 128, 1, 1}, 128B-swizzled (q >= Wo reads zeros)
// zero-padded copy for the padded row view: xp[n, h, w] = x[n, h - pad, w - pad] inside, 0 elsewhere;
// one 16-byte pixel (C = 8 bf16) per thread, xp rows Wpad pixels wide
__global__ void pad_rows_kernel(const uint4* __restrict__ x, uint4* __restrict__ xp, int64_t total, int H, int W,
                                int Hp, int Wpad, int pad) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < total; i += (int64_t)gridDim.x * blockDim.x) {
    const int w = (int)(i % Wpad);
    const int64_t t = i / Wpad;
    const int h = (int)(t % Hp);
    const int64_t n = t / Hp;
    const int hs = h - pad, ws = w - pad;
    xp[i] = (hs >= 0 && hs < H && ws >= 0 && ws < W) ? x[(n * H + hs) * W + ws] : make_uint4(0, 0, 0, 0);
  }
}

bool make_rowview_tmap(CUtensorMap* m, const void* x, int N, int H, int W, int C, int Wo) {
  const cuuint64_t dims[4] = {(cuuint64_t)BK, (cuuint64_t)Wo, (cuuint64_t)H, (cuuint64_t)N};
  const cuuint64_t strides[3] = {(cuuint64_t)C * 2, (cuuint64_t)W * C * 2, (cuuint64_t)H * W * C * 2};
  const cuuint32_t box[4] = {(cuuint32_t)BK, (cuuint32_t)BM, 1, 1};
  return encode_nd(m, x, 4, dims, strides, box) == CUDA_SUCCESS;
}

static int pick_bn(int Cg_out, int groups, int K) {
  // short-K layers are epilogue/HBM-bound: 128-wide tiles get a double-buffered output staging
  static const int k128 = getenv("VISTA_BN_K") ? atoi(getenv("VISTA_BN_K")) : 256;  // A/B of the threshold
  if (K <= k128 && Cg_out % 128 == 0) return 128;
  if (Cg_out % 256 == 0) return 256;
  if (Cg_out % 128 == 0) return 128;
  if (Cg_out % 64 == 0) return 64;
  if (groups == 1 && Cg_out < 128) return 128;  // one masked tile (e.g. AlexNet conv1, 96)
  return Cg_out > 128 ? 256 : 128;              // masked last tile (e.g. FC 1000)
}

void conv_layer_init(ConvLayer& L, const std::vector<uint16_t>& w, int Cin_real, const std::vector<float>& scale,
                     const std::vector<float>& shift) {
  if (L.Cin % L.groups || L.Cout % L.groups) fail(1, "conv: channels not divisible by groups");
  L.Cg_in = L.Cin / L.groups;
  L.Cg_out = L.Cout / L.groups;
  if (L.Cg_in % 8 || L.Cg_out % 8) fail(1, "conv: per-group channels must be multiples of 8");
  const int cg_real = Cin_real / L.groups;
  L.K = L.R * L.S * L.Cg_in;
  if (L.K_alg <= 0) L.K_alg = L.R * L.S * cg_real;
  // first layers (input padded to 8 or 16 channels, one filter row <= 64 elements): one k-block per
  // filter row (measured: for ResNet conv1 the row gather beats eight 2 KB im2col TMAs per k-block)
  L.row_mode = L.groups == 1 && (L.Cg_in == 8 || L.Cg_in == 16) && L.S * L.Cg_in <= BK &&
               L.R * 64 <= ((L.K + BK - 1) / BK * BK) * 2;
  // stride-1 unpadded conv whose filter row is exactly one 128-byte window: TMA row view
  L.rowview = L.row_mode && L.S * L.Cg_in == BK && L.stride == 1 && L.pad == 0;
  L.Kp = L.row_mode ? L.R * BK : (L.K + BK - 1) / BK * BK;
  L.BN = pick_bn(L.Cg_out, L.groups, L.K);
  // repack OHWI [Cout][R][S][cg_real] -> [Cout][Kp] with channel padding cg_real -> Cg_in and K padding
  std::vector<uint16_t> packed((size_t)L.Cout * L.Kp, 0);
  for (int o = 0; o < L.Cout; ++o)
    for (int r = 0; r < L.R; ++r)
      for (int s = 0; s < L.S; ++s)
        for (int c = 0; c < cg_real; ++c) {
          const size_t k = L.row_mode ? (size_t)r * BK + s * L.Cg_in + c : (size_t)(r * L.S + s) * L.Cg_in + c;
          packed[(size_t)o * L.Kp + k] = w[(((size_t)o * L.R + r) * L.S + s) * cg_real + c];
        }
  VCHECK(cudaMalloc(&L.w, packed.size() * 2));
  VCHECK(cudaMemcpy(L.w, packed.data(), packed.size() * 2, cudaMemcpyHostToDevice));
  VCHECK(cudaMalloc(&L.scale, L.Cout * sizeof(float)));
  VCHECK(cudaMalloc(&L.shift, L.Cout * sizeof(float)));
  VCHECK(cudaMemcpy(L.scale, scale.data(), L.Cout * sizeof(float), cudaMemcpyHostToDevice));
  VCHECK(cudaMemcpy(L.shift, shift.data(), L.Cout * sizeof(float), cudaMemcpyHostToDevice));
  make_tmap(&L.tmap_w, L.w, (uint64_t)L.Kp, (uint64_t)L.Cout, (uint32_t)L.BN);
  make_tmap(&L.tmap_w_half, L.w, (uint64_t)L.Kp, (uint64_t)L.Cout, (uint32_t)(L.BN / 2));
}

void conv_layer_free(ConvLayer& L) {
  if (L.w) cudaFree(L.w);
  if (L.scale) cudaFree(L.scale);
  if (L.shift) cudaFree(L.shift);
  L.w = nullptr;
  L.scale = L.shift = nullptr;
}

template <int BN, int AMODE, bool TE, int NB, int RKB = 0, bool CG2 = false>
static void launch_t(const ConvLayer& L, const CUtensorMap& ta, const CUtensorMap& ty, const CUtensorMap& tr,
                     const ConvParams& p, cudaStream_t st) {
  static_assert(NB >= 1 && NB <= 4, "staging buffers");
  auto kern = conv_tc_kernel<BN, AMODE, TE, NB, RKB, CG2>;
  constexpr int smem = Cfg<BN, TE, NB, AMODE == A_HALO, RKB, CG2>::kBytes;
  ensure_smem_attr((const void*)kern, smem);
  if (p.mc) {  // clusters of two CTAs walking pair tiles (see ConvParams::mc)
    if (RKB > 0 && !CG2) fail(1, "conv: multicast with resident weights");
    int pairs = std::min(p.n_tiles, num_sms() / 2);
    if (RKB > 0) {  // CTA pairs with resident weights: every pair keeps one N tile (pairs a multiple of n_nt)
      if (p.nkb > RKB || p.n_nt > pairs) fail(1, "conv: resident-weight pair launch misconfigured");
      pairs -= pairs % p.n_nt;
    }
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * pairs, 1, 1);
    cfg.blockDim = dim3(kThreads, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    VCHECK(cudaLaunchKernelEx(&cfg, kern, L.tmap_w_half, ta, ty, tr, p));
    LAUNCHED();
    return;
  }
  int grid = p.n_tiles < num_sms() ? p.n_tiles : num_sms();
  if (RKB > 0) {  // every CTA keeps one N tile: grid a multiple of the N-tile count (groups == 1)
    if (p.nkb > RKB || p.n_nt > grid) fail(1, "conv: resident-weight launch misconfigured");
    grid -= grid % p.n_nt;
  }
  if (p.amc) {  // A-multicast pairs: clusters of two CTAs with adjacent N tiles (n_nt even, so grid even)
    if (RKB == 0 || p.n_nt % 2) fail(1, "conv: A multicast needs resident weights and an even N-tile count");
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid, 1, 1);
    cfg.blockDim = dim3(kThreads, 1, 1);
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    VCHECK(cudaLaunchKernelEx(&cfg, kern, L.tmap_w, ta, ty, tr, p));
    LAUNCHED();
    return;
  }
  kern<<<grid, kThreads, smem, st>>>(L.tmap_w, ta, ty, tr, p);
  LAUNCHED();
}

template <int BN, bool TE, int NB>
static void launch_bn(const ConvLayer& L, int amode, const CUtensorMap& ta, const CUtensorMap& ty,
                      const CUtensorMap& tr, const ConvParams& p, cudaStream_t st, int rkb) {
  switch (amode) {
    case A_TMA:
      if constexpr (BN >= 128) {
        if (p.cg2 && rkb == 0) {
          launch_t<BN, A_TMA, TE, NB, 0, true>(L, ta, ty, tr, p, st);
          break;
        }
      }
      if constexpr (TE && BN <= 128) {
        if (rkb == 4) {
          if (p.cg2) launch_t<BN, A_TMA, TE, NB, 4, true>(L, ta, ty, tr, p, st);
          else launch_t<BN, A_TMA, TE, NB, 4>(L, ta, ty, tr, p, st);
          break;
        }
      }
      launch_t<BN, A_TMA, TE, NB>(L, ta, ty, tr, p, st);
      break;
    case A_CAT:
      if constexpr (BN >= 128) {
        if (p.cg2 && rkb == 0) {
          launch_t<BN, A_CAT, TE, NB, 0, true>(L, ta, ty, tr, p, st);
          break;
        }
      }
      if constexpr (TE && BN <= 128) {
        if (rkb == 4) {
          if (p.cg2) launch_t<BN, A_CAT, TE, NB, 4, true>(L, ta, ty, tr, p, st);
          else launch_t<BN, A_CAT, TE, NB, 4>(L, ta, ty, tr, p, st);
          break;
        }
      }
      launch_t<BN, A_CAT, TE, NB>(L, ta, ty, tr, p, st);
      break;
    case A_GATHER_FAST: launch_t<BN, A_GATHER_FAST, TE, NB>(L, ta, ty, tr, p, st); break;
    case A_GATHER_ROW: launch_t<BN, A_GATHER_ROW, TE, NB>(L, ta, ty, tr, p, st); break;
    case A_IM2COL:
      if constexpr (BN >= 128) {
        if (p.cg2) {
          launch_t<BN, A_IM2COL, TE, NB, 0, true>(L, ta, ty, tr, p, st);
          break;
        }
      }
      launch_t<BN, A_IM2COL, TE, NB>(L, ta, ty, tr, p, st);
      break;
    case A_IM2COL_C8: launch_t<BN, A_IM2COL_C8, TE, NB>(L, ta, ty, tr, p, st); break;
    case A_ROWVIEW:
      if constexpr (TE && BN <= 128) {
        if (rkb == 4) {
          launch_t<BN, A_ROWVIEW, TE, NB, 4>(L, ta, ty, tr, p, st);
          break;
        }
      }
      if constexpr (TE) launch_t<BN, A_ROWVIEW, TE, NB>(L, ta, ty, tr, p, st);
      else fail(1, "conv: row-view mode needs the TMA epilogue");
      break;
    case A_HALO:
      if constexpr (!TE && BN == 64) {
        if (rkb == 9) {
          if (p.cg2) launch_t<BN, A_HALO, TE, NB, 9, true>(L, ta, ty, tr, p, st);
          else launch_t<BN, A_HALO, TE, NB, 9>(L, ta, ty, tr, p, st);
          break;
        }
      }
      if constexpr (!TE && BN == 128) {
        if (p.cg2) {
          launch_t<BN, A_HALO, TE, NB, 0, true>(L, ta, ty, tr, p, st);
          break;
        }
      }
      if constexpr (!TE && BN <= 128) launch_t<BN, A_HALO, TE, NB>(L, ta, ty, tr, p, st);
      else fail(1, "conv: halo mode needs the register epilogue and BN <= 128");
      break;
    default: launch_t<BN, A_GATHER_GENERAL, TE, NB>(L, ta, ty, tr, p, st); break;
  }
}

// staging buffers of the TMA epilogue (VISTA_EPI_NB overrides for A/B measurements)
static const int g_epi_nb_env = [] {
  const char* e = getenv("VISTA_EPI_NB");
  return e ? atoi(e) : 0;
}();

bool conv_forward(const ConvLayer& L, const bf16* x, int N, int H, int W, const bf16* res, bf16* y,
                  cudaStream_t st, unsigned int* tapf) {
  ConvParams p{};
  p.x = x;
  p.y = y;
  p.res = res;
  p.tapf = nullptr;
  p.dbg = g_conv_dbg;
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
  p.segs = 1;
  const int64_t M = (int64_t)N * p.Ho * p.Wo;
  if (M <= 0) return tapf == nullptr;
  if (!res && !tapf && !g_conv_dbg && rowconv3x3_supported(L, H, W) && env_flag("VISTA_ROWCONV", true)) {
    rowconv3x3_forward(L, x, N, H, W, y, st);
    return true;
  }
  if (M > INT32_MAX - BM) fail(1, "conv: M too large for one launch");
  p.M = (int)M;
  p.relu = L.relu ? 1 : 0;
  p.n_mt = (p.M + BM - 1) / BM;
  p.n_nt = (L.Cg_out + L.BN - 1) / L.BN;
  const int64_t tiles = (int64_t)p.n_mt * p.n_nt * L.groups;
  if (tiles > INT32_MAX) fail(1, "conv: too many tiles");
  p.n_tiles = (int)tiles;
  // A operand path: a 1x1 stride-1 unpadded ungrouped conv (or FC) reads a plain [M, C] matrix -> TMA
  int amode;
  CUtensorMap ta, ty, tr;
  std::memset(&ta, 0, sizeof(ta));
  bool rowview = false;
  if (L.rowview && g_rowview_enabled && p.Wo <= BM && !res && L.R <= 8 && L.Cout % 8 == 0) {
    // overlapping 4-D view of the input: element (k, q, h, n) = x[n, h, q + k / Cin, k % Cin]
    const cuuint64_t odims[3] = {(cuuint64_t)L.Cout, (cuuint64_t)p.Wo, (cuuint64_t)N * p.Ho};
    const cuuint64_t ostr[2] = {(cuuint64_t)L.Cout * 2, (cuuint64_t)p.Wo * L.Cout * 2};
    const cuuint32_t obox[3] = {(cuuint32_t)BK, (cuuint32_t)BM, 1};
    if (make_rowview_tmap(&ta, x, N, H, W, L.Cin, p.Wo) &&
        encode_nd(&ty, y, 3, odims, ostr, obox) == CUDA_SUCCESS) {
      rowview = true;
      p.n_mt = N * p.Ho;  // one tile per output row; rows q >= Wo of a tile are padding
      p.M = p.n_mt * BM;
      p.n_tiles = p.n_mt * p.n_nt;
    }
  }
  // padded row view (first layers with Cin = 8 and padding, e.g. VGG16 conv1_1 3x3 pad 1 at 227 wide): the
  // cp.async gather is latency-bound there (one k-block group per 16 B per thread in flight, measured 1 TB/s),
  // so the input is first copied into a zero-padded buffer whose rows are wide enough for every 8-pixel
  // window, then read by the overlapping row view in ceil(Wo / 128) segments per output row
  bf16* xpad = nullptr;
  if (!rowview && L.row_mode && g_rowview_enabled && L.Cin == 8 && L.stride == 1 && L.pad > 0 && L.groups == 1 &&
      !res && L.R <= 8 && L.Cout % 8 == 0 && !tapf) {
    const int Hp = H + 2 * L.pad;
    const int Wpad = std::max(W + 2 * L.pad, p.Wo + BK / L.Cin - 1);
    const int64_t total = (int64_t)N * Hp * Wpad;
    if (cudaMallocAsync((void**)&xpad, (size_t)total * 16, st) == cudaSuccess) {
      pad_rows_kernel<<<num_sms() * 8, 256, 0, st>>>(reinterpret_cast<const uint4*>(x), reinterpret_cast<uint4*>(xpad),
                                                     total, H, W, Hp, Wpad, L.pad);
      LAUNCHED();
      const int segs = (p.Wo + BM - 1) / BM;
      const cuuint64_t odims[3] = {(cuuint64_t)L.Cout, (cuuint64_t)p.Wo, (cuuint64_t)N * p.Ho};
      const cuuint64_t ostr[2] = {(cuuint64_t)L.Cout * 2, (cuuint64_t)p.Wo * L.Cout * 2};
      const cuuint32_t obox[3] = {(cuuint32_t)BK, (cuuint32_t)BM, 1};
      if (make_rowview_tmap(&ta, xpad, N, Hp, Wpad, L.Cin, p.Wo) &&
          encode_nd(&ty, y, 3, odims, ostr, obox) == CUDA_SUCCESS) {
        rowview = true;
        p.segs = segs;
        p.n_mt = N * p.Ho * segs;
        p.M = p.n_mt * BM;
        p.n_tiles = p.n_mt * p.n_nt;
      }
    } else {
      cudaGetLastError();
      xpad = nullptr;
    }
  }
  // halo mode: 3x3 stride-1 pad-1 ungrouped, one N tile, both halo buffers fit the compile-time budget
  bool halo = false;
  if (!rowview && g_halo_enabled && L.R == 3 && L.S == 3 && L.stride == 1 && L.pad == 1 && L.groups == 1 &&
      L.Cin % BK == 0 && L.BN <= 128 && L.Cout == L.BN && !res && !tapf) {
    const int Wp = W + 2;
    const int hrows = (Wp - 1 + BM + 1 + 2 * Wp) / Wp + 1;  // padded rows touched by 128 positions + 2 rows + 2
    const int hsz = (hrows * Wp * 128 + 1023) & ~1023;
    const int cblocks = L.Cin / BK;
    const int half = L.BN == 64 ? 45056 : 61440;
    if (Wp <= 256 && hrows <= 256 && hsz * cblocks <= half && L.Kp / BK <= 36 &&
        (p.Ho * Wp + BM - 1) / BM <= 64) {
      const cuuint64_t dims[4] = {(cuuint64_t)L.Cin, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
      const cuuint64_t strides[3] = {(cuuint64_t)L.Cin * 2, (cuuint64_t)W * L.Cin * 2, (cuuint64_t)H * W * L.Cin * 2};
      const cuuint32_t box[4] = {(cuuint32_t)BK, (cuuint32_t)Wp, (cuuint32_t)hrows, 1};
      if (encode_nd(&ta, x, 4, dims, strides, box) == CUDA_SUCCESS) {
        halo = true;
        p.Wp = Wp;
        p.hrows = hrows;
        p.hsz = hsz;
        p.cblocks = cblocks;
        p.mt_per_img = (p.Ho * Wp + BM - 1) / BM;
        for (int r = 0; r < p.mt_per_img && r < 64; ++r) p.hofft[r] = (short)((r * BM) % Wp);
        for (int kb = 0; kb < p.nkb && kb < 36; ++kb) {
          const int tap = kb / cblocks, cb = kb % cblocks, r = tap / 3, sc = tap % 3;
          p.koff[kb] = ((r * Wp + sc) * 128 + cb * hsz) >> 4;
        }
        p.n_mt = N * p.mt_per_img;
        p.n_tiles = p.n_mt * p.n_nt;
      }
    } else if (g_hseg_enabled && L.Kp / BK <= 36) {
      // rows too wide for the padded-grid halo (VGG16 conv1_2 / conv2_1 at 227 / 113): row-segment tiles
      const int wb_max = half / (3 * 128 * cblocks);  // widest 3-row box of all channel blocks in one buffer
      const int nsegs = wb_max > 2 ? (p.Wo + wb_max - 3) / (wb_max - 2) : 0;
      const int seg_w = nsegs ? (p.Wo + nsegs - 1) / nsegs : 0;
      const int Wps = seg_w + 2, hszs = (3 * Wps * 128 + 1023) & ~1023;
      if (nsegs && seg_w >= 96 && seg_w <= BM && hszs * cblocks <= half) {
        const cuuint64_t dims[4] = {(cuuint64_t)L.Cin, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
        const cuuint64_t strides[3] = {(cuuint64_t)L.Cin * 2, (cuuint64_t)W * L.Cin * 2,
                                       (cuuint64_t)H * W * L.Cin * 2};
        const cuuint32_t box[4] = {(cuuint32_t)BK, (cuuint32_t)Wps, 3, 1};
        if (encode_nd(&ta, x, 4, dims, strides, box) == CUDA_SUCCESS) {
          halo = true;
          p.hseg = 1;
          p.segs = nsegs;
          p.seg_w = seg_w;
          p.Wp = Wps;
          p.hrows = 3;
          p.hsz = hszs;
          p.cblocks = cblocks;
          p.mt_per_img = p.Ho * nsegs;
          for (int kb = 0; kb < p.nkb && kb < 36; ++kb) {
            const int tap = kb / cblocks, cb = kb % cblocks, r = tap / 3, sc = tap % 3;
            p.koff[kb] = ((r * Wps + sc) * 128 + cb * hszs) >> 4;
          }
          p.n_mt = N * p.Ho * nsegs;
          p.n_tiles = p.n_mt * p.n_nt;
        }
      }
    }
  }
  if (halo) {
    amode = A_HALO;
  } else if (rowview) {
    amode = A_ROWVIEW;
  } else if (L.R == 1 && L.S == 1 && L.stride == 1 && L.pad == 0 && L.groups == 1 && L.Cin % BK == 0) {
    amode = A_TMA;
    make_tmap(&ta, x, (uint64_t)L.Cin, (uint64_t)M, BM);
  } else {
    amode = L.row_mode ? A_GATHER_ROW : ((L.Cg_in % BK) == 0 ? A_GATHER_FAST : A_GATHER_GENERAL);
    ta = L.tmap_w;  // unused
    // channel blocks of 64 per filter tap: the TMA unit gathers the implicit im2col rows
    if (amode == A_GATHER_FAST && g_im2col_enabled) {
      amode = A_IM2COL;
      make_tmap_im2col(&ta, x, N, H, W, L.Cin, L.R, L.S, L.stride, L.pad, BK, true);
    } else if (g_im2col_enabled && !L.row_mode && L.groups == 1 && L.Cg_in == 8) {
      amode = A_IM2COL_C8;
      make_tmap_im2col(&ta, x, N, H, W, L.Cin, L.R, L.S, L.stride, L.pad, 8, false);
    }
  }
  // epilogue: staged in smem and written by TMA (residual read by TMA) unless a group's last N tile
  // would spill into the next group's channels
  // (long-K layers keep the register epilogue: it is hidden behind the mainloop and frees the staging
  // smem for a deeper k-block ring)
  static const int tma_epi_nkb = getenv("VISTA_TMAEPI_NKB") ? atoi(getenv("VISTA_TMAEPI_NKB")) : 12;  // A/B (measured: K = 768 projection unit -0.25 ms with the TMA epilogue, K = 1024 +0.6 ms)
  const bool tma_epi =
      !halo && (rowview || ((L.groups == 1 || L.Cg_out % L.BN == 0) && L.Cout % 8 == 0 && p.nkb <= tma_epi_nkb));
  // the fused tap needs the staged tile, non-negative outputs (ReLU) and <= 4 images per 128-row tile
  const bool fuse_tap = tapf && tma_epi && !rowview && L.relu && p.Ho * p.Wo >= 43;
  if (fuse_tap) p.tapf = tapf;
  if (rowview) {
    tr = ty;  // output map built above; no residual
  } else if (tma_epi) {
    make_tmap(&ty, y, (uint64_t)L.Cout, (uint64_t)M, BM);
    if (res) make_tmap(&tr, res, (uint64_t)L.Cout, (uint64_t)M, BM);
    else tr = ty;
  } else {
    ty = tr = L.tmap_w;  // unused
  }
  const double flops = 2.0 * (double)M * L.Cout * L.K_alg;  // algorithmic (unpadded) MACs x 2
  // algorithmic bytes: the input once (a strided 1x1 conv reads only its sampled pixels: whole 16-byte-aligned
  // channel runs, so no other line is touched), the output, the residual, the weights
  const double in_px = (L.R == 1 && L.S == 1 && L.pad == 0) ? (double)M : (double)N * H * W;
  const double bytes = 2.0 * (in_px * L.Cin + (double)M * L.Cout * (res ? 2 : 1) + (double)L.Cout * L.Kp);
  // resident weights (see Cfg): 3x3 halo convs with Cout = 64 (9 k-blocks of 8 KB) and 1x1 TMA convs with
  // K <= 256 and BN <= 128 (<= 4 k-blocks); one N tile per CTA needs groups == 1 and n_nt <= the grid
  int rkb = 0;
  if (g_wres_enabled && L.groups == 1 && p.n_nt <= num_sms() && p.n_tiles >= num_sms()) {
    if (amode == A_HALO && L.BN == 64 && p.nkb == 9) rkb = 9;
    else if ((amode == A_TMA || amode == A_ROWVIEW) && tma_epi && L.BN <= 128 && p.nkb <= 4) rkb = 4;
  }
  // CTA pairs for the resident-weight 1x1 TMA-epilogue convs: two adjacent M tiles of one N tile per pair, each
  // CTA holding half of the N tile's weights (the freed shared memory deepens the A ring)
  const bool cg2_res = rkb == 4 && amode == A_TMA && !fuse_tap && !p.dbg && env_flag("VISTA_CG2_RES", true) &&
                       (int64_t)p.n_nt * ((p.n_mt + 1) / 2) >= num_sms() / 2 && p.n_nt <= num_sms() / 2;
  if (cg2_res) {
    p.mc = 1;
    p.cg2 = 2;
    p.n_tiles = p.n_nt * ((p.n_mt + 1) / 2);
  }
  if (rkb == 4 && amode == A_TMA && L.groups == 1 && !cg2_res) p.apf = g_apf;
  // CTA pairs for the resident-weight halo 3x3 (res2, Cout = 64): pair tile = one position in two consecutive
  // images (as the streamed-weight halo pairs), half of the 72 KB of resident weights per CTA
  if (rkb == 9 && !p.hseg && p.n_nt == 1 && !p.dbg && env_flag("VISTA_CG2_HALO64", true) &&
      (int64_t)((N + 1) / 2) * p.mt_per_img >= num_sms() / 2) {
    p.mc = 1;
    p.cg2 = 1;
    p.n_tiles = ((N + 1) / 2) * p.mt_per_img;
  }
  p.no_sthr = env_flag("VISTA_STORE_THR", true) ? 0 : 1;
  if (rkb == 4 && amode == A_TMA && !cg2_res && p.n_nt % 2 == 0 && !fuse_tap && !p.dbg && env_flag("VISTA_AMC", false)) {
    p.amc = 1;  // A multicast across the pair's two N tiles (see ConvParams::amc): half-row A boxes
    make_tmap(&ta, x, (uint64_t)L.Cin, (uint64_t)M, BM / 2);
  }
  if (!fuse_tap && use_mc(L, amode, rkb, p)) {
    p.mc = 1;
    p.n_tiles = p.n_nt * ((p.n_mt + 1) / 2);
    // CTA-pair MMA for the streamed-weight padded-grid halo convs (res3 3x3): pair tile = one position in
    // two consecutive images (VISTA_CG2=0 keeps the weight-multicast pairs)
    if (env_flag("VISTA_CG2", true) && amode == A_HALO && L.BN == 128 && rkb == 0 && !p.hseg && p.n_nt == 1 && !p.dbg) {
      p.cg2 = 1;
      p.n_tiles = ((N + 1) / 2) * p.mt_per_img;
    }
    // CTA-pair MMA (M = 256, N = 256) for the streamed-weight im2col / plain-TMA convs with the register
    // epilogue: the multicast pair tile (two adjacent M tiles), each CTA loading its A tile and half of B
    if (env_flag("VISTA_CG2", true) && (amode == A_IM2COL || amode == A_TMA) && L.BN >= 128 && !p.dbg &&
        !p.tapf)
      p.cg2 = 2;
  }
  unsigned long long* dbgb = nullptr;
  if (p.dbg & 8) {
    VCHECK(cudaMalloc(&dbgb, 148 * 8 * 8));
    VCHECK(cudaMemset(dbgb, 0, 148 * 8 * 8));
    p.dbg_buf = dbgb;
  }
  prof_begin(st);
  int nb = 1;
  if (tma_epi) {
    if (L.BN == 256) {
      launch_bn<256, true, 1>(L, amode, ta, ty, tr, p, st, rkb);
    } else if (L.BN == 128) {
      nb = g_epi_nb_env == 2 ? 2 : (g_epi_nb_env == 4 ? 4 : 3);
      if (nb == 2) launch_bn<128, true, 2>(L, amode, ta, ty, tr, p, st, rkb);
      else if (nb == 4) launch_bn<128, true, 4>(L, amode, ta, ty, tr, p, st, rkb);
      else launch_bn<128, true, 3>(L, amode, ta, ty, tr, p, st, rkb);
    } else {
      nb = g_epi_nb_env == 2 ? 2 : 4;
      if (nb == 2) launch_bn<64, true, 2>(L, amode, ta, ty, tr, p, st, rkb);
      else launch_bn<64, true, 4>(L, amode, ta, ty, tr, p, st, rkb);
    }
  } else {
    if (L.BN == 256) launch_bn<256, false, 1>(L, amode, ta, ty, tr, p, st, rkb);
    else if (L.BN == 128) launch_bn<128, false, 1>(L, amode, ta, ty, tr, p, st, rkb);
    else launch_bn<64, false, 1>(L, amode, ta, ty, tr, p, st, rkb);
  }
  if (xpad) VCHECK(cudaFreeAsync(xpad, st));  // stream-ordered: after the conv has read it
  char label[160] = {0};
  if (prof_labels())
    snprintf(label, sizeof(label), "conv R%d S%d s%d g%d Cin%d Cout%d HxW%dx%d M%d K%d BN%d amode%d epi%d nb%d rkb%d mc%d segs%d tiles%d%s",
             L.R, L.S, L.stride, L.groups, L.Cin, L.Cout, H, W, p.M, L.K, L.BN, amode, tma_epi ? 1 : 0, nb, rkb, p.mc,
             p.segs, p.n_tiles, res ? " res" : "");
  prof_end(st, 0, flops, bytes, label);
  if (dbgb) {
    unsigned long long h[148 * 8];
    VCHECK(cudaMemcpy(h, dbgb, sizeof(h), cudaMemcpyDeviceToHost));
    double a[6] = {0, 0, 0, 0, 0, 0};
    int n = 0;
    for (int b = 0; b < 148; ++b)
      if (h[b * 8 + 5]) {
        for (int k = 0; k < 6; ++k) a[k] += (double)h[b * 8 + k];
        ++n;
      }
    if (n)
      fprintf(stderr, "[conv dbg] CTAs %d tiles/CTA %.1f cycles/tile: total %.0f tempty %.0f decode %.0f hfull %.0f issue %.0f\n",
              n, a[5] / n, a[0] / a[5], a[1] / a[5], a[2] / a[5], a[3] / a[5], a[4] / a[5]);
    cudaFree(dbgb);
  }
  return tapf == nullptr || fuse_tap;
}

// Closing 1x1 conv of a projection unit with the projection folded into its K loop (A_CAT):
//   y = ReLU(s_c * ([b | x_s] . [Wc | Wp']^T) + t),  Wp' = bf16(Wp * s_p / s_c), t = t_c + t_p
// = ReLU(BN_c(b * Wc) + BN_p(x_s * Wp)) up to the bf16 rounding of the rescaled projection weights
// (reading R31).  b: [N, Ho, Wo, Kb] (Kb = L.Cin - Cx), x: [N, Hx, Wx, Cx], x_s = x sampled at stride
// `stride` (Ho = ceil(Hx / stride)).  The projection output (4 * mid channels per pixel) is never written
// to HBM nor read back as the residual.
void conv_cat_forward(const ConvLayer& L, int Cx, const bf16* b, const bf16* x, int N, int Hx, int Wx, int stride,
                      bf16* y, cudaStream_t st) {
  const int Kb = L.Cin - Cx;
  if (L.R != 1 || L.S != 1 || L.groups != 1 || Kb <= 0 || Kb % BK || Cx % BK || L.Kp != L.Cin)
    fail(1, "conv_cat: unsupported layer");
  ConvParams p{};
  p.x = b;
  p.y = y;
  p.res = nullptr;
  p.dbg = g_conv_dbg;
  p.scale = L.scale;
  p.shift = L.shift;
  p.H = p.Ho = conv_out_dim(Hx, 1, stride, 0);
  p.W = p.Wo = conv_out_dim(Wx, 1, stride, 0);
  p.Cin = L.Cin;
  p.Cout = L.Cout;
  p.R = p.S = 1;
  p.stride = stride;
  p.Cg_in = L.Cin;
  p.Cg_out = L.Cout;
  p.K = L.K;
  p.nkb = L.Kp / BK;
  p.nkb1 = Kb / BK;
  p.cat_im2col = stride != 1;
  p.no_sthr = env_flag("VISTA_STORE_THR", true) ? 0 : 1;
  const int64_t M = (int64_t)N * p.Ho * p.Wo;
  if (M <= 0) return;
  if (M > INT32_MAX - BM) fail(1, "conv_cat: M too large for one launch");
  p.M = (int)M;
  p.relu = L.relu ? 1 : 0;
  p.n_mt = (p.M + BM - 1) / BM;
  p.n_nt = (L.Cout + L.BN - 1) / L.BN;
  p.n_tiles = p.n_mt * p.n_nt;
  CUtensorMap ta, ty, tr;
  std::memset(&ty, 0, sizeof(ty));
  make_tmap(&ta, b, (uint64_t)Kb, (uint64_t)M, BM);
  if (stride != 1) make_tmap_im2col(&tr, x, N, Hx, Wx, Cx, 1, 1, stride, 0, BK, true);
  else make_tmap(&tr, x, (uint64_t)Cx, (uint64_t)M, BM);
  static const int tma_epi_nkb = getenv("VISTA_TMAEPI_NKB") ? atoi(getenv("VISTA_TMAEPI_NKB")) : 12;  // A/B (measured: K = 768 projection unit -0.25 ms with the TMA epilogue, K = 1024 +0.6 ms)
  const bool tma_epi = L.Cout % 8 == 0 && p.nkb <= tma_epi_nkb;
  if (tma_epi) make_tmap(&ty, y, (uint64_t)L.Cout, (uint64_t)M, BM);
  else ty = L.tmap_w;  // unused
  const int rkb = (g_wres_enabled && tma_epi && L.BN <= 128 && p.nkb <= 4 && p.n_nt <= num_sms() &&
                   p.n_tiles >= num_sms()) ? 4 : 0;
  const bool cg2_res = rkb == 4 && stride == 1 && !p.dbg && env_flag("VISTA_CG2_RES", true) &&
                       (int64_t)p.n_nt * ((p.n_mt + 1) / 2) >= num_sms() / 2 && p.n_nt <= num_sms() / 2;
  if (cg2_res) {  // CTA pairs with half of the resident weights each (see conv_forward)
    p.mc = 1;
    p.cg2 = 2;
    p.n_tiles = p.n_nt * ((p.n_mt + 1) / 2);
  }
  if (rkb == 4 && stride == 1 && !cg2_res && p.n_nt % 2 == 0 && !p.dbg && env_flag("VISTA_AMC", false)) {
    p.amc = 1;  // A multicast across the pair's two N tiles (see ConvParams::amc): half-row A boxes
    make_tmap(&ta, b, (uint64_t)Kb, (uint64_t)M, BM / 2);
    make_tmap(&tr, x, (uint64_t)Cx, (uint64_t)M, BM / 2);
  }
  if (use_mc(L, A_CAT, rkb, p)) {
    p.mc = 1;
    p.n_tiles = p.n_nt * ((p.n_mt + 1) / 2);
    if (env_flag("VISTA_CG2", true) && L.BN >= 128 && !p.dbg) p.cg2 = 2;  // CTA-pair MMA, see conv_forward
  }
  const double flops = 2.0 * (double)M * L.Cout * L.K_alg;
  const double bytes = 2.0 * ((double)M * (Kb + Cx + L.Cout) + (double)L.Cout * L.Kp);
  prof_begin(st);
  if (tma_epi) {
    if (L.BN == 256) launch_bn<256, true, 1>(L, A_CAT, ta, ty, tr, p, st, rkb);
    else if (L.BN == 128) launch_bn<128, true, 3>(L, A_CAT, ta, ty, tr, p, st, rkb);
    else launch_bn<64, true, 4>(L, A_CAT, ta, ty, tr, p, st, rkb);
  } else {
    if (L.BN == 256) launch_bn<256, false, 1>(L, A_CAT, ta, ty, tr, p, st, 0);
    else if (L.BN == 128) launch_bn<128, false, 1>(L, A_CAT, ta, ty, tr, p, st, 0);
    else launch_bn<64, false, 1>(L, A_CAT, ta, ty, tr, p, st, 0);
  }
  char label[160] = {0};
  if (prof_labels())
    snprintf(label, sizeof(label), "conv_cat c+proj s%d Cb%d Cx%d Cout%d HxW%dx%d K%d BN%d epi%d rkb%d mc%d", stride,
             Kb, Cx, L.Cout, p.Ho, p.Wo, L.K, L.BN, tma_epi ? 1 : 0, rkb, p.mc);
  prof_end(st, 0, flops, bytes, label);
}

// Plain "TN" GEMM on the same kernel (A_TMA mode, register epilogue):
//   y[m, n] = act(scale[n] * sum_k A[m, k] B[n, k] + shift[n]),  m < M, n < N, k < K
// A: bf16 [M rows, lda], B: bf16 [N rows, ldb] (both K-major, rows 16-byte aligned); columns k >= K
// (and B rows >= N) are read as zeros by the TMA, so K needs no padding.  y: [M, N] row-major, bf16 or
// fp32 (out_f32).  scale / shift: fp32 device [N] (per output column).
void gemm_tn(const bf16* A, int64_t M, int K, int lda, const bf16* B, int N, int ldb, const float* scale,
             const float* shift, bool relu, void* y, bool out_f32, cudaStream_t st, int prof_cls) {
  if (M <= 0 || N <= 0) return;
  if (K <= 0 || (lda % 8) || (ldb % 8) || (N % 8)) fail(1, "gemm_tn: K > 0, lda, ldb, N multiples of 8 required");
  if (M > INT32_MAX - BM) fail(1, "gemm_tn: M too large");
  ConvLayer L;
  L.Cin = L.Cg_in = L.K = K;
  L.Cout = L.Cg_out = N;
  L.Kp = (K + BK - 1) / BK * BK;
  L.K_alg = K;
  L.BN = N % 256 == 0 ? 256 : (N % 128 == 0 ? 128 : (N >= 256 ? 256 : 128));
  {
    const cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)N};
    const cuuint64_t strides[1] = {(cuuint64_t)ldb * 2};
    const cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)L.BN};
    if (encode_nd(&L.tmap_w, B, 2, dims, strides, box) != CUDA_SUCCESS) fail(5, "gemm_tn: B tensor map");
  }
  CUtensorMap ta;
  {
    const cuuint64_t dims[2] = {(cuuint64_t)K, (cuuint64_t)M};
    const cuuint64_t strides[1] = {(cuuint64_t)lda * 2};
    const cuuint32_t box[2] = {(cuuint32_t)BK, (cuuint32_t)BM};
    if (encode_nd(&ta, A, 2, dims, strides, box) != CUDA_SUCCESS) fail(5, "gemm_tn: A tensor map");
  }
  ConvParams p{};
  p.x = A;
  p.y = reinterpret_cast<bf16*>(y);
  p.scale = scale;
  p.shift = shift;
  p.H = p.W = p.Ho = p.Wo = 1;
  p.Cin = K;
  p.Cout = N;
  p.R = p.S = p.stride = 1;
  p.Cg_in = K;
  p.Cg_out = N;
  p.K = K;
  p.nkb = L.Kp / BK;
  p.M = (int)M;
  p.relu = relu ? 1 : 0;
  p.out_f32 = out_f32 ? 1 : 0;
  p.n_mt = (p.M + BM - 1) / BM;
  p.n_nt = (N + L.BN - 1) / L.BN;
  p.n_tiles = p.n_mt * p.n_nt;
  prof_begin(st);
  if (L.BN == 256) launch_bn<256, false, 1>(L, A_TMA, ta, ta, ta, p, st, 0);
  else launch_bn<128, false, 1>(L, A_TMA, ta, ta, ta, p, st, 0);
  char label[96] = {0};
  if (prof_labels()) snprintf(label, sizeof(label), "gemm_tn M%lld N%d K%d%s", (long long)M, N, K, out_f32 ? " f32" : "");
  prof_end(st, prof_cls, 2.0 * (double)M * N * K,
           2.0 * ((double)M * K + (double)N * K) + (double)M * N * (out_f32 ? 4 : 2), label);
}

}  // namespace vista
