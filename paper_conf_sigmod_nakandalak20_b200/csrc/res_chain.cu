// res_chain.cu — two chained 1x1 convolutions of consecutive ResNet bottleneck units in ONE kernel:
//   out    = ReLU(BN_c(b * Wc) + x)        (unit u's closing 1x1 conv + residual, Cout = 4 * MID)
//   a_next = ReLU(BN_a(out * Wa))          (unit u+1's opening 1x1 conv, Cout = MID)
// SURVEY.md §8a S1 (partial inference f^ as a chain of TensorOps, Def 3.7).
// Unfused, the a-conv re-reads `out` (4 * MID channels per pixel) from HBM right after the c-conv wrote
// it; here every 128-pixel x 128-channel chunk of `out` is staged in shared memory for its TMA store
// anyway (128B-swizzled, K-major: exactly the A-operand layout of tcgen05.mma), so the a-conv's MMAs read
// it from there and `out` is read zero times instead of once (-29 % HBM bytes for the pair at MID = 64).
//
// Per 128-pixel tile: c-chunks j = 0 .. 4*MID/128 - 1 (128 output channels each, two TMEM accumulators
// alternate) and the a-accumulator (MID columns) that sums over the chunks.  MMA issue order
// c(0), c(1), a(0), c(2), a(1), ... lets c(j+1) run while the epilogue finishes chunk j.
// Both GEMMs use the same instruction shapes and k order as conv_tc.cu's unfused launches (N = 128 for
// c, N = MID for a, K-steps of 16 in ascending k), and the same epilogue arithmetic, so the result is
// bit-identical to conv_forward(c) followed by conv_forward(a) (tested).
#include <cstring>

#include "internal.h"
#include "ptx.cuh"

namespace vista {

namespace {

constexpr int BMr = 128, BKr = 64;
// warps: 0 producer, 1 MMA issuer, 2..9 epilogue, 10 store warp (lane 0: the out / a_next TMA stores and the
// staging-buffer releases, so the epilogue warps never wait on store completion or on one another)
constexpr int kEpiW0 = 2, kEpiWn = 8, kEpiT = kEpiWn * 32, kStoreW = kEpiW0 + kEpiWn, kThr = (kStoreW + 1) * 32;

// V = 0: b tile double-buffered; V = 1: b single-buffered, the freed 16/32 KB spent on one more
// weight stage (MID = 64) or one more out/residual staging buffer (MID = 128: residual chunks in flight).
// MID = 256 (ResNet res4, Cout 1024): the closing conv alone (no a_next: a 1024-wide c accumulator and the
// a GEMM's 512 KB of weights per tile do not fit beside it), b single-buffered (64 KB); V = 0: two staging
// buffers and five weight stages, V = 1: three and three.
// CG2 (CTA pairs): each CTA holds half of every weight k-block, so weight stages are 8 KB and the space goes to a
// fourth out/residual staging buffer (more residual chunks in flight) and, at MID = 64, a fifth weight stage.
template <int MID, int V = 0, bool CG2 = false>
struct RC {
  static constexpr int NCH = 4 * MID / 128;       // c chunks of 128 channels
  static constexpr int KBC = MID / BKr;           // k-blocks of the c GEMM
  // (CG2, MID = 128: b single-buffered; V = 1 four staging buffers and three weight stages, V = 0 three and seven)
  static constexpr int NBB = (V || MID == 256 || (CG2 && MID == 128)) ? 1 : 2;  // b tile buffers
  static constexpr int NB = CG2 ? (MID == 128 ? (V ? 4 : 3) : 4)
                                : (MID == 64 ? 3 : (MID == 256 ? (V ? 3 : 2) : (V ? 3 : 2)));  // out/residual staging
  static constexpr int WS = CG2 ? (MID == 64 ? 5 : (V ? 3 : 7))
                                : (MID == 64 ? (V ? 5 : 4) : (MID == 256 ? (V ? 3 : 5) : 3));  // weight stages
  static constexpr int kWst = CG2 ? 8192 : 16384;  // weight stage bytes
  static constexpr int kB = KBC * BMr * 128;      // b tile bytes
  static constexpr int kO = BMr * 128 * 2;        // one out chunk: two 64-channel sub-tiles
  static constexpr int kA = MID == 256 ? 0 : BMr * MID * 2;  // a_next tile (none for MID = 256)
  static constexpr int offB = 0, offO = offB + NBB * kB, offA = offO + NB * kO, offW = offA + kA,
                       offS = offW + WS * kWst, offBar = offS + (5 * MID) * 2 * 4;
  static constexpr int nBar = 2 + 2 + NB * 3 + 2 * WS + 2 + 1 + 1 + 2 + NB + 2;
  static constexpr int kSmem = offBar + nBar * 8 + 16 + 1024;
  static_assert(kSmem <= 227 * 1024, "res_chain smem");
};

struct RCParams {
  const float* sc_c;
  const float* sh_c;
  const float* sc_a;
  const float* sh_a;
  int M, n_mt;
  int has_a;  // 0: closing conv only (last unit of a stage: no chained opening conv, no a_next)
  int sthr;   // 1: store warp (VISTA_STORE_THR, default on); 0: epilogue thread 0 issues the stores
};

// CG2: CTA pairs (2-CTA clusters) run every GEMM as ONE tcgen05.mma.cta_group::2 with M = 256 over the pair's
// two adjacent 128-pixel tiles (rank r: tile 2t + r; rank 1 past the last tile: phantom, TMA zero-fill and
// clipped stores).  Each CTA keeps its own b tile, residual chunks, staged out chunks and TMEM accumulators
// (its 128 rows) but loads only HALF of every weight k-block (B's N rows split between the pair): the weights
// are 256 of the 416 KB a MID = 128 tile brings into shared memory, and per-SM TMA ingest is what bounds the
// chain.  The leader (rank 0) waits for both CTAs' operands (its full barriers count both) and issues; commits
// multicast to both CTAs; both epilogues / store warps arrive on the leader's tempty / oready.
template <int MID, int V, bool CG2 = false>
__global__ void __launch_bounds__(kThr, 1)
    res_chain_kernel(const __grid_constant__ CUtensorMap tm_b, const __grid_constant__ CUtensorMap tm_res,
                     const __grid_constant__ CUtensorMap tm_out, const __grid_constant__ CUtensorMap tm_a,
                     const __grid_constant__ CUtensorMap tm_wc, const __grid_constant__ CUtensorMap tm_wa,
                     const RCParams p) {
  using C = RC<MID, V, CG2>;
  constexpr int NCH = C::NCH, KBC = C::KBC, NB = C::NB, WS = C::WS, NBB = C::NBB;
  constexpr bool kCanA = MID <= 128;  // MID = 256: closing conv only
  static_assert(!CG2 || kCanA, "CTA-pair chain: MID <= 128");
  // tile walk: CTA pairs walk pair tiles t (M tile 2t + rank); unpaired CTAs walk M tiles
  const uint32_t crank = CG2 ? (blockIdx.x & 1u) : 0u;
  const int t0 = CG2 ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int tstep = CG2 ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  const int n_t = CG2 ? (p.n_mt + 1) / 2 : p.n_mt;
  auto tile_m0 = [&](int t) { return (CG2 ? 2 * t + (int)crank : t) * BMr; };
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  uint8_t* gbase = smem_raw + (base - raw);
  const uint32_t sB = base + C::offB, sO = base + C::offO, sAo = base + C::offA, sW = base + C::offW;
  float* sc_c = reinterpret_cast<float*>(gbase + C::offS);  // [4 MID] scale, [4 MID] shift, [MID], [MID]
  float* sh_c = sc_c + 4 * MID;
  float* sc_a = sh_c + 4 * MID;
  float* sh_a = sc_a + MID;
  uint64_t* bar = reinterpret_cast<uint64_t*>(gbase + C::offBar);
  uint64_t* bfull = bar;            // [2] b tile landed
  uint64_t* bempty = bfull + 2;     // [2] b tile consumed by the c MMAs
  uint64_t* rfull = bempty + 2;     // [NB] residual chunk landed in staging buffer
  uint64_t* oready = rfull + NB;    // [NB] out chunk staged (a-MMA may read it)
  uint64_t* ofree = oready + NB;    // [NB] staging buffer free: store has read it AND a-MMA done (count 2)
  uint64_t* wfull = ofree + NB;     // [WS]
  uint64_t* wempty = wfull + WS;    // [WS]
  uint64_t* tfull_c = wempty + WS;  // [2]
  uint64_t* tfull_a = tfull_c + 2;  // [1]
  uint64_t* tempty_a = tfull_a + 1; // [1]
  uint64_t* tempty_c = tempty_a + 1;  // [2]
  uint64_t* staged = tempty_c + 2;  // [NB] store warp: the epilogue warps staged out chunk b
  uint64_t* astaged = staged + NB;  // [1] store warp: a_next tile staged
  uint64_t* afree = astaged + 1;    // [1] the previous a_next store has read the a_next staging tile
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(afree + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  constexpr uint32_t kPair = CG2 ? 2u : 1u;  // arrivals the leader's operand / drain barriers collect
  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&bfull[i], kPair);
      mbar_init(&bempty[i], 1);
      mbar_init(&tfull_c[i], 1);
      mbar_init(&tempty_c[i], kEpiWn * kPair);
    }
    for (int i = 0; i < NB; ++i) {
      mbar_init(&rfull[i], 1);
      mbar_init(&oready[i], kPair);
      mbar_init(&ofree[i], p.has_a ? 2 : 1);
    }
    for (int i = 0; i < WS; ++i) {
      mbar_init(&wfull[i], kPair);
      mbar_init(&wempty[i], 1);
    }
    mbar_init(tfull_a, 1);
    mbar_init(tempty_a, kEpiWn * kPair);
    for (int i = 0; i < NB; ++i) mbar_init(&staged[i], kEpiWn);
    mbar_init(astaged, kEpiWn);
    mbar_init(afree, 1);
    fence_mbar_init();
  }
  for (int i = threadIdx.x; i < 5 * MID * 2; i += blockDim.x) {
    float v;
    if (i < 4 * MID) v = p.sc_c[i];
    else if (i < 8 * MID) v = p.sh_c[i - 4 * MID];
    else if (i < 9 * MID) v = p.sc_a[i - 8 * MID];
    else v = p.sh_a[i - 9 * MID];
    sc_c[i] = v;
  }
  if constexpr (CG2) cluster_sync_all();  // both CTAs' barriers initialised; the pair allocates TMEM together
  if (warp == 1) {
    if constexpr (CG2) tmem_alloc_cg2(tmem_slot, 512);
    else tmem_alloc(tmem_slot, 512);
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;  // acc_c[0] cols 0..127, acc_c[1] 128..255, acc_a 256..256+MID (MID <= 128)

  if (warp == 0) {
    // ================= producer =================
    if (lane == 0) {
      uint32_t gw = 0, q = 0, it = 0;
      // bytes: one CTA's box (CG2: half of the k-block's N rows, rows offset by rank; the leader arms its
      // barrier for both boxes, the peer adds an arrival)
      auto push_w = [&](const CUtensorMap* m, int c0, int c1, uint32_t bytes) {
        const uint32_t st = gw % WS;
        if (gw >= (uint32_t)WS) mbar_wait(&wempty[st], ((gw / WS) - 1) & 1);
        if constexpr (CG2) {
          const uint32_t fl = mapa_u32(smem_u32(&wfull[st]), 0);
          if (crank == 0) mbar_arrive_expect_tx(&wfull[st], 2 * bytes);
          tma_load_2d_cg2(sW + st * C::kWst, m, c0, c1, fl);
          if (crank != 0) mbar_arrive_cluster(fl);
        } else {
          mbar_arrive_expect_tx(&wfull[st], bytes);
          tma_load_2d(sW + st * C::kWst, m, c0, c1, &wfull[st]);
        }
        ++gw;
      };
      auto push_res = [&](int m0, int j) {
        const uint32_t qq = q + j, ob = qq % NB;
        if (qq >= (uint32_t)NB) mbar_wait(&ofree[ob], ((qq / NB) - 1) & 1);
        mbar_arrive_expect_tx(&rfull[ob], C::kO);
        tma_load_2d(sO + ob * C::kO, &tm_res, j * 128, m0, &rfull[ob]);
        tma_load_2d(sO + ob * C::kO + BMr * 128, &tm_res, j * 128 + 64, m0, &rfull[ob]);
      };
      constexpr int kNc = CG2 ? 64 : 128, kNa = CG2 ? MID / 2 : MID;  // weight rows per CTA box
      auto push_c = [&](int j) {
        for (int kb = 0; kb < KBC; ++kb) push_w(&tm_wc, kb * BKr, j * 128 + (int)crank * kNc, kNc * 128);
      };
      auto push_a = [&](int j) {
        for (int h = 0; h < 2; ++h) push_w(&tm_wa, j * 128 + h * 64, (int)crank * kNa, kNa * 128);
      };
      for (int tile = t0; tile < n_t; tile += tstep, ++it, q += NCH) {
        const int m0 = tile_m0(tile);
        const uint32_t bb = it % NBB;
        if (it >= (uint32_t)NBB) mbar_wait(&bempty[bb], ((it / NBB) - 1) & 1);
        if constexpr (CG2) {
          const uint32_t fl = mapa_u32(smem_u32(&bfull[bb]), 0);
          if (crank == 0) mbar_arrive_expect_tx(&bfull[bb], 2 * C::kB);
          for (int kb = 0; kb < KBC; ++kb) tma_load_2d_cg2(sB + bb * C::kB + kb * BMr * 128, &tm_b, kb * BKr, m0, fl);
          if (crank != 0) mbar_arrive_cluster(fl);
        } else {
          mbar_arrive_expect_tx(&bfull[bb], C::kB);
          for (int kb = 0; kb < KBC; ++kb) tma_load_2d(sB + bb * C::kB + kb * BMr * 128, &tm_b, kb * BKr, m0, &bfull[bb]);
        }
        // weights in the order the MMA warp consumes them: c(0), then per j: c(j+1), a(j); each residual
        // chunk right after its c weights (its buffer frees up only once the a-MMA two chunks back is done)
        push_c(0);
        push_res(m0, 0);
        for (int j = 0; j < NCH; ++j) {
          if (j + 1 < NCH) {
            push_c(j + 1);
            push_res(m0, j + 1);
          }
          if (kCanA && p.has_a) push_a(j);
        }
      }
      // observe the completion of the staging buffers' last released uses (compute-sanitizer synccheck:
      // no mbarrier phase is left completed-but-unwaited); the final chunk's buffer is never released
      const uint32_t total = q;
      for (uint32_t u = total > (uint32_t)NB ? total - NB : 0; u + 1 < total; ++u)
        if (u + NB >= total) mbar_wait(&ofree[u % NB], (u / NB) & 1);
    }
  } else if (warp == 1) {
    // ================= MMA issuer (whole warp, elected lane issues; CG2: the leader, for the pair) =========
    if (!CG2 || crank == 0) {
    constexpr uint32_t idesc_c = umma_idesc_bf16(CG2 ? 2 * BMr : BMr, 128);
    constexpr uint32_t idesc_a = umma_idesc_bf16(CG2 ? 2 * BMr : BMr, MID);
    // MMA + commit for both forms (CG2: one pair MMA over both CTAs, commits multicast to both)
    auto mma4 = [&](uint32_t tacc, uint32_t a_addr, uint32_t b_addr, uint32_t idesc, uint32_t acc0) {
      if constexpr (CG2) {
        const uint32_t a = umma_desc_lo_sw128(a_addr), b = umma_desc_lo_sw128(b_addr);
        tc_mma_bf16_lo_warp_cg2(tacc, a, b, idesc, acc0);
        tc_mma_bf16_lo_warp_cg2(tacc, a + 2, b + 2, idesc, 1u);
        tc_mma_bf16_lo_warp_cg2(tacc, a + 4, b + 4, idesc, 1u);
        tc_mma_bf16_lo_warp_cg2(tacc, a + 6, b + 6, idesc, 1u);
      } else {
        const uint64_t da = umma_desc_k_sw128(a_addr), db = umma_desc_k_sw128(b_addr);
        tc_mma_bf16_warp(tacc, da, db, idesc, acc0);
        tc_mma_bf16_warp(tacc, da + 2, db + 2, idesc, 1u);
        tc_mma_bf16_warp(tacc, da + 4, db + 4, idesc, 1u);
        tc_mma_bf16_warp(tacc, da + 6, db + 6, idesc, 1u);
      }
    };
    auto commit = [&](uint64_t* bar) {
      if constexpr (CG2) tc_commit_cg2_warp(bar, (uint16_t)3);
      else tc_commit_warp(bar);
    };
    uint32_t gw = 0, it = 0;
    auto wait_w = [&]() -> uint32_t {
      const uint32_t st = gw % WS;
      mbar_wait(&wfull[st], (gw / WS) & 1);
      return st;
    };
    for (int tile = t0; tile < n_t; tile += tstep, ++it) {
      const uint32_t bb = it % NBB, qbase = it * NCH;
      mbar_wait(&bfull[bb], (it / NBB) & 1);
      auto issue_c = [&](const int j) {
        const uint32_t qq = qbase + j, acc = qq & 1;
        if (qq >= 2) mbar_wait(&tempty_c[acc], ((qq >> 1) - 1) & 1);
        tc_fence_after();
        const uint32_t tacc = tmem + acc * 128;
#pragma unroll
        for (int kb = 0; kb < KBC; ++kb) {
          const uint32_t st = wait_w();
          mma4(tacc, sB + bb * C::kB + kb * BMr * 128, sW + st * C::kWst, idesc_c, kb != 0 ? 1u : 0u);
          commit(&wempty[st]);
          ++gw;
        }
        commit(&tfull_c[acc]);
        if (j == NCH - 1) commit(&bempty[bb]);
      };
      auto issue_a = [&](const int j) {
        const uint32_t qq = qbase + j, ob = qq % NB;
        if (j == 0 && it >= 1) mbar_wait(tempty_a, (it - 1) & 1);
        mbar_wait(&oready[ob], (qq / NB) & 1);
        tc_fence_after();
        const uint32_t tacc = tmem + 256;
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const uint32_t st = wait_w();
          mma4(tacc, sO + ob * C::kO + h * BMr * 128, sW + st * C::kWst, idesc_a, (j | h) != 0 ? 1u : 0u);
          commit(&wempty[st]);
          ++gw;
        }
        commit(&ofree[ob]);
        if (j == NCH - 1) commit(tfull_a);
      };
      issue_c(0);
#pragma unroll
      for (int j = 0; j < NCH; ++j) {
        if (j + 1 < NCH) issue_c(j + 1);
        if (kCanA && p.has_a) issue_a(j);
      }
    }
    }
  } else if (warp == kStoreW) {
    // ================= store warp =================
    if (lane == 0 && p.sthr) {
      uint32_t it = 0;
      for (int tile = t0; tile < n_t; tile += tstep, ++it) {
        const int m0 = tile_m0(tile);
        for (int j = 0; j < NCH; ++j) {
          const uint32_t qq = it * NCH + j, ob = qq % NB;
          const uint32_t so = sO + ob * C::kO;
          mbar_wait(&staged[ob], (qq / NB) & 1);
          if (kCanA && p.has_a) {  // staged chunk may feed the a-MMA (CG2: the leader's, which reads both)
            if constexpr (CG2) mbar_arrive_cluster(mapa_u32(smem_u32(&oready[ob]), 0));
            else mbar_arrive(&oready[ob]);
          }
          tma_store_2d(&tm_out, j * 128, m0, so);
          tma_store_2d(&tm_out, j * 128 + 64, m0, so + BMr * 128);
          bulk_commit();
          if (qq >= 1) {
            bulk_wait_read<1>();  // every earlier store (the previous chunk's, the previous a_next) has read its tile
            mbar_arrive(&ofree[(qq - 1) % NB]);
            if (j == 0 && kCanA && p.has_a) mbar_arrive(afree);
          }
        }
        if (kCanA && p.has_a) {
          mbar_wait(astaged, it & 1);
          for (int s2 = 0; s2 < MID / 64; ++s2) tma_store_2d(&tm_a, s2 * 64, m0, sAo + s2 * BMr * 128);
          bulk_commit();
        }
      }
      bulk_wait0();
    }
  } else {
    // ================= epilogue (8 warps) =================
    const int et = threadIdx.x - kEpiW0 * 32;
    const int qd = warp & 3, half = (warp - kEpiW0) >> 2;
    const int row = qd * 32 + lane;
    uint32_t it = 0;
    auto arrive_leader = [&](uint64_t* bar) {  // the MMA-side drain barriers live in the leader
      if constexpr (CG2) mbar_arrive_cluster(mapa_u32(smem_u32(bar), 0));
      else mbar_arrive(bar);
    };
    for (int tile = t0; tile < n_t; tile += tstep, ++it) {
      const int m0 = tile_m0(tile);
#pragma unroll 1
      for (int j = 0; j < NCH; ++j) {
        const uint32_t qq = it * NCH + j, acc = qq & 1, ob = qq % NB;
        const uint32_t so = sO + ob * C::kO;
        mbar_wait(&rfull[ob], (qq / NB) & 1);
        mbar_wait(&tfull_c[acc], (qq >> 1) & 1);
        tc_fence_after();
#pragma unroll
        for (int cc = 0; cc < 2; ++cc) {  // two 32-column pieces of this warp's 64-column half
          const int cb = half * 2 + cc;    // 32-column block 0..3 of the 128-column chunk
          uint32_t v[32];
          tmem_ld_32x32b_x32(tmem + acc * 128 + cb * 32 + ((uint32_t)(qd * 32) << 16), v);
          tc_wait_ld();
          const uint32_t sub = so + (cb >> 1) * BMr * 128 + row * 128;
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            const int ch = j * 128 + cb * 32 + k * 8;
            const uint32_t addr = sub + (((uint32_t)((cb & 1) * 4 + k) ^ (uint32_t)(row & 7)) << 4);
            sts128(addr, epi8(v + k * 8, sc_c + ch, sh_c + ch, lds128(addr), true, true));
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) arrive_leader(&tempty_c[acc]);
        fence_proxy_async_smem();
        if (p.sthr) {  // hand the staged chunk to the store warp
          __syncwarp();
          if (lane == 0) mbar_arrive(&staged[ob]);
          continue;
        }
        named_bar_sync(1, kEpiT);
        if (et == 0) {
          // the previous chunk's store must have read its buffer before that buffer is refilled
          if (qq >= 1) {
            if (j == 0 && kCanA && p.has_a) bulk_wait_read<1>();  // the previous tile's a_next store was committed after it
            else bulk_wait_read<0>();
            mbar_arrive(&ofree[(qq - 1) % NB]);
          }
          if (kCanA && p.has_a) mbar_arrive(&oready[ob]);  // staged chunk may feed the a-MMA (waited only then)
          tma_store_2d(&tm_out, j * 128, m0, so);
          tma_store_2d(&tm_out, j * 128 + 64, m0, so + BMr * 128);
          bulk_commit();
        }
      }
      if (!kCanA || !p.has_a) continue;
      // ---- a_next = ReLU(BN_a(acc_a)) ----
      mbar_wait(tfull_a, it & 1);
      tc_fence_after();
      if (p.sthr) {
        if (it >= 1) mbar_wait(afree, (it - 1) & 1);  // the previous tile's a_next store has read the staging tile
      } else {
        if (et == 0) bulk_wait_read<NCH>();
        named_bar_sync(1, kEpiT);
      }
#pragma unroll
      for (int cc = 0; cc < MID / 64; ++cc) {
        const int cb = half * (MID / 64) + cc;  // 32-column block of the MID-wide accumulator
        uint32_t v[32];
        tmem_ld_32x32b_x32(tmem + 256 + cb * 32 + ((uint32_t)(qd * 32) << 16), v);
        tc_wait_ld();
        const uint32_t sub = sAo + (cb >> 1) * BMr * 128 + row * 128;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int ch = cb * 32 + k * 8;
          sts128(sub + (((uint32_t)((cb & 1) * 4 + k) ^ (uint32_t)(row & 7)) << 4),
                 epi8(v + k * 8, sc_a + ch, sh_a + ch, make_uint4(0, 0, 0, 0), false, true));
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) arrive_leader(tempty_a);
      fence_proxy_async_smem();
      if (p.sthr) {
        __syncwarp();
        if (lane == 0) mbar_arrive(astaged);
        continue;
      }
      named_bar_sync(1, kEpiT);
      if (et == 0) {
        for (int s = 0; s < MID / 64; ++s) tma_store_2d(&tm_a, s * 64, m0, sAo + s * BMr * 128);
        bulk_commit();
      }
    }
    if (et == 0 && !p.sthr) bulk_wait0();
  }
  tc_fence_before();
  __syncthreads();
  if constexpr (CG2) cluster_sync_all();  // no remote arrival or multicast commit may target an exited peer
  if (warp == 1) {
    if constexpr (CG2) tmem_dealloc_cg2(tmem, 512);
    else tmem_dealloc(tmem, 512);
  }
}

}  // namespace

bool res_chain_supported(const ConvLayer& Lc, const ConvLayer* La) {
  const int mid = Lc.Cin;
  // MID = 256 (res4 closing conv) measured 25.7 ms/step vs conv_tc's 20.5 on B200: opt-in (VISTA_CHAIN256=1)
  static const bool mid256 = getenv("VISTA_CHAIN256") && getenv("VISTA_CHAIN256")[0] == '1';
  const bool c_ok = (mid == 64 || mid == 128 || (mid == 256 && mid256 && !La)) && Lc.R == 1 && Lc.S == 1 &&
                    Lc.stride == 1 && Lc.pad == 0 && Lc.groups == 1 && Lc.Cout == 4 * mid && Lc.BN == 128 && Lc.relu;
  return c_ok && (!La || (La->R == 1 && La->S == 1 && La->stride == 1 && La->pad == 0 && La->groups == 1 &&
                          La->Cin == 4 * mid && La->Cout == mid && La->BN == mid && La->relu));
}

template <int MID, int V, bool CG2 = false>
static void launch_chain(const ConvLayer& Lc, const ConvLayer* La, const bf16* b, const bf16* res, bf16* out,
                         bf16* a_next, int M, cudaStream_t st) {
  CUtensorMap tb, tr, to, ta;
  if (!make_plain_tmap(&tb, b, MID, M) || !make_plain_tmap(&tr, res, 4 * MID, M) ||
      !make_plain_tmap(&to, out, 4 * MID, M) || !make_plain_tmap(&ta, La ? a_next : b, MID, M))
    fail(5, "res_chain: tensor map encoding failed");
  RCParams p;
  p.has_a = La ? 1 : 0;
  const bool sthr = !(getenv("VISTA_STORE_THR") && getenv("VISTA_STORE_THR")[0] == '0');
  p.sthr = sthr ? 1 : 0;
  p.sc_c = Lc.scale;
  p.sh_c = Lc.shift;
  p.sc_a = La ? La->scale : Lc.scale;  // (unused without a_next; any MID-long device array)
  p.sh_a = La ? La->shift : Lc.shift;
  p.M = M;
  p.n_mt = (M + BMr - 1) / BMr;
  auto kern = res_chain_kernel<MID, V, CG2>;
  ensure_smem_attr((const void*)kern, RC<MID, V, CG2>::kSmem);
  if constexpr (CG2) {  // 2-CTA clusters walking pair tiles; each CTA loads half-row weight boxes
    p.sthr = 1;
    const int pairs = std::min((p.n_mt + 1) / 2, num_sms() / 2);
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(2 * pairs, 1, 1);
    cfg.blockDim = dim3(kThr, 1, 1);
    cfg.dynamicSmemBytes = RC<MID, V, CG2>::kSmem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeClusterDimension;
    at[0].val.clusterDim.x = 2;
    at[0].val.clusterDim.y = 1;
    at[0].val.clusterDim.z = 1;
    cfg.attrs = at;
    cfg.numAttrs = 1;
    VCHECK(cudaLaunchKernelEx(&cfg, kern, tb, tr, to, ta, Lc.tmap_w_half, La ? La->tmap_w_half : Lc.tmap_w_half, p));
  } else {
    const int grid = p.n_mt < num_sms() ? p.n_mt : num_sms();
    kern<<<grid, kThr, RC<MID, V, CG2>::kSmem, st>>>(tb, tr, to, ta, Lc.tmap_w, La ? La->tmap_w : Lc.tmap_w, p);
  }
  LAUNCHED();
}

void res_chain_forward(const ConvLayer& Lc, const ConvLayer* La, const bf16* b, const bf16* res, bf16* out,
                       bf16* a_next, int N, int H, int W, cudaStream_t st) {
  const int64_t M64 = (int64_t)N * H * W;
  if (M64 <= 0) return;
  if (M64 > INT32_MAX - BMr) fail(1, "res_chain: M too large");
  const int M = (int)M64;
  const int mid = Lc.Cin;
  prof_begin(st);
  static const int v = [] {
    // measured (ResNet50 res3, 28x28): the MID = 128 chain is bound by residual chunks in flight, so its b
    // tile is single-buffered for a third staging buffer (20.98 -> 16.52 ms per step); MID = 64 keeps the
    // double-buffered b (its V = 1 variant was 1 % slower).  VISTA_CHAIN_V overrides (bit 0: 64, bit 1: 128)
    const char* e = getenv("VISTA_CHAIN_V");
    return e ? atoi(e) : 2;
  }();
  // CTA pairs (VISTA_CG2_CHAIN, default on): half of every weight k-block per CTA, one M = 256 MMA per K
  // step; measured per step (same box): c+a 56x56 13.2 -> 12.5 ms, c 56x56 11.9 -> 11.5, c+a 28x28 15.7 ->
  // 14.6 (three staging buffers, seven 8 KB weight stages), c 28x28 6.4 -> 5.8 (four staging buffers)
  const char* ce = getenv("VISTA_CG2_CHAIN");
  const bool cg2 = ce ? ce[0] == '1' : true;
  if (cg2 && mid == 64) {
    if (v & 1) launch_chain<64, 1, true>(Lc, La, b, res, out, a_next, M, st);
    else launch_chain<64, 0, true>(Lc, La, b, res, out, a_next, M, st);
  } else if (cg2 && mid == 128) {
    if (La) launch_chain<128, 0, true>(Lc, La, b, res, out, a_next, M, st);
    else launch_chain<128, 1, true>(Lc, La, b, res, out, a_next, M, st);
  } else if (mid == 64) {
    if (v & 1) launch_chain<64, 1>(Lc, La, b, res, out, a_next, M, st);
    else launch_chain<64, 0>(Lc, La, b, res, out, a_next, M, st);
  } else if (mid == 256) {
    if (La) fail(1, "res_chain: MID = 256 runs the closing conv only");
    if (v & 4) launch_chain<256, 1>(Lc, nullptr, b, res, out, a_next, M, st);
    else launch_chain<256, 0>(Lc, nullptr, b, res, out, a_next, M, st);
  } else {
    if (v & 2) launch_chain<128, 1>(Lc, La, b, res, out, a_next, M, st);
    else launch_chain<128, 0>(Lc, La, b, res, out, a_next, M, st);
  }
  const double flops = 2.0 * M64 * (double)(4 * mid) * mid * (La ? 2 : 1);  // both GEMMs (or the c GEMM)
  const double bytes = 2.0 * M64 * ((double)mid + 4 * mid + 4 * mid + (La ? mid : 0)) + 2.0 * (La ? 8 : 4) * mid * mid;
  char label[96] = {0};
  if (prof_labels()) snprintf(label, sizeof(label), "res_chain %s MID%d HxW%dx%d", La ? "c+a" : "c", mid, H, W);
  prof_end(st, 0, flops, bytes, prof_labels() ? label : nullptr);
}

}  // namespace vista
