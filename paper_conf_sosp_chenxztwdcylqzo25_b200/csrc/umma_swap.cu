// umma_swap.cu -- prefill grouped expert GEMM, swap-AB on CTA pairs.
//
// The expert FFN batches of PAPER.md L179 (gate+up fused, then down), recast
// for the 5th-gen tensor cores:
//   * swap-AB: the expert WEIGHTS are the tcgen05 A operand (M = 256 weight
//     rows per CTA pair, 128 per CTA) and the expert's TOKEN rows are the B
//     operand (N <= 256, a multiple of 16).  An expert segment is padded only
//     to 16 tokens instead of a 128-row M tile, so the tensor cores skip the
//     ~20 % padding rows a token-major tiling computes (V3, 8K tokens:
//     ~256 +- 16 rows per expert).
//   * cta_group::2: the two CTAs of a cluster each stage their own 128 weight
//     rows and HALF of the token tile; the leader issues one 256 x N MMA that
//     reads the peer's half from the peer's shared memory -- per SM the
//     shared-memory traffic per MMA is 2/3 of the 1-CTA 128x256 tile's.
//   * the stage handshake has no cross-CTA arrive: only the leader arrives
//     (expecting both CTAs' bytes); the peer's 2-SM TMA completes on the
//     leader's barrier; the MMA commit multicasts the stage release to both.
//     (A release.cluster arrive per stage serialised the producer: measured,
//     profiles/r01/pair_kernel.txt.)
//
// GEMM1 (EPI_SWIGLU): A = W13 tiles whose 128-row CTA halves hold, per lane
// quadrant, [gate f 0-31 | up f 0-31 | gate f 32-63 | up f 32-63] of the
// half's 64 h columns; the up quadrants hand their accumulators to the gate
// quadrants through shared memory, h = silu(g) * u is computed from fp32, and
// (FP8) requantised with a 1x128 UE8M0 scale per token whose amax spans both
// CTAs of the pair (DSMEM exchange) -- DESIGN.md readings R10/R11.
// GEMM2 (EPI_PLAIN): A = W2 tiles (256 H rows per pair), bf16 y rows.
//
// Work units = (expert, 256-row weight block, 256-token tile), expert-major
// then weight block then token tile, claimed from a device counter by the
// pair leader (the L181 dynamic task queue) and forwarded to the peer.
#include <cuda.h>

#include "common.cuh"
#include "kernels.h"
#include "sm100.cuh"

namespace moe {
using namespace sm100;

constexpr int SW_STAGES = 6, SW_THREADS = 320, SW_UQ = 4;
// stages are released in groups of SW_CE by one MMA commit: a tcgen05.commit costs the tensor
// pipe ~100 cycles at N = 256 (profiles/r02/mma_ring.txt: block-scaled pair MMA 153.5 cycles
// with a commit per k-block, 132.8 per 2, 128.0 per 4) -- but in this kernel SW_CE = 2
// measured 1-2 % slower than 1 twice (interleaved A/B: GEMM1 2.50 vs 2.47 ms, and 2.42 vs 2.37 ms
// after the two-box token halves): the coarser release shortens the producer's run-ahead, and
// the commit is not what binds inside this kernel (profiles/r02/swap_np.txt)
constexpr int SW_CE = 1;
static_assert(SW_STAGES % SW_CE == 0, "stage groups");
constexpr int SW_W_BYTES = 128 * 128;          // this CTA's 128 weight rows x 128 B
constexpr int SW_X_BYTES = 128 * 128;          // up to 128 token rows (half of N <= 256)
constexpr int SW_SFW_BYTES = 512, SW_SFX_BYTES = 1024;
constexpr int SW_XBOX = 32;                    // token rows per TMA box
constexpr uint32_t SW_TMEM_COLS = 512;
constexpr uint32_t SW_SFA_COL = 256, SW_SFB_COL = 264;   // + 16 for the second scale set
constexpr int SW_XCH = 8;                      // columns per up->gate exchange chunk
constexpr size_t SW_SMEM = 1024 + (size_t)SW_STAGES * (SW_W_BYTES + SW_X_BYTES + SW_SFW_BYTES + SW_SFX_BYTES) +
                           4 * 32 * SW_XCH * 4 +      // up -> gate exchange
                           2 * 2 * 4 * 128 * 4 +      // amax partials [parity][half][slot][128]
                           2 * 2 * 128 * 4 +          // per-token inverse scales [half][gate warp][128]
                           4 * 2048 +                 // SWIGLU: per gate warp 32 x 32 transpose tile
                           1024;                      // barriers, unit queue, TMEM base

struct SwapUnit {
  int valid, group, expert, row0, n, nb;
};

__device__ __forceinline__ SwapUnit swap_unit(const SwapParams &p, int u, int n_routed_units) {
  SwapUnit r{};
  if (u < n_routed_units) {
    const int nb_r = p.nb_r;
    const int4 any = p.tiles[u / nb_r];
    const int t0 = any.w & 0xFFFF, nt = any.w >> 16;
    const int local = u - t0 * nb_r;
    const int4 tl = p.tiles[t0 + local % nt];
    r.valid = 1; r.group = 0; r.expert = tl.x; r.row0 = tl.y; r.n = min(256, tl.z - tl.y); r.nb = local / nt;
    return r;
  }
  const int us = u - n_routed_units;
  const int nt = (p.T_shared + 255) / 256;
  if (p.T_shared > 0 && us < nt * p.nb_s) {
    r.valid = 1; r.group = 1; r.expert = 0; r.nb = us / nt;
    r.row0 = (us % nt) * 256; r.n = min(256, p.T_shared - r.row0);
  }
  return r;
}

template <bool FP8, int EPI, int NP>
__global__ void __launch_bounds__(SW_THREADS, 1) umma_swap_gemm(const __grid_constant__ SwapParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t *smem = reinterpret_cast<uint8_t *>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t *sW = smem;
  uint8_t *sX = sW + SW_STAGES * SW_W_BYTES;
  uint8_t *sSFW = sX + SW_STAGES * SW_X_BYTES;
  uint8_t *sSFX = sSFW + SW_STAGES * SW_SFW_BYTES;
  float *xbuf = reinterpret_cast<float *>(sSFX + SW_STAGES * SW_SFX_BYTES);   // [4 pairs][SW_XCH][32]
  float *am = xbuf + 4 * SW_XCH * 32;                                         // [2][2][4][128]
  float *isc = am + 2 * 2 * 4 * 128;                                          // [2 half][2 gate warp][128]
  uint8_t *trbuf = reinterpret_cast<uint8_t *>(isc + 2 * 2 * 128);            // [4 gate warps][2 KB]
  uint64_t *full = reinterpret_cast<uint64_t *>(trbuf + 4 * 2048);
  // PLAIN reuses xbuf .. trbuf (>= 16 KB) as 8 per-warp 2 KB transpose tiles
  static_assert(4 * 32 * SW_XCH * 4 + 2 * 2 * 4 * 128 * 4 + 2 * 2 * 128 * 4 + 4 * 2048 >= 8 * 2048, "tr tiles");
  uint64_t *empty = full + SW_STAGES;
  uint64_t *tmem_full = empty + SW_STAGES;
  uint64_t *tmem_empty = tmem_full + 1;
  uint64_t *uq_full = tmem_empty + 1;
  uint64_t *uq_empty = uq_full + SW_UQ;
  uint64_t *am_bar = uq_empty + SW_UQ;                                        // [2 parity][2 half]
  uint32_t *tmem_base_smem = reinterpret_cast<uint32_t *>(am_bar + 4);
  int *unit_q = reinterpret_cast<int *>(tmem_base_smem + 4);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  // NP CTA pairs per cluster: pair `pair` = cluster ranks 2*pair, 2*pair + 1 (the MMA
  // peers); with NP = 2 the pairs work on adjacent weight blocks of the same token tile
  // and each token box is loaded once and multicast to both pairs
  const uint32_t crank = cluster_rank();
  const uint32_t prank = crank & 1, pair = crank >> 1;
  const bool leader = crank == 0;                  // cluster leader: claims units
  const bool pleader = prank == 0;                 // pair leader: issues the MMAs
  const int n_routed_units = p.tiles ? (*p.n_tiles) * p.nb_r : 0;

  if (warp == 0 && lane == 0) {
    for (int i = 0; i < 2; ++i) {
      prefetch_tmap(&p.g[i].w_map); prefetch_tmap(&p.g[i].x_map); prefetch_tmap(&p.g[i].x_map128);
      if (FP8) { prefetch_tmap(&p.g[i].sfw_map); prefetch_tmap(&p.g[i].sfx_map); }
    }
    // a stage is released by every pair's MMA commit (its token box is in every pair's smem)
    for (int s = 0; s < SW_STAGES; ++s) mbar_init(&full[s], 1);
    for (int s = 0; s < SW_STAGES / SW_CE; ++s) mbar_init(&empty[s], NP);
    mbar_init(tmem_full, 1);
    mbar_init(tmem_empty, 16);                   // 8 epilogue warps x 2 CTAs (the leader's copy is used)
    // leader's uq_empty: per pair an MMA warp + 8 epilogue warps per CTA; the other CTAs' producers
    constexpr int kUqArrivals = NP * 17 + 2 * NP - 1;
    for (int i = 0; i < SW_UQ; ++i) {
      mbar_init(&uq_full[i], 1);
      mbar_init(&uq_empty[i], (kExperiments && p.debug_mode >= 4) ? kUqArrivals + 1 : kUqArrivals);
    }
    for (int i = 0; i < 4; ++i) mbar_init(&am_bar[i], 64);    // 2 gate warps here, per lane (+ peer bytes)
    fence_barrier_init();
  }
  if (warp == 1) tmem_alloc_pair(tmem_base_smem, SW_TMEM_COLS);
  tc_fence_before();
  __syncthreads();                               // the allocated TMEM address, CTA-local
  cluster_sync();                                // barriers of both CTAs initialised
  tc_fence_after();
  const uint32_t tmem = *tmem_base_smem;

  // unit queue: the leader's producer claims units; the peer receives the id
  // by st.async (completing on its uq_full); slot releases are plain arrives
  auto next_unit = [&](int &qs, uint32_t &qph) {
    mbar_wait(&uq_full[qs], qph);
    const int u = unit_q[qs];
    __syncwarp();
    if (lane == 0) {
      if (leader) mbar_arrive(&uq_empty[qs]);
      else mbar_arrive_remote(map_to_rank(&uq_empty[qs], 0));
    }
    if (++qs == SW_UQ) { qs = 0; qph ^= 1; }
    return u;
  };

  if (warp == 0) {
    // ============================ TMA producer (both CTAs) ============================
    if (lane == 0) {
      int stage = 0; uint32_t phase = 0;
      int qs = 0; uint32_t qph = 0;
      // the next unit is claimed one unit ahead, so the counter's round trip overlaps
      // this unit's loads instead of sitting between two units' load streams
      int u_next = leader ? atomicAdd(p.sched, 1) : 0;
      for (;;) {
        int u;
        if (leader) {
          u = u_next;
          u_next = atomicAdd(p.sched, 1);
          mbar_wait(&uq_empty[qs], qph ^ 1);
          unit_q[qs] = u;
          mbar_arrive(&uq_full[qs]);
#pragma unroll
          for (uint32_t r = 1; r < 2 * NP; ++r) {
            const uint32_t pbar = map_to_rank(&uq_full[qs], r);
            mbar_arrive_expect_tx_remote(pbar, 4);
            st_async_u32(map_to_rank(&unit_q[qs], r), (uint32_t)u, pbar);
          }
          if (++qs == SW_UQ) { qs = 0; qph ^= 1; }
        } else {
          mbar_wait(&uq_full[qs], qph);
          u = unit_q[qs];
          mbar_arrive_remote(map_to_rank(&uq_empty[qs], 0));
          if (++qs == SW_UQ) { qs = 0; qph ^= 1; }
        }
        const SwapUnit ui = swap_unit(p, u, n_routed_units);
        if (!ui.valid) break;
        const SwapGroup &g = p.g[ui.group];
        const int nb = ui.nb * NP + (int)pair;                 // this pair's weight block
        const int half_n = ((ui.n + 15) & ~15) >> 1;          // token rows per CTA
        const int nbox0 = (half_n + SW_XBOX - 1) / SW_XBOX;
        const int nbox = nbox0 > 2 ? 4 : nbox0;                // > 64 rows: one 128-row box (4 x 32 rows of bytes)
        const int xrow = ui.row0 + (int)prank * half_n;
        // NP = 1: the half in at most two boxes of 128 / 64 / 32 / 16 rows, at most 32 rows
        // over-read (one 128-row box above 96 rows, 64 + 32, 64, 32 + 16, 32, 16)
        const int xb0 = half_n > 96 ? 128 : half_n > 48 ? 64 : half_n > 16 ? 32 : 16;
        const int xb1 = (half_n > 64 && half_n <= 96) ? 32 : (half_n > 32 && half_n <= 48) ? 16 : 0;
        const CUtensorMap *xm0 = xb0 == 128 ? &g.x_map128 : xb0 == 64 ? &g.x_map64 : xb0 == 32 ? &g.x_map : &g.x_map16;
        const CUtensorMap *xm1 = xb1 == 32 ? &g.x_map : &g.x_map16;
        const uint32_t xbytes = NP == 1 ? (uint32_t)(xb0 + xb1) * 128 : (uint32_t)nbox * (SW_XBOX * 128);
        const int64_t wtile = ((int64_t)ui.expert * g.w_nblk + nb) * g.kblocks;
        const int G = (g.kblocks + 3) >> 2;
        for (int kb = 0; kb < g.kblocks; ++kb) {
          if (stage % SW_CE == 0) mbar_wait(&empty[stage / SW_CE], phase ^ 1);   // the group's release
          if (kExperiments && p.debug_mode == 3) {                 // timing experiment: MMAs on stale smem, no loads
            if (pleader) mbar_arrive(&full[stage]);
            if (++stage == SW_STAGES) { stage = 0; phase ^= 1; }
            continue;
          }
          const bool sf = FP8 && (kb & 3) == 0;
          const int kc = kb * (FP8 ? 128 : 64);
          if (kExperiments && p.debug_mode >= 4) {                 // timing experiments (loads only, per-CTA 1-SM TMA)
            const bool dw = p.debug_mode != 5, dx = p.debug_mode != 4;
            const uint32_t b1 = (dw ? SW_W_BYTES : 0) + (dx ? nbox * (SW_XBOX * 128) : 0);
            mbar_expect_tx(&full[stage], b1);
            if (dw) tma_load_2d(sW + stage * SW_W_BYTES, &g.w_map, &full[stage], 0, (int)((wtile + kb) * 16 + prank * 8));
            if (dx) {
              if (nbox > 2)
                tma_load_2d(sX + stage * SW_X_BYTES, &g.x_map128, &full[stage], kc, xrow);
              else
                for (int i = 0; i < nbox; ++i)
                  tma_load_2d(sX + stage * SW_X_BYTES + i * (SW_XBOX * 128), &g.x_map, &full[stage], kc, xrow + i * SW_XBOX);
            }
            if (++stage == SW_STAGES) { stage = 0; phase ^= 1; }
            continue;
          }
          const uint32_t bytes = SW_W_BYTES + xbytes + (sf ? SW_SFW_BYTES + SW_SFX_BYTES : 0);
          if (pleader) mbar_expect_tx(&full[stage], 2 * bytes);
          // the CTA's 16 KB half of the 256-row tile: 8 rows of 2 KB
          tma_load_2d_pair(sW + stage * SW_W_BYTES, &g.w_map, &full[stage], 0,
                           (int)((wtile + kb) * 16 + prank * 8));
          if constexpr (NP == 1) {                 // (rows past the half are never read)
            tma_load_2d_pair(sX + stage * SW_X_BYTES, xm0, &full[stage], kc, xrow);
            if (xb1) tma_load_2d_pair(sX + stage * SW_X_BYTES + xb0 * 128, xm1, &full[stage], kc, xrow + xb0);
          } else {
            // token half split between the two pairs, each part multicast to the CTA with
            // the same pair rank in both pairs: > 64 rows as 2 x 64-row boxes, else 32-row boxes
            const uint16_t mask = (uint16_t)(0x5u << prank);
            if (nbox > 2)
              tma_load_2d_pair_mc(sX + stage * SW_X_BYTES + pair * (64 * 128), &g.x_map64, &full[stage], kc,
                                  xrow + (int)pair * 64, mask);
            else if ((int)pair < nbox)
              tma_load_2d_pair_mc(sX + stage * SW_X_BYTES + pair * (SW_XBOX * 128), &g.x_map, &full[stage], kc,
                                  xrow + (int)pair * SW_XBOX, mask);
          }
          if (sf) {
            const int kg = kb >> 2;
            const int wr = g.sfw_per_cta ? (int)((((int64_t)ui.expert * G + kg) * g.w_nblk + nb) * 2 + prank)
                                         : (int)(((int64_t)ui.expert * G + kg) * g.w_nblk + nb);
            tma_load_2d_pair(sSFW + stage * SW_SFW_BYTES, &g.sfw_map, &full[stage], 0, wr);
            tma_load_2d_pair(sSFX + stage * SW_SFX_BYTES, &g.sfx_map, &full[stage], 0,
                             kg * g.sfx_tile_stride + (ui.row0 >> 7));
          }
          if (++stage == SW_STAGES) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ============================ MMA issuer (pair leader) ============================
    if (kExperiments && p.debug_mode >= 4) {                     // timing experiments: each CTA drains its own ring
      int stage = 0; uint32_t phase = 0;
      int qs = 0; uint32_t qph = 0;
      for (;;) {
        const int u = next_unit(qs, qph);
        const SwapUnit ui = swap_unit(p, u, n_routed_units);
        if (!ui.valid) break;
        const int kblocks = p.g[ui.group].kblocks;
        for (int kb = 0; kb < kblocks; ++kb) {
          mbar_wait(&full[stage], phase);
          if (lane == 0) {
            if (stage % SW_CE == SW_CE - 1) mbar_arrive(&empty[stage / SW_CE]);
            if (kb == kblocks - 1) mbar_arrive(tmem_full);
          }
          __syncwarp();
          if (++stage == SW_STAGES) { stage = 0; phase ^= 1; }
        }
      }
    } else if (pleader) {
      int stage = 0; uint32_t phase = 0; uint32_t acc_phase = 0;
      constexpr uint16_t kAllPairs = NP == 1 ? 0x3 : 0xF;
      const uint16_t my_pair = (uint16_t)(0x3u << (2 * pair));
      int qs = 0; uint32_t qph = 0;
      // MOE_DEBUG_TRACE: cycles waiting for a unit / the accumulator / loaded stages, and issuing
      long long c_unit = 0, c_tmem = 0, c_full = 0, c_issue = 0, n_units = 0, n_flop16 = 0;
      const bool trc = p.trace != nullptr && lane == 0;
      long long c0 = trc ? clock64() : 0;
      const long long c_start = c0;
      for (;;) {
        const int u = next_unit(qs, qph);
        const SwapUnit ui = swap_unit(p, u, n_routed_units);
        if (trc) { const long long c = clock64(); c_unit += c - c0; c0 = c; }
        if (!ui.valid) break;
        const int kblocks = p.g[ui.group].kblocks;
        const int N = (ui.n + 15) & ~15;
        mbar_wait(tmem_empty, acc_phase ^ 1);
        if (trc) { const long long c = clock64(); c_tmem += c - c0; c0 = c; ++n_units; n_flop16 += N / 16; }
        tc_fence_after();
        for (int kb = 0; kb < kblocks; ++kb) {
          mbar_wait(&full[stage], phase);
          if (trc) { const long long c = clock64(); c_full += c - c0; c0 = c; }
          tc_fence_after();
          if (kExperiments && lane == 0 && p.debug_mode == 1) {    // timing experiment: loads only (commit releases the stage)
            if (stage % SW_CE == SW_CE - 1) mma_commit_pair(&empty[stage / SW_CE]);
            if (kb == kblocks - 1) mma_commit_pair(tmem_full);
          } else if (lane == 0) {
            const uint32_t a0 = smem_u32(sW + stage * SW_W_BYTES);
            const uint32_t b0 = smem_u32(sX + stage * SW_X_BYTES);
            // one scale image covers 4 k-blocks (sf id = kb & 3); two TMEM column
            // sets alternate so a copy never overwrites scales in use.  The copy and the
            // MMAs are issued by this one thread into the tensor pipe, which executes its
            // tcgen05.cp / tcgen05.mma in issue order: the copy into set s at kb = 4j + 8 runs
            // after the MMAs of kb = 4j .. 4j + 3 that read set s, whatever SW_STAGES is
            const uint32_t set = FP8 ? ((kb >> 2) & 1) * 16 : 0;
            if (FP8 && (kb & 3) == 0) {
              tmem_cp_32x128b_x4_pair(tmem + SW_SFA_COL + set, sf_desc(smem_u32(sSFW + stage * SW_SFW_BYTES)));
              tmem_cp_32x128b_x4_pair(tmem + SW_SFB_COL + set, sf_desc(smem_u32(sSFX + stage * SW_SFX_BYTES)));
              if (N > 128)                         // tokens 128..255 (a cp costs the pipe ~100 cycles)
                tmem_cp_32x128b_x4_pair(tmem + SW_SFB_COL + set + 4,
                                        sf_desc(smem_u32(sSFX + stage * SW_SFX_BYTES + 512)));
            }
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const uint64_t ad = sw128_kmajor_desc(a0 + k * 32);
              const uint64_t bd = sw128_kmajor_desc(b0 + k * 32);
              const uint32_t acc = (kb | k) != 0;
              if (FP8)
                mma_mxf8_pair(tmem, ad, bd, idesc_mxf8(256, N, kb & 3, kb & 3), acc, tmem + SW_SFA_COL + set,
                              tmem + SW_SFB_COL + set);
              else
                mma_bf16_pair(tmem, ad, bd, idesc_bf16(256, N), acc);
            }
            if (stage % SW_CE == SW_CE - 1) mma_commit_pair_mc(&empty[stage / SW_CE], kAllPairs);
            if (kb == kblocks - 1) mma_commit_pair_mc(tmem_full, my_pair);
          }
          __syncwarp();
          if (trc) { const long long c = clock64(); c_issue += c - c0; c0 = c; }
          if (++stage == SW_STAGES) { stage = 0; phase ^= 1; }
        }
        acc_phase ^= 1;
      }
      if (trc) {
        unsigned long long *o = p.trace + 8 * (blockIdx.x >> 1);   // one record per CTA pair
        o[0] = c_unit; o[1] = c_tmem; o[2] = c_full; o[3] = c_issue; o[4] = n_units; o[5] = n_flop16;
        o[6] = clock64() - c_start;
      }
    }
  } else {
    // ============================ epilogue (8 warps, both CTAs) ============================
    // warp -> TMEM lane quadrant q = warp % 4 (weight rows 32q..32q+31 of this
    // CTA) and token-column half; each thread pulls its <= 128 accumulator
    // columns into registers and releases TMEM before any math.
    const int ew = warp - 2;
    const int q = warp & 3;
    const int half = ew >> 2;
    const uint32_t lane_base = (uint32_t)(q * 32) << 16;
    uint32_t acc_phase = 0, tile_i = 0;
    int qs = 0; uint32_t qph = 0;
    for (;;) {
      const int u = next_unit(qs, qph);
      const SwapUnit ui = swap_unit(p, u, n_routed_units);
      if (!ui.valid) break;
      const SwapGroup &g = p.g[ui.group];
      mbar_wait(tmem_full, acc_phase);
      tc_fence_after();
      const int c0 = half * 128;
      const int nvalid = max(0, min(128, ui.n - c0));
      const int nch = (nvalid + 31) >> 5;
      uint32_t r[128];
#pragma unroll
      for (int c = 0; c < 4; ++c)
        if (c < nch) tmem_ld_32x32b_x32(tmem + lane_base + c0 + c * 32, *reinterpret_cast<uint32_t(*)[32]>(r + 32 * c));
      tmem_ld_wait();
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (pleader) mbar_arrive(tmem_empty);
        else mbar_arrive_remote(map_to_rank(tmem_empty, crank & ~1u));
      }
      acc_phase ^= 1;
      const int64_t rbase = (int64_t)ui.row0 + c0;          // token row of this half's column 0
      const int nb = ui.nb * NP + (int)pair;                 // this pair's weight block
      if (kExperiments && p.debug_mode >= 1) { ++tile_i; continue; }        // timing experiments: no epilogue math
      if constexpr (EPI == GEMM_PLAIN) {
        // transpose 32 tokens x 32 H rows per step through a per-warp smem tile,
        // then 16-byte row stores (token t: 64 contiguous bytes of its y row)
        const int h0 = nb * 256 + (int)prank * 128 + q * 32;
        __nv_bfloat16 *tr = reinterpret_cast<__nv_bfloat16 *>(reinterpret_cast<uint8_t *>(xbuf) + ew * 2048);
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          if (c < nch) {
#pragma unroll
            for (int j = 0; j < 32; ++j) tr[j * 32 + lane] = __float2bfloat16_rn(__uint_as_float(r[32 * c + j]));
            __syncwarp();
#pragma unroll
            for (int it = 0; it < 4; ++it) {
              const int j = it * 8 + (lane >> 2), cc = lane & 3;
              if (32 * c + j < nvalid)
                *reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(g.out) + (rbase + 32 * c + j) * g.ldc + h0 +
                                           cc * 8) = *reinterpret_cast<const uint4 *>(tr + j * 32 + cc * 8);
            }
            __syncwarp();
          }
        }
      } else {
        // ---- up quadrants (odd q) hand their accumulators to the gate quadrants ----
        const int pi = (q >> 1) + 2 * half;
        const bool up = q & 1;
        float *xb = xbuf + pi * (SW_XCH * 32);
        const int nx = (nvalid + SW_XCH - 1) / SW_XCH;
#pragma unroll
        for (int c = 0; c < 128 / SW_XCH; ++c) {
          if (c < nx) {
            // (both warps reach each named barrier at the same instruction)
            if (up) {
#pragma unroll
              for (int j = 0; j < SW_XCH; ++j) xb[j * 32 + lane] = __uint_as_float(r[c * SW_XCH + j]);
            }
            asm volatile("bar.sync %0, 64;" ::"r"(1 + pi) : "memory");
            if (!up) {
#pragma unroll
              for (int j = 0; j < SW_XCH; ++j) {
                const float gt = __uint_as_float(r[c * SW_XCH + j]);
                r[c * SW_XCH + j] = __float_as_uint(silu_f(gt) * xb[j * 32 + lane]);
              }
            }
            asm volatile("bar.sync %0, 64;" ::"r"(5 + pi) : "memory");
          }
        }
        if (up) { ++tile_i; continue; }
        const int qg = q >> 1;                                // gate warp 0 / 1 of this half
        const int f = nb * 128 + (int)prank * 64 + qg * 32 + lane;
        const int f0 = f - lane;
        uint8_t *trw = trbuf + (half * 2 + qg) * 2048;
        if constexpr (!FP8) {
          __nv_bfloat16 *tr = reinterpret_cast<__nv_bfloat16 *>(trw);
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            if (c < nch) {
#pragma unroll
              for (int j = 0; j < 32; ++j) tr[j * 32 + lane] = __float2bfloat16_rn(__uint_as_float(r[32 * c + j]));
              __syncwarp();
#pragma unroll
              for (int it = 0; it < 4; ++it) {
                const int j = it * 8 + (lane >> 2), cc = lane & 3;
                if (32 * c + j < nvalid)
                  *reinterpret_cast<uint4 *>(reinterpret_cast<__nv_bfloat16 *>(g.out) + (rbase + 32 * c + j) * g.ldc + f0 +
                                             cc * 8) = *reinterpret_cast<const uint4 *>(tr + j * 32 + cc * 8);
              }
              __syncwarp();
            }
          }
        } else {
          // ---- per-token amax over the 128 h columns of block nb: 32 lanes x
          // 2 gate warps here x 2 in the peer.  Per 32-column chunk c a
          // butterfly reduce-scatter across lanes leaves lane l with the warp
          // max of column 32c + l (31 shuffles per chunk). ----
          float m4[4];
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            float v[32];
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] = 32 * c + j < nvalid ? fabsf(__uint_as_float(r[32 * c + j])) : 0.f;
#pragma unroll
            for (int o = 16; o >= 1; o >>= 1) {
              const bool hi = lane & o;
#pragma unroll
              for (int i = 0; i < o; ++i) {
                const float send = hi ? v[i] : v[i + o];
                const float keep = hi ? v[i + o] : v[i];
                v[i] = fmaxf(keep, __shfl_xor_sync(0xffffffffu, send, o));
              }
            }
            m4[c] = v[0];
          }
          const int par = tile_i & 1;
          const uint32_t ph = (tile_i >> 1) & 1;
          float *amh = am + (par * 2 + half) * 4 * 128;      // [slot][lane][chunk]
          // local partials by plain stores + arrive (this warp expects its peer
          // warp's 512 bytes); remote partials by st.async completing on the
          // peer's barrier
          *reinterpret_cast<float4 *>(amh + qg * 128 + 4 * lane) = make_float4(m4[0], m4[1], m4[2], m4[3]);
          uint64_t *bar = &am_bar[par * 2 + half];
          st_async_v4f32(map_to_rank(amh + (2 + qg) * 128 + 4 * lane, crank ^ 1), m4[0], m4[1], m4[2], m4[3],
                         map_to_rank(bar, crank ^ 1));
          if (lane == 0) mbar_expect_tx(bar, 32 * 16);
          else mbar_arrive(bar);
          mbar_wait(bar, ph);
          float *sc = isc + (half * 2 + qg) * 128;
          {
            const float4 a0 = *reinterpret_cast<const float4 *>(amh + 4 * lane);
            const float4 a1 = *reinterpret_cast<const float4 *>(amh + 128 + 4 * lane);
            const float4 a2 = *reinterpret_cast<const float4 *>(amh + 256 + 4 * lane);
            const float4 a3 = *reinterpret_cast<const float4 *>(amh + 384 + 4 * lane);
            const float mx[4] = {fmaxf(fmaxf(a0.x, a1.x), fmaxf(a2.x, a3.x)), fmaxf(fmaxf(a0.y, a1.y), fmaxf(a2.y, a3.y)),
                                 fmaxf(fmaxf(a0.z, a1.z), fmaxf(a2.z, a3.z)), fmaxf(fmaxf(a0.w, a1.w), fmaxf(a2.w, a3.w))};
#pragma unroll
            for (int c = 0; c < 4; ++c) {
              const int col = 32 * c + lane;
              const int e = ue8m0_exponent(mx[c]);
              sc[col] = exp2i(-e);
              if (pleader && qg == 0 && col < nvalid)
                g.out_sf[sf_img_off(rbase + col, nb, g.out_sf_tile_stride)] = (uint8_t)(e + 127);
            }
          }
          __syncwarp();
          // e4m3 codes: 32 tokens x 32 h columns per step through the smem tile,
          // then 16-byte stores (token t: 32 contiguous bytes of its h row)
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            if (c < nch) {
#pragma unroll
              for (int j = 0; j < 32; ++j) trw[j * 32 + lane] = f32_to_e4m3(__uint_as_float(r[32 * c + j]) * sc[32 * c + j]);
              __syncwarp();
#pragma unroll
              for (int it = 0; it < 2; ++it) {
                const int j = it * 16 + (lane >> 1), cc = lane & 1;
                if (32 * c + j < nvalid)
                  *reinterpret_cast<uint4 *>(reinterpret_cast<uint8_t *>(g.out) + (rbase + 32 * c + j) * g.ldc + f0 + cc * 16) =
                      *reinterpret_cast<const uint4 *>(trw + j * 32 + cc * 16);
              }
              __syncwarp();
            }
          }
        }
      }
      ++tile_i;
    }
  }
  tc_fence_before();
  cluster_sync();
  if (warp == 1) tmem_dealloc_pair(tmem, SW_TMEM_COLS);
}

// clusters of NP CTA pairs that can be co-resident (persistent grid = that many clusters)
template <bool FP8, int EPI, int NP>
static int swap_max_clusters() {
  auto k = umma_swap_gemm<FP8, EPI, NP>;
  if (set_kernel_attr((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SW_SMEM) != cudaSuccess) return 0;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(2 * NP);
  cfg.blockDim = dim3(SW_THREADS);
  cfg.dynamicSmemBytes = SW_SMEM;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2 * NP;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, (const void *)k, &cfg) != cudaSuccess) { cudaGetLastError(); return 0; }
  return n;
}

template <bool FP8, int EPI, int NP>
static cudaError_t launch_swap(const SwapParams &p, int grid, cudaStream_t st) {
  auto k = umma_swap_gemm<FP8, EPI, NP>;
  cudaError_t e = set_kernel_attr((const void *)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SW_SMEM);
  if (e != cudaSuccess) return e;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(grid & ~(2 * NP - 1));
  cfg.blockDim = dim3(SW_THREADS);
  cfg.dynamicSmemBytes = SW_SMEM;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2 * NP;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, p);
}

cudaError_t launch_umma_swap_gemm(bool fp8, int epi, const SwapParams &p, int grid, int np, cudaStream_t st) {
  if (np == 2) {
    grid = 4 * grid;                               // grid = clusters of 2 pairs (host: umma_swap_max_clusters4)
    if (fp8) return epi == GEMM_SWIGLU ? launch_swap<true, GEMM_SWIGLU, 2>(p, grid, st) : launch_swap<true, GEMM_PLAIN, 2>(p, grid, st);
    return epi == GEMM_SWIGLU ? launch_swap<false, GEMM_SWIGLU, 2>(p, grid, st) : launch_swap<false, GEMM_PLAIN, 2>(p, grid, st);
  }
  if (grid < 2) grid = 2;
  if (fp8) return epi == GEMM_SWIGLU ? launch_swap<true, GEMM_SWIGLU, 1>(p, grid, st) : launch_swap<true, GEMM_PLAIN, 1>(p, grid, st);
  return epi == GEMM_SWIGLU ? launch_swap<false, GEMM_SWIGLU, 1>(p, grid, st) : launch_swap<false, GEMM_PLAIN, 1>(p, grid, st);
}

int umma_swap_max_clusters4(bool fp8) {
  const int a = fp8 ? swap_max_clusters<true, GEMM_SWIGLU, 2>() : swap_max_clusters<false, GEMM_SWIGLU, 2>();
  const int b = fp8 ? swap_max_clusters<true, GEMM_PLAIN, 2>() : swap_max_clusters<false, GEMM_PLAIN, 2>();
  return a < b ? a : b;
}

size_t umma_swap_smem_bytes() { return SW_SMEM; }

}  // namespace moe
