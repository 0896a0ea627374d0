// monitor_tc.cuh -- BFAST-Monitor hot path on the 5th-generation tensor cores.
//
// Same algorithm and numerics contract as monitor_simt.cuh (Algorithm 1,
// PAPER.md L134; Fig. 12), re-mapped so that every contraction
// shared by a 128-pixel tile runs as a tcgen05.mma with fp32 accumulators
// in Tensor Memory, and the CUDA cores only do per-(pixel, date) scalar
// work:
//
//   masked Gram  A = sum_t v_t x_t x_t^T  (Alg. 1 l.2, Fig. 4)
//       The K(K+1)/2 entries are linear in NF = 2+6k masked moments
//       sum_t v_t f_q(t) of the functions f = {tau, tau^2, tau sin_j,
//       tau cos_j, sin_m, cos_m (m <= 2k)} (product-to-sum identities), so
//       the tile's Gram is ONE bf16 GEMM: D_G[128 x 3NF] += V[128 x 16] *
//       F[16 x 3NF] per 16 dates, with V the exact 0/1 mask and F split in
//       hi+mid+lo bf16 (24-bit mantissa: the products are exact, so the
//       Gram carries fp32 accumulation error only).
//   moment b = sum_t v_t y'_t x_t  (Alg. 1 l.4): D_b += [y'hi y'lo] * [xhi xlo]
//   yhat = X beta (Fig. 12 ker 6): D_y[128 x 16 dates] = [beta hi/mid/lo] *
//       [x hi/mid/lo] with the 6 cross terms of a 3-way bf16 split
//       (~24-bit accuracy, fp32 accumulate).
//   refinement db = sum_t v_t r0_t x_t, r0 = y' - x beta0: a sum with heavy
//       cancellation (db -> 0 as beta0 -> beta), so both r0 and x are split
//       3-way (24-bit): D_db[128 x 3K] += [r0 hi,mid,lo per date] * [x hi|mid|lo].
//   Because the refinement step re-solves with the residual moment, the
//   16-bit moment only sets beta0; the final beta carries fp32-level error
//   (DESIGN.md "Numerics").
//
// Roles (160 threads): warps 0-3 own one pixel per thread (TMEM lane =
// pixel row); warp 4 streams 16-date x 128-pixel boxes of the time-major
// stack (one 2-D TMA copy each) into a 4-stage ring that the consumer warps
// release as soon as they have read a box; warp 5 streams the chunk's
// B-operand tables (one 1-D bulk copy each, L2-resident) into a 3-stage ring
// released by tcgen05.commit of the MMAs that read them; warp 6 issues every
// tcgen05.mma.  All hand-offs are mbarriers (per-warp arrivals), so no warp
// ever waits at a CTA-wide barrier inside the date loops.  Thread 0 issues the MMAs after a
// named barrier and signals completion with tcgen05.commit on mbarriers.
// Per tile the chunk sequence is: history (Gram+moment), history again
// (residuals, sigma, refinement moment, MOSUM ring), monitoring (MOSUM,
// boundary, first break, mean).  The stack is read through a 2-D TMA tensor
// map whose out-of-bounds fill is NaN, so a ragged last tile needs no
// special case (its missing pixels are "all missing").
#pragma once
#include "monitor_simt.cuh"
#include "sm100.cuh"
#include <cuda.h>

namespace bfast {

// CTA = consumer warpgroup (warps 0-3, one pixel per thread) + producer
// warpgroup (warp 4 stack TMA, 5 table copies, 6 MMA issue, 7 idle).  At
// launch every thread holds 80 registers (3 CTAs x 256 threads); the
// producers drop to kTcAuxRegs, the consumers rise to kTcConsumerRegs
// (80*256 = 128*kTcAuxRegs + 128*kTcConsumerRegs).
constexpr int kTcThreads = 256;
constexpr int kTcLaunchRegs = 80;
#ifndef BFAST_TC_AUX_REGS
#define BFAST_TC_AUX_REGS 32
#endif
constexpr int kTcAuxRegs = BFAST_TC_AUX_REGS;
constexpr int kTcConsumerRegs = 2 * kTcLaunchRegs - kTcAuxRegs;

template <int K>
struct TcCfg {
  static constexpr int k = (K - 2) / 2;
  static constexpr int NF = 2 + 6 * k;                     // masked moment functions
  static constexpr int NGp = ((3 * NF + 15) / 16) * 16;    // Gram GEMM N (hi, mid, lo)
  static constexpr int KB = ((2 * K + 15) / 16) * 16;      // moment GEMM N
  static constexpr int KY = ((6 * K + 15) / 16) * 16;      // yhat GEMM K
  static constexpr int KB3 = ((3 * K + 15) / 16) * 16;     // refinement GEMM N (x hi|mid|lo)
  static constexpr int DC = 16;                            // dates per chunk
  // TMEM columns.  Pass 1 accumulates the Gram moments and the moment b;
  // pass 2 the refinement moment, two yhat slots and the beta operand (the
  // A operand of the yhat GEMM, bf16 pairs).  The consumers read G and b in
  // the solve before any pass-2 MMA is issued, so pass 2 reuses their columns.
  static constexpr int COL_G = 0, COL_B = NGp;
  static constexpr int COL_DB = 0, COL_Y = KB3, COL_A3 = KB3 + 2 * DC;
  static constexpr int COLS_P1 = NGp + KB, COLS_P2 = COL_A3 + KY / 2;
  static constexpr int COLS_USED = COLS_P1 > COLS_P2 ? COLS_P1 : COLS_P2;
  static constexpr int TMEM_COLS = COLS_USED <= 32 ? 32 : COLS_USED <= 64 ? 64 : COLS_USED <= 128 ? 128
                                   : COLS_USED <= 256 ? 256 : 512;
  static constexpr int B1_BYTES = NGp * DC * 2;            // [NGp x 16] bf16
  static constexpr int B2_BYTES = KB * 2 * DC * 2;         // [KB x 32] bf16
  static constexpr int B3_BYTES = DC * KY * 2;             // [16 x KY] bf16
  static constexpr int BR_BYTES = KB3 * 3 * DC * 2;        // [KB3 x 48] bf16 (refinement)
  static constexpr int TAB1 = B1_BYTES + B2_BYTES;         // pass 1 chunk tables
  static constexpr int TAB2 = BR_BYTES + B3_BYTES;         // pass 2a
  static constexpr int TAB3 = B3_BYTES;                    // pass 2b
  static constexpr int TABMAX = TAB1 > TAB2 ? TAB1 : TAB2;
  static constexpr int YBYTES = DC * 128 * 4;             // one [16 dates x 128 px] box
  static constexpr int TSTAGE = ((TABMAX + 127) / 128) * 128;
  static constexpr int SY_MAX = 4;                         // stack ring stages (released on read; 3 or 4)
  static constexpr int ST = 3;                             // table ring stages (released by MMA commit)
  static constexpr int A1_BYTES = 128 * DC * 2;
  static constexpr int A2_BYTES = 128 * 2 * DC * 2;
  static constexpr int A4_BYTES = 128 * 3 * DC * 2;        // r0 hi|mid|lo per date
  static constexpr int OPBUF = A1_BYTES + A2_BYTES > A4_BYTES ? A1_BYTES + A2_BYTES : A4_BYTES;
  static constexpr int RSLOT = 128 * 4;                   // ring slot: one residual per pixel
  static constexpr int VSLOT = 128 * 2;                   // validity mask: 16 bits per pixel per chunk
  // sy stack stages, nop operand buffers (2: the consumers fill one while the
  // MMA reads the other), the MOSUM ring of hcap slots, nch history masks
  static constexpr size_t smem_bytes(int hcap, int nch, int sy, int nop) {
    return (size_t)sy * YBYTES + (size_t)ST * TSTAGE + (size_t)nop * OPBUF + (size_t)hcap * RSLOT +
           (size_t)nch * VSLOT;
  }
};

struct TcTables {
  const uint8_t *tab1, *tab2, *tab3;  // per-chunk B operands, canonical K-major layout
  int nch, ncm;                       // history / monitoring chunks of 16 dates
  int sy, nop;                        // stack stages (3|4), operand buffers (1|2)
  int64_t ntiles;                     // 128-pixel tiles (the last may be ragged)
};

__device__ __forceinline__ void named_bar_sync_128() { asm volatile("bar.sync 1, 128;" ::: "memory"); }
__device__ __forceinline__ void sts_f32(uint32_t a, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(a), "f"(v) : "memory");
}
__device__ __forceinline__ void sts_u16(uint32_t a, uint16_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"(v) : "memory");
}
// store v if `inc` (the ring advance of this date: 0 for a missing one) is
// non-zero.  The advance is materialised anyway, so the predicate costs one
// compare instead of a re-evaluated NaN test (only 7 predicate registers).
__device__ __forceinline__ void sts_f32_inc(uint32_t a, float v, uint32_t inc) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p st.shared.f32 [%0], %1;\n\t}" ::"r"(a), "f"(v),
               "r"(inc)
               : "memory");
}
__device__ __forceinline__ float lds_f32(uint32_t a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ int lds_u16(uint32_t a) {
  uint16_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=h"(v) : "r"(a) : "memory");
  return v;
}
// producer-side wait with back-off so a waiting producer does not steal
// issue slots from the consumer warps of its SM sub-partition
#ifndef BFAST_AUX_WAIT
#define BFAST_AUX_WAIT 0
#endif
#ifndef BFAST_MMA_WAIT
#define BFAST_MMA_WAIT 0
#endif
template <int MODE>
__device__ __forceinline__ void mbar_wait_mode(uint64_t *bar, uint32_t parity) {
  if (MODE == 0) {
    while (!sm100::mbar_try_wait_suspend(bar, parity, 1000000u)) {
    }
  } else if (MODE == 1) {
    while (!sm100::mbar_try_wait(bar, parity)) {
    }
  } else {
    while (!sm100::mbar_try_wait_suspend(bar, parity, (uint32_t)MODE)) {
    }
  }
}
__device__ __forceinline__ void mbar_wait_sleep(uint64_t *bar, uint32_t parity) {
  mbar_wait_mode<BFAST_AUX_WAIT>(bar, parity);
}
__device__ __forceinline__ void mbar_wait_mma(uint64_t *bar, uint32_t parity) {
  mbar_wait_mode<BFAST_MMA_WAIT>(bar, parity);
}
// the rare branch of the boundary test (Alg. 1 l.10-12), kept out of line
// returns bit 0: |m| > B (a break), bit 1: |m|/B within kTieTol of 1
__device__ __noinline__ int boundary_rare(float m, int rank1, int nbar, float lam) {
  const float B = boundary_f32(lam, rank1, nbar);
  const float am = fabsf(m);
  return (am > B ? 1 : 0) | (fabsf(am - B) <= kTieTol * B ? 2 : 0);
}

// y split into hi and lo bf16 halves packed {lo16: hi part, hi16: lo part}
__device__ __forceinline__ uint32_t split2_bf16(float v) {
  const uint32_t w1 = sm100::pack_bf16x2(v, 0.f);
  const float hi = __uint_as_float(w1 << 16);
  return sm100::pack_bf16x2(v, v - hi);
}
// bf16 parts by truncation: hi = top 8 significant bits of v (exactly
// representable), v - hi exact.  Two words' upper halves -> one packed word.
__device__ __forceinline__ float bf16_trunc(float v) { return __uint_as_float(__float_as_uint(v) & 0xFFFF0000u); }
__device__ __forceinline__ uint32_t pack_hi16(float lo_elem, float hi_elem) {
  return __byte_perm(__float_as_uint(lo_elem), __float_as_uint(hi_elem), 0x7632);
}
__device__ __forceinline__ float bf16_round(float v) {
  return __uint_as_float(sm100::pack_bf16x2(v, 0.f) << 16);
}

template <int K>
__global__ void __launch_bounds__(kTcThreads, 3)
    monitor_tc_kernel(MonitorParams p, TcTables tb, const __grid_constant__ CUtensorMap ymap,
                      const __grid_constant__ CUtensorMap hmap) {
  using C = TcCfg<K>;
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t yfull[C::SY_MAX], yempty[C::SY_MAX], tfull[C::ST], tempty[C::ST], opfull[2],
      opfree[2], yhfull[2], yhfree[2], accready, betaready;
  __shared__ uint32_t tmem_base_s;
  const int hcap = p.hcap, SY = tb.sy, NOP = tb.nop;
  uint8_t *ystages = smem;
  uint8_t *tstages = ystages + SY * C::YBYTES;
  uint8_t *opb = tstages + C::ST * C::TSTAGE;
  uint8_t *ring = opb + NOP * C::OPBUF;
  uint8_t *vmask = ring + hcap * C::RSLOT;
  constexpr int NCW = 4;  // consumer warps

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  if (tid == 0) {
    for (int i = 0; i < C::SY_MAX; ++i) {
      sm100::mbar_init(&yfull[i], 1);
      sm100::mbar_init(&yempty[i], NCW);
    }
    for (int i = 0; i < C::ST; ++i) {
      sm100::mbar_init(&tfull[i], 1);
      sm100::mbar_init(&tempty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      sm100::mbar_init(&opfull[i], NCW);
      sm100::mbar_init(&opfree[i], 1);
      sm100::mbar_init(&yhfull[i], 1);
      sm100::mbar_init(&yhfree[i], NCW);
    }
    sm100::mbar_init(&accready, 1);
    sm100::mbar_init(&betaready, NCW);
    sm100::fence_mbar_init();
  }
  if (warp == 0) sm100::tmem_alloc(&tmem_base_s, C::TMEM_COLS);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tbase = tmem_base_s;
  const int n = p.n, N = p.N, nch = tb.nch, ncm = tb.ncm;

  if (warp >= NCW) {
    // producer warpgroup: three single-thread roles need few registers; hand
    // them to the consumer warpgroup (3 CTAs per SM fit the register file)
    sm100::setmaxnreg_dec<kTcAuxRegs>();
  if (warp == 4) {
    // ------------------------------------------------------------ stack producer
    if (lane == 0) {
      // one 2-D TMA box [16 dates x 128 px] per chunk.  History chunks read
      // through `hmap` (dates >= n are out of bounds), monitoring chunks
      // through `ymap`; out-of-bounds elements arrive as NaN = missing.
      sm100::prefetch_tmap(&ymap);
      sm100::prefetch_tmap(&hmap);
      const uint64_t pol_first = sm100::policy_evict_first();
      int ys = 0;
      uint32_t yph = 0;
      for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
        const int x0 = (int)(tile * 128);
        for (int phase = 0; phase < 3; ++phase) {
          const int nc = phase < 2 ? nch : ncm;
          const int tbeg = phase < 2 ? 0 : n;
          for (int c = 0; c < nc; ++c) {
            mbar_wait_sleep(&yempty[ys], yph ^ 1);
            uint8_t *yst = ystages + ys * C::YBYTES;
            sm100::mbar_arrive_expect_tx(&yfull[ys], C::YBYTES);
            if (phase == 0)
              sm100::tma_load_2d(yst, &hmap, x0, c * C::DC, &yfull[ys]);  // re-read in pass 2a (L2)
            else
              sm100::tma_load_2d_hint(yst, phase == 1 ? &hmap : &ymap, x0, tbeg + c * C::DC, &yfull[ys],
                                      pol_first);  // last use
            if (++ys == SY) {
              ys = 0;
              yph ^= 1;
            }
          }
        }
      }
    }
  } else if (warp == 5) {
    // ------------------------------------------------------------ table producer
    if (lane == 0) {
      int ts = 0;
      uint32_t tph = 0;
      for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
        for (int phase = 0; phase < 3; ++phase) {
          const int nc = phase < 2 ? nch : ncm;
          const uint32_t tabbytes = phase == 0 ? C::TAB1 : phase == 1 ? C::TAB2 : C::TAB3;
          const uint8_t *tabsrc = phase == 0 ? tb.tab1 : phase == 1 ? tb.tab2 : tb.tab3;
          for (int c = 0; c < nc; ++c) {
            mbar_wait_sleep(&tempty[ts], tph ^ 1);
            uint8_t *tst = tstages + ts * C::TSTAGE;
            sm100::mbar_arrive_expect_tx(&tfull[ts], tabbytes);
            sm100::bulk_g2s(tst, tabsrc + (size_t)c * tabbytes, tabbytes, &tfull[ts]);
            if (++ts == C::ST) {
              ts = 0;
              tph ^= 1;
            }
          }
        }
      }
    }
  } else if (warp == 6) {
    // ------------------------------------------------------------ MMA issuer
    if (lane == 0) {
      const uint32_t idG = sm100::idesc_bf16_f32(128, C::NGp);
      const uint32_t idB = sm100::idesc_bf16_f32(128, C::KB);
      const uint32_t idY = sm100::idesc_bf16_f32(128, C::DC);
      const uint32_t idR = sm100::idesc_bf16_f32(128, C::KB3);
      const uint32_t aop = sm100::smem_u32(opb), tss = sm100::smem_u32(tstages);
      int ts = 0;
      uint32_t tph = 0, opcnt = 0, yissue = 0, bcnt = 0;
      auto tslot = [&](int ahead, uint32_t &par) {
        int s = ts + ahead;
        par = tph;
        while (s >= C::ST) {
          s -= C::ST;
          par ^= 1;
        }
        return s;
      };
      auto tadvance = [&]() {
        if (++ts == C::ST) {
          ts = 0;
          tph ^= 1;
        }
      };
      // operand buffer of the opcnt-th chunk and its phase parity
      auto opwait = [&]() -> uint32_t {
        const uint32_t ob = NOP == 2 ? (opcnt & 1) : 0;
        const uint32_t par = NOP == 2 ? ((opcnt >> 1) & 1) : (opcnt & 1);
        mbar_wait_mma(&opfull[ob], par);
        return ob;
      };
      // yhat of the chunk `ahead` chunks after the current one (table offset)
      auto issue_yhat = [&](int ahead, uint32_t tab_off) {
        uint32_t par;
        const int s = tslot(ahead, par);
        const uint32_t slot = yissue & 1;
        mbar_wait_mma(&yhfree[slot], ((yissue >> 1) & 1) ^ 1);  // consumers done with the slot
        mbar_wait_mma(&tfull[s], par);
        sm100::tc_fence_after();
        const uint32_t b3 = tss + s * C::TSTAGE + tab_off;
#pragma unroll
        for (int q = 0; q < C::KY / 16; ++q)
          sm100::umma_bf16_ts(tbase + C::COL_Y + slot * C::DC, tbase + C::COL_A3 + 8 * q,
                              sm100::smem_desc(b3 + q * 2 * 256, 256, 128), idY, q > 0);
        sm100::umma_commit(&yhfull[slot]);
        ++yissue;
      };
      for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
        // pass 1: Gram + moment per chunk
        for (int c = 0; c < nch; ++c) {
          const uint32_t ob = opwait();
          mbar_wait_mma(&tfull[ts], tph);
          sm100::tc_fence_after();
          const uint32_t a1 = aop + ob * C::OPBUF, a2 = a1 + C::A1_BYTES;
          const uint32_t b1 = tss + ts * C::TSTAGE, b2 = b1 + C::B1_BYTES;
          sm100::umma_bf16(tbase + C::COL_G, sm100::smem_desc(a1, 2048, 128),
                           sm100::smem_desc(b1, C::NGp * 16, 128), idG, c > 0);
#pragma unroll
          for (int q = 0; q < 2; ++q)
            sm100::umma_bf16(tbase + C::COL_B, sm100::smem_desc(a2 + q * 2 * 2048, 2048, 128),
                             sm100::smem_desc(b2 + q * 2 * C::KB * 16, C::KB * 16, 128), idB, (c > 0 || q > 0));
          sm100::umma_commit(&opfree[ob]);
          sm100::umma_commit(&tempty[ts]);
          if (c == nch - 1) sm100::umma_commit(&accready);
          ++opcnt;
          tadvance();
        }
        // pass 2a: yhat0 two chunks ahead, refinement moment per chunk
        mbar_wait_mma(&betaready, bcnt & 1);
        ++bcnt;
        for (int a = 0; a < 2 && a < nch; ++a) issue_yhat(a, C::BR_BYTES);
        for (int c = 0; c < nch; ++c) {
          const uint32_t ob = opwait();
          mbar_wait_mma(&tfull[ts], tph);
          sm100::tc_fence_after();
          const uint32_t br = tss + ts * C::TSTAGE;
#pragma unroll
          for (int q = 0; q < 3; ++q)
            sm100::umma_bf16(tbase + C::COL_DB, sm100::smem_desc(aop + ob * C::OPBUF + q * 2 * 2048, 2048, 128),
                             sm100::smem_desc(br + q * 2 * C::KB3 * 16, C::KB3 * 16, 128), idR, (c > 0 || q > 0));
          sm100::umma_commit(&opfree[ob]);
          if (c + 2 < nch) issue_yhat(2, C::BR_BYTES);
          sm100::umma_commit(&tempty[ts]);
          if (c == nch - 1) sm100::umma_commit(&accready);
          ++opcnt;
          tadvance();
        }
        // pass 2b: yhat with the refined beta, two chunks ahead
        mbar_wait_mma(&betaready, bcnt & 1);
        ++bcnt;
        for (int a = 0; a < 2 && a < ncm; ++a) issue_yhat(a, 0);
        for (int c = 0; c < ncm; ++c) {
          if (c + 2 < ncm) issue_yhat(2, 0);
          sm100::umma_commit(&tempty[ts]);  // chunk c's table was read by its yhat MMA
          tadvance();
        }
      }
    }
  }  // warp 7 idles: it completes the producer warpgroup
  } else {
    // ------------------------------------------------------------ consumers
    sm100::setmaxnreg_inc<kTcConsumerRegs>();
    const uint32_t lanebase = tbase + ((uint32_t)(32 * warp) << 16);
    const float qnan = __int_as_float(0x7fc00000);
    // ring: slot s = 128 residuals f32, this thread's at rbase + s*RSLOT;
    // history validity: 16 bits per chunk, this thread's at vbase + c*VSLOT
    const uint32_t rbase = sm100::smem_u32(ring) + 4 * tid;
    const uint32_t rend = rbase + hcap * C::RSLOT;
    const uint32_t vbase = sm100::smem_u32(vmask) + 2 * tid;
    int ys = 0;
    uint32_t yph = 0, opcnt = 0, yuse = 0, acnt = 0;
    // 32-bit shared addresses of the barriers this warp waits on / arrives at
    const uint32_t a_yfull = sm100::smem_u32(&yfull[0]), a_yempty = sm100::smem_u32(&yempty[0]);
    const uint32_t a_opfull = sm100::smem_u32(&opfull[0]), a_opfree = sm100::smem_u32(&opfree[0]);
    const uint32_t a_yhfull = sm100::smem_u32(&yhfull[0]), a_yhfree = sm100::smem_u32(&yhfree[0]);
    const uint32_t a_accready = sm100::smem_u32(&accready), a_betaready = sm100::smem_u32(&betaready);
    const uint32_t ybuf0 = sm100::smem_u32(ystages);

    auto yadvance = [&]() {
      if (++ys == SY) {
        ys = 0;
        yph ^= 1;
      }
    };
    auto warp_arrive = [&](uint32_t bar) {
      __syncwarp();
      if (lane == 0) sm100::mbar_arrive_a(bar);
    };
    // wait until the MMA has released the operand buffer of chunk opcnt
    auto opbuf_acquire = [&]() -> uint8_t * {
      const uint32_t ob = NOP == 2 ? (opcnt & 1) : 0;
      const uint32_t par = NOP == 2 ? ((opcnt >> 1) & 1) : (opcnt & 1);
      sm100::mbar_wait_a(a_opfree + 8 * ob, par ^ 1);
      return opb + ob * C::OPBUF;
    };
    auto opbuf_publish = [&]() {
      const uint32_t ob = NOP == 2 ? (opcnt & 1) : 0;
      sm100::fence_proxy_async_smem();
      warp_arrive(a_opfull + 8 * ob);
      ++opcnt;
    };
    auto write_beta_operand = [&](const float (&bt)[K], float off) {
      // A3 row (TMEM) = [bh | bh | bh | bm | bm | bl | 0...] (6 blocks of K, KY bf16);
      // `off` would fold an offset into the intercept (kept at 0: the GEMM's
      // accumulation error scales with |yhat|, so the offset stays outside)
      float h[K], m[K], l[K];
#pragma unroll
      for (int i = 0; i < K; ++i) {
        const float bi = i == 0 ? bt[0] + off : bt[i];
        h[i] = bf16_round(bi);
        m[i] = bf16_round(bi - h[i]);
        l[i] = bi - h[i] - m[i];
      }
      uint32_t w[C::KY / 2];
#pragma unroll
      for (int j = 0; j < C::KY / 2; ++j) {
        float e[2];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
          const int col = 2 * j + u, blk = col / K, i = col % K;
          e[u] = col >= 6 * K ? 0.f : (blk < 3 ? h[i] : blk < 5 ? m[i] : l[i]);
        }
        w[j] = sm100::pack_bf16x2(e[0], e[1]);
      }
#pragma unroll
      for (int q = 0; q < C::KY / 16; ++q) {
        uint32_t w8[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) w8[i] = w[8 * q + i];
        sm100::tmem_st8(lanebase + C::COL_A3 + 8 * q, w8);  // this pixel's row of the A operand
      }
      sm100::tmem_st_wait();
      sm100::tc_fence_before();
      warp_arrive(a_betaready);
    };
    auto wait_yhat = [&]() {
      sm100::mbar_wait_a(a_yhfull + 8 * (yuse & 1), (yuse >> 1) & 1);
      sm100::tc_fence_after();
    };
    auto load_yhat8 = [&](int half, float (&yh)[8]) {
      sm100::tmem_ld8(lanebase + C::COL_Y + (yuse & 1) * C::DC + 8 * half, yh);
      sm100::tmem_ld_wait();
    };
    auto release_yhat = [&]() {
      sm100::tc_fence_before();
      warp_arrive(a_yhfree + 8 * (yuse & 1));
      ++yuse;
    };

    for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
      const int64_t pix = p.p0 + tile * 128 + tid;
      // ================= pass 1: masked Gram + moment on the tensor cores
      int nbar = 0;
      float c0 = qnan, ymax = 0.f;
      bool have = false;
      for (int c = 0; c < nch; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        const float *Ys = reinterpret_cast<const float *>(ystages + ys * C::YBYTES);
        // offset c = first valid value (warp-uniform pre-scan while a lane lacks it)
        if (__any_sync(0xffffffffu, !have)) {
          for (int d = 0; d < C::DC && !have; ++d) {
            const float y = Ys[d * 128 + tid];
            if (y == y) {
              c0 = y;
              have = true;
            }
          }
        }
        uint8_t *const ob = opbuf_acquire();
#pragma unroll 1
        for (int hf = 0; hf < 2; ++hf) {  // two halves of 8 dates: half the hot code
          float yv[8];
#pragma unroll
          for (int d = 0; d < 8; ++d) yv[d] = Ys[(8 * hf + d) * 128 + tid];  // dates >= n read as NaN (hmap)
          uint32_t mw[4], yw[8];
          float mf[8];
#pragma unroll
          for (int d = 0; d < 8; ++d) {
            const float y = yv[d];
            const bool v = (y == y);
            ymax = fmaxf(ymax, fabsf(y));  // NaN ignored
            nbar += v;
            const float yp = v ? y - c0 : 0.f;
            const float yh = bf16_trunc(yp);
            yw[d] = pack_hi16(yh, yp - yh);  // {y' hi, y' lo}
            mf[d] = v ? 1.0f : 0.0f;
          }
#pragma unroll
          for (int q = 0; q < 4; ++q) mw[q] = pack_hi16(mf[2 * q], mf[2 * q + 1]);
          *reinterpret_cast<uint4 *>(ob + sm100::kmajor_off(tid, 8 * hf, 128)) = make_uint4(mw[0], mw[1], mw[2], mw[3]);
#pragma unroll
          for (int q = 0; q < 2; ++q)
            *reinterpret_cast<uint4 *>(ob + C::A1_BYTES + sm100::kmajor_off(tid, 16 * hf + 8 * q, 128)) =
                make_uint4(yw[4 * q], yw[4 * q + 1], yw[4 * q + 2], yw[4 * q + 3]);
        }
        warp_arrive(a_yempty + 8 * ys);  // every loaded value has been consumed
        opbuf_publish();
        yadvance();
      }
      sm100::mbar_wait_a(a_accready, acnt & 1);
      ++acnt;
      sm100::tc_fence_after();

      // ================= solve (Alg. 1 l.3-4): Gram from the masked moments
      float A[Tri<K>::kN], b[K];
      {
        float F[C::NGp];
#pragma unroll
        for (int q = 0; q < C::NGp / 16; ++q) {
          float v16[16];
          sm100::tmem_ld16(lanebase + C::COL_G + 16 * q, v16);
          sm100::tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 16; ++i) F[16 * q + i] = v16[i];
        }
        float Bm[C::KB];
#pragma unroll
        for (int q = 0; q < C::KB / 16; ++q) {
          float v16[16];
          sm100::tmem_ld16(lanebase + C::COL_B + 16 * q, v16);
          sm100::tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 16; ++i) Bm[16 * q + i] = v16[i];
        }
        float G[C::NF];
#pragma unroll
        for (int q = 0; q < C::NF; ++q) G[q] = F[q] + F[C::NF + q] + F[2 * C::NF + q];
#pragma unroll
        for (int i = 0; i < K; ++i) b[i] = Bm[i] + Bm[K + i];
        const float nb = (float)nbar;
        auto Cf = [&](int m) -> float { return m == 0 ? nb : G[2 + 2 * C::k + 2 * ((m < 0 ? -m : m) - 1) + 1]; };
        auto Sf = [&](int m) -> float {
          return m == 0 ? 0.f : (m < 0 ? -G[2 + 2 * C::k + 2 * (-m - 1)] : G[2 + 2 * C::k + 2 * (m - 1)]);
        };
        A[Tri<K>::idx(0, 0)] = nb;
        A[Tri<K>::idx(0, 1)] = G[0];
        A[Tri<K>::idx(1, 1)] = G[1];
#pragma unroll
        for (int j = 1; j <= C::k; ++j) {
          A[Tri<K>::idx(0, 2 * j)] = Sf(j);
          A[Tri<K>::idx(0, 2 * j + 1)] = Cf(j);
          A[Tri<K>::idx(1, 2 * j)] = G[2 + 2 * (j - 1)];
          A[Tri<K>::idx(1, 2 * j + 1)] = G[3 + 2 * (j - 1)];
#pragma unroll
          for (int jb = j; jb <= C::k; ++jb) {
            A[Tri<K>::idx(2 * j, 2 * jb)] = 0.5f * (Cf(j - jb) - Cf(j + jb));          // s_j s_jb
            A[Tri<K>::idx(2 * j + 1, 2 * jb + 1)] = 0.5f * (Cf(j - jb) + Cf(j + jb));  // c_j c_jb
            A[Tri<K>::idx(2 * j, 2 * jb + 1)] = 0.5f * (Sf(j + jb) + Sf(j - jb));      // s_j c_jb
            if (jb > j) A[Tri<K>::idx(2 * j + 1, 2 * jb)] = 0.5f * (Sf(jb + j) + Sf(jb - j));  // c_j s_jb
          }
        }
      }
      const int h = window_h(nbar, p.hf);
      bool deg = (nbar < K + 1) || (h < 1);
      float beta[K];
      bool refit = false;
#ifdef BFAST_REFIT_WHY
      uint32_t why = 0;  // diagnostics build: which trigger sent the pixel to the refit
#define BFAST_WHY(b) why |= (b)
#else
#define BFAST_WHY(b)
#endif
      {
        const float minratio = chol_factor<K, float>(A);
        chol_solve<K, float>(A, b, beta);
        if (!deg && !(minratio >= (float)kRefitRatio)) {
          refit = true;
          BFAST_WHY(0x10);
        }
        if (deg) {
#pragma unroll
          for (int i = 0; i < K; ++i) beta[i] = 0.f;
        }
      }
      sm100::tc_fence_before();
      write_beta_operand(beta, 0.f);

      // ================= pass 2a: residuals r0, sigma, refinement moment, ring
      const int hh = deg ? 1 : h;
      float s2 = 0.f;
      int cr = 0;
      uint32_t wa = rbase;  // ring write address (slot of rank cr)
      for (int c = 0; c < nch; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        wait_yhat();
        const float *Ys = reinterpret_cast<const float *>(ystages + ys * C::YBYTES);
        uint8_t *const ob = opbuf_acquire();
        uint32_t vm = 0;  // validity of the chunk's 16 dates
#pragma unroll 1
        for (int hf = 0; hf < 2; ++hf) {
          float yh[8], yv[8];
          uint32_t m8 = 0;  // bit 9+d: date d valid (ring advances accumulated)
          load_yhat8(hf, yh);
#pragma unroll
          for (int d = 0; d < 8; ++d) yv[d] = Ys[(8 * hf + d) * 128 + tid];  // dates >= n read as NaN (hmap)
          float rs3[24];
#pragma unroll
          for (int d = 0; d < 8; ++d) {
            const float y = yv[d];
            const bool v = (y == y);
            const float r = v ? (y - c0) - yh[d] : 0.f;
            s2 = fmaf(r, r, s2);
            // exact 3-way bf16 split by truncation: r = rh + rm + rl
            const float rh = bf16_trunc(r), t1 = r - rh, rm = bf16_trunc(t1);
            rs3[3 * d] = rh;
            rs3[3 * d + 1] = rm;
            rs3[3 * d + 2] = t1 - rm;
            const uint32_t inc = v ? C::RSLOT : 0u;
            sts_f32_inc(wa, r, inc);
            m8 += inc << d;
            wa += inc;
            wa = (wa == rend) ? rbase : wa;
          }
          static_assert(C::RSLOT == 512, "m8 packs the advances as bit 9 + d");
          cr += __popc(m8);
          vm |= (m8 >> 9) << (8 * hf);
#pragma unroll
          for (int q = 0; q < 3; ++q)
            *reinterpret_cast<uint4 *>(ob + sm100::kmajor_off(tid, 24 * hf + 8 * q, 128)) =
                make_uint4(pack_hi16(rs3[8 * q], rs3[8 * q + 1]), pack_hi16(rs3[8 * q + 2], rs3[8 * q + 3]),
                           pack_hi16(rs3[8 * q + 4], rs3[8 * q + 5]), pack_hi16(rs3[8 * q + 6], rs3[8 * q + 7]));
        }
        sts_u16(vbase + c * C::VSLOT, (uint16_t)vm);
        release_yhat();
        warp_arrive(a_yempty + 8 * ys);  // every loaded value has been consumed
        opbuf_publish();
        yadvance();
      }
      sm100::mbar_wait_a(a_accready, acnt & 1);
      ++acnt;
      sm100::tc_fence_after();

      // ================= refinement: beta = beta0 + A^-1 db; sigma-hat
      float sigma, dbf[K];
      {
        float db[K], Dd[C::KB3];
#pragma unroll
        for (int q = 0; q < C::KB3 / 16; ++q) {
          float v16[16];
          sm100::tmem_ld16(lanebase + C::COL_DB + 16 * q, v16);
          sm100::tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 16; ++i) Dd[16 * q + i] = v16[i];
        }
#pragma unroll
        for (int i = 0; i < K; ++i) db[i] = Dd[i] + Dd[K + i] + Dd[2 * K + i];
        chol_solve<K, float>(A, db, dbf);
        float lin = 0.f;
#pragma unroll
        for (int i = 0; i < K; ++i) {
          if (deg) dbf[i] = 0.f;
          lin = fmaf(dbf[i], db[i], lin);
          beta[i] += dbf[i];
        }
        sigma = sqrtf(fmaxf(s2 - lin, 0.f) / (float)(nbar - K));
        // sigma^2 = s2 - lin cancels when the refinement step is large next to
        // the residual sum: the fp32 sigma-hat is then unreliable -> fp64 refit
        if (!(lin <= 1e-2f * s2)) {
          refit = true;
          BFAST_WHY(0x20);
        }
      }
      if (!deg && !(sigma > 1e-4f * ymax)) deg = true;
      // noise within 2e-3 of the signal scale: fp32 fitted values (~1e-7 |y|)
      // are no longer negligible next to sigma-hat -> fp64 refit (R12)
      if (!deg && !(sigma > 2e-3f * ymax)) {
        refit = true;
        BFAST_WHY(0x40);
      }
      const float inv_scale = 1.0f / (sigma * sqrtf((float)nbar));
      sm100::tc_fence_before();
      write_beta_operand(beta, 0.f);
      // MOSUM seed (m^fst, L518): the last h-1 history residuals, corrected
      // to the refined fit.  ra = slot of rank cr - hh (the next to drop).
      float W = 0.f;
      uint32_t ra;
      {
        // walk back from the newest history residual; its date is the
        // highest set bit of the chunk masks (scanned from the last chunk)
        const int nseed = deg ? 0 : hh - 1;
        uint32_t a = wa;
        int cm = nch;
        uint32_t bits = 0;
        for (int q = 0; q < nseed; ++q) {
          a = (a == rbase ? rend : a) - C::RSLOT;
          while (bits == 0 && cm > 0) bits = (uint32_t)lds_u16(vbase + (--cm) * C::VSLOT);
          const int d = 31 - __clz(bits);
          bits ^= 1u << d;
          const int t = cm * C::DC + d;
          const float *xr = p.X + (size_t)t * p.KP;
          float corr = 0.f;
#pragma unroll
          for (int i = 0; i < K; i += 2) {
            const float2 xx = __ldg(reinterpret_cast<const float2 *>(xr + i));
            corr = fmaf(dbf[i], xx.x, corr);
            corr = fmaf(dbf[i + 1], xx.y, corr);
          }
          const float r = lds_f32(a) - corr;
          sts_f32(a, r);
          W += r;
        }
        ra = (a == rbase ? rend : a) - C::RSLOT;  // rank cr - hh
        if (deg) ra = wa;
        // the window of j = 0 drops nothing: the slot of rank nbar - h (or
        // the write slot for invalid pixels) reads as 0 at the first step
        sts_f32(ra, 0.f);
      }

      // ================= pass 2b: monitoring (Alg. 1 l.6-12, Fig. 12 ker 9-10)
      float msum = 0.f, mfirst = 0.f;
      int brk = -1, first = -1;
      bool tie = false;
      // largest 1-based rank with B == lambda (rank/nbar <= e), evaluated with
      // the exact boundary formula around floor(e * nbar)
      int rank_flat;
      {
        int r0 = (int)(2.718281828f * (float)nbar) - 2;
        r0 = r0 < 0 ? 0 : r0;
        rank_flat = r0;
#pragma unroll
        for (int q = 1; q <= 4; ++q)
          if (nbar > 0 && boundary_f32(p.lambda, r0 + q, nbar) == p.lambda) rank_flat = r0 + q;
      }
      const float lam = p.lambda, lam_lo = lam * (1.0f - kTieTol), lam_hi = lam * (1.0f + kTieTol);
      for (int c = 0; c < ncm; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        wait_yhat();
        const float *Ys = reinterpret_cast<const float *>(ystages + ys * C::YBYTES);
        // B_j == lambda for every rank this chunk can reach (rank/nbar <= e):
        // warp-uniform fast path without the out-of-line boundary evaluation
        const bool fast = __all_sync(0xffffffffu, deg || cr + C::DC <= rank_flat);
        if (first >= 0 && brk < 0 && !tie) {  // resolve a fast-path candidate
          const float am = fabsf(mfirst);
          if (am > lam_hi) brk = first;
          else tie = true;
        }
#pragma unroll 1
        for (int hf = 0; hf < 2; ++hf) {
          float yh[8], yv[8];
          load_yhat8(hf, yh);
#pragma unroll
          for (int d = 0; d < 8; ++d) yv[d] = Ys[(8 * hf + d) * 128 + tid];  // dates >= N read as NaN (TMA OOB)
          if (fast) {
            uint32_t adv = 0;  // ring bytes advanced = valid dates * RSLOT
#pragma unroll
            for (int d = 0; d < 8; ++d) {
              const float y = yv[d];
              const bool v = (y == y);
              const float r = (y - c0) - yh[d];
              const float old = lds_f32(ra);  // rank cr - h (zeroed phantom at j = 0)
              const uint32_t inc = v ? C::RSLOT : 0u;
              sts_f32_inc(wa, r, inc);
              wa += inc;
              ra += inc;
              adv += inc;
              wa = (wa == rend) ? rbase : wa;
              ra = (ra == rend) ? rbase : ra;
              if (v) W += r - old;
              const float m = W * inv_scale;
              if (v) msum += m;
              // B_j == lambda here: the first |m| > lambda(1 - tol) decides --
              // a clear crossing is the break, a near tie goes to the fp64 refit
              const bool cand = v && first < 0 && fabsf(m) > lam_lo;
              first = cand ? c * C::DC + 8 * hf + d : first;
              mfirst = cand ? m : mfirst;
            }
            cr += adv >> 9;
          } else {
#pragma unroll
            for (int d = 0; d < 8; ++d) {
              const float y = yv[d];
              const bool v = (y == y);
              const float r = (y - c0) - yh[d];
              const float old = lds_f32(ra);
              sts_f32_inc(wa, r, v ? C::RSLOT : 0u);
              const uint32_t wn = wa + C::RSLOT, rn = ra + C::RSLOT;
              wa = v ? (wn == rend ? rbase : wn) : wa;
              ra = v ? (rn == rend ? rbase : rn) : ra;
              W = v ? W + (r - old) : W;
              const float m = W * inv_scale;
              msum += v ? m : 0.f;
              if (v && brk < 0 && !tie && first < 0 && fabsf(m) > lam_lo) {
                const int code = boundary_rare(m, cr + 1, nbar, lam);
                tie = tie || (code >> 1);
                brk = (code & 1) ? c * C::DC + 8 * hf + d : brk;
              }
              cr += v;
            }
          }
        }
        release_yhat();
        warp_arrive(a_yempty + 8 * ys);  // every loaded value has been consumed
        yadvance();
      }
      if (first >= 0 && brk < 0 && !tie) {
        if (fabsf(mfirst) > lam_hi) brk = first;
        else tie = true;
      }
      const int Nbar = cr;
      if (Nbar - nbar < 1) deg = true;

      // ================= epilogue
      const bool fit_ok = !((nbar < K + 1) || (h < 1) || (Nbar - nbar < 1));
      const bool inside = pix < p.p0 + p.P;  // the last tile may be ragged
      if (inside) {
        p.out_break[pix] = deg ? -2 : brk;
        p.out_mag[pix] = deg ? qnan : msum / (float)(Nbar - nbar);
        if (p.out_sigma) p.out_sigma[pix] = fit_ok ? sigma : qnan;
        if (p.out_nbar) p.out_nbar[pix] = nbar;
#ifdef BFAST_REFIT_WHY
        if (p.out_flags) p.out_flags[pix] = (deg ? 1u : 0u) | why | (tie ? 0x80u : 0u);
#else
        if (p.out_flags) p.out_flags[pix] = deg ? 1u : 0u;
#endif
        store_beta<K, float>(p, pix, beta, c0, fit_ok);
      }
      const bool want = (refit || tie) && fit_ok && inside;
      const unsigned mask = __ballot_sync(0xffffffffu, want);
      if (want) {
        const int leader = __ffs(mask) - 1;
        int base = 0;
        if (lane == leader) base = atomicAdd(p.refit_count, __popc(mask));
        base = __shfl_sync(mask, base, leader);
        p.refit_list[base + __popc(mask & ((1u << lane) - 1))] = (int32_t)pix;
      }
    }
  }
  sm100::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    sm100::tc_fence_after();
    sm100::tmem_dealloc(tbase, C::TMEM_COLS);
  }
}

}  // namespace bfast
