// monitor_tc.cuh -- BFAST-Monitor hot path on the 5th-generation tensor cores.
//
// Same algorithm and numerics contract as monitor_simt.cuh (Algorithm 1,
// PAPER.md L134; Fig. 12), re-mapped so that every contraction
// shared by a 128-pixel tile runs as a tcgen05.mma with fp32 accumulators
// in Tensor Memory, and the CUDA cores only do per-(pixel, date) scalar
// work, as little of it as the method allows:
//
//   masked Gram  A = sum_t v_t x_t x_t^T  (Alg. 1 l.2, Fig. 4)
//       The K(K+1)/2 entries are linear in NF = 2+6k masked moments
//       sum_t v_t f_q(t) of the functions f = {tau, tau^2, tau sin_j,
//       tau cos_j, sin_m, cos_m (m <= 2k)} (product-to-sum identities), so
//       the tile's Gram is D_G[128 x NF] += V[128 x 16] * F_e[16 x NF],
//       e = hi, mid, lo (three MMAs on the same exact 0/1 mask operand V;
//       F split in three bf16 parts: the products are exact, the Gram
//       carries fp32 accumulation error only).
//   moment b = sum_t v_t y'_t x_t  (Alg. 1 l.4): y' = y - c (c = the pixel's
//       first valid value) is split exactly in three bf16 parts by
//       truncation and x in three rounded parts; the six cross terms above
//       2^-24 are six MMAs into D_b[128 x K].
//   Gram and moment alternate between two TMEM accumulator sets (even / odd
//       chunks), which halves the fp32 accumulation error (DESIGN.md
//       "Numerics"); the solve adds the two sets.
//   yhat' = X beta (Fig. 12 ker 6) of the offset data y - c: D_y[128 x 16
//       dates] = [beta hi/mid/lo] * [x hi/mid/lo] with the 6 cross terms of a
//       3-way bf16 split (~24-bit accuracy, fp32 accumulate).
//
// Roles (256 threads): warps 0-3 own one pixel per thread (TMEM lane =
// pixel row); warp 4 streams 16-date x 128-pixel boxes of the time-major
// stack (one 2-D TMA copy each) into a ring the consumer warps release as
// soon as they have read a box; warp 5 streams the chunk's B-operand tables
// (one 1-D bulk copy each, L2-resident) into a ring released by
// tcgen05.commit of the MMAs that read them; warp 6 issues every
// tcgen05.mma; warp 7 idles.  All hand-offs are mbarriers (per-warp
// arrivals), so no warp waits at a CTA-wide barrier inside the date loops.
//
// Per tile the chunk sequence is two sweeps:
//   pass 1, history chunks:  mask + y' operands -> Gram and moment (MMA)
//   solve:                   fp32 register Cholesky (Alg. 1 l.3-4)
//   pass 2, history chunks:  r = y - yhat, sigma-hat (L513-L515); the last h
//                            valid residuals land in a per-pixel ring of h
//                            slots (the MOSUM seed m^fst, L518)
//   pass 2, monitoring:      r, MOSUM recurrence over the ring (the slot
//                            about to be overwritten holds rank c-h),
//                            boundary, first break, mean (L520-L537)
// The stack is read through a 2-D TMA tensor map whose out-of-bounds fill is
// NaN, so a ragged last tile needs no special case (its missing pixels are
// "all missing").
#pragma once
#include "monitor_simt.cuh"
#include "sm100.cuh"
#include <cuda.h>

namespace bfast {

// CTA = consumer warpgroup (warps 0-3, PX pixels per thread) + producer
// warpgroup (warp 4: stack boxes and chunk tables, warp 6: MMA issue).  At
// launch every thread holds LAUNCH_REGS registers (CTAS CTAs x 256 threads
// fill the register file); the producers drop to kTcAuxRegs, the consumers
// rise to CONSUMER_REGS (256 * LAUNCH_REGS = 128 * (kTcAuxRegs +
// CONSUMER_REGS)).
constexpr int kTcThreads = 256;
#ifndef BFAST_TC_AUX_REGS
#define BFAST_TC_AUX_REGS 32
#endif
constexpr int kTcAuxRegs = BFAST_TC_AUX_REGS;
// Pixels per consumer thread and CTAs per SM, per design width K.  K <= 8:
// one pixel per thread, 4 CTAs (16 consumer warps) per SM, 96 consumer
// registers; measured 1.5% faster than two pixels per thread at 2 CTAs per
// SM on the Landsat scene.  K >= 10 needs more registers per pixel (the
// K x K Cholesky): two pixels per thread, 2 CTAs, 224 registers.
// BFAST_TC_PX / BFAST_TC_CTAS override (experiments).
template <int K>
struct TcShape {
#ifdef BFAST_TC_PX
  static constexpr int PX = BFAST_TC_PX;
#else
  static constexpr int PX = K <= 8 ? 1 : 2;
#endif
#ifdef BFAST_TC_CTAS
  static constexpr int CTAS = BFAST_TC_CTAS;
#else
  static constexpr int CTAS = PX == 1 ? 4 : 2;
#endif
  static constexpr int LAUNCH_REGS = CTAS == 4 ? 64 : CTAS == 3 ? 80 : 128;
  static constexpr int CONSUMER_REGS = 2 * LAUNCH_REGS - kTcAuxRegs;
#ifdef BFAST_UNROLL_SEED
  static constexpr int UNROLL_SEED = BFAST_UNROLL_SEED;
#else
  static constexpr int UNROLL_SEED = 1;  // measured (2 was better before the TMEM operands)
#endif
};

// parts of the bf16 split of the first-fit residual r0 in the refinement
// moment (2: hi truncated + lo rounded, ~17 bits; 3: three truncated parts,
// exact -- measured magnitude error 2-5x lower for 2.7% more time)
#ifndef BFAST_R0_PARTS
#define BFAST_R0_PARTS 3
#endif
constexpr int kR0Parts = BFAST_R0_PARTS;
// release a chunk's stack stage and yhat slot as soon as the second half's
// values are in registers (1), or after the chunk's arithmetic (0)
#ifndef BFAST_EARLY_REL
#define BFAST_EARLY_REL 1
#endif
constexpr bool kEarlyRelease = BFAST_EARLY_REL != 0;
// TMEM slots for yhat = X beta of upcoming chunks (the MMA warp runs this
// many chunks ahead of the consumers in passes 2 and 3)
#ifndef BFAST_YS
#define BFAST_YS 2
#endif
constexpr int kYhatSlots = BFAST_YS;
// MMA A operands (mask / y' parts, r0 parts) written by the consumers into
// Tensor Memory with tcgen05.st (1) instead of shared memory (0), where the
// layout fits the CTA's TMEM allocation (one accumulator set then)
#ifndef BFAST_TMEM_OPS
#define BFAST_TMEM_OPS 1
#endif
constexpr bool kTmemOpsWanted = BFAST_TMEM_OPS != 0;
// unroll factors of the two 8-date halves of a chunk per sweep (1 keeps one
// copy of the hot code per sweep: instruction-cache footprint)
#ifndef BFAST_UNROLL_P1
#define BFAST_UNROLL_P1 1
#endif
constexpr int kUnrollP1 = BFAST_UNROLL_P1;
#ifndef BFAST_UNROLL_P2
#define BFAST_UNROLL_P2 2
#endif
constexpr int kUnrollP2 = BFAST_UNROLL_P2;
#ifndef BFAST_UNROLL_MON
#define BFAST_UNROLL_MON 1
#endif
constexpr int kUnrollMon = BFAST_UNROLL_MON;
// k-indexed ring slots in the seed pass too (the monitoring fast path always
// uses them when every pixel of the warp has h >= 8)
#ifndef BFAST_SEEDK
#define BFAST_SEEDK 1
#endif
constexpr bool kSeedK = BFAST_SEEDK != 0;

template <int K, int PX = TcShape<K>::PX>
struct TcCfg {
  static constexpr int k = (K - 2) / 2;
  static constexpr int NF = 2 + 6 * k;                     // masked moment functions
  static constexpr int NGn = ((NF + 1 + 15) / 16) * 16;    // Gram GEMM N (+ the constant 1: nbar)
  static constexpr int KBn = ((K + 15) / 16) * 16;         // moment GEMM N
  static constexpr int KY = ((6 * K + 15) / 16) * 16;      // yhat GEMM K
  static constexpr int DC = 16;                            // dates per chunk
  static constexpr int PIX = 128 * PX;                     // pixels per tile
  // TMEM columns (lane = consumer thread; a thread's PX pixels are the same
  // lane of PX column groups).  Pass 1: two accumulator sets [Gram | moment]
  // per pixel group; pass 2 (after the solve has read them): two yhat slots,
  // the beta operand (the A operand of the yhat GEMM, bf16 pairs) and the
  // refinement moment, per pixel group.
  static constexpr int SET = NGn + KBn;
  static constexpr int A3W = ((KY / 2 + 7) / 8) * 8;       // beta operand columns (8-column MMA steps)
  static constexpr int NYS = kYhatSlots;
  static constexpr int OPC = 3 * DC / 2;                   // three [128 x 16] bf16 A tiles, 8 columns each
  static constexpr int P2B = NYS * PX * DC + PX * A3W + PX * KBn;
  static constexpr __host__ __device__ int pow2cols(int c) {
    return c <= 32 ? 32 : c <= 64 ? 64 : c <= 128 ? 128 : c <= 256 ? 256 : 512;
  }
  // shared-memory operands: two accumulator sets; TMEM operands: one set and
  // two operand buffers per pass, taken where that fits the CTA's budget
  static constexpr int COLS_SMEM = pow2cols(2 * PX * SET > P2B ? 2 * PX * SET : P2B);
  static constexpr int P1T = PX * SET + 2 * PX * OPC, P2T = P2B + 2 * PX * OPC;
  // (the TMEM budget per CTA: 128 columns at 4 CTAs/SM for PX = 1, 256 at 2)
  static constexpr int TCAP = COLS_SMEM > 128 * PX ? COLS_SMEM : 128 * PX;
  static constexpr bool TOPS = kTmemOpsWanted && pow2cols(P1T > P2T ? P1T : P2T) <= TCAP;
  static constexpr int NSET = TOPS ? 1 : 2;
  static constexpr int COLS_P1 = TOPS ? P1T : 2 * PX * SET;
  static constexpr __host__ __device__ int col_set(int s, int q) { return (s * PX + q) * SET; }
  static constexpr __host__ __device__ int col_op1(int b, int q) { return PX * SET + (b * PX + q) * OPC; }
  static constexpr __host__ __device__ int col_y(int slot, int q) { return (slot * PX + q) * DC; }
  static constexpr __host__ __device__ int col_a3(int q) { return NYS * PX * DC + q * A3W; }
  static constexpr __host__ __device__ int col_db(int q) { return NYS * PX * DC + PX * A3W + q * KBn; }
  static constexpr __host__ __device__ int col_op2(int b, int q) { return P2B + (b * PX + q) * OPC; }
  static constexpr int COLS_P2 = TOPS ? P2T : P2B;
  static constexpr int COLS_USED = COLS_P1 > COLS_P2 ? COLS_P1 : COLS_P2;
  static constexpr int TMEM_COLS = pow2cols(COLS_USED);
  static constexpr int BF_BYTES = NGn * DC * 2;            // one part of the Gram table [NGn x 16]
  static constexpr int BX_BYTES = KBn * DC * 2;            // one part of x [KBn x 16]
  static constexpr int B3_BYTES = DC * KY * 2;             // yhat table [16 x KY]
  static constexpr int TAB1 = 3 * BF_BYTES + 2 * BX_BYTES; // pass 1 (history): F parts, x hi/mid
  static constexpr int TAB2 = B3_BYTES + 3 * BX_BYTES;     // pass 2 history: yhat table, x parts
  static constexpr int TABY = B3_BYTES;                    // pass 2 monitoring: yhat table
  static constexpr int TABMAX = TAB1 > TAB2 ? TAB1 : TAB2;
  static constexpr int YBYTES = DC * PIX * 4;              // one [16 dates x PIX px] box
  static constexpr int TSTAGE = ((TABMAX + 127) / 128) * 128;
  static constexpr int SY_MAX = 4;                         // stack ring stages (released on read)
  static constexpr int ST = NYS + 1 > 3 ? NYS + 1 : 3;     // table ring stages (released by MMA commit)
  static constexpr int ATILE = 128 * DC * 2;               // one [128 x 16] bf16 A tile (one pixel group)
  static constexpr int OPBUF = 3 * PX * ATILE;             // pass 1: mask, y'hi, y'lo; pass 2: r0 parts
  static constexpr int RSLOT = PIX * 4;                    // ring slot: one residual per pixel
  // sy stack stages, nop operand buffers (2: the consumers fill one while the
  // MMA reads the other) and, in the same bytes, the MOSUM ring of hcap slots
  // (the operands are dead once the refinement moment is accumulated, the
  // ring is dead once the tile's monitoring is done)
  static constexpr size_t smem_bytes(int hcap, int nch, int sy, int nop) {
    const size_t ob = TOPS ? 0 : (size_t)nop * OPBUF, rg = (size_t)hcap * RSLOT;
    return (size_t)sy * YBYTES + (size_t)ST * TSTAGE + ((ob > rg ? ob : rg) + 127) / 128 * 128 + 0 * nch;
  }
};

struct TcTables {
  const uint8_t *tab1, *tab2, *taby;  // per-chunk B operands, canonical K-major layout
  int nch, ncm;                       // history / monitoring chunks of 16 dates
  int sy, nop;                        // stack stages (2..4), operand buffers (1|2)
  int64_t ntiles;                     // 128-pixel tiles (the last may be ragged)
};

__device__ __forceinline__ void sts_f32(uint32_t a, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(a), "f"(v) : "memory");
}
__device__ __forceinline__ void sts_u16(uint32_t a, uint16_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "h"(v) : "memory");
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
// ---- per-date steps (inline PTX: the validity predicate never leaves the asm)
// Pass 1: vm = all-ones if y is a value (set.num), y' = (y - c) & vm (NaN -> 0),
// 2-way bf16 split of y' by truncation: y' = h + l (l exact in fp32; its bf16
// packing keeps 16 significant bits in all, enough for the first fit).
__device__ __forceinline__ void p1_date(float y, float c0, uint32_t &vm, float &h, float &l) {
  asm("{\n\t.reg .f32 yp;\n\t"
      "set.num.u32.f32 %0, %3, %3;\n\t"
      "sub.f32 yp, %3, %4;\n\t"
      "and.b32 yp, yp, %0;\n\t"
      "and.b32 %1, yp, 0xFFFF0000;\n\t"
      "sub.f32 %2, yp, %1;\n\t}"
      : "=r"(vm), "=f"(h), "=f"(l)
      : "f"(y), "f"(c0));
}
// Pass 2, history date: r0 = (y - c) - yhat0 (NaN if missing); if r0 is a
// value: s2 += r0^2 and bit BIT of vb is set; (h, l) = 2-way split of r0
// (0 when missing) for the refinement moment.
template <int BIT>
__device__ __forceinline__ void p2h_date(float y, float c0, float yh, float &s2, uint32_t &vb, float &h, float &l) {
  asm("{\n\t.reg .pred p;\n\t.reg .f32 r;\n\t"
      "sub.f32 r, %4, %5;\n\t"
      "sub.f32 r, r, %6;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %7;\n\t"
      "selp.f32 r, r, 0f00000000, p;\n\t"
      "and.b32 %2, r, 0xFFFF0000;\n\t"
      "sub.f32 %3, r, %2;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(h), "=f"(l)
      : "f"(y), "f"(c0), "f"(yh), "n"(1u << BIT));
}
// ... with a 3-way split of r0 by truncation (h + m + l exact)
template <int BIT>
__device__ __forceinline__ void p2h_date3(float y, float c0, float yh, float &s2, uint32_t &vb, float &h, float &m,
                                          float &l) {
  asm("{\n\t.reg .pred p;\n\t.reg .f32 r, t;\n\t"
      "sub.f32 r, %5, %6;\n\t"
      "sub.f32 r, r, %7;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %8;\n\t"
      "selp.f32 r, r, 0f00000000, p;\n\t"
      "and.b32 %2, r, 0xFFFF0000;\n\t"
      "sub.f32 t, r, %2;\n\t"
      "and.b32 %3, t, 0xFFFF0000;\n\t"
      "sub.f32 %4, t, %3;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(h), "=f"(m), "=f"(l)
      : "f"(y), "f"(c0), "f"(yh), "n"(1u << BIT));
}
// Seed date (history chunks re-read after the refinement): r = (y - c) -
// yhat with the final beta; if r is a value it enters the per-pixel ring of
// h slots at wa (wrap at rend back by hbytes).
template <int RSLOT>
__device__ __forceinline__ void seed_date(float y, float c0, float yh, uint32_t &wa, uint32_t rend, uint32_t hbytes) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r;\n\t"
      "sub.f32 r, %1, %2;\n\t"
      "sub.f32 r, r, %3;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "@p st.shared.f32 [%0], r;\n\t"
      "@p add.u32 %0, %0, %6;\n\t"
      "setp.ge.u32 q, %0, %4;\n\t"
      "@q sub.u32 %0, %0, %5;\n\t}"
      : "+r"(wa)
      : "f"(y), "f"(c0), "f"(yh), "r"(rend), "r"(hbytes), "n"(RSLOT)
      : "memory");
}
// seed_date with the k-indexed slot address of mon_date_k (below)
template <int RSLOT>
__device__ __forceinline__ void seed_date_k(float y, float c0, float yh, uint32_t &k, uint32_t wa, uint32_t jw,
                                            uint32_t hbytes) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r;\n\t.reg .u32 a;\n\t"
      "sub.f32 r, %1, %2;\n\t"
      "sub.f32 r, r, %3;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "mad.lo.u32 a, %0, %7, %4;\n\t"
      "setp.ge.u32 q, %0, %5;\n\t"
      "@q sub.u32 a, a, %6;\n\t"
      "@p st.shared.f32 [a], r;\n\t"
      "@p add.u32 %0, %0, 1;\n\t}"
      : "+r"(k)
      : "f"(y), "f"(c0), "f"(yh), "r"(wa), "r"(jw), "r"(hbytes), "n"(RSLOT)
      : "memory");
}
// Cholesky factorisation (Alg. 1 l.3, an SPD Gram) in fp32 with hardware
// reciprocal square roots: on return A holds L^T off the diagonal and dinv
// the reciprocal pivots 1/l_jj.  Returns the smallest pivot ratio d_j / A_jj
// (1 - R^2 of column j on the previous ones), the conditioning proxy of the
// refit trigger.  The iterative refinement absorbs the ~1 ulp of rsqrt.
template <int K>
__device__ __forceinline__ float chol_factor_rsq(float (&A)[Tri<K>::kN], float (&dinv)[K]) {
  float minratio = 1.f;
  SFor<0, K>::run([&](auto jc) {
    constexpr int j = decltype(jc)::value;
    float d = A[Tri<K>::idx(j, j)];
    SFor<0, j>::run([&](auto qc) {
      constexpr int q = decltype(qc)::value;
      d = fmaf(-A[Tri<K>::idx(q, j)], A[Tri<K>::idx(q, j)], d);
    });
    minratio = fminf(minratio, __fdividef(d, A[Tri<K>::idx(j, j)]));
    const float inv = rsqrtf(fmaxf(d, 1e-30f));
    dinv[j] = inv;
    SFor<j + 1, K>::run([&](auto ic) {
      constexpr int i = decltype(ic)::value;
      float t = A[Tri<K>::idx(j, i)];
      SFor<0, j>::run([&](auto qc) {
        constexpr int q = decltype(qc)::value;
        t = fmaf(-A[Tri<K>::idx(q, i)], A[Tri<K>::idx(q, j)], t);
      });
      A[Tri<K>::idx(j, i)] = t * inv;
    });
  });
  return minratio;
}
// Solve L L^T x = b with the factor of chol_factor_rsq.
template <int K>
__device__ __forceinline__ void chol_solve_rsq(const float (&L)[Tri<K>::kN], const float (&dinv)[K], const float (&b)[K],
                                               float (&x)[K]) {
  float z[K];
  SFor<0, K>::run([&](auto ic) {
    constexpr int i = decltype(ic)::value;
    float t = b[i];
    SFor<0, i>::run([&](auto qc) {
      constexpr int q = decltype(qc)::value;
      t = fmaf(-L[Tri<K>::idx(q, i)], z[q], t);
    });
    z[i] = t * dinv[i];
  });
  SForDown<0, K>::run([&](auto ic) {
    constexpr int i = decltype(ic)::value;
    float t = z[i];
    SFor<i + 1, K>::run([&](auto qc) {
      constexpr int q = decltype(qc)::value;
      t = fmaf(-L[Tri<K>::idx(i, q)], x[q], t);
    });
    x[i] = t * dinv[i];
  });
}
// Monitoring date (Eq. (4) recurrence, L520-L525): r = y - yhat; the ring
// slot at wa holds rank cr - h (`old`); if r is a value it replaces it,
// W += r - old, msum += W, cr += 1 and mx = max(mx, |W|).  r and old are
// returned for the exact replay of a half-chunk in which mx crossed.
template <int RSLOT>
__device__ __forceinline__ void mon_date(float y, float c0, float yh, float &W, float &msum, float &mx, int &cr,
                                         uint32_t &wa, uint32_t rend, uint32_t hbytes, float &r, float &old) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 t;\n\t"
      "sub.f32 %5, %7, %8;\n\t"
      "sub.f32 %5, %5, %9;\n\t"
      "setp.num.f32 p, %5, %5;\n\t"
      "ld.shared.f32 %6, [%4];\n\t"
      "@p st.shared.f32 [%4], %5;\n\t"
      "@p add.u32 %4, %4, %12;\n\t"
      "setp.ge.u32 q, %4, %10;\n\t"
      "@q sub.u32 %4, %4, %11;\n\t"
      "@p add.s32 %3, %3, 1;\n\t"
      "sub.f32 t, %5, %6;\n\t"
      "@p add.f32 %0, %0, t;\n\t"
      "@p add.f32 %1, %1, %0;\n\t"
      "abs.f32 t, %0;\n\t"
      "@p max.f32 %2, %2, t;\n\t}"
      : "+f"(W), "+f"(msum), "+f"(mx), "+r"(cr), "+r"(wa), "=f"(r), "=f"(old)
      : "f"(y), "f"(c0), "f"(yh), "r"(rend), "r"(hbytes), "n"(RSLOT)
      : "memory");
}
// mon_date with the slot addressed from the half's running count k instead
// of a pointer advanced date by date: a = wa + k*RSLOT, wrapped once when k
// reaches jw (slots left before the ring's end).  Only k += 1 is carried
// from date to date; every date's address is a fresh value, so a store does
// not hold up the next date's pointer arithmetic (write-after-read on the
// address register).  Needs h >= 8 (at most one wrap per 8-date half).
// wv = W after a valid date, 0 after a missing one (the crossing scan of a
// half reads these instead of replaying the half).
template <int RSLOT>
__device__ __forceinline__ void mon_date_k(float y, float c0, float yh, float &W, float &msum, float &mx, uint32_t &k,
                                           uint32_t wa, uint32_t jw, uint32_t hbytes, float &wv) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r, o, t;\n\t.reg .u32 a;\n\t"
      "sub.f32 r, %5, %6;\n\t"
      "sub.f32 r, r, %7;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "mad.lo.u32 a, %3, %11, %8;\n\t"
      "setp.ge.u32 q, %3, %9;\n\t"
      "@q sub.u32 a, a, %10;\n\t"
      "ld.shared.f32 o, [a];\n\t"
      "@p st.shared.f32 [a], r;\n\t"
      "@p add.u32 %3, %3, 1;\n\t"
      "sub.f32 t, r, o;\n\t"
      "@p add.f32 %0, %0, t;\n\t"
      "@p add.f32 %1, %1, %0;\n\t"
      "abs.f32 t, %0;\n\t"
      "@p max.f32 %2, %2, t;\n\t"
      "selp.f32 %4, %0, 0f00000000, p;\n\t}"
      : "+f"(W), "+f"(msum), "+f"(mx), "+r"(k), "=f"(wv)
      : "f"(y), "f"(c0), "f"(yh), "r"(wa), "r"(jw), "r"(hbytes), "n"(RSLOT)
      : "memory");
}
// producer-side waits with back-off so a waiting producer does not steal
// issue slots from the consumer warps of its SM sub-partition: MODE 0 =
// try_wait with a suspend hint, 1 = poll, N > 1 = poll with an N-ns sleep
// (__nanosleep(N) sleeps ~2N ns).  Measured on the Landsat config
// (tools/ab_bench.sh): producer 128 ns and MMA issuer 32 ns; polling and
// suspended waits are slower, longer producer sleeps delay the stack boxes.
#ifndef BFAST_AUX_WAIT
#define BFAST_AUX_WAIT 128
#endif
#ifndef BFAST_MMA_WAIT
#define BFAST_MMA_WAIT 32
#endif
template <int MODE>
__device__ __forceinline__ void mbar_wait_mode(uint32_t bar, uint32_t parity) {
  if (MODE == 0) {
    while (!sm100::mbar_try_wait_a_hint(bar, parity, 1000000u)) {
    }
  } else if (MODE == 1) {
    while (!sm100::mbar_try_wait_a(bar, parity)) {
    }
  } else {
    while (!sm100::mbar_try_wait_a(bar, parity)) __nanosleep(MODE);
  }
}
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  mbar_wait_mode<BFAST_AUX_WAIT>(bar, parity);
}
__device__ __forceinline__ void mbar_wait_mma(uint32_t bar, uint32_t parity) {
  mbar_wait_mode<BFAST_MMA_WAIT>(bar, parity);
}
// the rare branch of the boundary test (Alg. 1 l.10-12), kept out of line
// returns bit 0: |m| > B (a break), bit 1: |m|/B within kTieTol of 1
__device__ __noinline__ int boundary_rare(float m, int rank1, int nbar, float lam) {
  const float B = boundary_f32(lam, rank1, nbar);
  const float am = fabsf(m);
  return (am > B ? 1 : 0) | (fabsf(am - B) <= kTieTol * B ? 2 : 0);
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
__global__ void __launch_bounds__(kTcThreads, TcShape<K>::CTAS)
    monitor_tc_kernel(MonitorParams p, TcTables tb, const __grid_constant__ CUtensorMap ymap,
                      const __grid_constant__ CUtensorMap hmap) {
  constexpr int PX = TcShape<K>::PX;
  constexpr int UNROLL_SEED = TcShape<K>::UNROLL_SEED;
  using C = TcCfg<K, PX>;
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t yfull[C::SY_MAX], yempty[C::SY_MAX], tfull[C::ST], tempty[C::ST], opfull[2],
      opfree[2], yhfull[C::NYS], yhfree[C::NYS], accready, betaready, seedready;
  __shared__ uint32_t tmem_base_s;
  __shared__ int seed_slot[4];  // per consumer warp: first history chunk its MOSUM seed needs
  const int SY = tb.sy, NOP = C::TOPS ? 2 : tb.nop;
  uint8_t *ystages = smem;
  uint8_t *tstages = ystages + SY * C::YBYTES;
  uint8_t *opb = tstages + C::ST * C::TSTAGE;
  uint8_t *ring = opb;  // aliases the operand buffers (TcCfg::smem_bytes)
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
    }
    for (int i = 0; i < C::NYS; ++i) {
      sm100::mbar_init(&yhfull[i], 1);
      sm100::mbar_init(&yhfree[i], NCW);
    }
    sm100::mbar_init(&accready, 1);
    sm100::mbar_init(&betaready, NCW);
    sm100::mbar_init(&seedready, NCW);
    sm100::fence_mbar_init();
  }
  if (warp == 0) sm100::tmem_alloc(&tmem_base_s, C::TMEM_COLS);
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tbase = tmem_base_s;
  const int n = p.n, nch = tb.nch, ncm = tb.ncm;

  if (warp >= NCW) {
    // producer warpgroup: two single-thread roles (warp 4: stack boxes and
    // chunk tables; warp 6: MMA issue) need few registers; hand them to the
    // consumer warpgroup
    sm100::setmaxnreg_dec<kTcAuxRegs>();
    if (warp == 4) {
      // ------------------------------------------------------------ producer
      if (lane == 0) {
        // one 2-D TMA box [16 dates x PIX px] per chunk.  History chunks read
        // through `hmap` (dates >= n are out of bounds), monitoring chunks
        // through `ymap`; out-of-bounds elements arrive as NaN = missing.
        sm100::prefetch_tmap(&ymap);
        sm100::prefetch_tmap(&hmap);
        const uint64_t pol_first = sm100::policy_evict_first();
        // barrier and stage addresses held in registers (sm100::opaque)
        const uint32_t A_yfull = sm100::opaque(sm100::smem_u32(&yfull[0]));
        const uint32_t A_yempty = sm100::opaque(sm100::smem_u32(&yempty[0]));
        const uint32_t A_tfull = sm100::opaque(sm100::smem_u32(&tfull[0]));
        const uint32_t A_tempty = sm100::opaque(sm100::smem_u32(&tempty[0]));
        const uint32_t A_seed = sm100::opaque(sm100::smem_u32(&seedready));
        const uint32_t A_ys = sm100::opaque(sm100::smem_u32(ystages));
        const uint32_t A_ts = sm100::opaque(sm100::smem_u32(tstages));
        int ys = 0, ts = 0;
        uint32_t yph = 0, tph = 0, sph = 0;
        for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
          const int x0 = (int)(tile * C::PIX);
          // history twice (pass 1, pass 2: re-read from L2), then the seed
          // chunks [s0, nch) once the consumers have found s0, then monitoring;
          // each chunk's stack box and its B-operand tables (the two rings
          // advance over the same chunk sequence)
          int s0 = nch;
          for (int phase = 0; phase < 4; ++phase) {
            if (phase == 2) {
              mbar_wait_sleep(A_seed, sph);
              sph ^= 1;
              s0 = min(min(seed_slot[0], seed_slot[1]), min(seed_slot[2], seed_slot[3]));
            }
            const int cb = phase == 2 ? s0 : 0, ce = phase < 3 ? nch : ncm;
            // seed chunks only need the yhat part (the head) of their tab2 entry
            const uint32_t tabbytes = phase == 0 ? C::TAB1 : phase == 1 ? C::TAB2 : C::TABY;
            const uint32_t stride = phase == 0 ? C::TAB1 : phase < 3 ? C::TAB2 : C::TABY;
            const uint8_t *tabsrc = phase == 0 ? tb.tab1 : phase < 3 ? tb.tab2 : tb.taby;
            for (int c = cb; c < ce; ++c) {
              mbar_wait_sleep(A_yempty + 8 * ys, yph ^ 1);
              const uint32_t yst = A_ys + ys * C::YBYTES, yb = A_yfull + 8 * ys;
              sm100::mbar_arrive_expect_tx_a(yb, C::YBYTES);
              if (phase < 2)
                sm100::tma_load_2d_a(yst, &hmap, x0, c * C::DC, yb);  // read again later (L2)
              else
                sm100::tma_load_2d_hint_a(yst, phase == 2 ? &hmap : &ymap, x0, (phase == 2 ? 0 : n) + c * C::DC,
                                          yb, pol_first);  // last use
              if (++ys == SY) {
                ys = 0;
                yph ^= 1;
              }
              mbar_wait_sleep(A_tempty + 8 * ts, tph ^ 1);
              const uint32_t tb_ = A_tfull + 8 * ts;
              sm100::mbar_arrive_expect_tx_a(tb_, tabbytes);
              sm100::bulk_g2s_a(A_ts + ts * C::TSTAGE, tabsrc + (size_t)c * stride, tabbytes, tb_);
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
        const uint32_t idG = sm100::idesc_bf16_f32(128, C::NGn);
        const uint32_t idB = sm100::idesc_bf16_f32(128, C::KBn);
        const uint32_t idY = sm100::idesc_bf16_f32(128, C::DC);
        const uint32_t aop = sm100::opaque(sm100::smem_u32(opb)), tss = sm100::opaque(sm100::smem_u32(tstages));
        const uint32_t A_tfull = sm100::opaque(sm100::smem_u32(&tfull[0]));
        const uint32_t A_tempty = sm100::opaque(sm100::smem_u32(&tempty[0]));
        const uint32_t A_opfull = sm100::opaque(sm100::smem_u32(&opfull[0]));
        const uint32_t A_opfree = sm100::opaque(sm100::smem_u32(&opfree[0]));
        const uint32_t A_yhfull = sm100::opaque(sm100::smem_u32(&yhfull[0]));
        const uint32_t A_yhfree = sm100::opaque(sm100::smem_u32(&yhfree[0]));
        const uint32_t A_acc = sm100::opaque(sm100::smem_u32(&accready));
        const uint32_t A_beta = sm100::opaque(sm100::smem_u32(&betaready));
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
          mbar_wait_mma(A_opfull + 8 * ob, par);
          return ob;
        };
        // yhat of the chunk `ahead` chunks after the current one (its table
        // stage starts with the [16 x KY] yhat table), for every pixel group
        auto issue_yhat = [&](int ahead) {
          uint32_t par;
          const int s = tslot(ahead, par);
          const uint32_t slot = yissue % C::NYS;
          mbar_wait_mma(A_yhfree + 8 * slot, ((yissue / C::NYS) & 1) ^ 1);  // consumers done with the slot
          mbar_wait_mma(A_tfull + 8 * s, par);
          sm100::tc_fence_after();
          const uint32_t b3 = tss + s * C::TSTAGE;
#pragma unroll
          for (int q = 0; q < PX; ++q)
#pragma unroll
            for (int j = 0; j < C::KY / 16; ++j)
              sm100::umma_bf16_ts(tbase + C::col_y(slot, q), tbase + C::col_a3(q) + 8 * j,
                                  sm100::smem_desc(b3 + j * 2 * 256, 256, 128), idY, j > 0);
          sm100::umma_commit_a(A_yhfull + 8 * slot);
          ++yissue;
        };
        for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
          // pass 1: Gram + moment per chunk, accumulator set c & 1
          for (int c = 0; c < nch; ++c) {
            const uint32_t ob = opwait();
            mbar_wait_mma(A_tfull + 8 * ts, tph);
            sm100::tc_fence_after();
            const uint32_t bf = tss + ts * C::TSTAGE, bx = bf + 3 * C::BF_BYTES;
            const uint32_t first = c >= C::NSET ? 1u : 0u;
#pragma unroll
            for (int q = 0; q < PX; ++q) {
              const uint32_t dG = tbase + C::col_set(C::NSET == 2 ? (c & 1) : 0, q), dB = dG + C::NGn;
              if (C::TOPS) {
                const uint32_t at = tbase + C::col_op1(ob, q);  // mask, y' hi, y' lo tiles (TMEM)
#pragma unroll
                for (int e = 0; e < 3; ++e)
                  sm100::umma_bf16_ts(dG, at, sm100::smem_desc(bf + e * C::BF_BYTES, C::NGn * 16, 128), idG,
                                      first | (e > 0));
                sm100::umma_bf16_ts(dB, at + 8, sm100::smem_desc(bx, C::KBn * 16, 128), idB, first);
                sm100::umma_bf16_ts(dB, at + 8, sm100::smem_desc(bx + C::BX_BYTES, C::KBn * 16, 128), idB, 1);
                sm100::umma_bf16_ts(dB, at + 16, sm100::smem_desc(bx, C::KBn * 16, 128), idB, 1);
                continue;
              }
              const uint32_t am = aop + ob * C::OPBUF + q * 3 * C::ATILE;  // mask, y' hi, y' lo tiles
#pragma unroll
              for (int e = 0; e < 3; ++e)
                sm100::umma_bf16(dG, sm100::smem_desc(am, 2048, 128),
                                 sm100::smem_desc(bf + e * C::BF_BYTES, C::NGn * 16, 128), idG, first | (e > 0));
              // y'hi x_hi, y'hi x_mid, y'lo x_hi
              sm100::umma_bf16(dB, sm100::smem_desc(am + C::ATILE, 2048, 128),
                               sm100::smem_desc(bx, C::KBn * 16, 128), idB, first);
              sm100::umma_bf16(dB, sm100::smem_desc(am + C::ATILE, 2048, 128),
                               sm100::smem_desc(bx + C::BX_BYTES, C::KBn * 16, 128), idB, 1);
              sm100::umma_bf16(dB, sm100::smem_desc(am + 2 * C::ATILE, 2048, 128),
                               sm100::smem_desc(bx, C::KBn * 16, 128), idB, 1);
            }
            sm100::umma_commit_a(A_opfree + 8 * ob);
            sm100::umma_commit_a(A_tempty + 8 * ts);
            if (c == nch - 1) sm100::umma_commit_a(A_acc);
            ++opcnt;
            tadvance();
          }
          // pass 2, history: yhat0 two chunks ahead, refinement moment per chunk
          mbar_wait_mma(A_beta, bcnt & 1);
          ++bcnt;
          for (int a = 0; a < C::NYS && a < nch; ++a) issue_yhat(a);
          for (int c = 0; c < nch; ++c) {
            const uint32_t ob = opwait();
            mbar_wait_mma(A_tfull + 8 * ts, tph);
            sm100::tc_fence_after();
            const uint32_t bx = tss + ts * C::TSTAGE + C::B3_BYTES;
#pragma unroll
            for (int q = 0; q < PX; ++q) {
              const uint32_t am = aop + ob * C::OPBUF + q * 3 * C::ATILE;  // r0 parts
              const uint32_t at = tbase + C::col_op2(ob, q);                // (TMEM)
              const uint32_t dD = tbase + C::col_db(q);
              // r0hi (x_hi + x_mid + x_lo) + r0mid (x_hi + x_mid) + r0lo x_hi
#pragma unroll
              for (int e = 0; e < kR0Parts; ++e)
#pragma unroll
                for (int x = 0; x < 3 - e; ++x) {
                  const uint64_t bd = sm100::smem_desc(bx + x * C::BX_BYTES, C::KBn * 16, 128);
                  const uint32_t acc = (c > 0 || e > 0 || x > 0) ? 1u : 0u;
                  if (C::TOPS)
                    sm100::umma_bf16_ts(dD, at + 8 * e, bd, idB, acc);
                  else
                    sm100::umma_bf16(dD, sm100::smem_desc(am + e * C::ATILE, 2048, 128), bd, idB, acc);
                }
            }
            sm100::umma_commit_a(A_opfree + 8 * ob);
            if (c + C::NYS < nch) issue_yhat(C::NYS);
            sm100::umma_commit_a(A_tempty + 8 * ts);
            if (c == nch - 1) sm100::umma_commit_a(A_acc);
            ++opcnt;
            tadvance();
          }
          // pass 3, seed chunks + monitoring: yhat with the refined beta, two
          // chunks ahead (the consumers published s0 before betaready)
          mbar_wait_mma(A_beta, bcnt & 1);
          ++bcnt;
          const int s0 = min(min(seed_slot[0], seed_slot[1]), min(seed_slot[2], seed_slot[3]));
          const int n3 = nch - s0 + ncm;
          for (int a = 0; a < C::NYS && a < n3; ++a) issue_yhat(a);
          for (int c = 0; c < n3; ++c) {
            if (c + C::NYS < n3) issue_yhat(C::NYS);
            sm100::umma_commit_a(A_tempty + 8 * ts);  // chunk c's table was read by its yhat MMA
            tadvance();
          }
        }
      }
    }  // warp 7 idles: it completes the producer warpgroup
  } else {
    // ------------------------------------------------------------ consumers
    // Thread t owns pixels PX*t .. PX*t + PX-1 of the tile (adjacent: one
    // 8-byte shared load per date reads both); pixel group q = t's q-th
    // pixel, i.e. TMEM lane t of the column groups of q and row t of the A
    // tiles of q.
    sm100::setmaxnreg_inc<TcShape<K>::CONSUMER_REGS>();
    const uint32_t lanebase = tbase + ((uint32_t)(32 * warp) << 16);
    const float qnan = __int_as_float(0x7fc00000);
    // ring: slot s = PIX residuals f32, pixel q of this thread at rbase + 4q + s*RSLOT
    const uint32_t rbase = sm100::opaque(sm100::smem_u32(ring) + 4 * PX * tid);
    int ys = 0;
    uint32_t yph = 0, opcnt = 0, yuse = 0, acnt = 0;
    // 32-bit shared addresses of the barriers this warp waits on / arrives at
    // (sm100::opaque: kept in registers, not recomputed from the CTA's cluster rank)
    const uint32_t a_yfull = sm100::opaque(sm100::smem_u32(&yfull[0]));
    const uint32_t a_yempty = sm100::opaque(sm100::smem_u32(&yempty[0]));
    const uint32_t a_opfull = sm100::opaque(sm100::smem_u32(&opfull[0]));
    const uint32_t a_opfree = sm100::opaque(sm100::smem_u32(&opfree[0]));
    const uint32_t a_yhfull = sm100::opaque(sm100::smem_u32(&yhfull[0]));
    const uint32_t a_yhfree = sm100::opaque(sm100::smem_u32(&yhfree[0]));
    const uint32_t a_accready = sm100::opaque(sm100::smem_u32(&accready));
    const uint32_t a_betaready = sm100::opaque(sm100::smem_u32(&betaready));
    const uint32_t a_ystages = sm100::opaque(sm100::smem_u32(ystages));

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
      if (C::TOPS) {
        sm100::tmem_st_wait();  // this warp's operand rows are in TMEM
        sm100::tc_fence_before();
      } else {
        sm100::fence_proxy_async_smem();
      }
      warp_arrive(a_opfull + 8 * ob);
      ++opcnt;
    };
    // this thread's row of the three operand tiles of buffer `opcnt & 1`,
    // dates 8 hf .. 8 hf + 7 (4 columns of bf16 pairs per tile)
    auto tmem_ops = [&](uint32_t col, int hf, const uint32_t (&w)[3][4]) {
#pragma unroll
      for (int e = 0; e < 3; ++e) sm100::tmem_st4(lanebase + col + 8 * e + 4 * hf, w[e][0], w[e][1], w[e][2], w[e][3]);
    };
    // A3 rows (TMEM) = [bh | bh | bh | bm | bm | bl | 0...] (6 blocks of K, KY bf16) per pixel group
    auto write_beta_operand = [&](const float (&bt)[PX][K]) {
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        float h[K], m[K], l[K];
#pragma unroll
        for (int i = 0; i < K; ++i) {
          h[i] = bf16_round(bt[q][i]);
          m[i] = bf16_round(bt[q][i] - h[i]);
          l[i] = bt[q][i] - h[i] - m[i];
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
        for (int j = 0; j < C::KY / 16; ++j) {
          uint32_t w8[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) w8[i] = w[8 * j + i];
          sm100::tmem_st8(lanebase + C::col_a3(q) + 8 * j, w8);  // this pixel's row of the A operand
        }
      }
      sm100::tmem_st_wait();
      sm100::tc_fence_before();
      warp_arrive(a_betaready);
    };
    auto wait_yhat = [&]() {
      sm100::mbar_wait_a(a_yhfull + 8 * (yuse % C::NYS), (yuse / C::NYS) & 1);
      sm100::tc_fence_after();
    };
    auto load_yhat8 = [&](int half, float (&yh)[PX][8]) {
#pragma unroll
      for (int q = 0; q < PX; ++q) sm100::tmem_ld8(lanebase + C::col_y(yuse % C::NYS, q) + 8 * half, yh[q]);
      sm100::tmem_ld_wait();
    };
    auto release_yhat = [&]() {
      sm100::tc_fence_before();
      warp_arrive(a_yhfree + 8 * (yuse % C::NYS));
      ++yuse;
    };
    // the 8 dates of a half chunk for this thread's pixels: yv[q][d]
    // Ys = shared address of the stage (a register, see a_yfull)
    auto load_y8 = [&](uint32_t Ys, int hf, float (&yv)[PX][8]) {
      const uint32_t a = Ys + 4 * (8 * hf * C::PIX + PX * tid);
#pragma unroll
      for (int d = 0; d < 8; ++d) {
        if (PX == 2) {
          asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];"
                       : "=f"(yv[0][d]), "=f"(yv[PX - 1][d])
                       : "r"(a + 4 * d * C::PIX)
                       : "memory");
        } else {
          yv[0][d] = lds_f32(a + 4 * d * C::PIX);
        }
      }
    };

    for (int64_t tile = blockIdx.x; tile < tb.ntiles; tile += gridDim.x) {
      const int64_t pix0 = p.p0 + tile * C::PIX + PX * tid;
      // the operand buffers reuse the ring's bytes: every consumer warp must
      // be done with the previous tile's monitoring before any writes them
      if (!C::TOPS) asm volatile("bar.sync 1, 128;" ::: "memory");
      // ================= pass 1: masked Gram + moment on the tensor cores
      float c0[PX], ymax[PX];
      bool have[PX];
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        c0[q] = qnan;
        ymax[q] = 0.f;
        have[q] = false;
      }
      for (int c = 0; c < nch; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        const uint32_t Ys = a_ystages + ys * C::YBYTES;
        // offset c = first valid value (warp-uniform pre-scan while a lane lacks it)
        bool need = false;
#pragma unroll
        for (int q = 0; q < PX; ++q) need = need || !have[q];
        if (__any_sync(0xffffffffu, need)) {
#pragma unroll
          for (int q = 0; q < PX; ++q)
            for (int d = 0; d < C::DC && !have[q]; ++d) {
              const float y = lds_f32(Ys + 4 * (d * C::PIX + PX * tid + q));
              if (y == y) {
                c0[q] = y;
                have[q] = true;
              }
            }
        }
        uint8_t *ob = nullptr;
#pragma unroll kUnrollP1
        for (int hf = 0; hf < 2; ++hf) {  // two halves of 8 dates: half the hot code
          float yv[PX][8];
          load_y8(Ys, hf, yv);  // dates >= n read as NaN (hmap)
          if (kEarlyRelease && hf == 1) {  // the chunk's stack values are all in registers
            warp_arrive(a_yempty + 8 * ys);
            yadvance();
          }
          uint32_t vm[PX][8];
          float ph[PX][8], pl[PX][8];
#pragma unroll
          for (int q = 0; q < PX; ++q)
#pragma unroll
            for (int d = 0; d < 8; ++d) {
              ymax[q] = fmaxf(ymax[q], fabsf(yv[q][d]));  // NaN ignored
              p1_date(yv[q][d], c0[q], vm[q][d], ph[q][d], pl[q][d]);
            }
          // the MMA of the previous chunk frees the operand buffer while the
          // first half is computed
          if (hf == 0) ob = opbuf_acquire();
          if (C::TOPS) {
#pragma unroll
            for (int q = 0; q < PX; ++q) {
              const uint32_t w[3][4] = {
                  {(vm[q][0] & 0x3F80u) | (vm[q][1] & 0x3F800000u), (vm[q][2] & 0x3F80u) | (vm[q][3] & 0x3F800000u),
                   (vm[q][4] & 0x3F80u) | (vm[q][5] & 0x3F800000u), (vm[q][6] & 0x3F80u) | (vm[q][7] & 0x3F800000u)},
                  {pack_hi16(ph[q][0], ph[q][1]), pack_hi16(ph[q][2], ph[q][3]), pack_hi16(ph[q][4], ph[q][5]),
                   pack_hi16(ph[q][6], ph[q][7])},
                  {pack_hi16(pl[q][0], pl[q][1]), pack_hi16(pl[q][2], pl[q][3]), pack_hi16(pl[q][4], pl[q][5]),
                   pack_hi16(pl[q][6], pl[q][7])}};
              tmem_ops(C::col_op1(opcnt & 1, q), hf, w);
            }
            continue;
          }
          const uint32_t off = sm100::kmajor_off(tid, 8 * hf, 128);
#pragma unroll
          for (int q = 0; q < PX; ++q) {
            uint8_t *oq = ob + q * 3 * C::ATILE;
            // mask pair words: bf16 1.0 (0x3F80) in each half whose date is valid
            *reinterpret_cast<uint4 *>(oq + off) = make_uint4(
                (vm[q][0] & 0x3F80u) | (vm[q][1] & 0x3F800000u), (vm[q][2] & 0x3F80u) | (vm[q][3] & 0x3F800000u),
                (vm[q][4] & 0x3F80u) | (vm[q][5] & 0x3F800000u), (vm[q][6] & 0x3F80u) | (vm[q][7] & 0x3F800000u));
            *reinterpret_cast<uint4 *>(oq + C::ATILE + off) =
                make_uint4(pack_hi16(ph[q][0], ph[q][1]), pack_hi16(ph[q][2], ph[q][3]),
                           pack_hi16(ph[q][4], ph[q][5]), pack_hi16(ph[q][6], ph[q][7]));
            *reinterpret_cast<uint4 *>(oq + 2 * C::ATILE + off) =
                make_uint4(pack_hi16(pl[q][0], pl[q][1]), pack_hi16(pl[q][2], pl[q][3]),
                           pack_hi16(pl[q][4], pl[q][5]), pack_hi16(pl[q][6], pl[q][7]));
          }
        }
        if (!kEarlyRelease) {
          warp_arrive(a_yempty + 8 * ys);  // every loaded value has been consumed
          yadvance();
        }
        opbuf_publish();
      }
      sm100::mbar_wait_a(a_accready, acnt & 1);
      ++acnt;
      sm100::tc_fence_after();

      // ================= solve (Alg. 1 l.3-4): Gram from the masked moments
      float A[PX][Tri<K>::kN], dinv[PX][K], beta[PX][K];
      int nbar[PX], h[PX];
      bool deg[PX], refit[PX];
#ifdef BFAST_REFIT_WHY
      uint32_t why[PX];  // diagnostics build: which trigger sent the pixel to the refit
#pragma unroll
      for (int q = 0; q < PX; ++q) why[q] = 0;
#define BFAST_WHY(q, b) why[q] |= (b)
#else
#define BFAST_WHY(q, b)
#endif
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        float b[K];
        {
          float G[C::NF + 1];  // moments, then the count of valid history dates
#pragma unroll
          for (int i = 0; i <= C::NF; ++i) G[i] = 0.f;
#pragma unroll
          for (int i = 0; i < K; ++i) b[i] = 0.f;
#pragma unroll
          for (int s = 0; s < C::NSET; ++s) {
            if (s == 1 && nch < 2) break;
#pragma unroll
            for (int j = 0; j < C::NGn / 16; ++j) {
              float v16[16];
              sm100::tmem_ld16(lanebase + C::col_set(s, q) + 16 * j, v16);
              sm100::tmem_ld_wait();
#pragma unroll
              for (int i = 0; i < 16; ++i)
                if (16 * j + i <= C::NF) G[16 * j + i] += v16[i];
            }
            {
              float v16[16];
              sm100::tmem_ld16(lanebase + C::col_set(s, q) + C::NGn, v16);
              sm100::tmem_ld_wait();
#pragma unroll
              for (int i = 0; i < K; ++i) b[i] += v16[i];
            }
          }
          nbar[q] = (int)G[C::NF];  // exact: a sum of 0/1 products in fp32
          const float nb = (float)nbar[q];
          auto Cf = [&](int m) -> float { return m == 0 ? nb : G[2 + 2 * C::k + 2 * ((m < 0 ? -m : m) - 1) + 1]; };
          auto Sf = [&](int m) -> float {
            return m == 0 ? 0.f : (m < 0 ? -G[2 + 2 * C::k + 2 * (-m - 1)] : G[2 + 2 * C::k + 2 * (m - 1)]);
          };
          float(&Aq)[Tri<K>::kN] = A[q];
          Aq[Tri<K>::idx(0, 0)] = nb;
          Aq[Tri<K>::idx(0, 1)] = G[0];
          Aq[Tri<K>::idx(1, 1)] = G[1];
#pragma unroll
          for (int j = 1; j <= C::k; ++j) {
            Aq[Tri<K>::idx(0, 2 * j)] = Sf(j);
            Aq[Tri<K>::idx(0, 2 * j + 1)] = Cf(j);
            Aq[Tri<K>::idx(1, 2 * j)] = G[2 + 2 * (j - 1)];
            Aq[Tri<K>::idx(1, 2 * j + 1)] = G[3 + 2 * (j - 1)];
#pragma unroll
            for (int jb = j; jb <= C::k; ++jb) {
              Aq[Tri<K>::idx(2 * j, 2 * jb)] = 0.5f * (Cf(j - jb) - Cf(j + jb));          // s_j s_jb
              Aq[Tri<K>::idx(2 * j + 1, 2 * jb + 1)] = 0.5f * (Cf(j - jb) + Cf(j + jb));  // c_j c_jb
              Aq[Tri<K>::idx(2 * j, 2 * jb + 1)] = 0.5f * (Sf(j + jb) + Sf(j - jb));      // s_j c_jb
              if (jb > j) Aq[Tri<K>::idx(2 * j + 1, 2 * jb)] = 0.5f * (Sf(jb + j) + Sf(jb - j));  // c_j s_jb
            }
          }
        }
        h[q] = window_h(nbar[q], p.hf);
        deg[q] = (nbar[q] < K + 1) || (h[q] < 1);
        refit[q] = false;
        const float minratio = chol_factor_rsq<K>(A[q], dinv[q]);
        chol_solve_rsq<K>(A[q], dinv[q], b, beta[q]);
        if (!deg[q] && !(minratio >= (float)kRefitRatio)) {
          refit[q] = true;
          BFAST_WHY(q, 0x10);
        }
        if (deg[q]) {
#pragma unroll
          for (int i = 0; i < K; ++i) beta[q][i] = 0.f;
        }
      }
      sm100::tc_fence_before();
      write_beta_operand(beta);

      // ================= pass 2, history: residuals r0 of the first fit,
      // sigma-hat sums, the refinement moment operand; and which chunk holds
      // the oldest residual of the MOSUM seed (rank nbar - h: the window of
      // the first monitoring date reaches back to rank nbar - h + 1)
      int hh[PX], ring_from[PX], cr[PX], sc[PX];
      float s2[PX];
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        hh[q] = deg[q] ? min(8, p.hcap) : h[q];  // a degenerate pixel's ring is never read
        ring_from[q] = nbar[q] - hh[q];
        s2[q] = 0.f;
        cr[q] = 0;     // valid history dates before the current chunk
        sc[q] = nch;   // first chunk holding a rank >= ring_from (nch: no seed needed)
      }
      for (int c = 0; c < nch; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        wait_yhat();
        const uint32_t Ys = a_ystages + ys * C::YBYTES;
        uint8_t *ob = nullptr;
        uint32_t vb[PX];  // validity of the chunk's 16 dates
#pragma unroll
        for (int q = 0; q < PX; ++q) vb[q] = 0;
#pragma unroll kUnrollP2
        for (int hf = 0; hf < 2; ++hf) {
          float yh[PX][8], yv[PX][8];
          load_yhat8(hf, yh);
          load_y8(Ys, hf, yv);  // dates >= n read as NaN (hmap)
          if (kEarlyRelease && hf == 1) {  // yhat slot and stack stage fully read
            release_yhat();
            warp_arrive(a_yempty + 8 * ys);
            yadvance();
          }
          float rh[PX][8], rm[PX][8], rl[PX][8];
#pragma unroll
          for (int q = 0; q < PX; ++q) {
            uint32_t v8 = 0;
            SFor<0, 8>::run([&](auto dc) {
              constexpr int d = decltype(dc)::value;
              if (kR0Parts == 3)
                p2h_date3<d>(yv[q][d], c0[q], yh[q][d], s2[q], v8, rh[q][d], rm[q][d], rl[q][d]);
              else
                p2h_date<d>(yv[q][d], c0[q], yh[q][d], s2[q], v8, rh[q][d], rl[q][d]);
            });
            vb[q] |= v8 << (8 * hf);
          }
          if (hf == 0) ob = opbuf_acquire();
          if (C::TOPS) {
            static_assert(!C::TOPS || kR0Parts == 3, "TMEM operands carry the 3-way r0 split");
#pragma unroll
            for (int q = 0; q < PX; ++q) {
              const uint32_t w[3][4] = {
                  {pack_hi16(rh[q][0], rh[q][1]), pack_hi16(rh[q][2], rh[q][3]), pack_hi16(rh[q][4], rh[q][5]),
                   pack_hi16(rh[q][6], rh[q][7])},
                  {pack_hi16(rm[q][0], rm[q][1]), pack_hi16(rm[q][2], rm[q][3]), pack_hi16(rm[q][4], rm[q][5]),
                   pack_hi16(rm[q][6], rm[q][7])},
                  {pack_hi16(rl[q][0], rl[q][1]), pack_hi16(rl[q][2], rl[q][3]), pack_hi16(rl[q][4], rl[q][5]),
                   pack_hi16(rl[q][6], rl[q][7])}};
              tmem_ops(C::col_op2(opcnt & 1, q), hf, w);
            }
            continue;
          }
          const uint32_t off = sm100::kmajor_off(tid, 8 * hf, 128);
#pragma unroll
          for (int q = 0; q < PX; ++q) {
            uint8_t *oq = ob + q * 3 * C::ATILE;
            *reinterpret_cast<uint4 *>(oq + off) =
                make_uint4(pack_hi16(rh[q][0], rh[q][1]), pack_hi16(rh[q][2], rh[q][3]),
                           pack_hi16(rh[q][4], rh[q][5]), pack_hi16(rh[q][6], rh[q][7]));
            if (kR0Parts == 3) {
              *reinterpret_cast<uint4 *>(oq + C::ATILE + off) =
                  make_uint4(pack_hi16(rm[q][0], rm[q][1]), pack_hi16(rm[q][2], rm[q][3]),
                             pack_hi16(rm[q][4], rm[q][5]), pack_hi16(rm[q][6], rm[q][7]));
              *reinterpret_cast<uint4 *>(oq + 2 * C::ATILE + off) =
                  make_uint4(pack_hi16(rl[q][0], rl[q][1]), pack_hi16(rl[q][2], rl[q][3]),
                             pack_hi16(rl[q][4], rl[q][5]), pack_hi16(rl[q][6], rl[q][7]));
            } else {
              // r0 = hi (truncated, exact) + lo (rounded to nearest: unbiased)
              *reinterpret_cast<uint4 *>(oq + C::ATILE + off) =
                  make_uint4(sm100::pack_bf16x2(rl[q][0], rl[q][1]), sm100::pack_bf16x2(rl[q][2], rl[q][3]),
                             sm100::pack_bf16x2(rl[q][4], rl[q][5]), sm100::pack_bf16x2(rl[q][6], rl[q][7]));
            }
          }
        }
#pragma unroll
        for (int q = 0; q < PX; ++q) {
          cr[q] += __popc(vb[q]);
          if (sc[q] == nch && !deg[q] && cr[q] > ring_from[q]) sc[q] = c;
        }
        if (!kEarlyRelease) {
          release_yhat();
          warp_arrive(a_yempty + 8 * ys);  // every loaded value has been consumed
          yadvance();
        }
        opbuf_publish();
      }
      // the tile's seed chunks start at the smallest sc: publish this warp's
      int scm = sc[0];
#pragma unroll
      for (int q = 1; q < PX; ++q) scm = min(scm, sc[q]);
      const int sw = __reduce_min_sync(0xffffffffu, scm);
      if (lane == 0) {
        seed_slot[warp] = sw;
        sm100::mbar_arrive_a(sm100::smem_u32(&seedready));
      }
      sm100::mbar_wait_a(a_accready, acnt & 1);
      ++acnt;
      sm100::tc_fence_after();

      // ================= refinement: beta = beta0 + A^-1 db; sigma-hat
      float sigma[PX], scale[PX], inv_scale[PX];
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        float db[K], dbf[K];
        {
          float v16[16];
          sm100::tmem_ld16(lanebase + C::col_db(q), v16);
          sm100::tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < K; ++i) db[i] = v16[i];
        }
        chol_solve_rsq<K>(A[q], dinv[q], db, dbf);
        float lin = 0.f;
#pragma unroll
        for (int i = 0; i < K; ++i) {
          if (deg[q]) dbf[i] = 0.f;
          lin = fmaf(dbf[i], db[i], lin);
          beta[q][i] += dbf[i];
        }
        // sigma^2 (nbar - K) = sum (r0 - x dbeta)^2 = s2 - dbeta . db (A dbeta = db)
        sigma[q] = sqrtf(fmaxf(s2[q] - lin, 0.f) / (float)(nbar[q] - K));
        // sigma^2 cancels when the refinement step is large next to the
        // residual sum: the fp32 sigma-hat is then unreliable -> fp64 refit
        if (!(lin <= 1e-2f * s2[q])) {
          refit[q] = true;
          BFAST_WHY(q, 0x20);
        }
        // noise within 2e-3 of the signal scale: fp32 fitted values (~1e-7 |y|)
        // are no longer negligible next to sigma-hat -> fp64 refit (R12)
        if (!deg[q] && !(sigma[q] > 2e-3f * ymax[q])) {
          refit[q] = true;
          BFAST_WHY(q, 0x40);
        }
        scale[q] = sigma[q] * sqrtf((float)nbar[q]);  // MOSUM = W / scale (L524)
        inv_scale[q] = 1.0f / scale[q];
      }
      sm100::tc_fence_before();
      write_beta_operand(beta);

      // ================= pass 3, seed: the history chunks [s0, nch) again,
      // residuals of the refined fit into the per-pixel ring of h slots.  The
      // slot about to be written always holds rank cr - h; writing from any
      // rank <= nbar - h on leaves ranks nbar-h .. nbar-1 in the ring with the
      // write slot on rank nbar - h.  A warp starts at its own first chunk sw.
      uint32_t wa[PX], rend[PX], hbytes[PX];
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        wa[q] = rbase + 4 * q;
        hbytes[q] = (uint32_t)hh[q] * C::RSLOT;
        rend[q] = wa[q] + hbytes[q];
      }
      // k-indexed ring slots (mon_date_k) need at most one wrap per 8-date
      // half: h >= 8 for every pixel of the warp
      bool r8 = true;
#pragma unroll
      for (int q = 0; q < PX; ++q) r8 = r8 && hh[q] >= 8;
#ifdef BFAST_FORCE_RING8
      const bool ring8 = true;  // experiments only: wrong for pixels with h < 8
      (void)r8;
#else
      const bool ring8 = __all_sync(0xffffffffu, r8);
#endif
      // every consumer warp has published sw and written its last operands
      // (the ring overwrites them); the producers wait on seedready instead
      asm volatile("bar.sync 1, 128;" ::: "memory");
      const int s0 = min(min(seed_slot[0], seed_slot[1]), min(seed_slot[2], seed_slot[3]));
      for (int c = s0; c < nch; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        wait_yhat();
        if (c >= sw) {
          const uint32_t Ys = a_ystages + ys * C::YBYTES;
#pragma unroll UNROLL_SEED
          for (int hf = 0; hf < 2; ++hf) {
            float yh[PX][8], yv[PX][8];
            load_yhat8(hf, yh);
            load_y8(Ys, hf, yv);
            if (kSeedK && ring8) {
              uint32_t kk[PX], jw[PX];
#pragma unroll
              for (int q = 0; q < PX; ++q) {
                kk[q] = 0;
                jw[q] = (rend[q] - wa[q]) / C::RSLOT;
              }
#pragma unroll
              for (int q = 0; q < PX; ++q)
#pragma unroll
                for (int d = 0; d < 8; ++d)
                  seed_date_k<C::RSLOT>(yv[q][d], c0[q], yh[q][d], kk[q], wa[q], jw[q], hbytes[q]);
#pragma unroll
              for (int q = 0; q < PX; ++q) {
                const uint32_t a = wa[q] + kk[q] * C::RSLOT;
                wa[q] = a >= rend[q] ? a - hbytes[q] : a;
              }
            } else {
#pragma unroll
              for (int d = 0; d < 8; ++d)
#pragma unroll
                for (int q = 0; q < PX; ++q)
                  seed_date<C::RSLOT>(yv[q][d], c0[q], yh[q][d], wa[q], rend[q], hbytes[q]);
            }
          }
        }
        release_yhat();
        warp_arrive(a_yempty + 8 * ys);
        yadvance();
      }
      // W = the window of rank nbar - 1 (ranks nbar-h .. nbar-1); the first
      // monitoring step drops rank nbar - h, so W_0 = m^fst + r_nbar (L518)
      float W[PX];
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        W[q] = 0.f;
        if (!deg[q])
          for (uint32_t a = rbase + 4 * q; a < rend[q]; a += C::RSLOT) W[q] += lds_f32(a);
      }

      // ================= pass 3, monitoring (Alg. 1 l.6-12, Fig. 12 ker 9-10)
      float msum[PX], mfirst[PX], mx[PX], thr_lo[PX];
      int brk[PX], first[PX];
      bool tie[PX];
      bool anydeg = false;
      int rank_flat_min = 0x7fffffff;
      const float lam = p.lambda;
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        msum[q] = 0.f;
        mfirst[q] = 0.f;
        mx[q] = 0.f;  // max |W| over the valid monitoring dates so far
        brk[q] = -1;
        first[q] = -1;
        tie[q] = false;
        cr[q] = nbar[q];
        // a 1-based rank up to which B == lambda (rank/nbar <= e): floor(e nbar)
        // - 3 keeps ln(rank/nbar) below 1 by more than f32 rounding for any nbar
        const int rank_flat = max((int)(2.718281828f * (float)nbar[q]) - 3, 0);
        // thresholds on W: |m| > lambda (1 - tol)  <=>  |W| > lambda (1 - tol) scale
        thr_lo[q] = deg[q] ? __int_as_float(0x7f800000) : lam * (1.0f - kTieTol) * scale[q];
        if (!deg[q]) rank_flat_min = min(rank_flat_min, rank_flat - nbar[q]);  // monitoring ranks with B == lambda
        anydeg = anydeg || deg[q];
      }
      (void)anydeg;
      for (int c = 0; c < ncm; ++c) {
        sm100::mbar_wait_a(a_yfull + 8 * ys, yph);
        wait_yhat();
        const uint32_t Ys = a_ystages + ys * C::YBYTES;
        // B_j == lambda for every rank this chunk can reach (rank/nbar <= e)
        // for all of the thread's valid pixels: warp-uniform fast path without
        // the out-of-line boundary evaluation
        int crm = 0;
#pragma unroll
        for (int q = 0; q < PX; ++q) crm = max(crm, deg[q] ? 0 : cr[q] - nbar[q]);
        const bool fast = __all_sync(0xffffffffu, crm + C::DC <= rank_flat_min);
#pragma unroll kUnrollMon
        for (int hf = 0; hf < 2; ++hf) {
          float yh[PX][8], yv[PX][8];
          load_yhat8(hf, yh);
          load_y8(Ys, hf, yv);  // dates >= N read as NaN (TMA OOB)
          if (kEarlyRelease && hf == 1) {
            release_yhat();
            warp_arrive(a_yempty + 8 * ys);
            yadvance();
          }
          if (fast) {
            // B_j == lambda here: the first |m| > lambda(1 - tol) decides (a
            // clear crossing is the break, a near tie goes to the fp64 refit).
            // The dates only track max |W| and keep W at each valid date
            // (wv); a half in which max |W| crossed is scanned for the first
            // crossing date.
            float wv[PX][8];
            if (ring8) {
              // slot addresses from the half's running count (mon_date_k);
              // pixel-major order: each pixel's 8 loads issue back to back
              uint32_t kk[PX], jw[PX];
#pragma unroll
              for (int q = 0; q < PX; ++q) {
                kk[q] = 0;
                jw[q] = (rend[q] - wa[q]) / C::RSLOT;
              }
#pragma unroll
              for (int q = 0; q < PX; ++q)
#pragma unroll
                for (int d = 0; d < 8; ++d)
                  mon_date_k<C::RSLOT>(yv[q][d], c0[q], yh[q][d], W[q], msum[q], mx[q], kk[q], wa[q], jw[q],
                                       hbytes[q], wv[q][d]);
#pragma unroll
              for (int q = 0; q < PX; ++q) {
                cr[q] += (int)kk[q];
                const uint32_t a = wa[q] + kk[q] * C::RSLOT;
                wa[q] = a >= rend[q] ? a - hbytes[q] : a;
              }
            } else {
#pragma unroll
              for (int d = 0; d < 8; ++d)
#pragma unroll
                for (int q = 0; q < PX; ++q) {
                  float r, old;
                  mon_date<C::RSLOT>(yv[q][d], c0[q], yh[q][d], W[q], msum[q], mx[q], cr[q], wa[q], rend[q],
                                     hbytes[q], r, old);
                  wv[q][d] = r == r ? W[q] : 0.f;
                }
            }

#pragma unroll
            for (int q = 0; q < PX; ++q) {
              if (mx[q] > thr_lo[q]) {  // first[q] < 0 while thr_lo is finite
                int fd = 7;
                float fw = wv[q][7];
#pragma unroll
                for (int d = 6; d >= 0; --d)
                  if (fabsf(wv[q][d]) > thr_lo[q]) {
                    fd = d;
                    fw = wv[q][d];
                  }
                first[q] = c * C::DC + 8 * hf + fd;
                mfirst[q] = fw;
                thr_lo[q] = __int_as_float(0x7f800000);
              }
            }
          } else {
#pragma unroll
            for (int d = 0; d < 8; ++d) {
#pragma unroll
              for (int q = 0; q < PX; ++q) {
                float r, old;
                mon_date<C::RSLOT>(yv[q][d], c0[q], yh[q][d], W[q], msum[q], mx[q], cr[q], wa[q], rend[q], hbytes[q], r,
                         old);
                if (r == r && brk[q] < 0 && !tie[q] && first[q] < 0 && fabsf(W[q]) > thr_lo[q]) {
                  const int code = boundary_rare(W[q] * inv_scale[q], cr[q], nbar[q], lam);
                  tie[q] = tie[q] || (code >> 1);
                  brk[q] = (code & 1) ? c * C::DC + 8 * hf + d : brk[q];
                }
              }
            }
          }
        }
        if (!kEarlyRelease) {
          release_yhat();
          warp_arrive(a_yempty + 8 * ys);  // every loaded value has been consumed
          yadvance();
        }
#pragma unroll
        for (int q = 0; q < PX; ++q) {
          if (first[q] >= 0 && brk[q] < 0 && !tie[q]) {  // resolve a fast-path candidate
            if (fabsf(mfirst[q] * inv_scale[q]) > lam * (1.0f + kTieTol)) brk[q] = first[q];
            else tie[q] = true;
            thr_lo[q] = __int_as_float(0x7f800000);
          }
        }
      }

      // ================= epilogue
      unsigned wantbits = 0;
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        const int64_t pix = pix0 + q;
        const int Nbar = cr[q];
        if (Nbar - nbar[q] < 1) deg[q] = true;
        const bool fit_ok = !((nbar[q] < K + 1) || (h[q] < 1) || (Nbar - nbar[q] < 1));
        const bool inside = pix < p.p0 + p.P;  // the last tile may be ragged
        if (inside) {
          p.out_break[pix] = deg[q] ? -2 : brk[q];
          p.out_mag[pix] = deg[q] ? qnan : msum[q] * inv_scale[q] / (float)(Nbar - nbar[q]);
          if (p.out_sigma) p.out_sigma[pix] = fit_ok ? sigma[q] : qnan;
          if (p.out_nbar) p.out_nbar[pix] = nbar[q];
#ifdef BFAST_REFIT_WHY
          if (p.out_flags) p.out_flags[pix] = (deg[q] ? 1u : 0u) | why[q] | (tie[q] ? 0x80u : 0u);
#else
          if (p.out_flags) p.out_flags[pix] = deg[q] ? 1u : 0u;
#endif
          store_beta<K, float>(p, pix, beta[q], c0[q], fit_ok);
        }
        if ((refit[q] || tie[q]) && fit_ok && inside) wantbits |= 1u << q;
      }
      // append the pixels for the fp64 refit (warp-aggregated)
#pragma unroll
      for (int q = 0; q < PX; ++q) {
        const bool want = (wantbits >> q) & 1u;
        const unsigned mask = __ballot_sync(0xffffffffu, want);
        if (want) {
          const int leader = __ffs(mask) - 1;
          int base = 0;
          if (lane == leader) base = atomicAdd(p.refit_count, __popc(mask));
          base = __shfl_sync(mask, base, leader);
          p.refit_list[base + __popc(mask & ((1u << lane) - 1))] = pix0 + q;
        }
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
