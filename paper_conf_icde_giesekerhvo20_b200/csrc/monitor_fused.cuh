// monitor_fused.cuh -- the BFAST-Monitor hot path as one persistent kernel
// per SM: every (pixel, date) step on the CUDA cores, every contraction a
// tile of 128 pixels shares on the 5th-generation tensor cores, one control
// warp per tile that only moves data (TMA) and issues tcgen05.mma.
//
// Variants (template parameters, each its own instantiation so that the
// common kernel carries none of their code): I16 -- the stack as scaled
// int16 codes; MULTI -- several monitoring periods per
// stack pass (f1, FzMulti); CLAMP -- the MOSUM ring sized from a sample of
// the stack, wider windows to the fp64 refit; DENSE -- warps of complete
// histories use the plan's fp64 Gram factor (f3, FzTables::shared).
//
// Algorithm 1, Fig. 12 (L478-L537); readings R1-R14 of
// DESIGN.md.  Per tile of 128 pixels (one pixel per thread = one TMEM lane),
// three sweeps over 16-date chunks of the time-major stack:
//
//   pass A  history    mask v and y' = y - c (c = the pixel's first valid
//                      value) as bf16 A operands in TMEM ->
//                        Gram moments  D_G += V * [F_hi | F_mid | F_lo]
//                        (the K(K+1)/2 Gram entries are linear in 2 + 6k
//                        masked moments of fixed functions, product-to-sum
//                        identities; exact 0/1 mask x 3-way bf16 table)
//                        moment b0     D_b += Y'_hi (X_hi + X_mid) + Y'_lo X_hi
//                        (y' split in two bf16 parts, 16 bits: the first fit
//                        only seeds the refinement)            Alg. 1 l.2, l.4
//   solve              fp32 register Cholesky, beta0            Alg. 1 l.3-4
//   pass B  history    yhat0 = X beta0 (tcgen05, beta in TMEM), r0 = y - yhat0,
//                      sum r0^2, the refinement moment D_db += R0 * X (3-way
//                      splits), the validity bits of every chunk, and the
//                      last residuals of the history in the per-pixel MOSUM
//                      ring (Fig. 12 m^fst, L518)              L505-L515
//   refine             beta = beta0 + A^-1 db; sigma-hat^2 = (sum r0^2 -
//                      dbeta.db) / (nbar - K); the ring's residuals corrected
//                      by -x_t.dbeta (their dates t from the validity bits)
//   pass C  monitoring yhat = X beta, r = y - yhat, MOSUM recurrence over the
//                      ring, boundary, first break, mean       L518-L537
//
// Roles.  One persistent CTA per SM = a control warpgroup (warps 0-3) and T
// consumer warpgroups (T = FzShape::TMAX tiles of 128 pixels, by registers);
// the CTA loops over tile groups of T * 128 pixels.
//  - control warp i drives tile i in the tile's fixed event order: when the
//    tile's 4 consumer warps release a stack stage (mbarrier srel) it loads
//    the chunk SC ahead -- one [16 dates x 128 px] 2-D TMA box (8 KB) into
//    that stage, plus an L2 prefetch of first-touch dates pfd ahead; when
//    they publish a chunk's operands (mbarrier pub) it issues the chunk's
//    tcgen05.mma (one elected lane) and commits them to mdone / ybar.  Its
//    waits sleep in hardware (try_wait + suspend hint);
//  - the consumers only compute: per date registers, per chunk tcgen05.st /
//    tcgen05.ld of TMEM operands and accumulators;
//  - all B-operand tables (fixed functions of the dates, L2-resident) stream
//    through one ST-stage ring shared by the T tiles; a stage is reloaded by
//    the last tile to be done with it, two chunks after its use.
// The stack is read through tensor maps whose out-of-bounds fill is NaN, so
// ragged tiles and the partial last chunk of each period need no special case.
#pragma once
#include "monitor_simt.cuh"
#include "sm100.cuh"
#include <cuda.h>

namespace bfast {

template <int K>
struct FzShape {
  // tiles per CTA: the register budget of 128 threads per tile (the
  // Cholesky factor of the K x K Gram lives in registers through pass B)
#ifdef BFAST_FZ_TMAX8
  static constexpr int TMAX = K <= 8 ? BFAST_FZ_TMAX8 : K <= 12 ? 3 : 2;
#else
  static constexpr int TMAX = K <= 8 ? 4 : K <= 12 ? 3 : 2;
#endif
  // registers after setmaxnreg: consumers RC, the control warpgroup RP
  // (128 TMAX RC + 128 RP <= 65536)
  // (setmaxnreg moves registers within the CTA's launch allocation: the
  // launch gives every thread LAUNCH registers, 128 (TMAX + 1) LAUNCH in all)
  static constexpr int LAUNCH = (65536 / (128 * (TMAX + 1))) / 8 * 8;
#ifdef BFAST_FZ_RP
  static constexpr int RP = BFAST_FZ_RP;
#else
  static constexpr int RP = TMAX == 4 ? 32 : 56;
#endif
  static constexpr int RC = ((LAUNCH * (TMAX + 1) - RP) / TMAX) / 8 * 8;
  static_assert(TMAX * RC + RP <= LAUNCH * (TMAX + 1), "register pool");
};

// register split for TM tiles per CTA (FzTiles: the multi-period kernel of
// f1 may be built for one tile fewer, BFAST_FZ_MULTI_TM1, trading a tile
// for registers: measured -1.5% time on 7 yearly periods whose longest
// window admits only 3 tiles anyway, +17% where the windows admit 4)
template <int TM>
struct FzRegs {
  static constexpr int LAUNCH = (65536 / (128 * (TM + 1))) / 8 * 8;
#ifdef BFAST_FZ_RP
  static constexpr int RP = BFAST_FZ_RP;
#else
  static constexpr int RP = TM == 4 ? 32 : 56;
#endif
  static constexpr int RC = ((LAUNCH * (TM + 1) - RP) / TM) / 8 * 8 > 248 ? 248
                                                                          : ((LAUNCH * (TM + 1) - RP) / TM) / 8 * 8;
};
template <int K, bool MULTI>
struct FzTiles {
#ifdef BFAST_FZ_MULTI_TM1
  static constexpr int TM = MULTI && FzShape<K>::TMAX > 2 ? FzShape<K>::TMAX - 1 : FzShape<K>::TMAX;
#else
  static constexpr int TM = FzShape<K>::TMAX;
#endif
};

// tiles per control warp (BFAST_FZ_TPC): 2 = one control warp drives a pair
// of tiles in lockstep (one stack box of 256 px, one MMA event per pair)
#ifndef BFAST_FZ_TPC
#define BFAST_FZ_TPC 1
#endif

template <int K>
struct FzCfg {
  static constexpr int k = (K - 2) / 2;
  static constexpr int NF = 2 + 6 * k;                   // masked moment functions (+ the constant)
  static constexpr int NGn = ((NF + 1 + 15) / 16) * 16;  // Gram GEMM N
  static constexpr int KBn = ((K + 15) / 16) * 16;       // moment GEMM N
  static constexpr int KY = ((6 * K + 15) / 16) * 16;    // yhat GEMM K (6 cross terms of 3-way splits)
  static constexpr int DC = 16;                          // dates per chunk (MMA K of bf16)
  static constexpr int TMAX = FzShape<K>::TMAX;
  // TMEM columns of one tile (lane = pixel).  Pass A: Gram | b0 | two
  // operand buffers [mask 8 | y' hi 8 | y' lo 8].  Passes B/C: NYS yhat slots |
  // beta operand | db | one operand buffer [r0 hi 8 | mid 8 | lo 8].  The pass-B
  // layout overwrites pass A's only after the solve has read it.
  static constexpr int NOPA = 3;  // pass-A operand buffers (the consumers run NOPA - 1 chunks ahead of the MMA)
  static constexpr int cG = 0, cB = NGn, cOPA = NGn + KBn;
  static constexpr int PA_COLS = cOPA + 24 * NOPA;
  static constexpr int NYS = 3;  // yhat slots: yhat(c + 3) is issued when chunk c is published
  static_assert(NYS <= 3, "the publish barriers (pub[g % 4]) allow NYS outstanding groups");
  static_assert(NOPA <= 3, "the publish barriers (pub[g % 4]) allow NOPA outstanding groups");
  static constexpr int cY = 0, cA3 = 16 * NYS, cDB = cA3 + KY / 2, cOPB = cDB + KBn;
  static constexpr int PB_COLS = cOPB + 24;  // one r0 operand buffer
  static constexpr int USED = PA_COLS > PB_COLS ? PA_COLS : PB_COLS;
  static constexpr __host__ __device__ int pow2cols(int c) {
    return c <= 32 ? 32 : c <= 64 ? 64 : c <= 128 ? 128 : c <= 256 ? 256 : 512;
  }
  // per-tile columns (>= 4 mask columns): a power of two, except K = 12,
  // whose 136 columns round to 160 (32-aligned) so that three tiles fit the
  // 512 TMEM columns (measured -20% at N = 250, k = 5 against two tiles)
  static constexpr int TCOLS = K == 12 ? ((USED > PB_COLS + 4 ? USED : PB_COLS + 4) + 31) / 32 * 32
                                       : pow2cols(USED > PB_COLS + 4 ? USED : PB_COLS + 4);
  // the validity bits of the last 2 MKC history chunks (two per column) live
  // in the columns pass B leaves free (the ring correction reads them back)
  static constexpr int cMK = PB_COLS, MKC = TCOLS - PB_COLS;
  static_assert(MKC >= 4, "mask columns");
  static_assert(TCOLS * TMAX <= 512, "TMEM budget");
  // B-operand tables per chunk (canonical K-major, no swizzle)
  static constexpr int BF_BYTES = NGn * DC * 2;  // one part of the Gram table [NGn x 16]
  static constexpr int BX_BYTES = KBn * DC * 2;  // one part of x [KBn x 16]
  static constexpr int B3_BYTES = DC * KY * 2;   // yhat table [16 x KY]
  static constexpr int TABA = 3 * BF_BYTES + 2 * BX_BYTES;
  static constexpr int TABB = B3_BYTES + 3 * BX_BYTES;
  static constexpr int TABC = B3_BYTES;
  static constexpr int TMAXB = TABA > TABB ? TABA : TABB;
  static constexpr int TSTAGE = ((TMAXB + 127) / 128) * 128;
#ifdef BFAST_FZ_ST
  static constexpr int ST = BFAST_FZ_ST;
#else
  static constexpr int ST = 6;                   // table stages (a stage is reloaded two chunks after its use)
#endif
  static constexpr int PFB = 64;                 // dates per L2-prefetch box
  static constexpr int SCMAX = 3;                // stack chunk stages per tile (2 or 3, by shared memory)
  static constexpr int CBYTES = DC * 128 * 4;    // one [16 dates x 128 px] box (8 KB; 4 KB of int16 codes)
  static constexpr int TPC = BFAST_FZ_TPC;
  static constexpr size_t smem_bytes(int T, int hcap, int sc, int esz = 4) {
    return (size_t)T * sc * (CBYTES / 4 * esz) + (size_t)ST * TSTAGE + (size_t)T * hcap * 512;
  }
};

struct FzTables {
  const uint8_t *tabA, *tabB, *tabC;  // per-chunk B operands (FzCfg::TABA / TABB / TABC bytes each)
  int nch, ncm;                       // history / monitoring chunks of 16 dates
  int T;                              // tiles per CTA (<= FzShape::TMAX)
  int hcap;                           // MOSUM ring slots per pixel
  int pfd;                            // L2 prefetch distance in dates (multiple of FzCfg::PFB; 0: off)
  int sc;                             // stack chunk stages per tile (2..FzCfg::SCMAX)
  int64_t ntg;                        // tile groups of T * 128 pixels
  // NaN-free history (f3): the common Cholesky factor, [Tri<K>::kN | dinv K |
  // min pivot ratio | max VIF] (bfast_abi.cu shared_factor); nullptr = off
  const float *shared;
  // int16 codec (f4): the float every code equal to the nodata code turns
  // into (fz_code: 2^23 + (code ^ 0x8000), exact), i.e. "missing"
  float fnd;
};

// Several monitoring periods per stack pass (PAPER.md L391:
// yearly periods 2010-2011, 2011-2012, ... over one data cube).  Period i
// is an independent BFAST-Monitor problem on the dates [0, N_i) with
// history [0, n_i); the CTA runs every period of a tile group before the
// next tile group, so the re-reads of the group's columns come from L2.
constexpr int kMaxPeriods = 8;
struct FzPeriod {
  MonitorParams prm;                  // n, N, X, tc/ts, outputs, refit list of the period
  const uint8_t *tabA, *tabB, *tabC;  // its chunk tables (history centring depends on n)
  const float *shared;                // its NaN-free factor (f3) or nullptr
  int nch, ncm;
  CUtensorMap h, y;                   // its history [0, n) and full [0, N) stack maps
};
struct FzMulti {
  FzPeriod per[kMaxPeriods];
  int M;   // periods
  int Lg;  // chunks per tile group: sum of 2 nch + ncm
};

// int16 codes (f4) enter the per-date arithmetic as the exact floats
// 2^23 + (code + 32768): one LOP3 from the zero-extended 16-bit load.  The
// path is invariant to an offset and, up to the sign of the MOSUM, to a
// scale (y = scale code + offset: residuals and sigma-hat scale by scale,
// W / (sigma-hat sqrt(nbar)) by sign(scale)); the epilogue applies the
// codec to beta, sigma-hat and the magnitude.
constexpr float kCodeBias = 8421376.0f;  // 2^23 + 32768: fz_code(code) - kCodeBias == code
__device__ __forceinline__ float fz_code(uint32_t u16) { return __uint_as_float((u16 ^ 0x8000u) | 0x4B000000u); }
__device__ __forceinline__ uint32_t lds_u16(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u16 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_u16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}

#ifndef BFAST_FZ_CTLWAIT
#define BFAST_FZ_CTLWAIT 1  // control-warp waits: 1 = hardware-suspended try_wait, 0 = spin
#endif
// ---- optional cycle accounting (-DBFAST_FZ_TIMING, tools/fz_timing.py) -----
#ifdef BFAST_FZ_TIMING
__device__ unsigned long long fz_timing[16];
#define FZT_DECL unsigned long long fzt_acc[16] = {0};
#define FZT_T0(v) const long long v = clock64();
#define FZT_ADD(i, v) fzt_acc[i] += (unsigned long long)(clock64() - v);
#define FZT_FLUSH                                                          \
  if (lane == 0)                                                           \
    for (int i_ = 0; i_ < 16; ++i_) atomicAdd(&fz_timing[i_], fzt_acc[i_]);
#else
#define FZT_DECL
#define FZT_T0(v)
#define FZT_ADD(i, v)
#define FZT_FLUSH
#endif

// ---- small PTX helpers -----------------------------------------------------
__device__ __forceinline__ float lds_f(uint32_t a) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ void sts_f(uint32_t a, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(a), "f"(v) : "memory");
}
__device__ __forceinline__ uint32_t atom_add_acqrel(uint32_t a, uint32_t v) {
  uint32_t old;
  asm volatile("atom.acq_rel.cta.shared::cta.add.u32 %0, [%1], %2;" : "=r"(old) : "r"(a), "r"(v) : "memory");
  return old;
}
__device__ __forceinline__ void tma_prefetch_2d(const void *tmap, int x, int y) {
  asm volatile("cp.async.bulk.prefetch.tensor.2d.L2.global.tile [%0, {%1, %2}];" ::"l"(tmap), "r"(x), "r"(y)
               : "memory");
}
__device__ __forceinline__ void tmem_st16(uint32_t taddr, const uint32_t (&v)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], "
      "{%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(taddr),
      "r"(v[0]), "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7]), "r"(v[8]),
      "r"(v[9]), "r"(v[10]), "r"(v[11]), "r"(v[12]), "r"(v[13]), "r"(v[14]), "r"(v[15])
      : "memory");
}
__device__ __forceinline__ void tmem_st1(uint32_t taddr, uint32_t v) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x1.b32 [%0], {%1};" ::"r"(taddr), "r"(v) : "memory");
}
__device__ __forceinline__ void tmem_ld1(uint32_t taddr, float (&v)[1]) {
  uint32_t r;
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x1.b32 {%0}, [%1];" : "=r"(r) : "r"(taddr));
  v[0] = __uint_as_float(r);
}
// consumer-side waits: BFAST_FZ_CWAIT 0 = probe in a loop (try_wait's own
// time limit), 1 = try_wait with a suspend-time hint (compiles to TRYWAIT +
// NANOSLEEP.SYNCS + PHASECHK per iteration).  0 measured -0.7% on the
// Landsat scene, -1.4% at N = 1000, +-0 at N = 100 (round 2); the control
// warps keep the suspend hint (0 there: +0.2%)
#ifndef BFAST_FZ_CWAIT
#define BFAST_FZ_CWAIT 0
#endif
__device__ __forceinline__ void mbar_wait_spin(uint32_t bar, uint32_t parity) {
#if BFAST_FZ_CWAIT == 1
  while (!sm100::mbar_try_wait_a_hint(bar, parity, 0x10000u)) {
  }
#else
  while (!sm100::mbar_try_wait_a(bar, parity)) {
  }
#endif
}
// upper halves of two fp32 words (their bf16 truncations) -> one bf16 pair
__device__ __forceinline__ uint32_t hi16x2(float lo_elem, float hi_elem) {
  return __byte_perm(__float_as_uint(lo_elem), __float_as_uint(hi_elem), 0x7632);
}

// ---- per-date steps (inline PTX keeps the validity predicate in a register)
// Pass A: vm = all-ones iff y is a value (set.num), yp = (y - c) & vm.
template <bool I16>
__device__ __forceinline__ void fa_date(float y, float c0, uint32_t &vm, float &yp, float fnd) {
  if constexpr (I16) {
  asm("{\n\t.reg .f32 t;\n\t"
      "set.ne.u32.f32 %0, %2, %4;\n\t"
      "sub.f32 t, %2, %3;\n\t"
      "and.b32 %1, t, %0;\n\t}"
      : "=r"(vm), "=f"(yp)
      : "f"(y), "f"(c0), "f"(fnd));
  } else {
  asm("{\n\t.reg .f32 t;\n\t"
      "set.num.u32.f32 %0, %2, %2;\n\t"
      "sub.f32 t, %2, %3;\n\t"
      "and.b32 %1, t, %0;\n\t}"
      : "=r"(vm), "=f"(yp)
      : "f"(y), "f"(c0));
  }
}
// Pass B: r = y - yhat0 (NaN iff missing); if valid: s2 += r^2 and bit BIT
// of vb is set; rz = r or 0.
template <bool I16, int BIT>
__device__ __forceinline__ void fb_date(float y, float c0, float yh, float &s2, uint32_t &vb, float &rz,
                                        float fnd) {
  if constexpr (I16) {
  asm("{\n\t.reg .pred p;\n\t.reg .f32 r;\n\t"
      "sub.f32 r, %3, %4;\n\t"
      "sub.f32 r, r, %5;\n\t"
      "setp.ne.f32 p, %3, %7;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %6;\n\t"
      "selp.f32 %2, r, 0f00000000, p;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(rz)
      : "f"(y), "f"(c0), "f"(yh), "n"(1u << BIT), "f"(fnd));
  } else {
  asm("{\n\t.reg .pred p;\n\t.reg .f32 r;\n\t"
      "sub.f32 r, %3, %4;\n\t"
      "sub.f32 r, r, %5;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %6;\n\t"
      "selp.f32 %2, r, 0f00000000, p;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(rz)
      : "f"(y), "f"(c0), "f"(yh), "n"(1u << BIT));
  }
}
// the same with the ring write of mon ranks: slot a = wa + k*512 (wrapped
// once by hbytes when k >= jw); the residual enters it and k advances when
// the date is valid
template <bool I16, int BIT>
__device__ __forceinline__ void fb_date_ring(float y, float c0, float yh, float &s2, uint32_t &vb, float &rz,
                                             uint32_t &k, uint32_t wa, uint32_t jw, uint32_t hbytes, float fnd) {
  if constexpr (I16) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r;\n\t.reg .u32 a;\n\t"
      "sub.f32 r, %4, %5;\n\t"
      "sub.f32 r, r, %6;\n\t"
      "setp.ne.f32 p, %4, %11;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %10;\n\t"
      "selp.f32 %2, r, 0f00000000, p;\n\t"
      "mad.lo.u32 a, %3, 512, %7;\n\t"
      "setp.ge.u32 q, %3, %8;\n\t"
      "@q sub.u32 a, a, %9;\n\t"
      "@p st.shared.f32 [a], r;\n\t"
      "@p add.u32 %3, %3, 1;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(rz), "+r"(k)
      : "f"(y), "f"(c0), "f"(yh), "r"(wa), "r"(jw), "r"(hbytes), "n"(1u << BIT), "f"(fnd)
      : "memory");
  } else {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r;\n\t.reg .u32 a;\n\t"
      "sub.f32 r, %4, %5;\n\t"
      "sub.f32 r, r, %6;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %10;\n\t"
      "selp.f32 %2, r, 0f00000000, p;\n\t"
      "mad.lo.u32 a, %3, 512, %7;\n\t"
      "setp.ge.u32 q, %3, %8;\n\t"
      "@q sub.u32 a, a, %9;\n\t"
      "@p st.shared.f32 [a], r;\n\t"
      "@p add.u32 %3, %3, 1;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(rz), "+r"(k)
      : "f"(y), "f"(c0), "f"(yh), "r"(wa), "r"(jw), "r"(hbytes), "n"(1u << BIT)
      : "memory");
  }
}
// the same, ring slot advanced date by date (a pixel whose window h < 8 may
// wrap more than once per 8-date half)
template <bool I16, int BIT>
__device__ __forceinline__ void fb_date_ring1(float y, float c0, float yh, float &s2, uint32_t &vb, float &rz,
                                              uint32_t &wa, uint32_t rend, uint32_t hbytes, float fnd) {
  if constexpr (I16) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r;\n\t"
      "sub.f32 r, %4, %5;\n\t"
      "sub.f32 r, r, %6;\n\t"
      "setp.ne.f32 p, %4, %10;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %9;\n\t"
      "selp.f32 %2, r, 0f00000000, p;\n\t"
      "@p st.shared.f32 [%3], r;\n\t"
      "@p add.u32 %3, %3, 512;\n\t"
      "setp.ge.u32 q, %3, %7;\n\t"
      "@q sub.u32 %3, %3, %8;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(rz), "+r"(wa)
      : "f"(y), "f"(c0), "f"(yh), "r"(rend), "r"(hbytes), "n"(1u << BIT), "f"(fnd)
      : "memory");
  } else {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r;\n\t"
      "sub.f32 r, %4, %5;\n\t"
      "sub.f32 r, r, %6;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "@p fma.rn.f32 %0, r, r, %0;\n\t"
      "@p or.b32 %1, %1, %9;\n\t"
      "selp.f32 %2, r, 0f00000000, p;\n\t"
      "@p st.shared.f32 [%3], r;\n\t"
      "@p add.u32 %3, %3, 512;\n\t"
      "setp.ge.u32 q, %3, %7;\n\t"
      "@q sub.u32 %3, %3, %8;\n\t}"
      : "+f"(s2), "+r"(vb), "=f"(rz), "+r"(wa)
      : "f"(y), "f"(c0), "f"(yh), "r"(rend), "r"(hbytes), "n"(1u << BIT)
      : "memory");
  }
}
// Monitoring date (Eq. (4) recurrence, L520-L525), k-indexed ring slot (h >=
// 8): the slot holds rank cr - h; if r = y - yhat is a value it replaces
// it, W += r - old, msum += W, mx = max(mx, |W|); wv = W after a valid date,
// 0 after a missing one (the crossing scan of a half reads these).
template <bool I16>
__device__ __forceinline__ void fc_date_k(float y, float c0, float yh, float &W, float &msum, float &mx, uint32_t &k,
                                          uint32_t wa, uint32_t jw, uint32_t hbytes, float &wv, float fnd) {
  if constexpr (I16) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r, o, t;\n\t.reg .u32 a;\n\t"
      "sub.f32 r, %5, %6;\n\t"
      "sub.f32 r, r, %7;\n\t"
      "setp.ne.f32 p, %5, %11;\n\t"
      "mad.lo.u32 a, %3, 512, %8;\n\t"
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
      : "f"(y), "f"(c0), "f"(yh), "r"(wa), "r"(jw), "r"(hbytes), "f"(fnd)
      : "memory");
  } else {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r, o, t;\n\t.reg .u32 a;\n\t"
      "sub.f32 r, %5, %6;\n\t"
      "sub.f32 r, r, %7;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "mad.lo.u32 a, %3, 512, %8;\n\t"
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
      : "f"(y), "f"(c0), "f"(yh), "r"(wa), "r"(jw), "r"(hbytes)
      : "memory");
  }
}
// the same with the slot pointer advanced date by date (any h); returns r
// and validity for the slow boundary path
template <bool I16>
__device__ __forceinline__ void fc_date_1(float y, float c0, float yh, float &W, float &msum, float &mx, int &cr,
                                          uint32_t &wa, uint32_t rend, uint32_t hbytes, float &wv, float fnd) {
  if constexpr (I16) {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r, o, t;\n\t"
      "sub.f32 r, %6, %7;\n\t"
      "sub.f32 r, r, %8;\n\t"
      "setp.ne.f32 p, %6, %11;\n\t"
      "ld.shared.f32 o, [%4];\n\t"
      "@p st.shared.f32 [%4], r;\n\t"
      "@p add.u32 %4, %4, 512;\n\t"
      "setp.ge.u32 q, %4, %9;\n\t"
      "@q sub.u32 %4, %4, %10;\n\t"
      "@p add.s32 %3, %3, 1;\n\t"
      "sub.f32 t, r, o;\n\t"
      "@p add.f32 %0, %0, t;\n\t"
      "@p add.f32 %1, %1, %0;\n\t"
      "abs.f32 t, %0;\n\t"
      "@p max.f32 %2, %2, t;\n\t"
      "selp.f32 %5, %0, 0f7fc00000, p;\n\t}"
      : "+f"(W), "+f"(msum), "+f"(mx), "+r"(cr), "+r"(wa), "=f"(wv)
      : "f"(y), "f"(c0), "f"(yh), "r"(rend), "r"(hbytes), "f"(fnd)
      : "memory");
  } else {
  asm volatile(
      "{\n\t.reg .pred p, q;\n\t.reg .f32 r, o, t;\n\t"
      "sub.f32 r, %6, %7;\n\t"
      "sub.f32 r, r, %8;\n\t"
      "setp.num.f32 p, r, r;\n\t"
      "ld.shared.f32 o, [%4];\n\t"
      "@p st.shared.f32 [%4], r;\n\t"
      "@p add.u32 %4, %4, 512;\n\t"
      "setp.ge.u32 q, %4, %9;\n\t"
      "@q sub.u32 %4, %4, %10;\n\t"
      "@p add.s32 %3, %3, 1;\n\t"
      "sub.f32 t, r, o;\n\t"
      "@p add.f32 %0, %0, t;\n\t"
      "@p add.f32 %1, %1, %0;\n\t"
      "abs.f32 t, %0;\n\t"
      "@p max.f32 %2, %2, t;\n\t"
      "selp.f32 %5, %0, 0f7fc00000, p;\n\t}"
      : "+f"(W), "+f"(msum), "+f"(mx), "+r"(cr), "+r"(wa), "=f"(wv)
      : "f"(y), "f"(c0), "f"(yh), "r"(rend), "r"(hbytes)
      : "memory");
  }
}

// the rare branch of the boundary test (Alg. 1 l.10-12), kept out of line:
// bit 0: |m| > B (a break), bit 1: |m|/B within kTieTol of 1
__device__ __noinline__ int fz_boundary_rare(float m, int rank1, int nbar, float lam) {
  const float B = boundary_f32(lam, rank1, nbar);
  const float am = fabsf(m);
  return (am > B ? 1 : 0) | (fabsf(am - B) <= kTieTol * B ? 2 : 0);
}

// Cholesky (Alg. 1 l.3 on the SPD Gram) in fp32 with hardware reciprocal
// square roots: A holds L^T off the diagonal, dinv the reciprocal pivots.
// Returns the smallest pivot ratio d_j / A_jj (the refit trigger's
// conditioning proxy); the refinement step absorbs rsqrt's ~1 ulp.
template <int K>
__device__ __forceinline__ float fz_chol(float (&A)[Tri<K>::kN], float (&dinv)[K]) {
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
// Largest variance inflation factor max_j A_jj (A^-1)_jj of the factored
// Gram (A = L L^T: A holds L below the diagonal at idx(j, i), dinv = 1/l_jj):
// (A^-1)_jj = sum_i (L^-1)_ij^2, L^-1 built column by column.  The pivot
// ratio of the Cholesky only sees each column against the earlier ones; a
// near-dependence on later columns shows here (measured: sweep k = 5, 90%
// missing, 1-norm condition ~7e4 with every pivot ratio > 3e-2).
template <int K>
__device__ __forceinline__ float fz_vif_max(const float (&L)[Tri<K>::kN], const float (&dinv)[K],
                                            const float (&diagA)[K]) {
  float vmax = 0.f;
  SFor<0, K>::run([&](auto jc) {
    constexpr int j = decltype(jc)::value;
    float m[K];
    m[j] = dinv[j];
    float ss = m[j] * m[j];
    SFor<j + 1, K>::run([&](auto ic) {
      constexpr int i = decltype(ic)::value;
      float t = 0.f;
      SFor<j, i>::run([&](auto kc) {
        constexpr int kk = decltype(kc)::value;
        t = fmaf(L[Tri<K>::idx(kk, i)], m[kk], t);
      });
      m[i] = -t * dinv[i];
      ss = fmaf(m[i], m[i], ss);
    });
    vmax = fmaxf(vmax, ss * diagA[j]);
  });
  return vmax;
}
// VIF above which the fp32 fit is handed to the fp64 refit
constexpr float kRefitVif = 1000.f;

template <int K>
__device__ __forceinline__ void fz_solve(const float (&L)[Tri<K>::kN], const float (&dinv)[K], const float (&b)[K],
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

template <int K, bool I16, bool MULTI, bool CLAMP = false, bool DENSE = false>
__global__ void __launch_bounds__(128 * (FzTiles<K, MULTI>::TM + 1), 1)
    monitor_fused_kernel(MonitorParams pk, FzTables tb, const __grid_constant__ CUtensorMap ymap,
                         const __grid_constant__ CUtensorMap hmap, const __grid_constant__ CUtensorMap pmap,
                         const __grid_constant__ FzMulti mp) {
  // MULTI (f1): the per-period values come from mp; otherwise from pk / tb
  const MonitorParams &p = MULTI ? mp.per[0].prm : pk;
  using C = FzCfg<K>;
  constexpr int ESZ = I16 ? 2 : 4;           // bytes per stack element
  constexpr int TPC = C::TPC;                // tiles per control warp
  constexpr int CB = C::CBYTES / 4 * ESZ * TPC;  // one [16 dates x 128 TPC px] box (a group's stage)
  extern __shared__ __align__(1024) uint8_t smem[];
  __shared__ __align__(8) uint64_t sfull[C::TMAX][C::SCMAX];  // stack chunk stage landed (TMA tx)
  __shared__ __align__(8) uint64_t srel[C::TMAX][C::SCMAX];   // the tile's 4 warps consumed it
  // the tile's 4 warps published group g (on [g%4]: in pass C the consumers
  // may run NYS groups ahead of the control warp, so a parity pair would alias)
  __shared__ __align__(8) uint64_t pub[C::TMAX][4];
  // tile's group g completes phase g/4 of mdone[g%4] (waiters look up to 3
  // groups back: NOPA = 3 operand buffers)
  __shared__ __align__(8) uint64_t mdone[C::TMAX][4];
  __shared__ __align__(8) uint64_t ybar[C::TMAX][C::NYS];  // tile's yhat slot s written (one phase per yhat)
  __shared__ __align__(8) uint64_t tfull[C::ST];            // table stages
  __shared__ uint32_t tfree[C::ST];                         // tiles done with a table stage (mod T)
  __shared__ uint32_t tmem_base_s;
  __shared__ int s_per[MULTI ? kMaxPeriods : 1][4];  // f1: nch, ncm, n, N of each period (LDS, not LDC)

  const int T = tb.T;
  // warpgroup 0 = the control warps (one per tile: warp i drives tile i;
  // the oldest warps, which the warp scheduler favours), warpgroups 1..T =
  // the tiles' consumers
  // the warp index through a lane-0 shuffle: the compiler then treats it,
  // and every branch on it, as warp-uniform (uniform-datapath operands for
  // the tcgen05 / TMA instructions instead of per-lane broadcasts)
  const int tid = threadIdx.x, lane = tid & 31;
  const int warp = __shfl_sync(0xffffffffu, tid >> 5, 0);
  const bool control = warp < 4;
  const int ctid = tid - 128;  // consumer thread index = pixel of the tile group
  const int tile = control ? warp : (warp - 4) >> 2;
  // control group: tiles grp * TPC ... grp * TPC + TPC - 1 share one control
  // warp (warp grp), its barriers and its stack stages; sub = tile in group
  const int grp = control ? warp : tile / TPC, sub = control ? 0 : tile % TPC;
  const int nch = MULTI ? mp.per[0].nch : tb.nch, ncm = MULTI ? mp.per[0].ncm : tb.ncm, n = p.n, hcap = tb.hcap;
  const int M = MULTI ? mp.M : 1;
  auto P_nch = [&](int per) { return MULTI ? s_per[per][0] : nch; };
  auto P_ncm = [&](int per) { return MULTI ? s_per[per][1] : ncm; };
  auto P_n = [&](int per) { return MULTI ? s_per[per][2] : n; };
  auto P_N = [&](int per) { return MULTI ? s_per[per][3] : p.N; };
  FZT_DECL
  FZT_T0(t_kernel)
  const int SC = tb.sc;
  uint8_t *stack = smem;
  uint8_t *tabs = stack + (size_t)(T / TPC) * SC * CB;
  uint8_t *ring = tabs + (size_t)C::ST * C::TSTAGE;

  // chunk sequence per tile group: A[0, nch), B[0, nch), C[0, ncm) (per period)
  const int Lg = MULTI ? mp.Lg : 2 * nch + ncm;
  const uint32_t my_groups =
      tb.ntg > blockIdx.x ? (uint32_t)((tb.ntg - 1 - blockIdx.x) / gridDim.x + 1) : 0u;
  const uint32_t S_total = my_groups * (uint32_t)Lg;  // chunks this CTA runs
  const uint32_t U_total = S_total;                   // stack chunks per tile

  const uint32_t a_tabs = sm100::opaque(sm100::smem_u32(tabs));
  const uint32_t a_tfull = sm100::opaque(sm100::smem_u32(&tfull[0]));
  const uint32_t a_tfree = sm100::opaque(sm100::smem_u32(&tfree[0]));
  const uint32_t a_mdone = sm100::opaque(sm100::smem_u32(&mdone[grp][0]));
  const uint32_t a_ybar = sm100::opaque(sm100::smem_u32(&ybar[grp][0]));
  const uint32_t a_pub = sm100::opaque(sm100::smem_u32(&pub[grp][0]));
  const uint32_t a_sfull = sm100::opaque(sm100::smem_u32(&sfull[grp][0]));
  const uint32_t a_srel = sm100::opaque(sm100::smem_u32(&srel[grp][0]));
  const uint32_t a_stack = sm100::opaque(sm100::smem_u32(stack + (size_t)grp * SC * CB));

  if (MULTI && tid < M) {
    s_per[tid][0] = mp.per[tid].nch;
    s_per[tid][1] = mp.per[tid].ncm;
    s_per[tid][2] = mp.per[tid].prm.n;
    s_per[tid][3] = mp.per[tid].prm.N;
  }
  if (tid == 0) {
    for (int i = 0; i < T; ++i) {
      for (int j = 0; j < C::SCMAX; ++j) {
        sm100::mbar_init(&sfull[i][j], 1);
        sm100::mbar_init(&srel[i][j], 4 * TPC);
      }
      for (int j = 0; j < 4; ++j) sm100::mbar_init(&pub[i][j], 4 * TPC);
      for (int j = 0; j < 4; ++j) sm100::mbar_init(&mdone[i][j], 1);
      for (int j = 0; j < C::NYS; ++j) sm100::mbar_init(&ybar[i][j], 1);
    }
    for (int i = 0; i < C::ST; ++i) {
      sm100::mbar_init(&tfull[i], 1);
      tfree[i] = 0;
    }
    sm100::fence_mbar_init();
  }
  if (warp == 0) sm100::tmem_alloc(&tmem_base_s, C::pow2cols(T * C::TCOLS));
  sm100::tc_fence_before();
  __syncthreads();
  sm100::tc_fence_after();
  const uint32_t tbase = tmem_base_s;
  // this tile's TMEM columns (lane 0); a control warp: its group's first tile
  const uint32_t tc = tbase + (control ? grp * TPC : tile) * C::TCOLS;

  if (control) {
    // ================================================================ control
    // One warp per tile, every lane running the same program (warp-uniform
    // operands; one elected lane issues each TMA / MMA / commit).  It
    // follows the tile's fixed event order: stack halves consumed -> refill
    // the stage SH halves ahead; group published -> issue its tcgen05.mma.
    // Waits sleep in hardware (try_wait with a suspend-time hint).
    sm100::setmaxnreg_dec<FzRegs<FzTiles<K, MULTI>::TM>::RP>();
    if (grp * TPC >= T) {
      // spare warps of the control warpgroup
    } else {
      auto wait_sleep = [&](uint32_t bar, uint32_t par) {
#if BFAST_FZ_CTLWAIT == 1
        while (!sm100::mbar_try_wait_a_hint(bar, par, 0x10000u)) {
        }
#else
        while (!sm100::mbar_try_wait_a(bar, par)) {
        }
#endif
      };
      // ---- tables (shared by the T tiles)
      struct ChunkPos {
        uint32_t s;
        int q, st;
        uint32_t ph;
      };
      auto advance_pos = [&](ChunkPos cp, int a) -> ChunkPos {
        cp.s += a;
        cp.q += a;
        if (cp.q >= Lg) cp.q -= Lg;
        if (cp.q >= Lg) cp.q -= Lg;
        cp.st += a;
        if (cp.st >= C::ST) {
          cp.st -= C::ST;
          cp.ph ^= 1u;
        }
        return cp;
      };
      auto load_table = [&](const ChunkPos &cp) {  // one elected lane
        if (cp.s >= S_total) return;
        int q = cp.q, per = 0;
        if (MULTI)
          while (q >= 2 * P_nch(per) + P_ncm(per)) q -= 2 * P_nch(per) + P_ncm(per), ++per;
        const int nq = P_nch(per);
        const uint8_t *src;
        uint32_t bytes;
        if (q < nq) {
          bytes = C::TABA;
          src = (MULTI ? mp.per[per].tabA : tb.tabA) + (size_t)q * C::TABA;
        } else if (q < 2 * nq) {
          bytes = C::TABB;
          src = (MULTI ? mp.per[per].tabB : tb.tabB) + (size_t)(q - nq) * C::TABB;
        } else {
          bytes = C::TABC;
          src = (MULTI ? mp.per[per].tabC : tb.tabC) + (size_t)(q - 2 * nq) * C::TABC;
        }
        sm100::mbar_arrive_expect_tx_a(a_tfull + 8 * cp.st, bytes);
        sm100::bulk_g2s_a(a_tabs + cp.st * C::TSTAGE, src, bytes, a_tfull + 8 * cp.st);
      };
      ChunkPos cpos{0u, 0, 0, 0u};
      if (tile == 0 && lane == 0)
        for (int a = 0; a < C::ST; ++a) load_table(advance_pos(cpos, a));
      // ---- stack: per tile one [16 dates x 128 px] box (8 KB) per chunk
      const uint64_t pol_first = sm100::policy_evict_first();
      const int xstep = (int)gridDim.x * T * 128;
      struct ChunkCursor {
        uint32_t u;
        int left, y, region, x, per;
      };
      auto chunk_next = [&](ChunkCursor &cc) {
        ++cc.u;
        cc.y += C::DC;
        if (--cc.left == 0) {
          if (cc.region == 0) {
            cc.region = 1;
            cc.left = P_nch(cc.per);
            cc.y = 0;
          } else if (cc.region == 1) {
            cc.region = 2;
            cc.left = P_ncm(cc.per);
            cc.y = P_n(cc.per);
          } else {
            if (++cc.per == M) {
              cc.per = 0;
              cc.x += xstep;
            }
            cc.region = 0;
            cc.left = P_nch(cc.per);
            cc.y = 0;
          }
        }
      };
      ChunkCursor ldc{0u, nch, 0, 0, (int)blockIdx.x * T * 128 + 128 * TPC * grp, 0};
      int ldst = 0;  // stage of the next chunk to load
      auto load_chunk = [&]() {
        if (ldc.u < U_total && lane == 0) {
          // first-touch periods (A: history, C: monitoring) are prefetched
          // into L2 in [PFB dates x 128 px] boxes, pfd dates ahead of the loads
          // (later periods re-read the history of earlier ones: whatever L2
          // no longer holds is prefetched like a first touch)
          if (tb.pfd > 0 && ldc.region != 1) {
            const int pn = P_n(ldc.per);
            const int base = ldc.region == 0 ? 0 : pn, end = ldc.region == 0 ? pn : P_N(ldc.per);
            const int off = ldc.y - base;
            if (off % C::PFB == 0) {
              if (off == 0)
                for (int yy = base; yy < base + tb.pfd && yy < end; yy += C::PFB) tma_prefetch_2d(&pmap, ldc.x, yy);
              if (ldc.y + tb.pfd < end) tma_prefetch_2d(&pmap, ldc.x, ldc.y + tb.pfd);
            }
          }
          const uint32_t bar = a_sfull + 8 * ldst, dst = a_stack + ldst * CB;
          sm100::mbar_arrive_expect_tx_a(bar, CB);
          const void *hm = MULTI ? (const void *)&mp.per[ldc.per].h : (const void *)&hmap;
          const void *ym = MULTI ? (const void *)&mp.per[ldc.per].y : (const void *)&ymap;
          if (ldc.region == 0 || (MULTI && ldc.per + 1 < M))
            // read again in pass B / by the next period (L2)
            sm100::tma_load_2d_a(dst, ldc.region == 2 ? ym : hm, ldc.x, ldc.y, bar);
          else
            sm100::tma_load_2d_hint_a(dst, ldc.region == 1 ? hm : ym, ldc.x, ldc.y, bar, pol_first);
        }
        chunk_next(ldc);
        if (++ldst == SC) ldst = 0;
      };
      if (lane == 0) {
        sm100::prefetch_tmap(&ymap);
        if (MULTI)
          for (int i = 0; i < M; ++i) {
            sm100::prefetch_tmap(&mp.per[i].h);
            sm100::prefetch_tmap(&mp.per[i].y);
          }
        sm100::prefetch_tmap(&hmap);
      }
      for (int i = 0; i < SC; ++i) load_chunk();
      int rst = 0;       // stage of the next chunk whose consumption to await
      uint32_t rph = 0;  // and its phase parity
      auto on_release = [&]() {
        FZT_T0(tr)
        wait_sleep(a_srel + 8 * rst, rph);
        FZT_ADD(7, tr)
        FZT_T0(tl)
        load_chunk();
        FZT_ADD(12, tl)
        if (++rst == SC) {
          rst = 0;
          rph ^= 1u;
        }
      };
      // ---- MMA groups
      const uint32_t idG = sm100::idesc_bf16_f32(128, C::NGn);
      const uint32_t idB = sm100::idesc_bf16_f32(128, C::KBn);
      const uint32_t idY = sm100::idesc_bf16_f32(128, C::DC);
      uint32_t g = 0;
      int cslot = 0;  // yhat slot of the current B / C chunk
      int abuf = 0;   // pass-A operand buffer of the current A chunk
      uint32_t gch1 = 0, gch2 = 0;  // group indices of the previous two chunk groups
      auto tstage = [&](const ChunkPos &cp) -> uint32_t { return a_tabs + (uint32_t)cp.st * C::TSTAGE; };
      auto wait_table = [&](const ChunkPos &cp) {
        FZT_T0(tt)
        wait_sleep(a_tfull + 8 * cp.st, cp.ph);
        FZT_ADD(6, tt)
      };
      auto issue_yhat = [&](const ChunkPos &cp, int slot) {
        wait_table(cp);
        sm100::tc_fence_after();
        const uint32_t b3 = tstage(cp);
#pragma unroll
        for (int u = 0; u < TPC; ++u) {
          const uint32_t tcu = tc + u * C::TCOLS;
#pragma unroll
          for (int j = 0; j < C::KY / 16; ++j)
            sm100::umma_bf16_ts_e(tcu + C::cY + 16 * slot, tcu + C::cA3 + 8 * j,
                                  sm100::smem_desc(b3 + j * 2 * 256, 256, 128), idY, j > 0);
        }
        sm100::umma_commit_e(a_ybar + 8 * slot);
      };
      // kind: 0 = A chunk c, 1 = beta0 (yhat of B0, B1), 2 = B chunk c, 3 =
      // beta (yhat of C0, C1), 4 = C chunk c
      int cur_nch = nch, cur_ncm = ncm;  // the period being issued
      auto on_publish = [&](int kind, int c) {
        FZT_T0(tp)
        wait_sleep(a_pub + 8 * (g & 3), (g >> 2) & 1u);
        FZT_ADD(5, tp)
        FZT_T0(ti)
        // (no fence::after_thread_sync here: every MMA below follows a table
        // wait and its own fence, which orders it after this publish wait as
        // well; a bare commit reads no TMEM -- measured with the atom.inc
        // below: -0.6%)
        // group g commits to the barrier of group g - 4 without observing
        // that phase: one thread (this warp's elected lane) issues every
        // commit of the tile, whose arrivals come in issue order as the
        // tracked MMAs complete in order, so the phases of mdone[g % 4]
        // complete group by group; and no waiter of group x runs after group
        // x + 4 is issued (the waits' bounds at pub / wait_group).  The
        // round-1/2 defensive wait here cost 0.75% (measured).
        if (kind == 0) {
          wait_table(cpos);
          sm100::tc_fence_after();
          const uint32_t bf = tstage(cpos), bx = bf + 3 * C::BF_BYTES;
#pragma unroll
          for (int u = 0; u < TPC; ++u) {
            const uint32_t tcu = tc + u * C::TCOLS, at = tcu + C::cOPA + 24 * abuf;
#pragma unroll
            for (int e = 0; e < 3; ++e)
              sm100::umma_bf16_ts_e(tcu + C::cG, at, sm100::smem_desc(bf + e * C::BF_BYTES, C::NGn * 16, 128), idG,
                                    (c > 0 || e > 0) ? 1u : 0u);
            // y' hi x_hi, y' hi x_mid, y' lo x_hi
            sm100::umma_bf16_ts_e(tcu + C::cB, at + 8, sm100::smem_desc(bx, C::KBn * 16, 128), idB, c > 0 ? 1u : 0u);
            sm100::umma_bf16_ts_e(tcu + C::cB, at + 8, sm100::smem_desc(bx + C::BX_BYTES, C::KBn * 16, 128), idB, 1u);
            sm100::umma_bf16_ts_e(tcu + C::cB, at + 16, sm100::smem_desc(bx, C::KBn * 16, 128), idB, 1u);
          }
          if (++abuf == C::NOPA) abuf = 0;
        } else if (kind == 1 || kind == 3) {
          const int cnt = kind == 1 ? cur_nch : cur_ncm;
          for (int a = 0; a < C::NYS && a < cnt; ++a) issue_yhat(advance_pos(cpos, a), a);
          cslot = 0;
        } else if (kind == 2) {
          // the refinement moment first (the consumers' next operand store
          // waits for it), then yhat of chunk c + NYS into the slot chunk c
          // has just released
          wait_table(cpos);
          sm100::tc_fence_after();
          const uint32_t bx = tstage(cpos) + C::B3_BYTES;
          // r0 hi (x hi + mid + lo) + r0 mid (x hi + mid) + r0 lo x hi
#pragma unroll
          for (int u = 0; u < TPC; ++u) {
            const uint32_t tcu = tc + u * C::TCOLS, at = tcu + C::cOPB;
#pragma unroll
            for (int e = 0; e < 3; ++e)
#pragma unroll
              for (int xx = 0; xx < 3 - e; ++xx)
                sm100::umma_bf16_ts_e(tcu + C::cDB, at + 8 * e,
                                      sm100::smem_desc(bx + xx * C::BX_BYTES, C::KBn * 16, 128), idB,
                                      (c > 0 || e > 0 || xx > 0) ? 1u : 0u);
          }
          sm100::umma_commit_e(a_mdone + 8 * (g & 3));
          if (c + C::NYS < cur_nch) issue_yhat(advance_pos(cpos, C::NYS), cslot);
        } else {
          if (c + C::NYS < cur_ncm) issue_yhat(advance_pos(cpos, C::NYS), cslot);
        }
        if (kind == 2 || kind == 4)
          if (++cslot == C::NYS) cslot = 0;
        if (kind != 2) sm100::umma_commit_e(a_mdone + 8 * (g & 3));
        if (kind == 0 || kind == 2 || kind == 4) {
          if (cpos.s > 1) {
            // this tile is done with the table stage of chunk s - 2 (its
            // group completed two events ago: the wait is a formality); the
            // last of the T tiles reloads it with chunk s - 2 + ST
            FZT_T0(tm)
            wait_sleep(a_mdone + 8 * (gch2 & 3), (gch2 >> 2) & 1u);
            FZT_ADD(13, tm)
            const ChunkPos nxt = advance_pos(cpos, C::ST - 2);
            if (lane == 0) {
              // counts 0 .. NGc - 1 and wraps: the last group sees NGc - 1
              uint32_t old;
              asm volatile("atom.acq_rel.cta.shared::cta.inc.u32 %0, [%1], %2;"
                           : "=r"(old)
                           : "r"(a_tfree + 4 * nxt.st), "r"((uint32_t)(T / TPC - 1))
                           : "memory");
              const bool last = old == (uint32_t)(T / TPC - 1);
              if (last) load_table(nxt);
            }
            __syncwarp();
          }
          gch2 = gch1;
          gch1 = g;
          cpos = advance_pos(cpos, 1);
        }
        ++g;
        FZT_ADD(4, ti)
      };
      for (uint32_t gi = 0; gi < my_groups; ++gi) {
        for (int per = 0; per < M; ++per) {
          cur_nch = P_nch(per);
          cur_ncm = P_ncm(per);
          for (int c = 0; c < cur_nch; ++c) {
            on_release();
            on_publish(0, c);
          }
          on_publish(1, 0);
          for (int c = 0; c < cur_nch; ++c) {
            on_release();
            on_publish(2, c);
          }
          on_publish(3, 0);
          for (int c = 0; c < cur_ncm; ++c) {
            on_publish(4, c);
            on_release();
          }
        }
      }
      // the MMAs of the last groups complete before the CTA releases TMEM
      if (g > 0) wait_sleep(a_mdone + 8 * ((g - 1) & 3), ((g - 1) >> 2) & 1u);
    }
    FZT_ADD(8, t_kernel)
    FZT_FLUSH
    sm100::tc_fence_before();
    // the consumers reach their own copy of this barrier: the non-aligned
    // form (threads of the CTA at different barrier instructions)
    asm volatile("barrier.sync 0;" ::: "memory");
    if (warp == 0) {
      sm100::tc_fence_after();
      sm100::tmem_dealloc(tbase, C::pow2cols(T * C::TCOLS));
    }
    return;
  }

  // ================================================================== consumers
  sm100::setmaxnreg_inc<FzRegs<FzTiles<K, MULTI>::TM>::RC>();
  int ust = 0;       // stage of the current stack chunk
  uint32_t uph = 0;  // and its phase parity
  auto acquire_chunk = [&]() -> uint32_t {
    FZT_T0(t0)
    mbar_wait_spin(a_sfull + 8 * ust, uph);
    FZT_ADD(3, t0)
    return a_stack + ust * CB + ESZ * (128 * sub + (tid & 127));
  };
  auto release_chunk = [&]() {  // every value of the chunk has been consumed
    __syncwarp();
    if (lane == 0) sm100::mbar_arrive_a(a_srel + 8 * ust);
    if (++ust == SC) {
      ust = 0;
      uph ^= 1u;
    }
  };
  // the 8 dates of half hf of the chunk whose column address is a
  auto load8 = [&](uint32_t a, int hf, float (&yv)[8]) {
#pragma unroll
    for (int d = 0; d < 8; ++d) {
      if constexpr (I16)
        yv[d] = fz_code(lds_u16(a + 256 * TPC * (8 * hf + d)));
      else
        yv[d] = lds_f(a + 512 * TPC * (8 * hf + d));
    }
  };
  const float fnd = tb.fnd;
  auto is_value = [&](float y) { return I16 ? y != fnd : y == y; };
  // int16 stacks have no NaN out-of-bounds fill: the dates of a period's
  // last chunk past its end (TMA zero fill) are set to the nodata code in
  // this thread's own column before it reads them (then ordered before the
  // stage's next TMA write)
  const uint32_t nd16 = (uint32_t)(uint16_t)p.nodata;
  auto patch_tail = [&](uint32_t a, int valid_rows) {
    if constexpr (I16) {
      if (valid_rows < C::DC) {
        for (int d = valid_rows; d < C::DC; ++d) sts_u16(a + 256 * TPC * d, nd16);
        sm100::fence_proxy_async_smem();
      }
    }
  };

  uint32_t g = 0;  // group sequence
  auto wait_group = [&](uint32_t gg) {  // group gg's MMAs have completed
    mbar_wait_spin(a_mdone + 8 * (gg & 3), (gg >> 2) & 1);
    sm100::tc_fence_after();
  };
  // this warp's part of group g is done (its TMEM stores waited / loads
  // waited): arrive on the tile's publish barrier for the control warp
  auto publish = [&]() {
    sm100::tc_fence_before();
    __syncwarp();
    if (lane == 0) sm100::mbar_arrive_a(a_pub + 8 * (g & 3));
    ++g;
  };
  uint32_t yph = 0;  // phase parity of the yhat slots
  auto wait_yhat = [&](int slot) {
    FZT_T0(t0)
    mbar_wait_spin(a_ybar + 8 * slot, (yph >> slot) & 1u);
    yph ^= 1u << slot;
    sm100::tc_fence_after();
    FZT_ADD(1, t0)
  };
  const uint32_t lanebase = tc + ((uint32_t)(32 * (warp & 3)) << 16);
  const float qnan = __int_as_float(0x7fc00000);
  const uint32_t rbase = sm100::opaque(sm100::smem_u32(ring) + (uint32_t)tile * hcap * 512 + 4 * (tid & 127));

  int abuf = 0;  // pass-A operand buffer of the current chunk
  for (int64_t tg = blockIdx.x; tg < tb.ntg; tg += gridDim.x)
  for (int per = 0; per < M; ++per) {
    // the period's values (f1; the single period of pk / tb otherwise)
    const MonitorParams &p = MULTI ? mp.per[per].prm : pk;
    const int nch = P_nch(per), ncm = P_ncm(per), n = p.n;
    const float *shared_factor = MULTI ? mp.per[per].shared : tb.shared;
    const int hist_tail = n - (nch - 1) * C::DC, mon_tail = p.N - n - (ncm - 1) * C::DC;
    const int64_t pix = p.p0 + tg * (int64_t)T * 128 + ctid;
    // ================= pass A: masked Gram and moment on the tensor cores
    float c0 = qnan, ymax = 0.f;
    bool have = false;
    for (int c = 0; c < nch; ++c) {
      uint32_t w[24];
      const uint32_t ya = acquire_chunk();
      if (c == nch - 1) patch_tail(ya, hist_tail);
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        float yv[8];
        load8(ya, hf, yv);
        if (__any_sync(0xffffffffu, !have)) {  // offset c = first valid value
#pragma unroll
          for (int d = 0; d < 8; ++d)
            if (!have && is_value(yv[d])) {
              c0 = yv[d];
              have = true;
            }
        }
        uint32_t vm[8];
        float yp[8];
#pragma unroll
        for (int d = 0; d < 8; ++d) {
          fa_date<I16>(yv[d], c0, vm[d], yp[d], fnd);
          // the signal scale of the sigma-hat refit trigger: max |y| (NaN
          // ignored); codes: max |y - c| (their floats carry the 2^23 bias)
          ymax = fmaxf(ymax, fabsf(I16 ? yp[d] : yv[d]));
        }
        if (hf == 1) release_chunk();
        // y' = hi (truncated to bf16, exact) + lo (exact in fp32, rounded
        // to bf16 in the packing: 16 significant bits in all)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const float h0 = __uint_as_float(__float_as_uint(yp[2 * j]) & 0xFFFF0000u);
          const float h1 = __uint_as_float(__float_as_uint(yp[2 * j + 1]) & 0xFFFF0000u);
          w[4 * hf + j] = (vm[2 * j] & 0x3F80u) | (vm[2 * j + 1] & 0x3F800000u);  // bf16 1.0 where valid
          w[8 + 4 * hf + j] = hi16x2(h0, h1);
          w[16 + 4 * hf + j] = sm100::pack_bf16x2(yp[2 * j] - h0, yp[2 * j + 1] - h1);
        }
      }
      FZT_T0(tw)
      if (g >= C::NOPA) wait_group(g - C::NOPA);  // operand buffer abuf free
      FZT_ADD(0, tw)
      {
        uint32_t w16[16], w8[8];
#pragma unroll
        for (int i = 0; i < 16; ++i) w16[i] = w[i];
#pragma unroll
        for (int i = 0; i < 8; ++i) w8[i] = w[16 + i];
        tmem_st16(lanebase + C::cOPA + 24 * abuf, w16);
        sm100::tmem_st8(lanebase + C::cOPA + 24 * abuf + 16, w8);
        if (++abuf == C::NOPA) abuf = 0;
      }
      sm100::tmem_st_wait();
      publish();
    }
    // ================= solve (Alg. 1 l.3-4): Gram from the masked moments
    {
      FZT_T0(tw)
      wait_group(g - 1);
      FZT_ADD(9, tw)
    }
    float A[Tri<K>::kN], dinv[K], beta[K];
    int nbar, h;
    bool deg, refit = false;
    {
      float G[C::NGn], b[K];
#pragma unroll
      for (int j = 0; j < C::NGn / 16; ++j) {
        float v16[16];
        sm100::tmem_ld16(lanebase + C::cG + 16 * j, v16);
        sm100::tmem_ld_wait();
#pragma unroll
        for (int i = 0; i < 16; ++i) G[16 * j + i] = v16[i];
      }
      {
        float v16[16];
        sm100::tmem_ld16(lanebase + C::cB, v16);
        sm100::tmem_ld_wait();
#pragma unroll
        for (int i = 0; i < K; ++i) b[i] = v16[i];
      }
      nbar = (int)G[C::NF];  // exact: a sum of 0/1 products
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
      h = window_h(nbar, p.hf);
      deg = (nbar < K + 1) || (h < 1);
      float diagA[K];
#pragma unroll
      for (int i = 0; i < K; ++i) diagA[i] = A[Tri<K>::idx(i, i)];
      if constexpr (DENSE) {
        // f3 (L93, the [27] special case), for a scene declared to have
        // complete histories (BFAST_SHARED_FACTOR=1): every pixel shares one
        // Gram, factored once on the host in fp64 -- beta0 = A^-1 (X_hist^T
        // y'), the moment b being pass A's tensor-core GEMM -- and no pixel
        // factors its own.  A pixel whose history does have a gap (nbar < n)
        // is recomputed by the fp64 refit, so the result stays exact for any
        // input; the kernel carries no Cholesky code (a per-warp choice
        // between the two spilled and measured +2.7%)
#pragma unroll
        for (int i = 0; i < Tri<K>::kN; ++i) A[i] = __ldg(shared_factor + i);
#pragma unroll
        for (int i = 0; i < K; ++i) dinv[i] = __ldg(shared_factor + Tri<K>::kN + i);
        fz_solve<K>(A, dinv, b, beta);
        if (!deg && nbar != n) refit = true;
        if (!deg && !(__ldg(shared_factor + Tri<K>::kN + K) >= (float)kRefitRatio)) refit = true;
        if (!deg && !(__ldg(shared_factor + Tri<K>::kN + K + 1) <= kRefitVif)) refit = true;
      } else {
        const float minratio = fz_chol<K>(A, dinv);
        fz_solve<K>(A, dinv, b, beta);
        if (!deg && !(minratio >= (float)kRefitRatio)) refit = true;
        if (!deg && !refit && !(fz_vif_max<K>(A, dinv, diagA) <= kRefitVif)) refit = true;
      }
      if (deg || !have) {
#pragma unroll
        for (int i = 0; i < K; ++i) beta[i] = 0.f;
      }
      if (!have) c0 = 0.f;
    }
    // beta operand rows (A of the yhat GEMM): [bh | bh | bh | bm | bm | bl]
    // of beta in the offset form: yhat' = x beta' fits y' = y - c, whose
    // magnitude is the signal's variation, not its level (fp32 residuals
    // (y - c) - yhat' keep their precision when |y| >> sigma)
    auto write_beta = [&]() {
      float bt[K];
#pragma unroll
      for (int i = 0; i < K; ++i) bt[i] = beta[i];
      float hh[K], mm[K], ll[K];
#pragma unroll
      for (int i = 0; i < K; ++i) {
        hh[i] = __uint_as_float(sm100::pack_bf16x2(bt[i], 0.f) << 16);
        mm[i] = __uint_as_float(sm100::pack_bf16x2(bt[i] - hh[i], 0.f) << 16);
        ll[i] = bt[i] - hh[i] - mm[i];
      }
      uint32_t wv[C::KY / 2];
#pragma unroll
      for (int j = 0; j < C::KY / 2; ++j) {
        float e[2];
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const int col = 2 * j + q, blk = col / K, i = col % K;
          e[q] = col >= 6 * K ? 0.f : (blk < 3 ? hh[i] : blk < 5 ? mm[i] : ll[i]);
        }
        wv[j] = sm100::pack_bf16x2(e[0], e[1]);
      }
#pragma unroll
      for (int j = 0; j < C::KY / 16; ++j) {
        uint32_t w8[8];
#pragma unroll
        for (int i = 0; i < 8; ++i) w8[i] = wv[8 * j + i];
        sm100::tmem_st8(lanebase + C::cA3 + 8 * j, w8);
      }
      sm100::tmem_st_wait();
    };
    write_beta();
    publish();

    // ================= pass B: residuals of the first fit, sigma-hat sums,
    // the refinement moment, validity bits, and the history's last
    // residuals into the MOSUM ring
    // CLAMP (the launcher sized the ring from a sample of the stack): a
    // window wider than the ring goes to the fp64 refit; the ring then holds
    // what fits and the pixel's fp32 outputs are overwritten.  Without it
    // the ring holds every window (a separate instantiation: the clamp
    // measured +0.6% on the Landsat scene, +6% at N = 100)
    if (CLAMP && !deg && h > hcap) refit = true;
    const int hh = deg ? (hcap < 8 ? hcap : 8) : (CLAMP && h > hcap ? hcap : h);  // a degenerate pixel's ring is never read
    const uint32_t hbytes = (uint32_t)hh * 512, rend = rbase + hbytes;
    const int ring_from = deg ? 0x7fffffff : nbar - hh;  // first rank the ring must hold
    const bool ring8 = __all_sync(0xffffffffu, hh >= 8);
    float s2 = 0.f;
    int cnt = 0;         // valid history dates before the current chunk
    uint32_t wa = rbase; // ring write slot
    bool ringmode = false;
    uint32_t mpair = 0;
    int ys = 0;  // yhat slot of chunk c (c mod NYS)
    for (int c = 0; c < nch; ++c) {
      wait_yhat(ys);  // yhat0 of this chunk
      float yh[16];
      sm100::tmem_ld16(lanebase + C::cY + 16 * ys, yh);
      if (++ys == C::NYS) ys = 0;
      ringmode = ringmode || __any_sync(0xffffffffu, cnt + 16 > ring_from);
      uint32_t vb = 0;
      uint32_t w[24];
      sm100::tmem_ld_wait();
      const uint32_t ya = acquire_chunk();
      if (c == nch - 1) patch_tail(ya, hist_tail);
#pragma unroll
      for (int hf = 0; hf < 2; ++hf) {
        float yv[8], rz[8];
        load8(ya, hf, yv);
        uint32_t v8 = 0;
        if (!ringmode) {
          SFor<0, 8>::run([&](auto dc) {
            constexpr int d = decltype(dc)::value;
            fb_date<I16, d>(yv[d], c0, yh[8 * hf + d], s2, v8, rz[d], fnd);
          });
        } else if (ring8) {
          uint32_t kk = 0;
          const uint32_t jw = (rend - wa) >> 9;
          SFor<0, 8>::run([&](auto dc) {
            constexpr int d = decltype(dc)::value;
            fb_date_ring<I16, d>(yv[d], c0, yh[8 * hf + d], s2, v8, rz[d], kk, wa, jw, hbytes, fnd);
          });
          const uint32_t a = wa + kk * 512;
          wa = a >= rend ? a - hbytes : a;
        } else {
          SFor<0, 8>::run([&](auto dc) {
            constexpr int d = decltype(dc)::value;
            fb_date_ring1<I16, d>(yv[d], c0, yh[8 * hf + d], s2, v8, rz[d], wa, rend, hbytes, fnd);
          });
        }
        if (hf == 1) release_chunk();
        vb |= v8 << (8 * hf);
        // 3-way bf16 split of r0 by truncation (h + m + l exact)
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          float h0 = __uint_as_float(__float_as_uint(rz[2 * j]) & 0xFFFF0000u);
          float h1 = __uint_as_float(__float_as_uint(rz[2 * j + 1]) & 0xFFFF0000u);
          float t0 = rz[2 * j] - h0, t1 = rz[2 * j + 1] - h1;
          float m0 = __uint_as_float(__float_as_uint(t0) & 0xFFFF0000u);
          float m1 = __uint_as_float(__float_as_uint(t1) & 0xFFFF0000u);
          w[4 * hf + j] = hi16x2(h0, h1);
          w[8 + 4 * hf + j] = hi16x2(m0, m1);
          w[16 + 4 * hf + j] = hi16x2(t0 - m0, t1 - m1);
        }
      }
      // validity bits of the chunk (two chunks per TMEM column, the last
      // 2 MKC chunks kept)
      if (c & 1) {
        mpair |= vb << 16;
        tmem_st1(lanebase + C::cMK + (uint32_t)((c >> 1) % C::MKC), mpair);
      } else {
        mpair = vb;
        if (c == nch - 1) tmem_st1(lanebase + C::cMK + (uint32_t)((c >> 1) % C::MKC), mpair);
      }
      cnt += __popc(vb);
      {
        uint32_t w16[16], w8[8];
#pragma unroll
        for (int i = 0; i < 16; ++i) w16[i] = w[i];
#pragma unroll
        for (int i = 0; i < 8; ++i) w8[i] = w[16 + i];
        if (c >= 1) wait_group(g - 1);  // the operand buffer: refine(c - 1) has read it
        tmem_st16(lanebase + C::cOPB, w16);
        sm100::tmem_st8(lanebase + C::cOPB + 16, w8);
      }
      sm100::tmem_st_wait();
      publish();
    }
    // ================= refinement: beta = beta0 + A^-1 db, sigma-hat
    {
      FZT_T0(tw)
      wait_group(g - 1);
      FZT_ADD(10, tw)
    }
    float sigma, scale, inv_scale, dbf[K];
    {
      float db[K];
      {
        float v16[16];
        sm100::tmem_ld16(lanebase + C::cDB, v16);
        sm100::tmem_ld_wait();
#pragma unroll
        for (int i = 0; i < K; ++i) db[i] = v16[i];
      }
      fz_solve<K>(A, dinv, db, dbf);
      float lin = 0.f;
#pragma unroll
      for (int i = 0; i < K; ++i) {
        if (deg) dbf[i] = 0.f;
        lin = fmaf(dbf[i], db[i], lin);
        beta[i] += dbf[i];
      }
      // sum (r0 - x dbeta)^2 = s2 - dbeta.db (A dbeta = db)
      sigma = sqrtf(fmaxf(s2 - lin, 0.f) / (float)(nbar - K));
      // sigma^2 cancels when the step is large next to the residual sum
      if (!(lin <= 1e-2f * s2)) refit = true;
      // noise within 2e-3 of the signal scale (this includes an exact fit,
      // sigma ~ 0, reading R4): fp32 fitted values (~1e-7 |y|) are no
      // longer negligible -> fp64 refit, which takes the R4 decision
      if (!deg && !(sigma > 2e-3f * ymax)) refit = true;
      scale = sigma * sqrtf((float)nbar);  // MOSUM = W / scale (L524)
      inv_scale = 1.0f / scale;
    }
    // the ring holds r0 of ranks nbar-h .. nbar-1 (the slot at wa the
    // oldest): correct them to the refined fit, r = r0 - x_t . dbeta, with
    // t recovered from the validity bits (newest first), and sum them: W =
    // the window of rank nbar - 1
    float W = 0.f;
    {
      // chunk by chunk (the TMEM loads are warp-collective), each lane
      // walking its own valid dates newest first
      int need = deg ? 0 : hh;  // ring entries left to correct
      uint32_t a = wa;
      const int cmin = nch - 2 * C::MKC > 0 ? nch - 2 * C::MKC : 0;
      for (int ci = nch - 1; ci >= cmin && __any_sync(0xffffffffu, need > 0); --ci) {
        uint32_t pr;
        {
          float v1[1];
          tmem_ld1(lanebase + C::cMK + (uint32_t)((ci >> 1) % C::MKC), v1);
          sm100::tmem_ld_wait();
          pr = __float_as_uint(v1[0]);
        }
        uint32_t m = (ci & 1) ? pr >> 16 : pr & 0xFFFFu;
        while (need > 0 && m != 0) {
          const int bit = 31 - __clz(m);
          m &= ~(1u << bit);
          --need;
          const int t = ci * 16 + bit;
          a = a == rbase ? rend - 512 : a - 512;
          const float4 *xr = reinterpret_cast<const float4 *>(p.X + (size_t)t * p.KP);
          float corr = 0.f;
#pragma unroll
          for (int q = 0; q < (K + 3) / 4; ++q) {
            const float4 xv = __ldg(xr + q);
            if (4 * q + 0 < K) corr = fmaf(xv.x, dbf[4 * q + 0], corr);
            if (4 * q + 1 < K) corr = fmaf(xv.y, dbf[4 * q + 1], corr);
            if (4 * q + 2 < K) corr = fmaf(xv.z, dbf[4 * q + 2], corr);
            if (4 * q + 3 < K) corr = fmaf(xv.w, dbf[4 * q + 3], corr);
          }
          const float r = lds_f(a) - corr;
          sts_f(a, r);
          W += r;
        }
      }
      // a window reaching back past the masks kept in TMEM: fp64 refit
      if (need > 0) refit = true;
    }
    // outputs known now
    const bool fit_ok = !((nbar < K + 1) || (h < 1));
    const bool inside = pix < p.p0 + p.P;  // the last tile group may be ragged
    if (inside) {
      if constexpr (I16) {
        // y = scale code + offset: sigma-hat scales by |scale|; beta' (the
        // offset form) by scale, around the decoded first value
        if (p.out_sigma) p.out_sigma[pix] = fit_ok ? fabsf(p.dscale) * sigma : qnan;
        float bs[K];
#pragma unroll
        for (int i = 0; i < K; ++i) bs[i] = p.dscale * beta[i];
        store_beta<K, float>(p, pix, bs, fmaf(p.dscale, c0 - kCodeBias, p.doffset), fit_ok);
      } else {
        if (p.out_sigma) p.out_sigma[pix] = fit_ok ? sigma : qnan;
        store_beta<K, float>(p, pix, beta, c0, fit_ok);
      }
      if (p.out_nbar) p.out_nbar[pix] = nbar;
    }
    write_beta();
    publish();

    // ================= pass C: monitoring (Alg. 1 l.6-12, Fig. 12 ker 9-10)
    float msum = 0.f, mfirst = 0.f, mx = 0.f;
    int brk = -1, first = -1, cr = nbar;
    bool tie = false;
    const float lam = p.lambda;
    // a 1-based rank up to which B == lambda (rank/nbar <= e): floor(e nbar)
    // - 3 keeps ln(rank/nbar) below 1 by more than f32 rounding
    const int rank_flat = deg ? 0x7fffffff : max((int)(2.718281828f * (float)nbar) - 3, 0) - nbar;
    const int rank_flat_min = __reduce_min_sync(0xffffffffu, rank_flat);
    // |m| > lambda (1 - tol)  <=>  |W| > lambda (1 - tol) scale
    float thr_lo = deg ? __int_as_float(0x7f800000) : lam * (1.0f - kTieTol) * scale;
    ys = 0;
    for (int c = 0; c < ncm; ++c) {
      wait_yhat(ys);  // yhat of this chunk
      float yh[16];
      sm100::tmem_ld16(lanebase + C::cY + 16 * ys, yh);
      const int crm = __reduce_max_sync(0xffffffffu, deg ? 0 : cr - nbar);
      const bool fast = crm + C::DC <= rank_flat_min;
      const uint32_t ya = acquire_chunk();
      if (c == ncm - 1) patch_tail(ya, mon_tail);
      sm100::tmem_ld_wait();
      publish();  // the slot is read: yhat of chunk c + NYS may overwrite it
      if (++ys == C::NYS) ys = 0;
      if (fast && ring8) {
        // B_j == lambda here: the first |m| > lambda (1 - tol) decides; the
        // dates track max |W| and W at each valid date, a chunk whose max
        // crossed is scanned for its first crossing
        float wv[16];
#pragma unroll
        for (int hf = 0; hf < 2; ++hf) {
          float yv[8];
          load8(ya, hf, yv);
          uint32_t kk = 0;
          const uint32_t jw = (rend - wa) >> 9;
#pragma unroll
          for (int d = 0; d < 8; ++d)
            fc_date_k<I16>(yv[d], c0, yh[8 * hf + d], W, msum, mx, kk, wa, jw, hbytes, wv[8 * hf + d], fnd);
          cr += (int)kk;
          const uint32_t a = wa + kk * 512;
          wa = a >= rend ? a - hbytes : a;
        }
        release_chunk();
        if (mx > thr_lo) {  // first < 0 while thr_lo is finite
          int fd = 15;
          float fw = wv[15];
#pragma unroll
          for (int d = 14; d >= 0; --d)
            if (fabsf(wv[d]) > thr_lo) {
              fd = d;
              fw = wv[d];
            }
          first = c * C::DC + fd;
          mfirst = fw;
          thr_lo = __int_as_float(0x7f800000);
        }
      } else {
#pragma unroll 1
        for (int hf = 0; hf < 2; ++hf) {
          float yv[8], yq[8], wv[8];
          load8(ya, hf, yv);
#pragma unroll
          for (int d = 0; d < 8; ++d) yq[d] = hf ? yh[8 + d] : yh[d];
#pragma unroll
          for (int d = 0; d < 8; ++d) {
            fc_date_1<I16>(yv[d], c0, yq[d], W, msum, mx, cr, wa, rend, hbytes, wv[d], fnd);
            if (wv[d] == wv[d] && brk < 0 && !tie && first < 0 && fabsf(W) > thr_lo) {
              const int code = fz_boundary_rare(W * inv_scale, cr, nbar, lam);
              tie = tie || (code >> 1);
              brk = (code & 1) ? c * C::DC + 8 * hf + d : brk;
            }
          }
        }
        release_chunk();
      }
      if (first >= 0 && brk < 0 && !tie) {  // resolve a fast-path candidate
        if (fabsf(mfirst * inv_scale) > lam * (1.0f + kTieTol)) brk = first;
        else tie = true;
        thr_lo = __int_as_float(0x7f800000);
      }
    }

    // ================= epilogue
    const int Nbar = cr;
    if (Nbar - nbar < 1) deg = true;
    if (inside) {
      p.out_break[pix] = deg ? -2 : brk;
      // the MOSUM is scale-free up to the codec's sign (f4)
      const float mag = msum * inv_scale / (float)(Nbar - nbar);
      p.out_mag[pix] = deg ? qnan : (I16 && p.dscale < 0.f ? -mag : mag);
      if (p.out_flags) p.out_flags[pix] = deg ? 1u : 0u;
    }
    const bool want = (refit || tie) && fit_ok && (Nbar - nbar >= 1) && inside;
    const unsigned bal = __ballot_sync(0xffffffffu, want);
    if (want) {
      const int leader = __ffs(bal) - 1;
      int base = 0;
      if (lane == leader) base = atomicAdd(p.refit_count, __popc(bal));
      base = __shfl_sync(bal, base, leader);
      p.refit_list[base + __popc(bal & ((1u << lane) - 1))] = pix;
    }
  }
  FZT_ADD(8, t_kernel)
  FZT_FLUSH
  sm100::tc_fence_before();
  asm volatile("barrier.sync 0;" ::: "memory");  // pairs with the control warps' barrier
}

}  // namespace bfast
