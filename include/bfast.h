/*
 * include/bfast.h -- C ABI of the B200-native BFAST-Monitor library
 * (libbfast.so, built from paper_conf_icde_giesekerhvo20_b200/csrc/).
 *
 * The operation is BFAST-Monitor with missing values as defined by
 * Gieseke et al., ICDE 2020 (/root/reference/PAPER.md, "L<n>" = line n):
 * the season-trend model of Eq. (1)-(3) (L51-L68), fitted by least squares
 * on the valid values of the history period (Eq. (5)-(6), L85, L122), the
 * MOSUM process of Eq. (4) (L72-L75) over the compacted residuals, the
 * boundary lambda*sqrt(log+(t/nbar)) and the first-break / magnitude
 * outputs of Algorithm 1 (L128-L136) and of the entry point
 * `bfast k n f lambda hf Y -> [M](i32, f32)` of Fig. 12 (L491-L537).
 * Where the paper is silent or garbled, DESIGN.md "Readings" (R1-R14)
 * states the interpretation implemented; the tags are cited below.
 *
 * Conventions for every entry point:
 *  - extern "C", no exceptions cross the ABI, no C++ types.
 *  - The caller allocates and frees every array.  The library owns only
 *    plan-internal device constants (design matrix, scratch counters).
 *  - Return value: BFAST_OK (0) or a negative bfast_status.  On any
 *    non-OK status nothing has been written to the outputs and
 *    bfast_last_error() returns a thread-local message.
 *  - Argument errors (BFAST_EINVAL) are detected on the host before any
 *    CUDA call: N < 2; n_hist outside [1, N-1]; k < 0; hf outside (0, 1];
 *    lambda <= 0 or not finite; dates not finite or not strictly
 *    increasing; P < 0; ldY < P; a required pointer NULL with P > 0.
 *  - BFAST_EUNSUPPORTED: k > BFAST_K_MAX_HARMONICS, or a size beyond the
 *    kernel's on-chip limits (see bfast_plan_create).
 *  - Per-pixel ill-posedness is data, not an error (reading R4): such a
 *    pixel gets out_break = BFAST_INVALID_PIXEL and a NaN magnitude.
 *  - P == 0 is a valid no-op.
 */
#ifndef BFAST_H
#define BFAST_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define BFAST_ABI_VERSION 1

/* Largest supported number of harmonics k; K = 2k + 2 <= 14 (L77). */
#define BFAST_K_MAX_HARMONICS 6

typedef enum bfast_status {
  BFAST_OK = 0,
  BFAST_EINVAL = -1,       /* invalid argument, nothing written            */
  BFAST_EUNSUPPORTED = -2, /* valid but beyond the implementation's limits  */
  BFAST_ECUDA = -3,        /* CUDA runtime/driver failure                    */
  BFAST_ENOMEM = -4        /* device or pinned host allocation failed        */
} bfast_status;

/* Per-pixel values of out_break besides offsets >= 0 (Fig. 12: -1
   when no break is found; -2 for ill-posed pixels, reading R4). */
#define BFAST_NO_BREAK (-1)
#define BFAST_INVALID_PIXEL (-2)

/* Bits of out_flags. */
#define BFAST_FLAG_DEGENERATE 0x01u /* out_break == -2                      */
#define BFAST_FLAG_REFIT_FP64 0x02u /* fp32 fit ill-conditioned: refitted in fp64 */

/*
 * bfast_args -- one invocation over P pixels.
 *
 * Y         device pointer, float32, time-major: value of pixel p at date t
 *           (0-based) is Y[t * ldY + p] (the paper's Y^T, L185; Fig. 12
 *           types Y as [M][N]f32, L491).  NaN (any payload) = missing
 *           (L164, reading R9).  +-Inf is undefined input.
 * N         number of dates (>= 2).
 * P         number of pixels (>= 0).
 * ldY       leading dimension in elements (>= P).  Rows must be 16-byte
 *           aligned (ldY % 4 == 0 and Y 16-byte aligned) for the TMA path;
 *           other strides use the plain-load kernel.
 * dates     HOST pointer, float64[N], strictly increasing acquisition times
 *           in seasonal cycles (years).  Harmonic j at date t uses
 *           2*pi*j*dates[t]; dates[t] = (t+1)/f reproduces Eq. (3) with
 *           frequency f (L53, L65-L68, reading R11).  The trend regressor is
 *           the 1-based date index t (L53, L65).
 * n_hist    history length n: dates [0, n) form the stable history, dates
 *           [n, N) the monitoring period (L70).
 * k         number of harmonic terms (L53); K = 2k + 2 regressors (L77).
 * h         MOSUM window as a fraction of the valid history, hf in (0, 1]:
 *           the window is t32(r32(nbar) * hf) valid dates, computed in f32
 *           as in Fig. 12 L516 (reading R3).  Pixels with a zero window are
 *           ill-posed.
 * lambda    boundary scale (> 0): B_j = lambda*sqrt(log+((nbar+1+j)/nbar)),
 *           log+(x) = max(1, ln x) (L75, Alg. 1 l.10, reading R6).
 * out_break device int32[P]: offset, in dates, of the first break from the
 *           start of the monitoring period (the original date index of the
 *           first compacted monitoring value whose |MOSUM| exceeds the
 *           boundary, minus n; Alg. 1 l.12-13, Fig. 12, reading
 *           R7); BFAST_NO_BREAK; or BFAST_INVALID_PIXEL.
 * out_magnitude device float32[P]: mean of the MOSUM process over the
 *           whole monitoring period (L136, L405, reading R8); NaN for
 *           invalid pixels.
 * out_beta  optional device float32[P][K]: fitted coefficients in the
 *           basis (1, t, sin 2 pi d, cos 2 pi d, ..., sin 2 pi k d,
 *           cos 2 pi k d) with t 1-based (Eq. (3)); NaN for pixels whose
 *           fit is undefined.
 * out_sigma optional device float32[P]: sigma-hat (L515, reading R1).
 * out_nbar  optional device int32[P]: number of valid history values.
 * out_flags optional device uint8[P]: BFAST_FLAG_* bits.
 * stream    cudaStream_t to launch on; NULL = the legacy default stream.
 */
typedef struct bfast_args {
  const float *Y;
  int64_t N, P, ldY;
  const double *dates;
  int32_t n_hist, k;
  float h, lambda;
  int32_t *out_break;
  float *out_magnitude;
  float *out_beta;
  float *out_sigma;
  int32_t *out_nbar;
  uint8_t *out_flags;
  void *stream;
} bfast_args;

/*
 * bfast_monitor -- the north-star entry.
 * Synchronous: returns after the results are in out_break/out_magnitude.
 * Y, out_break, out_magnitude are DEVICE pointers on the current device;
 * dates is a HOST pointer.  Uses (and caches) a plan for the current
 * device.
 */
int bfast_monitor(const float *Y, int64_t N, int64_t P, const double *dates,
                  int32_t n_hist, int32_t k, float h, float lambda,
                  int32_t *out_break, float *out_magnitude);

/* Extended form: leading dimension, optional outputs, stream.  Asynchronous
   with respect to the host: returns after enqueueing on a->stream -- except
   when a complete history's MOSUM window (floor(h * n_hist) slots per pixel)
   would cost the fused kernel a tile per CTA (long histories, e.g. N = 700):
   the call then samples the stack on a->stream (window_probe_kernel, 2048
   groups of 32 pixels), synchronises the stream once to size the window ring
   from the widest sampled window, and pixels whose window is wider are
   recomputed by the fp64 refit (results unchanged; BFAST_WINDOW_PROBE=0
   keeps the full ring and the asynchrony).  The same holds for
   bfast_plan_execute and the entries built on them.
   BFAST_SHARED_FACTOR=1: warps whose 32
   pixels have no missing history value use the plan's Gram factor,
   computed once in fp64, instead of factoring their own (a separate
   kernel instantiation, off by default: its per-warp test costs scenes
   with gaps; results identical up to fp32 rounding). */
int bfast_monitor_ex(const bfast_args *a);

/*
 * Plans: the per-(N, dates, n_hist, k, h, lambda) device constants -- the
 * design matrix of Eq. (3) built in fp64 on the host and rounded to fp32,
 * with the trend regressor centred and scaled for conditioning (DESIGN.md
 * "Numerics") -- uploaded once to `device`.  A plan may be executed from
 * several host threads and streams of its device; executions sharing a
 * plan are ordered on the device (they share the plan's refit scratch),
 * so use one plan per stream for concurrency.  bfast_plan_create
 * returns BFAST_EUNSUPPORTED if the MOSUM ring for floor(h * n_hist)
 * residuals per pixel does not fit the kernel's shared memory.
 */
typedef struct bfast_plan bfast_plan;
int bfast_plan_create(bfast_plan **out, int device, int64_t N, const double *dates,
                      int32_t n_hist, int32_t k, float h, float lambda);
/* a->N, a->dates, a->n_hist, a->k, a->h, a->lambda must equal the plan's. */
int bfast_plan_execute(const bfast_plan *plan, const bfast_args *a);
void bfast_plan_destroy(bfast_plan *plan);

/*
 * bfast_monitor_host -- end-to-end form on HOST buffers.  The device
 * slabs, streams and events it pipelines with belong to the device's
 * cached plan and are reused by later calls (a stream of tiles allocates
 * once).  Y_host is
 * float32 [N][ldY] (pinned memory gives full PCIe bandwidth; pageable
 * memory works but is slower); out_break_host int32[P] and
 * out_magnitude_host float32[P] are host arrays.  The call uploads the
 * stack in pixel slabs, overlapping the host-to-device copy of slab i+1
 * with the kernel on slab i (two streams, double-buffered device slabs),
 * and copies the results back; synchronous.  `device` < 0 = current
 * device.  Device memory used: about 2 * N * slab * 4 bytes.
 */
int bfast_monitor_host(const float *Y_host, int64_t N, int64_t P, int64_t ldY,
                       const double *dates, int32_t n_hist, int32_t k, float h,
                       float lambda, int32_t *out_break_host, float *out_magnitude_host,
                       int device);

/*
 * bfast_monitor_multi -- shard the pixels of a HOST stack over `ndev`
 * devices (contiguous pixel ranges, multiples of 128 pixels).  Pixels are
 * independent (L142), so there is no collective: each device runs
 * bfast_monitor_host on its slice from its own host thread and writes its
 * slice of the host outputs (the break-map gather).  Synchronous.
 */
int bfast_monitor_multi(const float *Y_host, int64_t N, int64_t P, int64_t ldY,
                        const double *dates, int32_t n_hist, int32_t k, float h,
                        float lambda, const int *devices, int ndev,
                        int32_t *out_break_host, float *out_magnitude_host);

/*
 * bfast_monitor_shards -- device-resident pixel shards on several devices,
 * gathered into ONE output map (pixels are independent,
 * L142, so the only exchange is the break map).  Shard i is the stack
 * Y_dev[i] (device pointer on devices[i], float32 [N][ldY[i]] with P[i]
 * pixels, layout as in bfast_args); its results land at offset
 * P[0] + ... + P[i-1] of out_break / out_magnitude, which are device
 * arrays on `gather_device`.  Each shard's kernel stores its outputs
 * straight into the gather device's memory (peer access over NVLink,
 * enabled by the call): the gather is the epilogue's stores, no copy
 * afterwards.  One host thread per shard, each with its device's cached
 * plan; synchronous.  Several shards may live on the same device.
 * Errors: BFAST_EINVAL for a bad shard description (nothing written);
 * BFAST_ECUDA if peer access between a shard device and gather_device is
 * impossible.
 */
int bfast_monitor_shards(const float *const *Y_dev, const int64_t *P, const int64_t *ldY,
                         const int *devices, int nshards, int64_t N, const double *dates,
                         int32_t n_hist, int32_t k, float h, float lambda, int gather_device,
                         int32_t *out_break, float *out_magnitude);

/*
 * ---- Several monitoring periods per stack pass ------
 * the large-scale runs vary "the start and the end of the
 * monitoring periods ... each lasting one year (2010-2011, 2011-2012, ...)".
 * Period i is the BFAST-Monitor problem on the dates [0, N_end[i]) with
 * history [0, n_hist[i]) (each period its own fit, Alg. 1).
 * bfast_monitor_periods runs all M periods in ONE fused launch: each
 * persistent CTA runs every period of a pixel tile group before the next
 * group, so the stack is read from HBM about once and re-read from L2.
 * a: the stack and scalars as in bfast_monitor_ex (a->n_hist is ignored,
 * a->N >= every N_end[i]); the outputs are period-major: out_break int32
 * [M][P], out_magnitude float [M][P], optional out_beta [M][P][K],
 * out_sigma / out_nbar / out_flags [M][P].  Result of period i = that of
 * bfast_monitor_ex on the first N_end[i] dates with n_hist[i].
 * Environment: BFAST_PERIODS=split runs the periods as separate launches
 * instead (the same results bit for bit; each period then reads its slice
 * of the stack from HBM -- measured faster on B200).
 * Requirements: 1 <= M <= 8 distinct periods, each valid as a bfast_args
 * (n_hist[i] in [1, N_end[i] - 1], N_end[i] <= a->N); the fused kernel
 * (16-byte aligned Y, ldY % 4 == 0).  Errors: BFAST_EINVAL (NULL arrays,
 * a period that fails validation, equal periods); BFAST_EUNSUPPORTED (M >
 * 8, alignment, SIMT-only plans).  Asynchronous on a->stream.
 */
int bfast_monitor_periods(const bfast_args *a, const int32_t *n_hist, const int32_t *N_end, int32_t M);

/*
 * ---- Compact input codec (not from the paper) --------
 * Landsat NDMI products are delivered as scaled int16 with a nodata code;
 * reading the codes halves the stack bytes per date.
 *   y = fmaf(scale, (float)code, offset)  for code != nodata (one rounding)
 *   code == nodata -> missing (the NaN of L164)
 * bfast_monitor_i16 runs the hot path of bfast_monitor_ex on such a stack:
 * codec->Y is the DEVICE stack int16 [N][ldY] (a->ldY counts int16
 * elements; a->Y must be NULL), every other argument and output as in
 * bfast_args, in the units of y.  The result is that of bfast_monitor_ex on
 * the decoded float32 stack up to the parity tolerances: the
 * path runs on the codes and applies the codec to beta, sigma-hat and the
 * MOSUM's sign; flagged pixels are refitted in fp64 on the decoded values.
 * Requirements: a 16-byte aligned codec->Y and ldY % 8 == 0 (TMA rows), the
 * fused tensor-core kernel (not BFAST_KERNEL=simt).  Errors: BFAST_EINVAL
 * (NULL codec/args, a->Y != NULL, scale zero or not finite, offset not
 * finite, nodata outside [-32768, 32767], and every bfast_args rule);
 * BFAST_EUNSUPPORTED (alignment, SIMT-only plan).  Asynchronous on a->stream.
 */
typedef struct {
  const int16_t *Y; /* device [N][ldY] codes */
  float scale;      /* y = fmaf(scale, code, offset) */
  float offset;
  int32_t nodata;   /* the missing-value code, in [-32768, 32767] */
} bfast_codec_i16;
int bfast_monitor_i16(const bfast_codec_i16 *codec, const bfast_args *a);

/*
 * ---- Preprocessing before the hot path --------------
 * after a chunk is copied to the GPU, "removal of slices only
 * containing NaN values"; L379: a Landsat image of Africa spans 6873 dates
 * of which only about 350 slices contain any data, and they "are extracted
 * efficiently before applying the core algorithm".  The monitoring entries
 * never renumber dates (reading R13); these two calls do it explicitly.
 * The caller then runs bfast_monitor* on the compacted stack with the kept
 * dates and n_hist' = #kept dates < n_hist (the trend regressor is then
 * the 1-based index in the compacted stack, as in the paper's pipeline); a
 * break offset b >= 0 maps back to the original date keep_idx[n_hist' + b].
 *
 * bfast_valid_dates -- keep[t] = 1 iff some pixel p < P of date slice t of
 * the DEVICE stack Y (float32 [N][ldY], NaN = missing, any payload) holds
 * a value, else 0.  keep: device int32[N].  Asynchronous on `stream`
 * (NULL = legacy default stream).  A slice stops being read once a value
 * is found, so the cost is about one 32 KB segment per slice with data and
 * the whole slice (4 P bytes) per empty one.  Errors: BFAST_EINVAL (N < 0,
 * P < 0, ldY < P, NULL pointer); BFAST_EUNSUPPORTED (N > 2^31 - 1 or P >
 * 2^29); nothing is written on error.
 */
int bfast_valid_dates(const float *Y, int64_t N, int64_t P, int64_t ldY, int32_t *keep, void *stream);

/*
 * bfast_gather_dates -- Yc[i][p] = Y[idx[i]][p] for i < Nc, p < P: the
 * kept slices (idx: device int32[Nc], normally increasing) of the DEVICE
 * stack Y float32 [N][ldY] as a compact DEVICE stack Yc float32 [Nc][ldYc].
 * A row whose idx[i] is outside [0, N) is filled with NaN (the kernel never
 * reads outside the stack).  Y and Yc must not overlap.  Asynchronous on
 * `stream`.  Errors: BFAST_EINVAL (N < 0, P < 0, Nc < 0, ldY < P, ldYc < P,
 * NULL pointer); BFAST_EUNSUPPORTED (Nc > 65535).
 */
int bfast_gather_dates(const float *Y, int64_t N, int64_t ldY, int64_t P, const int32_t *idx, int64_t Nc,
                       float *Yc, int64_t ldYc, void *stream);

/*
 * bfast_monitor_host_resume -- a scene streamed tile by tile with
 * tile-level resume (the paper splits scenes that do
 * not fit in memory into chunks on the host, L291).  Processes the pixels
 * [*done, P) of the HOST stack (arguments as bfast_monitor_host) in tiles
 * of `tile` pixels, at most `max_tiles` of them (< 0: all), and advances
 * *done past each tile whose results are in the host arrays.  A call that
 * returns early (error, interruption, max_tiles) is resumed by calling it
 * again with the same *done; the results are identical to one
 * uninterrupted call.  Errors: as bfast_monitor_host, plus BFAST_EINVAL for
 * done == NULL, *done outside [0, P] or tile < 1.
 */
int bfast_monitor_host_resume(const float *Y_host, int64_t N, int64_t P, int64_t ldY,
                              const double *dates, int32_t n_hist, int32_t k, float h,
                              float lambda, int32_t *out_break_host, float *out_magnitude_host,
                              int device, int64_t tile, int64_t max_tiles, int64_t *done);

/*
 * Cross-process break-map gather (one process per GPU, torchrun): the
 * process owning the map exports its device allocation as a CUDA IPC
 * handle of BFAST_IPC_HANDLE_BYTES bytes; every other process opens it and
 * passes the mapped pointer (plus its shard offset) as out_break /
 * out_magnitude of bfast_plan_execute, so each rank's kernel writes its
 * slice of the map directly into the owner's GPU memory.  The handle
 * carries no synchronisation: the ranks order their writes before the
 * owner's reads with a barrier (bench.py, tests/test_multi_ipc.py).
 * bfast_ipc_open maps on `device` (< 0: current); bfast_ipc_close unmaps.
 * The exporting allocation must come from cudaMalloc (e.g. a torch
 * tensor's storage base) and outlive every mapping.
 */
#define BFAST_IPC_HANDLE_BYTES 72 /* CUDA IPC handle of the allocation + byte offset */
int bfast_ipc_export(const void *dev_ptr, unsigned char *handle);
int bfast_ipc_open(const unsigned char *handle, int device, void **dev_ptr);
int bfast_ipc_close(void *dev_ptr);

/* Host-side helper (no CUDA): the [begin, end) pixel range of shard
   `rank` of `world` for P pixels, aligned to 128-pixel tiles. */
void bfast_shard_range(int64_t P, int rank, int world, int64_t *begin, int64_t *end);

/*
 * Profiling hook (used by bench.py for the roofline): while enabled on the
 * calling thread, every bfast_plan_execute / bfast_monitor_ex records a CUDA
 * event pair around its fused monitor kernel on the launch stream.
 * bfast_profile_collect synchronizes the recorded events, writes the
 * elapsed milliseconds of up to `max` launches (oldest first) to ms_out,
 * clears the record and returns how many were written (or a negative
 * status).  bfast_profile_enable(0) disables and clears.
 */
int bfast_profile_enable(int on);
int bfast_profile_collect(float *ms_out, int max);

/* Number of device kernels the calling thread's last successful
   bfast_monitor* / bfast_plan_execute call enqueued. */
int bfast_last_launch_count(void);

/* Thread-local description of the last non-OK status ("" if none). */
const char *bfast_last_error(void);
const char *bfast_status_string(int status);
int bfast_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* BFAST_H */
