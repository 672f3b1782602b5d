/*
 * photon.h — C ABI of libphoton, the B200 (sm_100a) hot path of Photon's online analysis.
 *
 * Source of the method: Liu, Sun, Carlson, "Photon: A Fine-grained Sampled Simulation Methodology for GPU
 * Workloads", MICRO '23 (text at PAPER.md; "L<n>" below = a line of that text plus its section/figure/equation).
 * Readings of passages the paper leaves silent or garbled are tagged [P-n]; the register is DESIGN.md §3.
 *
 * Conventions (apply to every entry point):
 *  - Every array pointer is a DEVICE pointer unless its comment says HOST.  The caller owns all inputs, outputs
 *    and workspaces; the library never allocates or frees device memory.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).  Calls only ENQUEUE work on it and
 *    never synchronise, except photon_check (documented below) and the *_count helpers that say "syncs".
 *  - Return value: PHOTON_OK or a negative photon_status.  Host-detectable errors (NULL pointers, sizes, params,
 *    workspace too small) return immediately and enqueue nothing.  Errors only the device can see (a BB id out of
 *    range, non-monotone offsets, a full hash table, an exactness bound exceeded, ...) are LATCHED in the call's
 *    workspace (first error wins: code + element index) and reported by photon_check().
 *  - Outputs are bit-identical across runs, devices, shard counts, and to the CPU oracle (oracle/).
 *  - A photon_ctx is owned by one host thread and one CUDA device.  No C++ exception crosses this ABI.
 */
#ifndef PHOTON_H
#define PHOTON_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define PHOTON_ABI_VERSION 1
#if defined(__GNUC__)
#define PHOTON_API __attribute__((visibility("default")))
#else
#define PHOTON_API
#endif
#define PHOTON_BINS 16 /* "project these BBVs into fixed-size BBVs (We use 16)" — L178 §3 Obs. 5 */

typedef enum {
  PHOTON_OK = 0,
  PHOTON_EINVAL = -1,    /* bad host-side argument: NULL pointer, size or parameter out of range             */
  PHOTON_ECUDA = -2,     /* CUDA runtime / launch error; text via photon_last_error                             */
  PHOTON_ERANGE = -3,    /* device-detected bad input: bb >= n_bb, offsets not monotone, retire < issue,
                            records not retire-sorted, time >= 2^40, per-warp insts >= 2^32, N_k >= 2^50       */
  PHOTON_ECAPACITY = -4, /* a workspace table (warp types, candidate pairs) is full: retry with a larger one    */
  PHOTON_EWORKSPACE = -5 /* ws_bytes smaller than the matching photon_*_workspace_bytes()                       */
} photon_status;

typedef struct photon_ctx photon_ctx; /* opaque host object; owns no device memory */

PHOTON_API int photon_abi_version(void);
/* Creates a context bound to `cuda_device` (reads its SM count).  Returns PHOTON_ECUDA without a usable device. */
PHOTON_API int photon_create(photon_ctx **out, int cuda_device);
PHOTON_API void photon_destroy(photon_ctx *ctx);
/* Host string describing the most recent error of this ctx; valid until the next call on it. */
PHOTON_API const char *photon_last_error(const photon_ctx *ctx);
/* SYNCHRONISES `stream`, then reads the device error latch of the most recent call that used a workspace.
 * Returns that call's device status (PHOTON_OK if none); *bad_index (may be NULL) receives the offending element
 * index (event, warp, record, kernel or slot, per the code) or -1. */
PHOTON_API int photon_check(photon_ctx *ctx, void *stream, int64_t *bad_index);
/* Same as photon_check for an explicit workspace (one of several calls in flight). SYNCHRONISES `stream`. */
PHOTON_API int photon_ws_status(photon_ctx *ctx, const void *ws, void *stream, int64_t *bad_index);

/* Diagnostics.  photon_profile(ctx, 1) resets and enables in-stream CUDA-event timing of each launch section
 * below (events are recorded on the call's stream around the section's kernels); photon_profile_read SYNCHRONISES
 * `stream` and writes, per section, the summed milliseconds and the number of timed sections.
 * photon_launch_count() = libphoton kernel launches since the library was loaded (all contexts). */
enum {
  PHOTON_PROF_BBV_FUSED = 0,    /* fused A1+A2 streaming kernel (photon_warp_group, warp_bbv16 == NULL) */
  PHOTON_PROF_BBV = 1,          /* A1 streaming kernel (photon_bbv_build)                               */
  PHOTON_PROF_KBB = 2,          /* kernel_bb_insts                                                      */
  PHOTON_PROF_GROUP_UNFUSED = 3,/* A2 insertion from materialised BBVs                                 */
  PHOTON_PROF_CANON = 4,        /* canonical type tables + warp remap                                   */
  PHOTON_PROF_SIG = 5,          /* A3 signatures                                                         */
  PHOTON_PROF_SCAN = 6,         /* A4 pair filter + exact check                                          */
  PHOTON_PROF_RESOLVE = 7,      /* A4 launch-order resolution                                            */
  PHOTON_PROF_STABLE = 8,       /* A5 (all kernels)                                                      */
  PHOTON_PROF_PREP = 9,         /* photon_warp_group set-up: table clear, BB table, work items            */
  PHOTON_PROF_N = 10
};
PHOTON_API int photon_profile(photon_ctx *ctx, int enable);
PHOTON_API int photon_profile_read(photon_ctx *ctx, void *stream, double *ms /*[PHOTON_PROF_N] HOST*/,
                                   uint64_t *sections /*[PHOTON_PROF_N] HOST*/);
PHOTON_API uint64_t photon_launch_count(void);

/* ------------------------------------------------------------------------------------------------------------
 * Input 1: the functional basic-block trace of the analysed (sampled) warps, CSR by kernel then by warp.
 * Paper: the online analysis functionally simulates a sample of warps (1%, L208/L258) and records, per warp, the
 * sequence of executed basic blocks; a BB is identified by its start PC (L105, L161) and has a length in
 * instructions.  The trace IS that sample [P-21]: W counts the traced warps.
 * ---------------------------------------------------------------------------------------------------------- */
typedef struct {
  uint32_t n_kernels;              /* K >= 1, kernels in launch order                                              */
  uint32_t n_bb;                   /* B, 1 <= B <= 65536 (global BB-id space)                                      */
  uint64_t n_warps;                /* W  (< 2^40)                                                                  */
  uint64_t n_events;               /* E  (< 2^48)                                                                  */
  const uint64_t *kernel_warp_off; /* [K+1] non-decreasing, [0]=0, [K]=W: kernel k owns warps [off[k],off[k+1])    */
  const uint64_t *warp_event_off;  /* [W+1] non-decreasing, [0]=0, [W]=E: warp w owns events [off[w],off[w+1])     */
  const uint16_t *bb;              /* [E] BB id per event, execution order within a warp; 16-byte aligned          */
  const uint32_t *bb_len;          /* [B] instructions per BB, 1 <= len < 2^17                                    */
  const uint8_t *bb_bin;           /* [B] projection bin (< 16) of each BB [P-2]; NULL => bin(b) = b & 15          */
} photon_trace;

/* Canonical warp-type tables (output of photon_warp_group / photon_types_merge).  Capacity is `capacity` rows
 * (types), at most n_warps are ever needed.  Row order: kernel-major (CSR by kernel_type_off), within a kernel by
 * (count descending, key lexicographically ascending) [P-4]; row 0 of a kernel is its dominant type. */
typedef struct {
  uint64_t capacity;          /* rows allocated in type_key/type_count/type_first_warp                          */
  uint32_t *warp_type;        /* [W] kernel-local canonical type id of each warp (0 = dominant); may be NULL for
                                 photon_types_merge                                                             */
  uint64_t *kernel_type_off;  /* [K+1] CSR: kernel k owns rows [off[k], off[k+1]); off[K] = total types T       */
  uint32_t *type_key;         /* [capacity][16] projected 16-bin BBV of the type (L178) [P-3]                   */
  uint64_t *type_count;       /* [capacity] warps of the type, c_t (L178 "portion of warps")                   */
  uint64_t *type_first_warp;  /* [capacity] lowest (global) warp index with this type                          */
  uint8_t *warp_sampling_ok;  /* [K] 1 iff 100*c_0 > 95*W_k: dominant type holds MORE than 95% (L249) [P-15]   */
} photon_types;

/* ---- A1: per-warp BBV projected to 16 bins (L154, L161, L178) [P-1][P-2] -------------------------------------
 * p_w[j] = sum over events e of warp w with bin(bb[e]) == j of bb_len[bb[e]]    (u32; warp_insts I_w = sum_j p_w[j])
 * kernel_bb_insts[k][b] = sum over warps w of kernel k of count_w(b) * bb_len[b]  (the BB distribution, L208-210)
 * Any output may be NULL (not computed).  Device errors: ERANGE (bb >= n_bb: index = event; non-monotone
 * warp_event_off / kernel_warp_off: index = warp / kernel; I_w >= 2^32: index = warp). */
PHOTON_API size_t photon_bbv_workspace_bytes(const photon_trace *trace);
PHOTON_API int photon_bbv_build(photon_ctx *ctx, const photon_trace *trace, void *ws, size_t ws_bytes,
                     uint32_t *warp_bbv16 /*[W][16] or NULL*/, uint64_t *warp_insts /*[W] or NULL*/,
                     uint64_t *kernel_bb_insts /*[K][B] or NULL*/, void *stream);

/* ---- A2: warp-type grouping + dominance decision (L154, L178, L249) ------------------------------------------
 * Warps of one kernel with equal projected keys form one type [P-3]; canonical order [P-4]; weight_t = c_t / W_k
 * (L178); warp_sampling_ok per L249 [P-15].  warp_bbv16 == NULL runs the fused single-pass path (A1+A2 in one
 * streaming kernel); otherwise keys are read from warp_bbv16 (the unfused path).  The workspace holds an
 * open-addressing hash table sized from `type_capacity_hint` (expected total types; 0 => a default of
 * min(W, 2^20)); if it fills, the call latches PHOTON_ECAPACITY and the caller retries with a larger hint.
 * out->capacity must be >= the number of types found (ECAPACITY otherwise). */
PHOTON_API size_t photon_group_workspace_bytes(const photon_trace *trace, uint64_t type_capacity_hint);
PHOTON_API int photon_warp_group(photon_ctx *ctx, const photon_trace *trace, const uint32_t *warp_bbv16 /*or NULL*/, void *ws,
                      size_t ws_bytes, photon_types *out, void *stream);
/* The same call with its last step -- writing out->warp_type from the canonical ids -- issued on `remap_stream`
 * (after an event wait on `stream`): everything but warp_type is complete in `stream` order when the call's work
 * there is; warp_type is complete in `remap_stream` order.  Lets later per-type work (A3/A4) on `stream` overlap
 * the per-warp write; the caller joins the streams before reading warp_type. */
PHOTON_API int photon_warp_group2(photon_ctx *ctx, const photon_trace *trace, const uint32_t *warp_bbv16 /*or NULL*/,
                                  void *ws, size_t ws_bytes, photon_types *out, void *stream, void *remap_stream);
/* SYNCS the stream and returns kernel_type_off[K] (total types) in *total_types (HOST). */
PHOTON_API int photon_types_total(photon_ctx *ctx, const photon_types *types, uint32_t n_kernels, uint64_t *total_types,
                       void *stream);

/* ---- A3 + A4: GPU-BBV signature and kernel matching (L159 Fig 5, L178, L271 Fig 12) ---------------
 * Signature of kernel k [P-4][P-5]: g_k = concat over its types r = 0..T_k-1 (canonical order) of c_r*key_r[0..15]
 * (u64); mass N_k = sum g_k.  The normalised GPU BBV is g_k / N_k.
 * Distance [P-6]: D(k,r) = sum_i |g_k[i]/N_k - g_r[i]/N_r| over position-aligned, zero-padded signatures.
 * Close: D < theta = theta_num/theta_den [P-7][P-15], decided exactly as
 *        theta_den * sum_i |g_k[i]*N_r - g_r[i]*N_k| < theta_num * N_k * N_r   (u128; N = 0 never matches [P-19]).
 * Warp rule [P-10] (L271 Fig 12 note, L277): (W_k == W_r) or min(W_k, W_r) >= n_cores, with W = warps_total.
 * For k in launch order: cand = { r < k : r in pool, close, warp rule } where pool = representatives (kernels
 * that were not themselves matched) [P-8] or all prior kernels when pool_all_prior = 1.  cand empty => k is a
 * representative, match[k] = -1; else match[k] = argmin over cand of (|W_k - W_r|, r) [P-9] ("closest warp
 * count", L271 Step 3).  match_dist[k] = D(k, match[k]) in fp64 (rel. err < 1e-6); for a representative the
 * minimum D to any earlier member of the pool (warp rule ignored), +inf when there is none or N_k = 0 [P-19]
 * (SURVEY.md §8(a) A4 output).  match_dist is a report: it never changes a decision, and NULL skips it (the
 * representatives' minimum is an extra pass over the pool).
 * The A3 outputs themselves (sig, N = mass; sig_off = 16 * kernel_type_off) are produced by photon_sig_build
 * below with k_lo = 0, k_hi = K: photon_kernel_match recomputes them into its workspace.
 * Device errors: ERANGE (N_k >= 2^50, index = kernel); ECAPACITY (candidate-pair table full). */
typedef struct {
  uint32_t theta_num, theta_den; /* theta = num/den; default 1/20; 1 <= den <= 2^20, num <= 2*den               */
  uint64_t n_cores;              /* equal-warp rule below this count; default 64 (R9 Nano CUs, Table 1)    */
  uint32_t pool_all_prior;       /* 0 = representatives only (default) [P-8]; 1 = every prior kernel           */
} photon_match_params;

/* Workspace for K kernels, T total types and room for `pair_capacity` close pairs (0 => default 16*K + 65536). */
PHOTON_API size_t photon_match_workspace_bytes(uint32_t n_kernels, uint64_t total_types, uint64_t pair_capacity);
PHOTON_API int photon_kernel_match(photon_ctx *ctx, uint32_t n_kernels, const photon_types *types,
                        const uint64_t *warps_total /*[K]*/, photon_match_params params, void *ws, size_t ws_bytes,
                        int64_t *match /*[K]*/, double *match_dist /*[K] or NULL*/, void *stream);

/* A3 (L178, Fig 5) and the split form of photon_kernel_match used by the multi-GPU driver (signatures
 * all-reduced, pair lists all-gathered between the steps).  photon_sig_build is the A3 entry point: it writes g_k
 * (sig, u64, the rows' order: sig_off = 16 * kernel_type_off) and N_k (mass, u64) for kernels [k_lo, k_hi)
 * and zeros for every other kernel (so the buffers of ranks owning disjoint kernel ranges sum, by an all-reduce,
 * to the whole table); ERANGE when N_k >= 2^50.
 * match_scan appends the close pairs (k, r) with k in [k_lo, k_hi) to pairs[] (u64: k << 32 | r), count in
 * *n_pairs (DEVICE u64, zeroed by the call; > pair_capacity means pairs were dropped); `pair_capacity` entries
 * fit and every entry past the last pair holds PHOTON_PAIR_PAD, so fixed-capacity buffers of several ranks can be
 * all-gathered as they are.  match_resolve takes the union of all pair lists (any order; PHOTON_PAIR_PAD entries
 * are skipped) and runs the launch-order resolution; its result does not depend on pair order. */
#define PHOTON_PAIR_PAD 0xFFFFFFFFFFFFFFFFull
PHOTON_API int photon_sig_build(photon_ctx *ctx, uint32_t n_kernels, const uint64_t *kernel_type_off, const uint32_t *type_key,
                     const uint64_t *type_count, uint32_t k_lo, uint32_t k_hi, uint64_t *sig /*[16*T]*/,
                     uint64_t *mass /*[K]*/, void *ws /* >= 256 bytes: error latch */, size_t ws_bytes, void *stream);
PHOTON_API int photon_match_scan(photon_ctx *ctx, uint32_t n_kernels, const uint64_t *kernel_type_off, const uint64_t *sig,
                      const uint64_t *mass, const uint64_t *warps_total, photon_match_params params, uint32_t k_lo,
                      uint32_t k_hi, void *ws, size_t ws_bytes, uint64_t *pairs, uint64_t pair_capacity,
                      uint64_t *n_pairs, void *stream);
/* Diagnostics of the most recent photon_kernel_match on `ws` (K and T as passed there; SYNCS): stats[0] = pairs
 * that passed the conservative fp32 filter, [1] = close pairs (exact), [2] = resolution rounds, [3] = pair capacity. */
PHOTON_API int photon_match_stats(photon_ctx *ctx, uint32_t n_kernels, uint64_t total_types_bound, const void *ws,
                                  size_t ws_bytes, uint64_t *stats /*[4] HOST*/, void *stream);
PHOTON_API int photon_match_resolve(photon_ctx *ctx, uint32_t n_kernels, const uint64_t *kernel_type_off, const uint64_t *sig,
                         const uint64_t *mass, const uint64_t *warps_total, photon_match_params params,
                         const uint64_t *pairs, uint64_t n_pairs, void *ws, size_t ws_bytes, int64_t *match,
                         double *match_dist, void *stream);

/* The chain A1 -> A2 -> A3 -> A4 in one call: photon_warp_group (fused, warp_bbv16 = NULL) into `out` with the
 * group workspace `gws` (photon_group_workspace_bytes), then photon_kernel_match with the match workspace `mws`
 * (photon_match_workspace_bytes(K, out->capacity, ...)) -- the same results and device errors (each workspace
 * latches its own part's).  The library runs independent parts on two internal streams (the filter profiles,
 * pair filter and its candidate segments beside the canonical sort, which also writes A3's g and g/N; the
 * warp_type write beside A4) with event forks and
 * joins: all work is ordered after earlier work on `stream`, and later work on `stream` sees every output.  The
 * fork / join is captured with the rest when `stream` is being captured into a CUDA graph. */
PHOTON_API int photon_analyse(photon_ctx *ctx, const photon_trace *trace, void *group_ws, size_t group_ws_bytes,
                              photon_types *out, const uint64_t *warps_total /*[K]*/, photon_match_params params,
                              void *match_ws, size_t match_ws_bytes, int64_t *match /*[K]*/,
                              double *match_dist /*[K] or NULL*/, void *stream);

/* ---- A5: per-BB stability test + BB-sampling switch (L208-210 Fig 7, L220-229 Eq. 1) -------------------
 * Timing stream: one record per retired BB execution of the detailed simulation, CSR by kernel, each kernel's
 * records sorted by retire time (ties keep input order) [P-18]; times are integer ticks < 2^40 [P-16].
 * For each kernel k and BB type b, walk b's executions in stream order.  At its j-th execution (1-based) with
 * j >= 2n (n = window_n, L229) [P-11], over the last n executions (x = issue, y = retire):
 *   cond1 (Eq. 1; |1-a| < delta, L229):  den > 0 and delta_den*|den - num| < delta_num*den,
 *          num = n*Sxy - Sx*Sy, den = n*Sxx - Sx^2   (exact i128)                                  [P-16]
 *   cond2 (mean check, L229) [P-12][P-17]:  S_2n > 0 and delta_den*|2*S_n - S_2n| < delta_num*S_2n,
 *          S_m = sum of (retire - issue) over the last m executions.
 * The first such execution latches b stable [P-13]: first_stable[k][b] = its position in kernel k's stream
 * (0-based record index relative to kernel_rec_off[k]) and stable_dur_sum[k][b] = S_n; else -1 / 0.
 * Switch (L208, Fig 7) [P-14][P-15]: order k's stable BBs by position; switch_at[k] = the first position at
 * which 100 * sum of their weights > 95 * (total weight), weights = kernel_bb_insts[k][*]; -1 if never or if
 * the total is 0.  rate_num/rate_den replaces 95/100.
 * Device errors: ERANGE (bb >= n_bb, retire < issue, retire decreasing within a kernel, time >= 2^40,
 * non-monotone kernel_rec_off; index = record or kernel). */
typedef struct {
  uint32_t n_kernels, n_bb;        /* K, B as in the trace; K*B < 2^31 (batch kernels otherwise) -> else EINVAL */
  uint64_t n_records;              /* R (< 2^32)                                                                */
  const uint64_t *kernel_rec_off;  /* [K+1]                                                                     */
  const uint16_t *bb;              /* [R]                                                                       */
  const uint64_t *issue, *retire;  /* [R] ticks                                                                 */
} photon_timing;
typedef struct {
  uint32_t window_n;             /* n, default 2048 (L229); 2 <= n <= 8192                                     */
  uint32_t delta_num, delta_den; /* delta, default 3/100 (L229); 1 <= den <= 2^16, num <= den                  */
  uint32_t rate_num, rate_den;   /* switch rate, default 95/100 (L208); 1 <= den <= 2^16, num <= den           */
} photon_stable_params;

PHOTON_API size_t photon_stable_workspace_bytes(const photon_timing *timing);
PHOTON_API int photon_bb_stable(photon_ctx *ctx, const photon_timing *timing, const uint64_t *kernel_bb_insts /*[K][B]*/,
                     photon_stable_params params, void *ws, size_t ws_bytes, int64_t *first_stable /*[K][B]*/,
                     uint64_t *stable_dur_sum /*[K][B] or NULL*/, int64_t *switch_at /*[K]*/, void *stream);

/* ---- N1: warp-level stability + warp-sampling switch (L249, L262, Fig 10 Step 3) -------------------------------
 * Warp stream: one record per warp of the detailed simulation (x = the warp's issue, y = its retire time), CSR by
 * kernel (timing->kernel_rec_off), each kernel's records sorted by retire (ties keep input order) [P-18]; times are
 * integer ticks < 2^40 [P-16]; timing->bb and timing->n_bb are ignored (every record belongs to the kernel's one
 * warp stream: "the issue and retired time for all warps", L262) [N1-c].
 * Kernel k is tested only when warp_sampling_ok[k] != 0 (one warp type holds more than 95% of the warps, L249; the
 * A2 output; NULL = every kernel) [N1-d].  At its j-th warp retirement (1-based) with j >= 2n (n = window_n,
 * default 1024, L262), over the last n warps: cond1 (Eq. 1 slope, |1-a| < delta) and cond2 (mean duration of the
 * last n vs the last 2n: "n and n0" read as n and 2n) [N1-b], both exactly as in photon_bb_stable.  The first such
 * retirement is the switch to warp sampling: switch_at[k] = its 0-based position in kernel k's stream and
 * dur_sum[k] = S_n there, so the predicted time of every later warp is S_n / n ("the average time of the last n1
 * warps", n1 read as n) [N1-e]; else -1 / 0.
 * Workspace: photon_warp_stable_workspace_bytes(warps) bytes, caller-owned.  Device errors (photon_check): ERANGE
 * (retire < issue, retire decreasing within a kernel, time >= 2^40, bad kernel_rec_off; index = record or kernel).
 * Host errors: EINVAL (NULL arrays, K = 0, n outside [2, 8192], bad delta), EWORKSPACE. */
typedef struct {
  uint32_t window_n;             /* n, default 1024 (L262); 2 <= n <= 8192                                     */
  uint32_t delta_num, delta_den; /* delta, default 3/100 (L229, L262); 1 <= den <= 2^16, num <= den           */
} photon_warp_stable_params;

PHOTON_API size_t photon_warp_stable_workspace_bytes(const photon_timing *warps);
PHOTON_API int photon_warp_stable(photon_ctx *ctx, const photon_timing *warps, const uint8_t *warp_sampling_ok /*[K]|NULL*/,
                                  photon_warp_stable_params params, void *ws, size_t ws_bytes,
                                  int64_t *switch_at /*[K]*/, uint64_t *dur_sum /*[K] or NULL*/, void *stream);

/* ---- N3: kernel- and BB-level prediction (Fig 12 Step 4 / L279-281; Fig 7 Step 3, caption L201 / L208) ---------------------
 * photon_kernel_predict: for a kernel k matched to r = match[k] >= 0 (photon_kernel_match), "#insts = #insts^K' *
 * #insts_sample / #insts^K'_sample" and "the IPC of K is predicted to be the same as K'" (L279-281):
 *   pred_insts[k]  = round_half_up(full_insts[r]  * mass[k] / mass[r]),
 *   pred_cycles[k] = round_half_up(full_cycles[r] * mass[k] / mass[r])   (same IPC => same ratio for cycles),
 * with mass = the instructions of each kernel's analysed sample (N_k, photon_sig_build's mass) and full_* the
 * detailed-simulation counts of the representative (as given by the caller) [N3-a]; a representative
 * (match[k] < 0) copies its own full_*.  Exact u128; ERANGE (index k) when r >= k, mass[r] = 0, mass >= 2^50 or a
 * result >= 2^64.  All arrays [K] device, caller-owned; ws >= 256 bytes (error latch).
 * photon_bb_predict: per analysed warp w of kernel k, "accumulating the predicted time of their basic blocks"
 * (L208, Fig 7 caption L201): pred_dur_sum[w] = sum over w's events e of stable_dur_sum[k][bb_e] for the types with
 * first_stable[k][bb_e] >= 0 (photon_bb_stable's outputs; the predicted time is pred_dur_sum[w] / n ticks), and
 * unpredicted[w] = the number of w's events whose type never became stable (rare BBs: the interval model of
 * L231-245, out of scope) [N3-b].  ERANGE: bb >= n_bb (index = event), a warp sum >= 2^64 or decreasing
 * warp_event_off (index = warp).  EINVAL when n_kernels >= 2^24 or n_warps >= 2^40 (the long-warp work list
 * packs both ids in one u64).  ws >= photon_bb_predict_workspace_bytes(trace) (error latch + a work list of
 * the long warps). */
PHOTON_API int photon_kernel_predict(photon_ctx *ctx, uint32_t n_kernels, const int64_t *match, const uint64_t *mass,
                                     const uint64_t *full_insts, const uint64_t *full_cycles, void *ws, size_t ws_bytes,
                                     uint64_t *pred_insts, uint64_t *pred_cycles, void *stream);
PHOTON_API size_t photon_bb_predict_workspace_bytes(const photon_trace *trace);
PHOTON_API int photon_bb_predict(photon_ctx *ctx, const photon_trace *trace, const int64_t *first_stable /*[K][B]*/,
                                 const uint64_t *stable_dur_sum /*[K][B]*/, void *ws, size_t ws_bytes,
                                 uint64_t *pred_dur_sum /*[W]*/, uint32_t *unpredicted /*[W]*/, void *stream);

/* ---- N2: full-BBV exact grouping and tagged-stream ingest (L154, L161) -----------------------------------------
 * photon_warp_group_full: warp types keyed on the FULL BBV -- the execution count of every BB id, "warps that
 *   execute the same instruction sequence ... have the same BBV" (L154, L161) -- instead of the 16-bin projection
 *   of L178 [P-3]: warps w, v of one kernel share a type iff their event multisets are equal.  Outputs as
 *   photon_warp_group (out->capacity >= the number of types, else ECAPACITY); type_key = the 16-bin projection of
 *   the type (warp_bbv16 from photon_bbv_build, identical for all members); rows ordered by (count desc, key asc,
 *   lowest warp asc) [N2-a]; warp_sampling_ok as A2 (L249).  Decided by a 128-bit order-independent hash and then
 *   VERIFIED exactly: every member's event multiset is compared with its type's lowest warp's (equal sequences
 *   at once, else by event counts); a hash collision (probability ~2^-128 per pair) latches PHOTON_ERANGE with the
 *   warp index instead of a result.  ERANGE also for bb >= n_bb and bad offsets.
 *   ws >= photon_group_full_workspace_bytes(trace, hint): its hash table holds 2 x hint types (hint 0: 2 x W,
 *   always enough); the call uses the largest table that fits ws_bytes and latches PHOTON_ECAPACITY if the
 *   types outgrow it (the caller retries with a larger hint).  The error latch is at the workspace's start.
 * photon_ingest_tagged: n tagged events (warp[i] u32 < n_warps: the analysed-warp index, bb[i] u16), interleaved
 *   in any order (as a functional simulator retires them), to the CSR of photon_trace: bb_out[n] = the events
 *   stably sorted by warp (each warp keeps its events' stream order, L125) and warp_event_off[n_warps + 1].
 *   n < 2^32, n_warps < 2^32 (else EINVAL).  ERANGE (index = event): warp[i] >= n_warps.
 *   ws >= photon_ingest_workspace_bytes(n, n_warps). */
PHOTON_API size_t photon_group_full_workspace_bytes(const photon_trace *trace, uint64_t type_capacity_hint);
PHOTON_API int photon_warp_group_full(photon_ctx *ctx, const photon_trace *trace, const uint32_t *warp_bbv16 /*[W][16]*/,
                                      void *ws, size_t ws_bytes, photon_types *out, void *stream);
PHOTON_API size_t photon_ingest_workspace_bytes(uint64_t n_events, uint64_t n_warps);
PHOTON_API int photon_ingest_tagged(photon_ctx *ctx, uint64_t n_events, uint64_t n_warps, const uint32_t *warp /*[n]*/,
                                    const uint16_t *bb /*[n]*/, void *ws, size_t ws_bytes, uint16_t *bb_out /*[n]*/,
                                    uint64_t *warp_event_off /*[n_warps+1]*/, void *stream);

/* ---- N4: persisted signature pool, offline reuse of the analysis (L402, §6.3 "Online/Offline Tradeoff") -------
 * "All data that is generated by the online analysis ... is micro-architecture agnostic.  Hardware researchers can
 * reuse these data" (L402).  Reading [N4-a]: a pool holds the REPRESENTATIVE kernels (match[k] < 0) of one or more
 * earlier runs -- their canonical type rows and launched warp counts -- in launch order; a later run is matched as
 * if the pool's kernels had been launched before its own kernels (the A4 rule above, unchanged), so one of its
 * kernels that is close to a pooled representative reuses that representative's simulation.
 * photon_pool_export: pool <- the representatives of a run (K kernels, types as from photon_warp_group, match as
 *   from photon_kernel_match).  pool->kernel_type_off needs K+1 entries, type_key/type_count pool->capacity rows
 *   (>= the run's total types suffices); warp_type, type_first_warp and warp_sampling_ok of `pool` are unused (may
 *   be NULL).  pool_warps_total [K], pool_kernel_id [K] (the run's index of each pooled kernel) and *n_pool (DEVICE
 *   u32: pooled kernels) are written; ws >= photon_pool_export_workspace_bytes(K).  No device errors.
 * photon_kernel_match_pooled: match[] / match_dist[] over the combined index space [0, Kp + K): indices < Kp are
 *   the pool's kernels (in pool order), Kp + k is this run's kernel k; params and semantics as photon_kernel_match
 *   (a pooled kernel is never matched to a later one; reading [P-8] applies to pool and run alike).  `pool` holds
 *   Kp kernels and Tp_bound >= its total types, `types` the run's K kernels and T_bound >= their total; ws >=
 *   photon_pool_match_workspace_bytes(Kp, Tp_bound, K, T_bound, 0).  Device errors as photon_kernel_match. */
PHOTON_API size_t photon_pool_export_workspace_bytes(uint32_t n_kernels);
PHOTON_API int photon_pool_export(photon_ctx *ctx, uint32_t n_kernels, const photon_types *types,
                                  const uint64_t *warps_total /*[K]*/, const int64_t *match /*[K]*/, void *ws,
                                  size_t ws_bytes, photon_types *pool, uint64_t *pool_warps_total /*[K]*/,
                                  uint32_t *pool_kernel_id /*[K]*/, uint32_t *n_pool /*DEVICE [1]*/, void *stream);
PHOTON_API size_t photon_pool_match_workspace_bytes(uint32_t n_pool, uint64_t pool_types_bound, uint32_t n_kernels,
                                                    uint64_t types_bound, uint64_t pair_capacity);
PHOTON_API int photon_kernel_match_pooled(photon_ctx *ctx, uint32_t n_pool, const photon_types *pool,
                                          const uint64_t *pool_warps_total /*[Kp]*/, uint64_t pool_types_bound,
                                          uint32_t n_kernels, const photon_types *types,
                                          const uint64_t *warps_total /*[K]*/, uint64_t types_bound,
                                          photon_match_params params, void *ws, size_t ws_bytes,
                                          int64_t *match /*[Kp+K]*/, double *match_dist /*[Kp+K] or NULL*/,
                                          void *stream);

/* ---- Multi-GPU merge helpers ------------------------------------------------------------------
 * A shard is a contiguous warp range of the global trace; its local kernel l is global kernel kernel_base + l and
 * its local warp v is global warp warp_base + v.  Rows exchanged between ranks (88 bytes each):       */
typedef struct {
  uint32_t kernel;     /* global kernel id */
  uint32_t pad;
  uint32_t key[16];
  uint64_t count;
  uint64_t first_warp; /* global warp index */
} photon_type_row;
/* Writes the local types as rows (global ids) to rows[0..min(T_local, row_capacity)) and padding rows (kernel =
 * PHOTON_ROW_PAD, skipped by photon_types_merge) to rows[T_local..row_capacity); T_local =
 * local->kernel_type_off[K_local] is stored to *n_rows (DEVICE u64, may be NULL) -- T_local > row_capacity means
 * rows were dropped.  Fixed-capacity row buffers of all ranks can thus be all-gathered without a host sync. */
#define PHOTON_ROW_PAD 0xFFFFFFFFu
PHOTON_API int photon_types_export(photon_ctx *ctx, uint32_t n_kernels_local, const photon_types *local, uint32_t kernel_base,
                        uint64_t warp_base, photon_type_row *rows, uint64_t row_capacity, uint64_t *n_rows,
                        void *stream);
/* Merges rows of all shards (any order; rows with equal (kernel, key) add counts and take the min first_warp)
 * into canonical global tables for K kernels; `kernel_warps` [K] = analysed warps per kernel (for the dominance
 * decision).  global->warp_type is ignored. */
PHOTON_API size_t photon_merge_workspace_bytes(uint64_t n_rows, uint32_t n_kernels);
PHOTON_API int photon_types_merge(photon_ctx *ctx, const photon_type_row *rows, uint64_t n_rows, uint32_t n_kernels,
                       const uint64_t *kernel_warps, void *ws, size_t ws_bytes, photon_types *global, void *stream);
/* warp_type_global[v] = global canonical id of local warp v's type, looked up in the merged table that
 * photon_types_merge left in `merge_ws` (pass the same buffer, unmodified, with the merge's n_rows and K). */
PHOTON_API int photon_types_remap(photon_ctx *ctx, uint32_t n_kernels_local, uint64_t n_warps_local,
                       const uint64_t *kernel_warp_off_local /*[K_local+1]*/, const photon_types *local,
                       uint32_t kernel_base, uint64_t n_rows_merged, uint32_t n_kernels_global, const void *merge_ws,
                       size_t ws_bytes, uint32_t *warp_type_global, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* PHOTON_H */
