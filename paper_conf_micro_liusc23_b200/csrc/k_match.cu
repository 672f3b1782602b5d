// k_match.cu — A3 (GPU-BBV signature) and A4 (kernel matching).
//
// PAPER.md L178 / Fig 5 (L159): the GPU BBV lists the weighted per-type BBVs in descending weight order; [P-5] it is
// scaled to unit L1 mass, so with g_k = concat_t (c_t * key_t) (integers) and N_k = sum g_k the GPU BBV is g_k/N_k.
// Fig 12 (L271) Step 2: "finds all prior kernels whose distance is less than the threshold" [P-6 L1, P-7 theta,
// P-8 pool = representatives, P-15 strict]; Step 3: "selects kernels whose warp count is closest" [P-9]; note:
// warp counts must be equal below the GPU core count [P-10] (also L277).
//
// Design: the decision is exact in u128: theta_den * sum_i |g_k[i] N_r - g_r[i] N_k| <
// theta_num * N_k * N_r.  To avoid the O(K^2 L) exact work, pairs are first filtered with a provably conservative
// fp32 lower bound: the per-bin profile distance sum_j |P_k[j] - P_r[j]| (P = per-bin sums of g/N) is <= D by the
// triangle inequality; a pair is dropped only if that bound exceeds theta by more than its worst rounding error.
// Survivors get the exact u128 check (one warp per pair).  Launch-order resolution (leader clustering) is then a
// parallel fixed point: k is a representative iff none of its close predecessors is one.
#include <cooperative_groups.h>
#include <math.h>

#include "internal.h"

#ifndef PHOTON_UNR
#define PHOTON_UNR 8  // exact-check unroll (profiling builds may override)
#endif
namespace photon {
constexpr int kExactUnroll = PHOTON_UNR;
}

namespace photon {

namespace {

// ---- A3: g = count * key, N = sum g (one warp per kernel) ------------------------------------------------
__global__ void k_sig(uint32_t K, uint32_t k_lo, uint32_t k_hi, const uint64_t* __restrict__ kto,
                      const uint32_t* __restrict__ key, const uint64_t* __restrict__ count, uint64_t* __restrict__ sig,
                      uint64_t* __restrict__ mass, DevErr* err) {
  uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  uint32_t k = warp;
  if (k >= K) return;
  uint64_t r0 = kto[k], r1 = kto[k + 1];
  if (k < k_lo || k >= k_hi) {  // not this caller's kernel: zero (rank buffers then sum to the whole table)
    for (uint64_t i = r0 * 16 + lane; i < r1 * 16; i += 32) sig[i] = 0;
    if (lane == 0) mass[k] = 0;
    return;
  }
  uint64_t acc = 0;
  bool over = false;
  for (uint64_t i = r0 * 16 + lane; i < r1 * 16; i += 32) {
    uint64_t c = count[i >> 4];
    uint64_t g;
    over |= c >= (1ull << 32);
    g = c * (uint64_t)key[i];
    sig[i] = g;
    over |= g >= kMassLimit;
    acc += g;
    over |= acc >= kMassLimit;
  }
  for (int o = 16; o > 0; o >>= 1) {
    acc += __shfl_xor_sync(0xffffffffu, acc, o);
    over |= __shfl_xor_sync(0xffffffffu, (int)over, o) != 0;
  }
  if (lane == 0) {
    if (over || acc >= kMassLimit) latch(err, PHOTON_ERANGE, (int64_t)k);
    mass[k] = acc;
  }
}

// per-bin profile P_k[j] = sum_t g[16t+j] / N_k (filter only), one warp per kernel
__global__ void k_prof(uint32_t K, const uint64_t* __restrict__ kto, const uint64_t* __restrict__ sig,
                       const uint64_t* __restrict__ mass, float* __restrict__ prof, double* __restrict__ invn,
                       uint32_t* __restrict__ prof8, float* __restrict__ sigf) {
  uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= K) return;
  uint32_t k = warp;
  uint64_t r0 = kto[k], r1 = kto[k + 1];
  uint64_t acc = 0;
  const double inv = mass[k] ? 1.0 / (double)mass[k] : 0.0;
  for (uint64_t r = r0 + (lane >> 4); r < r1; r += 2) {
    const uint64_t g = sig[r * 16 + (lane & 15)];
    acc += g;
    if (sigf) sigf[r * 16 + (lane & 15)] = (float)((double)g * inv);
  }
  acc += __shfl_xor_sync(0xffffffffu, acc, 16);
  const uint64_t N = mass[k];
  const double P = N ? (double)acc / (double)N : 0.0;
  // u8 quantisation for the coarse filter: q = round(255 P) in [0, 255], four bins per word (bin j in byte j & 3)
  uint32_t q = (uint32_t)rint(P * 255.0);
  q = q > 255u ? 255u : q;
  uint32_t w = q << (8 * (lane & 3));
  w |= __shfl_xor_sync(0xffffffffu, w, 1);
  w |= __shfl_xor_sync(0xffffffffu, w, 2);
  if (lane < 16) {
    prof[(uint64_t)k * 16 + lane] = (float)P;
    if ((lane & 3) == 0) prof8[(uint64_t)k * 4 + (lane >> 2)] = w;
    if (lane == 0) invn[k] = N ? 1.0 / (double)N : 0.0;
  }
}

// A3 fused with the filter profiles (the single-GPU photon_kernel_match: every kernel, one pass over the type
// rows): g = count x key, N = sum g with the 2^50 bound (as k_sig), then P_k[j], its u8 quantisation, 1/N and the
// normalised copy sigf = g / N (as k_prof).  Lane l covers bin l & 15 of every other row.
__global__ void k_sig_prof(uint32_t K, const uint64_t* __restrict__ kto, const uint32_t* __restrict__ key,
                           const uint64_t* __restrict__ count, uint64_t* __restrict__ sig, uint64_t* __restrict__ mass,
                           float* __restrict__ prof, double* __restrict__ invn, uint32_t* __restrict__ prof8,
                           float* __restrict__ sigf, DevErr* err) {
  const uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (k >= K) return;
  const uint64_t r0 = kto[k], r1 = kto[k + 1];
  uint64_t acc = 0;
  bool over = false;
  for (uint64_t r = r0 + (lane >> 4); r < r1; r += 2) {
    const uint64_t i = r * 16 + (lane & 15);
    const uint64_t c = count[r];
    over |= c >= (1ull << 32);
    const uint64_t g = c * (uint64_t)key[i];
    sig[i] = g;
    over |= g >= kMassLimit;
    acc += g;
    over |= acc >= kMassLimit;
  }
  uint64_t bin = acc + __shfl_xor_sync(0xffffffffu, acc, 16);  // this lane's bin over all rows
  uint64_t N = bin;
  for (int o = 8; o > 0; o >>= 1) N += __shfl_xor_sync(0xffffffffu, N, o);  // 16 bins (lanes 0-15 == 16-31)
  over = __any_sync(0xffffffffu, over) || N >= kMassLimit;
  if (lane == 0) {
    if (over) latch(err, PHOTON_ERANGE, (int64_t)k);
    mass[k] = N;
  }
  const double inv = N ? 1.0 / (double)N : 0.0;
  if (sigf)
    for (uint64_t r = r0 + (lane >> 4); r < r1; r += 2) {
      const uint64_t i = r * 16 + (lane & 15);
      sigf[i] = (float)((double)sig[i] * inv);  // this lane's own store, read back
    }
  const double P = N ? (double)bin / (double)N : 0.0;
  uint32_t q = (uint32_t)rint(P * 255.0);
  q = q > 255u ? 255u : q;
  uint32_t w = q << (8 * (lane & 3));
  w |= __shfl_xor_sync(0xffffffffu, w, 1);
  w |= __shfl_xor_sync(0xffffffffu, w, 2);
  if (lane < 16) {
    prof[(uint64_t)k * 16 + lane] = (float)P;
    if ((lane & 3) == 0) prof8[(uint64_t)k * 4 + (lane >> 2)] = w;
    if (lane == 0) invn[k] = inv;
  }
}

// photon_analyse's split of k_sig_prof, so the filter need not wait for the canonical sort:
// k_prof_slots -- the filter profiles, 1/N and N from the UNSORTED type table (the per-kernel slot lists of the
// canonicalisation; the bin sums are exact integers, so they equal the sorted rows' sums bit for bit);
// g and its fp32 copy g / N in the canonical row order are written by the canonical sort itself (k_types.cu
// emit_sig_row: the sorting warp / CTA sums N_k, the same exact integer).
// zero (optional): the per-k counters the filter and the exact check fill next (kcnt, ccnt) and the survivor count
// and filter ticket (n_maybe, ticket) -- zeroed here instead of by separate memset nodes
struct SegZero {
  uint32_t* kcnt;
  uint32_t* ccnt;
  uint64_t* n_maybe;
  uint32_t* ticket;
  uint64_t* n_pairs;  // the exact check's close-pair count
};
__global__ void k_prof_slots(uint32_t K, const uint64_t* __restrict__ kto, const uint32_t* __restrict__ list,
                             HashTable ht, uint64_t* __restrict__ mass, float* __restrict__ prof,
                             double* __restrict__ invn, uint32_t* __restrict__ prof8, DevErr* err, SegZero z) {
  const uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (z.kcnt && blockIdx.x == 0 && threadIdx.x == 0) {
    *z.n_maybe = 0;
    *z.ticket = 0;
    *z.n_pairs = 0;
  }
  if (k >= K) return;
  if (z.kcnt && lane == 0) {
    z.kcnt[k] = 0u;
    z.ccnt[k] = 0u;
  }
  const uint64_t r0 = kto[k], r1 = kto[k + 1];
  uint64_t acc = 0;
  bool over = false;
  for (uint64_t r = r0 + (lane >> 4); r < r1; r += 2) {
    const uint32_t sl = list[r];
    const uint64_t g = (uint64_t)ht.count[sl] * (uint64_t)ht.key[(uint64_t)sl * 16 + (lane & 15)];
    over |= g >= kMassLimit;
    acc += g;
    over |= acc >= kMassLimit;
  }
  const uint64_t bin = acc + __shfl_xor_sync(0xffffffffu, acc, 16);
  uint64_t N = bin;
  for (int o = 8; o > 0; o >>= 1) N += __shfl_xor_sync(0xffffffffu, N, o);
  over = __any_sync(0xffffffffu, over) || N >= kMassLimit;
  const double inv = N ? 1.0 / (double)N : 0.0;
  const double P = N ? (double)bin / (double)N : 0.0;
  uint32_t q = (uint32_t)rint(P * 255.0);
  q = q > 255u ? 255u : q;
  uint32_t w = q << (8 * (lane & 3));
  w |= __shfl_xor_sync(0xffffffffu, w, 1);
  w |= __shfl_xor_sync(0xffffffffu, w, 2);
  if (lane < 16) {
    prof[(uint64_t)k * 16 + lane] = (float)P;
    if ((lane & 3) == 0) prof8[(uint64_t)k * 4 + (lane >> 2)] = w;
    if (lane == 0) {
      invn[k] = inv;
      mass[k] = N;
      if (over) latch(err, PHOTON_ERANGE, (int64_t)k);
    }
  }
}

// ---- pair filter: 64 x 64 tiles of (k, r < k) --------------------------------------------------------------
constexpr int FT = 64;
struct ScanArgs {
  uint32_t K, k_lo, k_hi;
  const uint64_t* kto;
  const uint64_t* sig;
  const uint64_t* mass;
  const uint64_t* wt;
  const float* prof;
  const uint32_t* prof8;
  uint32_t thr8;  // coarse reject: sum_j |q_k[j] - q_r[j]| >= thr8 implies D >= theta
  const double* invn;
  const float* sigf;
  photon_match_params p;
  float bound;  // reject if profile distance >= bound
  uint64_t* maybe;
  uint64_t* n_maybe;
  uint64_t cap;
  DevErr* err;
  // fused path: close pairs go straight into k's segment [cbeg[k], cbeg[k] + ccnt[k]) of cand (else: pairs list)
  uint32_t* cand;
  const uint64_t* cbeg;
  uint32_t* ccnt;
  // band order (single-GPU path): kernels sorted by the projection f (band_f); tiles of the sorted order whose f
  // ranges differ by >= thr8 are never enumerated
  const uint32_t* order;    // [NB * FT] sorted position -> kernel (>= K: padding)
  const uint32_t* bandlo;   // [NB] first r-block that can hold a partner of k-block kb
  const uint64_t* job_off;  // [NB + 1] jobs before k-block kb
  uint32_t* kcnt;           // survivors per k (the sizes of the candidate segments), or nullptr
  uint32_t* ticket;         // with kcnt: the CTAs' completion counter; the last one scans kcnt into seg_off / seg_cur
  uint64_t* seg_off;
  uint32_t* seg_cur;
};

// Jobs: one k-block (FT kernels) against a run of up to FR r-blocks (rb <= kb).  S(kb) = jobs before k-block kb
//   = sum_{y=1..kb} ceil(y / FR) = FR q(q+1)/2 + rem (q+1), q = kb / FR, rem = kb % FR.
constexpr int FR = 8;
constexpr uint32_t kBandMaxK = 1u << 24;  // band-ordered filter up to this K (one-CTA sort and job scan)
#ifndef PHOTON_BAND
#define PHOTON_BAND 1
#endif
#ifndef PHOTON_FRB
#define PHOTON_FRB 4
#endif
constexpr int FRB = PHOTON_FRB;  // r-blocks per band job (the band's tiles are few: short jobs keep the GPU full)
__host__ __device__ __forceinline__ uint64_t filter_jobs_before(uint64_t kb) {
  const uint64_t q = kb / FR, rem = kb % FR;
  return FR * q * (q + 1) / 2 + rem * (q + 1);
}

// Each thread scores a 4 x 4 block of (k, r) pairs per tile.  Coarse level: the u8-quantised profiles, 4 bins per
// word, give sum_j |q_k[j] - q_r[j]| with four VABSDIFF4.ACC per pair (the k-side words stay in registers for the
// whole job); a sum >= thr8 proves D >= theta.  Fine level, only for pairs the coarse level keeps: the fp32
// profile distance (bin-major shared tiles).  The k-block stays in shared memory for the job; the next r-block is
// fetched into registers while the current one is scored.  A tile's survivors are collected in a shared list of
// tile-local (i, j) (it cannot overflow) and appended after the tile with one global atomic.
constexpr int FTP = FT + 4;  // row stride (floats) of the bin-major profile tiles
__device__ __forceinline__ uint32_t sad4(uint32_t a, uint32_t b, uint32_t acc) { return __vsadu4(a, b) + acc; }

// Band order.  f(k) = sum_{j < 8} q_k[j] - sum_{j >= 8} q_k[j] (u8 profile) satisfies |f(k) - f(r)| <=
// sum_j |q_k[j] - q_r[j]|, so a pair with |f(k) - f(r)| >= thr8 fails the coarse test: with the kernels sorted by f,
// only tiles near the diagonal of the sorted order can hold survivors (C5: ~1/5 of the pairs).
__device__ __forceinline__ int band_f(uint4 q) {
  return (int)(__vsadu4(q.x, 0u) + __vsadu4(q.y, 0u)) - (int)(__vsadu4(q.z, 0u) + __vsadu4(q.w, 0u));
}
constexpr int kBandOff = 2048;  // f + kBandOff in [0, 4096)
// One CTA: counting sort of the kernels by f (order within equal f is immaterial; padding to whole tiles), then per
// k-block the first r-block whose largest f is within thr8 of the block's smallest f, the job count
// ceil((kb - rb_lo + 1) / FRB) and the job prefix.  The projections are read once (8 kernels per thread in flight)
// and kept, with the sorted ones, in shared memory when K fits (kBandSmemK), so the scatter and the binary searches
// touch no global memory.
constexpr uint32_t kBandSmemK = 16384;
template <bool SM>
__global__ void __launch_bounds__(1024) k_band_sort_jobs(uint32_t K, const uint32_t* __restrict__ prof8,
                                                         uint32_t NB, uint32_t* __restrict__ order, int* fsort,
                                                         int thr8, uint32_t* bandlo, uint32_t* job_cnt,
                                                         uint64_t* job_off) {
  extern __shared__ int sm_f[];  // SM: [K] f by kernel, [K] f by sorted position
  __shared__ uint32_t hist[4096];
  __shared__ uint32_t wsum[32];
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  int* fk = SM ? sm_f : nullptr;
  int* fs = SM ? sm_f + K : fsort;
  for (uint32_t i = tid; i < 4096; i += 1024) hist[i] = 0u;
  __syncthreads();
  constexpr int IT = 8;
  for (uint32_t base = 0; base < K; base += 1024u * IT) {
    int f[IT];
#pragma unroll
    for (int u = 0; u < IT; ++u) {
      const uint32_t k = base + u * 1024u + tid;
      f[u] = k < K ? band_f(__ldg((const uint4*)(prof8 + 4ull * k))) : 0;
    }
#pragma unroll
    for (int u = 0; u < IT; ++u) {
      const uint32_t k = base + u * 1024u + tid;
      if (k < K) {
        atomicAdd(&hist[f[u] + kBandOff], 1u);
        if (SM) fk[k] = f[u];
      }
    }
  }
  __syncthreads();
  // exclusive scan of hist: 4 bins per thread
  uint32_t v[4], sum = 0;
#pragma unroll
  for (int j = 0; j < 4; ++j) { v[j] = hist[tid * 4 + j]; sum += v[j]; }
  uint32_t x = sum;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if ((int)lane >= o) x += y;
  }
  if (lane == 31) wsum[wid] = x;
  __syncthreads();
  uint32_t w = wsum[lane];
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, w, o);
    if ((int)lane >= o) w += y;
  }
  uint32_t run = __shfl_sync(0xffffffffu, w, wid) - wsum[wid] + x - sum;
  __syncthreads();
#pragma unroll
  for (int j = 0; j < 4; ++j) { hist[tid * 4 + j] = run; run += v[j]; }
  __syncthreads();
  for (uint32_t k = tid; k < K; k += 1024) {
    const int f = SM ? fk[k] : band_f(__ldg((const uint4*)(prof8 + 4ull * k)));
    const uint32_t pos = atomicAdd(&hist[f + kBandOff], 1u);
    order[pos] = k;
    fs[pos] = f;
  }
  for (uint32_t pos = K + tid; pos < NB * FT; pos += 1024) order[pos] = UINT32_MAX;
  __syncthreads();  // fs (shared or this block's global writes) complete
  for (uint32_t kb = tid; kb < NB; kb += 1024) {
    const int fmin = fs[kb * FT];
    uint32_t lo = 0, hi = kb;  // first rb with fmax(rb) > fmin - thr8 (rb = kb always qualifies)
    while (lo < hi) {
      const uint32_t mid = (lo + hi) >> 1;
      const uint32_t last = mid * FT + FT - 1 < K ? mid * FT + FT - 1 : K - 1;
      if (fs[last] > fmin - thr8) hi = mid; else lo = mid + 1;
    }
    bandlo[kb] = lo;
    job_cnt[kb] = (kb - lo) / FRB + 1;
  }
  __syncthreads();
  cta_scan_counts(job_cnt, NB, job_off, nullptr);
}

template <bool BAND>
__device__ void pair_filter_job(const ScanArgs& a, uint64_t job, uint32_t kb_lo, uint32_t kb_hi) {
  uint32_t kb, rb0, rb1;
  if constexpr (BAND) {
    uint32_t lo = 0, hi = kb_hi - 1;  // last kb with job_off[kb] <= job
    while (lo < hi) {
      const uint32_t mid = (lo + hi + 1) >> 1;
      if (a.job_off[mid] <= job) lo = mid; else hi = mid - 1;
    }
    kb = lo;
    rb0 = a.bandlo[kb] + (uint32_t)(job - a.job_off[kb]) * FRB;
    rb1 = rb0 + FRB - 1 < kb ? rb0 + FRB - 1 : kb;  // inclusive
  } else {
    uint32_t lo = kb_lo, hi = kb_hi - 1;  // last kb with filter_jobs_before(kb) <= job
    while (lo < hi) {
      const uint32_t mid = (lo + hi + 1) >> 1;
      if (filter_jobs_before(mid) <= job) lo = mid; else hi = mid - 1;
    }
    kb = lo;
    rb0 = (uint32_t)(job - filter_jobs_before(kb)) * FR;
    rb1 = rb0 + FR - 1 < kb ? rb0 + FR - 1 : kb;  // inclusive
  }
  // tile row / column -> kernel (identity, or the band order; >= K: none)
  auto kid_of = [&](uint32_t pos) -> uint32_t { return BAND ? a.order[pos] : pos; };

  const uint32_t k0 = kb * FT;
  __shared__ __align__(16) float pk[16][FTP];
  __shared__ __align__(16) uint4 q8rb[2][FT];
  __shared__ uint64_t wk[FT], wrb[2][FT];
  __shared__ uint32_t okk[FT], okrb[2][FT];  // mass > 0 [P-19]
  __shared__ uint32_t kidk[FT], kidr[2][FT];  // the kernels of the tile rows / columns
  // band order: the r-block's fp32 profiles staged too (its tiles are dense in coarse survivors); row stride 17
  __shared__ float prs[BAND ? 2 : 1][BAND ? FT * 17 : 1];
  __shared__ uint16_t s_loc[FT * FT];       // the tile's survivors, tile-local (i, j)
  __shared__ uint32_t s_n;
  __shared__ unsigned long long s_base;
  const int tid = threadIdx.x;
  if (tid == 0) s_n = 0;
  const uint32_t kpad = BAND ? (kb + 1) * FT : a.K;  // rows past K (identity) / padding (band) hold no kernel
  for (int i = tid; i < FT * 16; i += 256) {
    const int row = i >> 4, j = i & 15;
    const uint32_t k = k0 + row < kpad ? kid_of(k0 + row) : UINT32_MAX;
    pk[j][row] = k < a.K ? a.prof[(uint64_t)k * 16 + j] : 0.f;
  }
  if (tid < FT) {
    const uint32_t k = k0 + tid < kpad ? kid_of(k0 + tid) : UINT32_MAX;
    kidk[tid] = k;
    wk[tid] = k < a.K ? a.wt[k] : 0;
    okk[tid] = k < a.K && a.mass[k] != 0;
  }
  const int i0 = (tid >> 4) * 4, j0 = (tid & 15) * 4;
  uint4 qk[4];  // u8 profiles of this thread's 4 k rows
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const uint32_t k = k0 + i0 + u < kpad ? kid_of(k0 + i0 + u) : UINT32_MAX;
    qk[u] = k < a.K ? *(const uint4*)(a.prof8 + (uint64_t)k * 4) : make_uint4(0, 0, 0, 0);
  }
  // register stage of one r-block: one u8 word per thread, (wt, mass != 0) for tid < FT (the fp32 r profiles are
  // read from L1 / L2 by the fine check of the rare coarse survivors only)
  uint32_t sq = 0;
  uint64_t swr = 0;
  uint32_t sok = 0, srid = 0;
  float4 spf = make_float4(0.f, 0.f, 0.f, 0.f);
  auto fetch = [&](uint32_t rb) {
    {
      const uint32_t r = rb * FT + (tid >> 2) < kpad ? kid_of(rb * FT + (tid >> 2)) : UINT32_MAX;
      sq = r < a.K ? a.prof8[(uint64_t)r * 4 + (tid & 3)] : 0u;
      if (BAND && r < a.K) spf = __ldg((const float4*)(a.prof + (uint64_t)r * 16) + (tid & 3));
    }
    if (tid < FT) {
      const uint32_t r = rb * FT + tid < kpad ? kid_of(rb * FT + tid) : UINT32_MAX;
      srid = r;
      swr = r < a.K ? a.wt[r] : 0;
      sok = r < a.K && a.mass[r] != 0;
    }
  };
  auto store = [&](int buf) {
    ((uint32_t*)q8rb[buf])[tid] = sq;
    if (BAND) {
      float* d = &prs[BAND ? buf : 0][(tid >> 2) * 17 + (tid & 3) * 4];
      d[0] = spf.x; d[1] = spf.y; d[2] = spf.z; d[3] = spf.w;
    }
    if (tid < FT) { wrb[buf][tid] = swr; okrb[buf][tid] = sok; kidr[buf][tid] = srid; }
  };
  fetch(rb0);
  store(0);
  __syncthreads();
  int cur = 0;
  for (uint32_t rb = rb0; rb <= rb1; ++rb, cur ^= 1) {
    if (rb < rb1) fetch(rb + 1);  // in flight while this block is scored
    const uint4* q8r = q8rb[cur];
    const uint64_t* wr = wrb[cur];
    const uint32_t* okr = okrb[cur];
    const uint32_t* ridr = kidr[cur];
    const uint32_t r0 = rb * FT;
    // coarse level for all 16 pairs (four VABSDIFF4.ACC each); the per-pair eligibility rules only for survivors
    uint32_t keep = 0;  // bit 4u+v
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      const uint4 qr = q8r[j0 + v];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t sad = sad4(qk[u].w, qr.w, sad4(qk[u].z, qr.z, sad4(qk[u].y, qr.y, __vsadu4(qk[u].x, qr.x))));
        keep |= (sad < a.thr8 ? 1u : 0u) << (4 * u + v);
      }
    }
    for (uint32_t m = keep; m; m &= m - 1) {
      const int bit = __ffs(m) - 1, i = i0 + (bit >> 2), j = j0 + (bit & 3);
      const uint64_t Wk = wk[i], Wr = wr[j];
      // each unordered pair once: the identity order needs r < k; the band order takes the tile triangle (sorted
      // position of the row > that of the column) and either launch order
      const bool tri = BAND ? (rb < kb || j < i) : (r0 + j < k0 + i && k0 + i >= a.k_lo && k0 + i < a.k_hi);
      const bool ok = okr[j] && tri && okk[i] && (Wk == Wr || (Wk < Wr ? Wk : Wr) >= a.p.n_cores);  // [P-10]
      if (!ok) keep &= ~(1u << bit);
    }
    // fine level for the coarse survivors: fp32 profile distance
    for (uint32_t m = keep; m; m &= m - 1) {
      const int bit = __ffs(m) - 1, i = i0 + (bit >> 2), j = j0 + (bit & 3);
      float pr[16];
      if (BAND) {
#pragma unroll
        for (int b = 0; b < 16; ++b) pr[b] = prs[BAND ? cur : 0][j * 17 + b];
      } else {
        const float4* rp = (const float4*)(a.prof + (uint64_t)(r0 + j) * 16);  // r < K (eligible)
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          const float4 v = __ldg(rp + q);
          pr[4 * q] = v.x; pr[4 * q + 1] = v.y; pr[4 * q + 2] = v.z; pr[4 * q + 3] = v.w;
        }
      }
      float d = 0.f;
#pragma unroll
      for (int b = 0; b < 16; ++b) d += fabsf(pk[b][i] - pr[b]);
      if (!(d < a.bound)) keep &= ~(1u << bit);
    }
    // survivors of this tile go to a shared list as tile-local (i, j) (at most FT * FT, so it never overflows) and
    // are flushed to the global list after the tile: one global atomic per tile with survivors
    for (uint32_t m = keep; m; m &= m - 1) {
      const int bit = __ffs(m) - 1;
      const uint32_t sp = atomicAdd(&s_n, 1u);
      s_loc[sp] = (uint16_t)((i0 + (bit >> 2)) * FT + j0 + (bit & 3));
    }
    __syncthreads();
    const uint32_t ns = s_n;
    if (ns) {
      if (tid == 0) s_base = atomicAdd((unsigned long long*)a.n_maybe, (unsigned long long)ns);
      __syncthreads();
      for (uint32_t t = tid; t < ns; t += 256) {
        const uint32_t ij = s_loc[t], i = ij / FT, j = ij % FT;
        uint32_t k = k0 + i, r = r0 + j;
        if (BAND) {
          const uint32_t x = kidk[i], y = ridr[j];
          k = x > y ? x : y;
          r = x > y ? y : x;
        }
        const unsigned long long pos = s_base + t;
        if (pos < a.cap) {
          a.maybe[pos] = ((uint64_t)k << 32) | r;
          if (a.kcnt) atomicAdd(&a.kcnt[k], 1u);
        } else {
          latch(a.err, PHOTON_ECAPACITY, (int64_t)pos);
        }
      }
      __syncthreads();  // the list is read before it is reset
      if (tid == 0) s_n = 0;
    }
    if (rb < rb1) store(cur ^ 1);  // that buffer was last read before the previous barrier
    __syncthreads();
  }
}

#ifndef PHOTON_FMINB
#define PHOTON_FMINB 0  // > 0: __launch_bounds__(256, PHOTON_FMINB)
#endif
#if PHOTON_FMINB > 0
#define PHOTON_FMINB_LB __launch_bounds__(256, PHOTON_FMINB)
#else
#define PHOTON_FMINB_LB __launch_bounds__(256)
#endif
template <bool BAND>
__global__ void PHOTON_FMINB_LB k_pair_filter(ScanArgs a, uint64_t job0, uint32_t kb_lo, uint32_t kb_hi) {
  const uint64_t job = job0 + blockIdx.x;
  // band: the grid is sized for every tile of the triangle, the band needs fewer jobs
  if (!BAND || job < a.job_off[kb_hi]) pair_filter_job<BAND>(a, job, kb_lo, kb_hi);
  if (a.ticket) {  // the last CTA to finish scans the per-k survivor counts into the candidate segments
    __shared__ bool s_last;
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(a.ticket, 1u) + 1 == gridDim.x;
    __syncthreads();
    if (s_last) {
      __threadfence();
      cta_scan_counts(a.kcnt, a.K, a.seg_off, a.seg_cur);
    }
  }
}

// exact Dnum = sum_i |g_k[i] N_r - g_r[i] N_k| (zero padded), by a group of G lanes (G | 32, aligned); all lanes
// of the group return the total
template <int G>
__device__ u128 group_dnum(const uint64_t* sig, const uint64_t* kto, const uint64_t* mass, uint32_t k, uint32_t r,
                          bool act = true) {
  const uint32_t l = threadIdx.x & (G - 1);
  uint64_t ok = 0, orr = 0, Lk = 0, Lr = 0, Nk = 0, Nr = 0;
  if (act) {  // inactive groups only join the shuffles
    ok = kto[k] * 16;
    orr = kto[r] * 16;
    Lk = (kto[k + 1] - kto[k]) * 16;
    Lr = (kto[r + 1] - kto[r]) * 16;
    Nk = mass[k];
    Nr = mass[r];
  }
  const uint64_t L = Lk > Lr ? Lk : Lr;
  u128 acc = 0;
#pragma unroll 4
  for (uint64_t i = l; i < L; i += G) {
    const uint64_t gk = i < Lk ? sig[ok + i] : 0, gr = i < Lr ? sig[orr + i] : 0;
    const u128 x = (u128)gk * Nr, y = (u128)gr * Nk;
    acc += x > y ? x - y : y - x;
  }
  uint64_t lo = (uint64_t)acc, hi = (uint64_t)(acc >> 64);
  for (int o = G / 2; o > 0; o >>= 1) {
    const uint64_t lo2 = __shfl_xor_sync(0xffffffffu, lo, o), hi2 = __shfl_xor_sync(0xffffffffu, hi, o);
    const uint64_t sm = lo + lo2;
    hi = hi + hi2 + (sm < lo ? 1 : 0);
    lo = sm;
  }
  return ((u128)hi << 64) | lo;
}
__device__ __forceinline__ u128 warp_dnum(const uint64_t* sig, const uint64_t* kto, const uint64_t* mass, uint32_t k,
                                          uint32_t r) {
  return group_dnum<32>(sig, kto, mass, k, r);
}

// Screen of D = sum_i |g_k[i]/N_k - g_r[i]/N_r| by a group of G lanes (all lanes return the sum and its error
// bound).  With the fp32 copy sigf (each value RN32(g / N), relative error <= 2^-24, unit mass per kernel) the fp32
// |a - b| terms and their fp32 sum are within (L + 8) * 2^-21 of D.  Without it every term is RN(RN(g) * RN(1/N))
// in fp64 (g < 2^50 is exact), within (L + 8) * 2^-50.
template <int G>
__device__ double group_dfp(const uint64_t* __restrict__ sig, const float* __restrict__ sigf,
                            const uint64_t* __restrict__ kto, const double* __restrict__ invn, uint32_t k, uint32_t r,
                            bool act, double& eps) {
  const uint32_t l = threadIdx.x & (G - 1);
  uint64_t Lk = 0, Lr = 0, ok = 0, orr = 0;
  double ik = 0.0, ir = 0.0;
  if (act) {
    ok = kto[k];
    orr = kto[r];
    Lk = (kto[k + 1] - ok) * 16;
    Lr = (kto[r + 1] - orr) * 16;
    ik = invn[k];
    ir = invn[r];
  }
  const uint64_t L = Lk > Lr ? Lk : Lr;
  double acc = 0.0;
  if (sigf) {
    const float* pk = sigf + ok * 16;
    const float* pr = sigf + orr * 16;
    float af = 0.f;
#pragma unroll kExactUnroll
    for (uint64_t i = l; i < L; i += G) {
      const float a = i < Lk ? pk[i] : 0.f;
      const float b = i < Lr ? pr[i] : 0.f;
      af += fabsf(a - b);
    }
    acc = af;
    eps = (double)(L + 8) * 0x1p-21;
  } else {
    const uint64_t* pk = sig + ok * 16;
    const uint64_t* pr = sig + orr * 16;
#pragma unroll kExactUnroll
    for (uint64_t i = l; i < L; i += G) {
      const double a = i < Lk ? (double)pk[i] * ik : 0.0;
      const double b = i < Lr ? (double)pr[i] * ir : 0.0;
      acc += fabs(a - b);
    }
    eps = (double)(L + 8) * 0x1p-50;
  }
  for (int o = G / 2; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  return acc;
}

// one group of XG lanes per filtered pair: close <=> theta_den * Dnum < theta_num * N_k * N_r (Fig 12, [P-15]).
// The fp64 screen decides every pair whose distance is farther than its error bound from theta; the rest (ties
// within ~1e-9) take the exact u128 sum.
#ifndef PHOTON_XG
#define PHOTON_XG 8  // lanes per pair (profiling builds may override)
#endif
constexpr int XG = PHOTON_XG;
#ifndef PHOTON_XGRID
#define PHOTON_XGRID 5  // k_pair_exact CTAs per SM (grid-stride rounds; all resident)
#endif
#ifndef PHOTON_XMINB
#define PHOTON_XMINB 5  // k_pair_exact: minimum resident CTAs per SM (a register cap without spills)
#endif
__global__ void __launch_bounds__(256, PHOTON_XMINB) k_pair_exact(ScanArgs a, uint64_t* pairs, uint64_t pair_cap,
                                                    uint64_t* n_pairs) {
  uint64_t n = *a.n_maybe;
  if (n > a.cap) n = a.cap;
  const uint64_t g = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) / XG;
  const uint64_t ng = ((uint64_t)gridDim.x * blockDim.x) / XG;
  const uint64_t rounds = (n + ng - 1) / ng;  // every lane runs the same number of rounds (shuffles stay converged)
  const double theta = (double)a.p.theta_num / (double)a.p.theta_den;
  for (uint64_t it = 0; it < rounds; ++it) {
    const uint64_t q = g + it * ng;
    const bool act = q < n;
    const uint64_t pr = act ? a.maybe[q] : 0;
    const uint32_t k = (uint32_t)(pr >> 32), r = (uint32_t)pr;
    double eps = 0.0;
    const double d = group_dfp<XG>(a.sig, a.sigf, a.kto, a.invn, k, r, act, eps);
    eps += theta * 0x1p-50;
    bool close = d < theta - eps;
    const bool unsure = act && !close && !(d > theta + eps);
    if (__any_sync(0xffffffffu, unsure)) {  // rare: exact u128 decision for this round's unsure pairs
      const u128 dn = group_dnum<XG>(a.sig, a.kto, a.mass, k, r, unsure);
      if (unsure) close = (u128)a.p.theta_den * dn < (u128)a.p.theta_num * ((u128)a.mass[k] * a.mass[r]);
    }
    if (act && close && (threadIdx.x & (XG - 1)) == 0) {
      const unsigned long long pos = atomicAdd((unsigned long long*)n_pairs, 1ull);
      if (a.cand) {  // fused path: the close r into k's candidate segment (sized by k's filter survivors)
        const uint64_t pos_c = a.cbeg[k] + atomicAdd(&a.ccnt[k], 1u);
        PHOTON_DCHECK(pos_c < a.cbeg[k + 1], "close pair past k's candidate segment", k);
        a.cand[pos_c] = r;
      } else if (pos < pair_cap) {
        pairs[pos] = pr;
      } else {
        latch(a.err, PHOTON_ECAPACITY, (int64_t)pos);
      }
    }
  }
}

// ---- resolve -------------------------------------------------------------------------------------------------
__device__ __forceinline__ uint64_t pair_count(uint64_t n_host, const uint64_t* n_dev) {
  return n_dev ? umin64(*n_dev, n_host) : n_host;
}

__global__ void k_cand_count(const uint64_t* pairs, uint64_t n_host, const uint64_t* n_dev, uint32_t K, uint32_t* cnt,
                             DevErr* err) {
  uint64_t n = pair_count(n_host, n_dev);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    if (pairs[i] == PHOTON_PAIR_PAD) continue;  // padding of a fixed-capacity exchange
    uint32_t k = (uint32_t)(pairs[i] >> 32), r = (uint32_t)pairs[i];
    if (k >= K || r >= k) { latch(err, PHOTON_EINVAL, (int64_t)i); continue; }
    atomicAdd(&cnt[k], 1u);
  }
}

__global__ void __launch_bounds__(1024) k_cand_scan(const uint32_t* cnt, uint32_t K, uint64_t* off, uint32_t* cur) {
  cta_scan_counts(cnt, K, off, cur);
}

__global__ void k_cand_scatter(const uint64_t* pairs, uint64_t n_host, const uint64_t* n_dev, uint32_t K,
                               const uint64_t* off, uint32_t* cur, uint32_t* cand) {
  uint64_t n = pair_count(n_host, n_dev);
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  uint32_t k = (uint32_t)(pairs[i] >> 32), r = (uint32_t)pairs[i];
  if (k >= K || r >= k) return;
  const uint64_t pos = off[k] + atomicAdd(&cur[k], 1u);
  PHOTON_DCHECK(pos < off[k + 1], "candidate past k's segment", k);
  cand[pos] = r;
}


// Fixed point of the launch-order rule (small K, one CTA): state 1 = representative, 2 = matched, 0 = undecided.
// Round-synchronous: every round reads the states of the previous round only (barrier), decides each undecided
// kernel whose candidates allow it (a representative among them -> matched; none undecided -> representative),
// and writes the decisions after a second barrier -- no thread reads a state another thread is writing.  The
// result is the same fixed point (states are monotone); the rounds are at most the longest chain of undecided
// predecessors.  pool_all: every prior kernel counts, so any candidate decides (matched) at once.
constexpr uint32_t kResolveSmemK = 4096;
__global__ void k_pool_all_states(uint32_t K, const uint32_t* cnt, uint8_t* state, uint32_t* flag) {
  const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k < K) state[k] = cnt[k] > 0 ? 2 : 1;
  if (k == 0) flag[0] = 1;
}  // kernels per thread-owned slice: K <= 4 x 1024
__global__ void __launch_bounds__(1024) k_resolve_rounds(uint32_t K, const uint64_t* beg, const uint32_t* cnt,
                                                         const uint32_t* cand, uint8_t* state, uint32_t* flag,
                                                         uint32_t pool_all) {
  __shared__ uint8_t st[kResolveSmemK];
  for (uint32_t k = threadIdx.x; k < K; k += blockDim.x) st[k] = pool_all ? (cnt[k] > 0 ? 2 : 1) : 0;
  uint32_t rounds = 0;
  if (!pool_all) {
    for (;;) {
      ++rounds;
      __syncthreads();  // the previous round's decisions are visible
      uint8_t dec[kResolveSmemK / 1024];
      int open = 0;
#pragma unroll
      for (int j = 0; j < (int)(kResolveSmemK / 1024); ++j) {
        const uint32_t k = threadIdx.x + j * 1024;
        dec[j] = 0;
        if (k >= K || st[k] != 0) continue;
        const uint64_t o0 = beg[k], o1 = o0 + cnt[k];
        bool rep = false, und = false;
        for (uint64_t i = o0; i < o1 && !rep; ++i) {
          const uint8_t s = st[cand[i]];
          rep = s == 1;
          und |= s == 0;
        }
        dec[j] = rep ? 2 : (und ? 0 : 1);
        open |= dec[j] == 0;
      }
      const int any_open = __syncthreads_or(open);  // every read of this round is done
#pragma unroll
      for (int j = 0; j < (int)(kResolveSmemK / 1024); ++j) {
        const uint32_t k = threadIdx.x + j * 1024;
        if (k < K && dec[j] != 0) st[k] = dec[j];
      }
      if (!any_open) break;
    }
  }
  __syncthreads();
  for (uint32_t k = threadIdx.x; k < K; k += blockDim.x) state[k] = st[k];
  if (threadIdx.x == 0) flag[0] = rounds;
}

// The same fixed point in ONE pass over the whole GPU, without barriers: warp j decides kernels j, j + nw, ... in
// increasing order, each by the sequential rule (k is a representative iff none of its close predecessors is one),
// waiting on a predecessor that is still undecided.  A predecessor r < k belongs to an earlier iteration of some
// warp (or the same iteration of a warp with a smaller index), and the smallest undecided kernel never waits, so
// with every warp resident (cooperative launch) the waits always end.  A kernel stops at its first representative.
__global__ void __launch_bounds__(256) k_resolve_spin(uint32_t K, const uint64_t* __restrict__ beg,
                                                      const uint32_t* __restrict__ cnt,
                                                      const uint32_t* __restrict__ cand, uint8_t* state,
                                                      uint32_t* flag) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  volatile uint8_t* vs = state;
  for (uint64_t k = gw; k < K; k += nw) {
    const uint64_t o0 = beg[k], o1 = o0 + cnt[k];
    bool rep_found = false;
    for (;;) {  // a sweep over all candidates: any representative decides at once; else wait while any is open
      bool open = false;
      for (uint64_t i0 = o0; i0 < o1; i0 += 32) {
        const uint64_t i = i0 + lane;
        const uint8_t st = i < o1 ? vs[cand[i]] : (uint8_t)2;
        if (__ballot_sync(0xffffffffu, st == 1)) { rep_found = true; break; }
        open |= __ballot_sync(0xffffffffu, st == 0) != 0;
      }
      if (rep_found || !open) break;
      __nanosleep(100);  // back off: many waiting warps poll L2
    }
    __syncwarp();
    if (lane == 0) vs[k] = rep_found ? 2 : 1;
  }
  if (gw == 0 && lane == 0) flag[0] = 1;
}


// match[k] = argmin over eligible candidates of (|W_k - W_r|, r); match_dist exact -> fp64 (one warp per kernel)
__global__ void k_resolve_match(uint32_t K, const uint64_t* beg, const uint32_t* cnt, const uint32_t* cand,
                                const uint8_t* state,
                                uint32_t pool_all, const uint64_t* wt, const uint64_t* kto, const uint64_t* sig,
                                const uint64_t* mass, int64_t* match, double* dist) {
  uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= K) return;
  uint32_t k = warp;
  uint64_t best_dw = ~0ull;
  uint32_t best_r = UINT32_MAX;
  if (state[k] == 2) {
    for (uint64_t i = beg[k] + lane; i < beg[k] + cnt[k]; i += 32) {
      uint32_t r = cand[i];
      if (!pool_all && state[r] != 1) continue;
      uint64_t dw = wt[k] > wt[r] ? wt[k] - wt[r] : wt[r] - wt[k];
      if (dw < best_dw || (dw == best_dw && r < best_r)) { best_dw = dw; best_r = r; }
    }
  }
  for (int o = 16; o > 0; o >>= 1) {
    uint64_t dw2 = __shfl_xor_sync(0xffffffffu, best_dw, o);
    uint32_t r2 = __shfl_xor_sync(0xffffffffu, best_r, o);
    if (dw2 < best_dw || (dw2 == best_dw && r2 < best_r)) { best_dw = dw2; best_r = r2; }
  }
  if (best_r == UINT32_MAX) {
    if (lane == 0) { match[k] = -1; if (dist) dist[k] = INFINITY; }
    return;
  }
  if (lane == 0) match[k] = (int64_t)best_r;
  if (dist) {
    u128 d = warp_dnum(sig, kto, mass, k, best_r);
    if (lane == 0) {
      u128 den = (u128)mass[k] * mass[best_r];
      double dn = (double)(uint64_t)(d >> 64) * 18446744073709551616.0 + (double)(uint64_t)d;
      double dd = (double)(uint64_t)(den >> 64) * 18446744073709551616.0 + (double)(uint64_t)den;
      dist[k] = dn / dd;
    }
  }
}

// match_dist of a representative (match[k] < 0): the minimum D to any earlier member of the pool [P-8] (warp rule
// ignored; SURVEY.md §8(a) A4 output), +inf when there is none or N_k = 0 [P-19].  One warp per kernel: an fp64
// pass over the pool (each D within (L + 8) * 2^-50 of exact) finds the minimum, then the exact u128 numerator of
// every candidate within twice that bound of it picks the exact minimum.  Only when match_dist is requested.
__device__ __forceinline__ double warp_d64(const uint64_t* sig, const uint64_t* kto, const uint64_t* mass, uint32_t k,
                                           uint32_t r, double& eps) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t ok = kto[k], orr = kto[r];
  const uint64_t Lk = (kto[k + 1] - ok) * 16, Lr = (kto[r + 1] - orr) * 16, L = Lk > Lr ? Lk : Lr;
  const double ik = 1.0 / (double)mass[k], ir = 1.0 / (double)mass[r];
  double acc = 0.0;
  for (uint64_t i = lane; i < L; i += 32) {
    const double a = i < Lk ? (double)sig[ok * 16 + i] * ik : 0.0;
    const double b = i < Lr ? (double)sig[orr * 16 + i] * ir : 0.0;
    acc += fabs(a - b);
  }
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  eps = (double)(L + 8) * 0x1p-50;
  return acc;
}
__device__ __forceinline__ double u128_to_double(u128 x) {
  return (double)(uint64_t)(x >> 64) * 18446744073709551616.0 + (double)(uint64_t)x;
}
__global__ void k_rep_mindist(uint32_t K, const int64_t* match, uint32_t pool_all, const uint64_t* kto,
                              const uint64_t* sig, const uint64_t* mass, double* dist) {
  const uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (k >= K || match[k] >= 0) return;
  const uint32_t lane = threadIdx.x & 31;
  if (mass[k] == 0) return;  // +inf already written
  double best = INFINITY, best_eps = 0.0;
  for (uint32_t r = 0; r < k; ++r) {
    if ((!pool_all && match[r] >= 0) || mass[r] == 0) continue;
    double eps;
    const double d = warp_d64(sig, kto, mass, k, r, eps);
    if (d < best) { best = d; best_eps = eps; }
  }
  if (best == INFINITY) return;
  double exact = INFINITY;
  for (uint32_t r = 0; r < k; ++r) {
    if ((!pool_all && match[r] >= 0) || mass[r] == 0) continue;
    double eps;
    const double d = warp_d64(sig, kto, mass, k, r, eps);
    if (d > best + best_eps + eps) continue;
    const u128 dn = warp_dnum(sig, kto, mass, k, r);
    const double v = u128_to_double(dn) / u128_to_double((u128)mass[k] * mass[r]);
    if (v < exact) exact = v;
  }
  if (lane == 0) dist[k] = exact;
}

}  // namespace

cudaError_t launch_sig_build(uint32_t K, const uint64_t* kto, const uint32_t* type_key, const uint64_t* type_count,
                             uint32_t k_lo, uint32_t k_hi, uint64_t* sig, uint64_t* mass, DevErr* err, cudaStream_t s) {
  if (K == 0) return cudaSuccess;
  note_launch(), k_sig<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, s>>>(K, k_lo, k_hi, kto, type_key,
                                                                                 type_count, sig, mass, err);
  return cudaGetLastError();
}

cudaError_t launch_sig_prof(uint32_t K, const uint64_t* kto, const uint32_t* type_key, const uint64_t* type_count,
                            uint64_t* sig, uint64_t* mass, const MatchWs& mw, DevErr* err, cudaStream_t s) {
  if (K == 0) return cudaSuccess;
  note_launch(), k_sig_prof<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, s>>>(
      K, kto, type_key, type_count, sig, mass, mw.prof, mw.invn, mw.prof8, mw.sigf, err);
  return cudaGetLastError();
}

namespace {
ScanArgs scan_args(uint32_t K, uint32_t k_lo, uint32_t k_hi, const uint64_t* kto, const uint64_t* sig,
                   const uint64_t* mass, const uint64_t* wt, photon_match_params p, const MatchWs& mw, DevErr* err) {
  ScanArgs a{};
  a.K = K; a.k_lo = k_lo; a.k_hi = k_hi; a.kto = kto; a.sig = sig; a.mass = mass; a.wt = wt; a.prof = mw.prof; a.invn = mw.invn; a.prof8 = mw.prof8; a.sigf = mw.sigf;
  a.p = p;
  // rigorous margin: each |P_k - P_r| term carries <= 3 fp32 roundings of values in [0, 1] plus 16 additions
  a.bound = (float)((double)p.theta_num / (double)p.theta_den) + 1e-5f;
  // |q - 255 P| <= 1/2 + 2^-40 per value, so sum_j |q_k - q_r| <= 255 sum_j |P_k - P_r| + 16 + 2^-30 <= 255 D + 17:
  // a pair with sum >= 255 theta + 17 has D >= theta
  a.thr8 = (uint32_t)ceil(255.0 * (double)p.theta_num / (double)p.theta_den + 17.0);
  a.maybe = mw.maybe; a.n_maybe = mw.n_maybe; a.cap = mw.pair_cap; a.err = err;
  return a;
}
void launch_filter(const ScanArgs& a, cudaStream_t s) {
  const uint32_t kb_hi = (uint32_t)ceil_div(a.k_hi, FT), kb_lo = a.k_lo / FT;
  const uint64_t j0 = filter_jobs_before(kb_lo), j1 = filter_jobs_before(kb_hi);
  if (j1 > j0) note_launch(), k_pair_filter<false><<<(unsigned)(j1 - j0), 256, 0, s>>>(a, j0, kb_lo, kb_hi);
}
// the whole triangle through the band order: sort by f, the band's jobs, then the filter over those jobs only (the
// grid is sized for every tile of the triangle; the jobs past the band's count return at once)
void launch_filter_band(ScanArgs a, const MatchWs& mw, cudaStream_t s) {
  const uint32_t K = a.K, NB = (uint32_t)ceil_div(K, FT);
  if (NB == 0) return;
  if (K <= kBandSmemK) {
    const int smem = (int)(2 * (size_t)K * sizeof(int));
    cudaFuncSetAttribute(k_band_sort_jobs<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    note_launch(), k_band_sort_jobs<true><<<1, 1024, smem, s>>>(K, a.prof8, NB, mw.border, mw.bfs, (int)a.thr8,
                                                                 mw.bandlo, mw.bjobs, mw.bjob_off);
  } else {
    note_launch(), k_band_sort_jobs<false><<<1, 1024, 0, s>>>(K, a.prof8, NB, mw.border, mw.bfs, (int)a.thr8,
                                                               mw.bandlo, mw.bjobs, mw.bjob_off);
  }
  a.order = mw.border;
  a.bandlo = mw.bandlo;
  a.job_off = mw.bjob_off;
  const uint64_t jobs = (uint64_t)(NB / FRB) * (NB / FRB + 1) / 2 * FRB + (uint64_t)(NB % FRB) * (NB / FRB + 1);
  note_launch(), k_pair_filter<true><<<(unsigned)jobs, 256, 0, s>>>(a, 0, 0, NB);
}
// the split path's candidate segments (fused = true): one per k, sized by k's filter survivors (the exact check
// writes the close ones into it)
void launch_segments(uint32_t K, const MatchWs& mw, DevErr* err, int num_sms, cudaStream_t s) {
  const unsigned gb = (unsigned)umin64(ceil_div(mw.pair_cap, 256), (uint64_t)num_sms * 64);
  cudaMemsetAsync(mw.close_cnt, 0, sizeof(uint32_t) * K, s);
  cudaMemsetAsync(mw.cand_cnt, 0, sizeof(uint32_t) * K, s);
  note_launch(), k_cand_count<<<gb, 256, 0, s>>>(mw.maybe, mw.pair_cap, mw.n_maybe, K, mw.cand_cnt, err);
  note_launch(), k_cand_scan<<<1, 1024, 0, s>>>(mw.cand_cnt, K, mw.cand_off, mw.cand_cur);
}
void launch_exact(ScanArgs a, bool fused, const MatchWs& mw, uint64_t* pairs, uint64_t pair_cap, uint64_t* n_pairs,
                  int num_sms, cudaStream_t s) {
  if (fused) {
    a.cand = mw.cand;  // the survivors are checked in the filter's order (band tiles keep a k-block's pairs together)
    a.cbeg = mw.cand_off;
    a.ccnt = mw.close_cnt;
  }
  note_launch(), k_pair_exact<<<(unsigned)num_sms * PHOTON_XGRID, 256, 0, s>>>(a, pairs, pair_cap, n_pairs);
}
}  // namespace

cudaError_t launch_match_scan(uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                              const uint64_t* wt, photon_match_params p, uint32_t k_lo, uint32_t k_hi,
                              const MatchWs& mw, uint64_t* pairs, uint64_t pair_cap, uint64_t* n_pairs, DevErr* err,
                              int num_sms, cudaStream_t s, bool prof_ready, bool fused) {
  cudaMemsetAsync(n_pairs, 0, 8, s);
  cudaMemsetAsync(mw.n_maybe, 0, 8, s);
  if (K == 0 || k_hi <= k_lo) return cudaGetLastError();
  if (!prof_ready)
    note_launch(), k_prof<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, s>>>(K, kto, sig, mass, mw.prof,
                                                                                  mw.invn, mw.prof8, mw.sigf);
  const ScanArgs a = scan_args(K, k_lo, k_hi, kto, sig, mass, wt, p, mw, err);
  launch_filter(a, s);
  if (fused) launch_segments(K, mw, err, num_sms, s);
  launch_exact(a, fused, mw, pairs, pair_cap, n_pairs, num_sms, s);
  return cudaGetLastError();
}

// photon_analyse's split: A3 profiles + filter + candidate segments from the unsorted table (stream sb), then -- after the
// sort, on the main stream -- g / N in row order and the exact check
cudaError_t launch_analyse_filter(uint32_t K, const uint64_t* kto, const uint32_t* list, const HashTable& ht,
                                  uint64_t* mass, const uint64_t* wt, photon_match_params p, const MatchWs& mw,
                                  uint64_t* n_pairs, DevErr* err, cudaStream_t sb) {
  const SegZero z{mw.cand_cnt, mw.close_cnt, mw.n_maybe, mw.flag + 2, n_pairs};
  note_launch(), k_prof_slots<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, sb>>>(K, kto, list, ht, mass,
                                                                                       mw.prof, mw.invn, mw.prof8,
                                                                                       err, z);
  ScanArgs a = scan_args(K, 0, K, kto, nullptr, mass, wt, p, mw, err);
  a.kcnt = mw.cand_cnt;  // the filter counts its survivors per k (no separate count pass) and its last CTA scans
  a.ticket = mw.flag + 2;  // the counts into the candidate segments (no separate scan launch)
  a.seg_off = mw.cand_off;
  a.seg_cur = mw.cand_cur;
  if (PHOTON_BAND && K <= kBandMaxK) launch_filter_band(a, mw, sb);  // f in [-2040, 2040]: the counting sort's 4096 bins
  else launch_filter(a, sb);
  return cudaGetLastError();  // the candidate segments: counted and scanned by the filter, close_cnt zeroed above
}
cudaError_t launch_analyse_exact(uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                                 const uint64_t* wt, photon_match_params p, const MatchWs& mw, uint64_t* pairs,
                                 uint64_t pair_cap, uint64_t* n_pairs, DevErr* err, int num_sms, cudaStream_t s) {
  // n_pairs was zeroed by k_prof_slots (launch_analyse_filter), which precedes this on the joined streams
  launch_exact(scan_args(K, 0, K, kto, sig, mass, wt, p, mw, err), true, mw, pairs, pair_cap, n_pairs, num_sms, s);
  return cudaGetLastError();
}

cudaError_t launch_match_resolve(uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                                 const uint64_t* wt, photon_match_params p, const uint64_t* pairs, uint64_t n_pairs,
                                 const uint64_t* n_pairs_dev, const MatchWs& mw, int64_t* match, double* match_dist,
                                 DevErr* err, int num_sms, cudaStream_t s, bool fused, bool zeroed) {
  if (K == 0) return cudaSuccess;
  // candidate segments: fused -- written by k_pair_exact into k's segment (cand_off, close_cnt); else built here
  // from the pair list (cand_off, cand_cnt)
  const uint32_t* ccnt = fused ? mw.close_cnt : mw.cand_cnt;
  if (!fused) cudaMemsetAsync(mw.cand_cnt, 0, sizeof(uint32_t) * K, s);
  if (!fused && n_pairs) {
    note_launch(), k_cand_count<<<(unsigned)ceil_div(n_pairs, 256), 256, 0, s>>>(pairs, n_pairs, n_pairs_dev, K, mw.cand_cnt, err);
  }
  if (!fused) note_launch(), k_cand_scan<<<1, 1024, 0, s>>>(mw.cand_cnt, K, mw.cand_off, mw.cand_cur);
  if (!fused && n_pairs) {
    note_launch(), k_cand_scatter<<<(unsigned)ceil_div(n_pairs, 256), 256, 0, s>>>(pairs, n_pairs, n_pairs_dev, K, mw.cand_off,
                                                                    mw.cand_cur, mw.cand);
  }
  if (!p.pool_all_prior && K > 2048) {  // large K: the whole GPU, one pass (every warp resident: cooperative launch)
    static int per_sm = 0;
    if (!per_sm) {
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_resolve_spin, 256, 0);
      if (per_sm < 1) per_sm = 1;
    }
    unsigned grid = (unsigned)umin64((uint64_t)per_sm * num_sms, ceil_div((uint64_t)K * 32, 256));
    if (!zeroed) cudaMemsetAsync(mw.state, 0, K, s);
    const uint64_t* off = mw.cand_off;
    const uint32_t* cand = mw.cand;
    void* args[] = {(void*)&K, (void*)&off, (void*)&ccnt, (void*)&cand, (void*)&mw.state, (void*)&mw.flag};
    note_launch();
    cudaError_t e = cudaLaunchCooperativeKernel((void*)k_resolve_spin, grid, 256, args, 0, s);
    if (e != cudaSuccess) return e;
  } else if (K <= kResolveSmemK) {
    note_launch(), k_resolve_rounds<<<1, 1024, 0, s>>>(K, mw.cand_off, ccnt, mw.cand, mw.state, mw.flag,
                                                       p.pool_all_prior);
  } else {  // pool_all with a large K: every kernel with a candidate is matched
    note_launch(), k_pool_all_states<<<(unsigned)ceil_div(K, 256), 256, 0, s>>>(K, ccnt, mw.state, mw.flag);
  }
  note_launch(), k_resolve_match<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, s>>>(K, mw.cand_off, ccnt, mw.cand, mw.state,
                                                                           p.pool_all_prior, wt, kto, sig, mass,
                                                                           match, match_dist);
  if (match_dist)
    note_launch(), k_rep_mindist<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, s>>>(K, match, p.pool_all_prior,
                                                                                          kto, sig, mass, match_dist);
  return cudaGetLastError();
}

}  // namespace photon
