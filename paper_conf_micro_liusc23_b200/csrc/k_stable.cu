// k_stable.cu — A5: per-BB stability test (Eq. 1 rolling slope + mean check) and the BB-sampling switch.
//
// PAPER.md L125 (BB executions indexed by retirement time), L229 ("rolling slope value a of the least-squares
// method for the last n basic blocks from the same type (we use 2048) ... |1-a| less than the threshold delta (we
// use 3%) ... also checking the average ... with the last 2n"), Eq. 1 (L222-225), L208 / Fig 7 (switch when the
// rate of stable basic blocks is larger than 95%).  Readings [P-11]..[P-18].
//
// Design:
//   1. validate records and build composite keys (kernel << bbits | bb), one CTA per (kernel, 4096-record chunk);
//   2. stable LSD radix sort of (key, record index), 8-bit digits: per-tile digit histograms -> device scan ->
//      scatter with a stable in-tile rank (warp __match_any_sync + per-warp digit prefix);
//   3. gather (issue, retire) into group order; find group heads; split every group with >= 2n executions into
//      work items of 2048 positions;
//   4. per work item (one CTA, 8 consecutive positions per thread): the window sums ending just before the item
//      by a block reduction, per-thread deltas by a block scan, then each thread slides over its 8 positions and
//      evaluates cond1/cond2 exactly in i128; the first passing position per group is an atomicMin;
//   5. S_n at the latched position, first_stable/stable_dur_sum, and the per-kernel switch point.
#include "internal.h"

namespace photon {

namespace {

constexpr int RT = 256;        // radix threads per CTA
constexpr int RIPT = 16;       // keys per thread
constexpr int RTILE = RT * RIPT;
constexpr int RBITS = 8;
constexpr int RNB = 1 << RBITS;
constexpr int REC_CHUNK = 4096;
constexpr int WT = 256;        // window threads
constexpr int WPT = 8;         // positions per thread
constexpr int WITEM = WT * WPT;

// ---- generic device-wide exclusive scan of u32 (values and total < 2^32) --------------------------------------
constexpr int SB = 4096;
__global__ void __launch_bounds__(256) k_scan_reduce(const uint32_t* in, uint64_t n, uint32_t* bsum) {
  __shared__ uint32_t ws[8];
  uint64_t base = (uint64_t)blockIdx.x * SB;
  uint32_t s = 0;
  for (int i = threadIdx.x; i < SB; i += 256) {
    uint64_t j = base + i;
    if (j < n) s += in[j];
  }
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    uint32_t t = 0;
    for (int w = 0; w < 8; ++w) t += ws[w];
    bsum[blockIdx.x] = t;
  }
}
__global__ void __launch_bounds__(1024) k_scan_single(uint32_t* a, uint64_t n, uint32_t* total) {
  __shared__ uint32_t ws[32];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint64_t base = 0; base < n; base += 1024) {
    uint64_t i = base + threadIdx.x;
    uint32_t v = i < n ? a[i] : 0, x = v;
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint32_t s = ws[lane];
      for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += y;
      }
      ws[lane] = s;
    }
    __syncthreads();
    uint32_t ex = carry + (wid ? ws[wid - 1] : 0) + x - v;
    if (i < n) a[i] = ex;
    __syncthreads();
    if (threadIdx.x == 1023) carry = ex + v;
    __syncthreads();
  }
  if (threadIdx.x == 0 && total) *total = carry;
}
__global__ void __launch_bounds__(256) k_scan_apply(const uint32_t* in, uint64_t n, const uint32_t* bsum,
                                                    uint32_t* out) {
  __shared__ uint32_t ws[8];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = bsum[blockIdx.x];
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint64_t base = (uint64_t)blockIdx.x * SB;
  for (int c = 0; c < SB; c += 256) {
    uint64_t i = base + c + threadIdx.x;
    uint32_t v = i < n ? in[i] : 0, x = v;
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[wid] = x;
    __syncthreads();
    uint32_t pre = 0;
    for (int w = 0; w < wid; ++w) pre += ws[w];
    uint32_t ex = carry + pre + x - v;
    if (i < n) out[i] = ex;
    __syncthreads();
    if (threadIdx.x == 255) carry = ex + v;
    __syncthreads();
  }
}
// out may alias in; bsum needs ceil(n/SB) entries; total (device) receives the sum
void scan_u32(const uint32_t* in, uint32_t* out, uint64_t n, uint32_t* bsum, uint32_t* total, cudaStream_t s) {
  uint64_t nb = ceil_div(n ? n : 1, SB);
  note_launch(), k_scan_reduce<<<(unsigned)nb, 256, 0, s>>>(in, n, bsum);
  note_launch(), k_scan_single<<<1, 1024, 0, s>>>(bsum, nb, total);
  note_launch(), k_scan_apply<<<(unsigned)nb, 256, 0, s>>>(in, n, bsum, out);
}

// ---- 1. per-kernel record chunks + validation + keys -------------------------------------------------------
__global__ void __launch_bounds__(1024) k_rec_chunks(const uint64_t* kro, uint32_t K, uint64_t R, uint64_t* coff,
                                                     DevErr* err) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) {
    carry = 0;
    if (kro[0] != 0 || kro[K] != R) latch(err, PHOTON_ERANGE, 0);
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t base = 0; base < K; base += 1024) {
    uint32_t k = base + threadIdx.x;
    uint64_t v = 0;
    if (k < K) {
      uint64_t a = kro[k], b = kro[k + 1];
      if (b < a) latch(err, PHOTON_ERANGE, (int64_t)k);
      v = b > a ? ceil_div(b - a, REC_CHUNK) : 0;
    }
    uint64_t x = v;
    for (int o = 1; o < 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint64_t s = ws[lane];
      for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += y;
      }
      ws[lane] = s;
    }
    __syncthreads();
    uint64_t ex = carry + (wid ? ws[wid - 1] : 0) + x - v;
    if (k < K) coff[k] = ex;
    __syncthreads();
    if (threadIdx.x == 1023) carry = ex + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) coff[K] = carry;
}

__device__ __forceinline__ uint32_t upper_idx(const uint64_t* a, uint32_t n, uint64_t v) {
  // last i in [0, n-1] with a[i] <= v
  uint32_t lo = 0, hi = n - 1;
  while (lo < hi) {
    uint32_t mid = (lo + hi + 1) >> 1;
    if (a[mid] <= v) lo = mid; else hi = mid - 1;
  }
  return lo;
}

__global__ void __launch_bounds__(256) k_rec_prep(photon_timing t, const uint64_t* coff, uint32_t bbits,
                                                  uint64_t* key, DevErr* err) {
  const uint64_t total = coff[t.n_kernels];
  for (uint64_t job = blockIdx.x; job < total; job += gridDim.x) {
    uint32_t k = upper_idx(coff, t.n_kernels, job);
    uint64_t c = job - coff[k];
    uint64_t a = t.kernel_rec_off[k], b = t.kernel_rec_off[k + 1];
    uint64_t cs = a + c * REC_CHUNK, ce = umin64(cs + REC_CHUNK, b);
    for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
      uint32_t bb = t.bb[i];
      uint64_t x = t.issue[i], y = t.retire[i];
      if (bb >= t.n_bb || x >= kTimeLimit || y >= kTimeLimit || y < x || (i > a && t.retire[i - 1] > y)) {
        latch(err, PHOTON_ERANGE, (int64_t)i);
        bb = 0;
      }
      key[i] = ((uint64_t)k << bbits) | bb;
    }
  }
}

// ---- 2. stable LSD radix sort of (key u64, value u32) -------------------------------------------------------
__global__ void __launch_bounds__(RT) k_radix_up(const uint64_t* key, uint64_t n, uint32_t shift, uint32_t* hist,
                                                 uint64_t n_tiles) {
  __shared__ uint32_t cnt[RNB];
  for (int i = threadIdx.x; i < RNB; i += RT) cnt[i] = 0;
  __syncthreads();
  uint64_t base = (uint64_t)blockIdx.x * RTILE;
  for (int it = 0; it < RIPT; ++it) {
    uint64_t j = base + (uint64_t)it * RT + threadIdx.x;
    bool v = j < n;
    uint32_t d = v ? (uint32_t)((key[j] >> shift) & (RNB - 1)) : RNB;  // RNB = invalid
    unsigned peers = __match_any_sync(0xffffffffu, d);
    if (v && (threadIdx.x & 31) == (unsigned)(__ffs(peers) - 1)) atomicAdd(&cnt[d], (uint32_t)__popc(peers));
  }
  __syncthreads();
  for (int d = threadIdx.x; d < RNB; d += RT) hist[(uint64_t)d * n_tiles + blockIdx.x] = cnt[d];
}

__global__ void __launch_bounds__(RT) k_radix_down(const uint64_t* key, const uint32_t* val, uint64_t n,
                                                   uint32_t shift, const uint32_t* off, uint64_t n_tiles,
                                                   uint64_t* okey, uint32_t* oval, int iota) {
  __shared__ uint32_t wcnt[RT / 32][RNB];
  __shared__ uint32_t wpre[RT / 32][RNB];
  __shared__ uint32_t dbase[RNB];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (int d = threadIdx.x; d < RNB; d += RT) {
    dbase[d] = off[(uint64_t)d * n_tiles + blockIdx.x];
    for (int w = 0; w < RT / 32; ++w) wcnt[w][d] = 0xFFFFFFFFu;
  }
  __syncthreads();
  uint64_t base = (uint64_t)blockIdx.x * RTILE;
  const unsigned lt = (1u << lane) - 1u;
  for (int it = 0; it < RIPT; ++it) {
    uint64_t j = base + (uint64_t)it * RT + threadIdx.x;
    bool v = j < n;
    uint64_t kk = v ? key[j] : 0;
    uint32_t vv = v ? (iota ? (uint32_t)j : val[j]) : 0;
    uint32_t d = v ? (uint32_t)((kk >> shift) & (RNB - 1)) : RNB;
    unsigned peers = __match_any_sync(0xffffffffu, d);
    uint32_t rank = (uint32_t)__popc(peers & lt);
    if (v && rank == 0) wcnt[wid][d] = ((uint32_t)it << 16) | (uint32_t)__popc(peers);
    __syncthreads();
    for (int dd = threadIdx.x; dd < RNB; dd += RT) {
      uint32_t run = dbase[dd];
      for (int w = 0; w < RT / 32; ++w) {
        uint32_t e = wcnt[w][dd];
        wpre[w][dd] = run;
        if ((e >> 16) == (uint32_t)it) run += e & 0xFFFFu;
      }
      dbase[dd] = run;
    }
    __syncthreads();
    if (v) {
      uint32_t dest = wpre[wid][d] + rank;
      okey[dest] = kk;
      oval[dest] = vv;
    }
  }
}

// ---- 3. gather + groups + work items -------------------------------------------------------------------------
__global__ void k_gather(const uint32_t* idx, uint64_t n, const uint64_t* issue, const uint64_t* retire, uint64_t* X,
                         uint64_t* Y) {
  uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  uint32_t i = idx[p];
  X[p] = issue[i];
  Y[p] = retire[i];
}

__global__ void k_heads(const uint64_t* key, uint64_t n, uint32_t* flag) {
  uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  flag[p] = (p == 0 || key[p] != key[p - 1]) ? 1u : 0u;
}

__global__ void k_group_start(const uint64_t* key, uint64_t n, const uint32_t* gidx, uint64_t* gstart) {
  uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  if (p == 0 || key[p] != key[p - 1]) gstart[gidx[p]] = p;
}

__global__ void k_group_end(uint64_t* gstart, const uint32_t* G, uint64_t n) { gstart[*G] = n; }

__global__ void k_work_count(const uint64_t* gstart, const uint32_t* G, uint32_t n2, uint32_t* nwork,
                             uint64_t* gfirst, uint64_t gcap) {
  uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (g >= gcap) return;
  uint32_t ng = *G;
  if (g >= ng) { nwork[g] = 0; return; }
  uint64_t sz = gstart[g + 1] - gstart[g];
  nwork[g] = sz >= n2 ? (uint32_t)ceil_div(sz - n2 + 1, WITEM) : 0u;
  gfirst[g] = ~0ull;
}

// ---- 4. windowed exact test ----------------------------------------------------------------------------------
struct Sums {
  int64_t sx, sy, sn, s2n;
  i128 sxy, sxx;
};
__device__ __forceinline__ void sums_add(Sums& a, const Sums& b) {
  a.sx += b.sx; a.sy += b.sy; a.sn += b.sn; a.s2n += b.s2n; a.sxy += b.sxy; a.sxx += b.sxx;
}
__device__ __forceinline__ void sums_zero(Sums& a) { a.sx = a.sy = a.sn = a.s2n = 0; a.sxy = a.sxx = 0; }
__device__ __forceinline__ i128 shfl_i128(i128 v, int src, bool up, int delta) {
  uint64_t lo = (uint64_t)v, hi = (uint64_t)((u128)v >> 64);
  if (up) {
    lo = __shfl_up_sync(0xffffffffu, lo, delta);
    hi = __shfl_up_sync(0xffffffffu, hi, delta);
  } else {
    lo = __shfl_sync(0xffffffffu, lo, src);
    hi = __shfl_sync(0xffffffffu, hi, src);
  }
  return (i128)(((u128)hi << 64) | lo);
}
__device__ __forceinline__ Sums shfl_up_sums(const Sums& s, int delta) {
  Sums r;
  r.sx = __shfl_up_sync(0xffffffffu, s.sx, delta);
  r.sy = __shfl_up_sync(0xffffffffu, s.sy, delta);
  r.sn = __shfl_up_sync(0xffffffffu, s.sn, delta);
  r.s2n = __shfl_up_sync(0xffffffffu, s.s2n, delta);
  r.sxy = shfl_i128(s.sxy, 0, true, delta);
  r.sxx = shfl_i128(s.sxx, 0, true, delta);
  return r;
}
__device__ __forceinline__ Sums shfl_xor_sums(const Sums& s, int m) {
  Sums r;
  r.sx = __shfl_xor_sync(0xffffffffu, s.sx, m);
  r.sy = __shfl_xor_sync(0xffffffffu, s.sy, m);
  r.sn = __shfl_xor_sync(0xffffffffu, s.sn, m);
  r.s2n = __shfl_xor_sync(0xffffffffu, s.s2n, m);
  uint64_t lo = (uint64_t)s.sxy, hi = (uint64_t)((u128)s.sxy >> 64);
  lo = __shfl_xor_sync(0xffffffffu, lo, m); hi = __shfl_xor_sync(0xffffffffu, hi, m);
  r.sxy = (i128)(((u128)hi << 64) | lo);
  lo = (uint64_t)s.sxx; hi = (uint64_t)((u128)s.sxx >> 64);
  lo = __shfl_xor_sync(0xffffffffu, lo, m); hi = __shfl_xor_sync(0xffffffffu, hi, m);
  r.sxx = (i128)(((u128)hi << 64) | lo);
  return r;
}

struct WinArgs {
  const uint64_t* X;
  const uint64_t* Y;
  const uint64_t* gstart;
  const uint32_t* G;
  const uint32_t* work_off;  // exclusive scan of nwork, [gcap]
  const uint32_t* n_work;    // total
  uint64_t gcap;
  uint32_t n;
  uint32_t dnum, dden;
  uint64_t* gfirst;
};

__global__ void __launch_bounds__(WT) k_window(WinArgs a) {
  __shared__ Sums part[WT / 32];
  __shared__ Sums wtot[WT / 32];
  __shared__ uint64_t best;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint32_t total = *a.n_work;
  const uint32_t G = *a.G;
  const int64_t n = a.n;
  for (uint32_t item = blockIdx.x; item < total; item += gridDim.x) {
    // group of this work item: last g with work_off[g] <= item (and a non-empty item count)
    uint32_t lo = 0, hi = G - 1;
    while (lo < hi) {
      uint32_t mid = (lo + hi + 1) >> 1;
      if (a.work_off[mid] <= item) lo = mid; else hi = mid - 1;
    }
    uint32_t g = lo;
    const int64_t gs = (int64_t)a.gstart[g], ge = (int64_t)a.gstart[g + 1];
    const int64_t c = item - a.work_off[g];
    const int64_t Q0 = gs + 2 * n - 1 + c * WITEM;
    const int64_t Q1 = Q0 + WITEM < ge ? Q0 + WITEM : ge;
    auto X = [&](int64_t q) -> int64_t { return q >= gs ? (int64_t)a.X[q] : 0; };
    auto D = [&](int64_t q) -> int64_t { return q >= gs ? (int64_t)(a.Y[q] - a.X[q]) : 0; };
    auto Y = [&](int64_t q) -> int64_t { return q >= gs ? (int64_t)a.Y[q] : 0; };
    // base: windows ending at Q0-1 ([Q0-n, Q0-1] and [Q0-2n, Q0-1]); positions < gs contribute 0
    Sums s;
    sums_zero(s);
    for (int64_t q = Q0 - 2 * n + tid; q < Q0; q += WT) {
      int64_t d = D(q);
      s.s2n += d;
      if (q >= Q0 - n) {
        int64_t x = X(q), y = Y(q);
        s.sx += x; s.sy += y; s.sn += d;
        s.sxy += (i128)x * y; s.sxx += (i128)x * x;
      }
    }
    for (int o = 16; o > 0; o >>= 1) sums_add(s, shfl_xor_sums(s, o));
    if (lane == 0) part[wid] = s;
    // per-thread deltas over its 8 positions
    Sums dl;
    sums_zero(dl);
    const int64_t q0 = Q0 + (int64_t)tid * WPT;
    int64_t xs[WPT], ys[WPT], xo[WPT], yo[WPT], do2[WPT];
#pragma unroll
    for (int u = 0; u < WPT; ++u) {
      int64_t q = q0 + u;
      if (q < Q1) {
        xs[u] = X(q); ys[u] = Y(q); xo[u] = X(q - n); yo[u] = Y(q - n); do2[u] = D(q - 2 * n);
      } else {
        xs[u] = ys[u] = xo[u] = yo[u] = do2[u] = 0;
      }
      dl.sx += xs[u] - xo[u];
      dl.sy += ys[u] - yo[u];
      dl.sn += (ys[u] - xs[u]) - (yo[u] - xo[u]);
      dl.s2n += (ys[u] - xs[u]) - do2[u];
      dl.sxy += (i128)xs[u] * ys[u] - (i128)xo[u] * yo[u];
      dl.sxx += (i128)xs[u] * xs[u] - (i128)xo[u] * xo[u];
    }
    // block exclusive scan of dl
    Sums incl = dl;
    for (int o = 1; o < 32; o <<= 1) {
      Sums t = shfl_up_sums(incl, o);
      if (lane >= o) sums_add(incl, t);
    }
    if (lane == 31) wtot[wid] = incl;
    if (tid == 0) best = ~0ull;
    __syncthreads();
    Sums w;
    sums_zero(w);
    for (int k = 0; k < WT / 32; ++k) sums_add(w, part[k]);  // base
    for (int k = 0; k < wid; ++k) sums_add(w, wtot[k]);
    // exclusive = w + incl - dl
    sums_add(w, incl);
    w.sx -= dl.sx; w.sy -= dl.sy; w.sn -= dl.sn; w.s2n -= dl.s2n; w.sxy -= dl.sxy; w.sxx -= dl.sxx;
    uint64_t mine = ~0ull;
#pragma unroll
    for (int u = 0; u < WPT; ++u) {
      int64_t q = q0 + u;
      if (q >= Q1) break;
      w.sx += xs[u] - xo[u];
      w.sy += ys[u] - yo[u];
      w.sn += (ys[u] - xs[u]) - (yo[u] - xo[u]);
      w.s2n += (ys[u] - xs[u]) - do2[u];
      w.sxy += (i128)xs[u] * ys[u] - (i128)xo[u] * yo[u];
      w.sxx += (i128)xs[u] * xs[u] - (i128)xo[u] * xo[u];
      if (mine != ~0ull) continue;
      // cond1: den > 0 and dden*|den - num| < dnum*den  (Eq. 1: a = num/den)
      i128 num = (i128)n * w.sxy - (i128)w.sx * w.sy;
      i128 den = (i128)n * w.sxx - (i128)w.sx * w.sx;
      bool c1 = false;
      if (den > 0) {
        i128 diff = den - num;
        if (diff < 0) diff = -diff;
        c1 = (i128)a.dden * diff < (i128)a.dnum * den;
      }
      bool c2 = false;
      if (c1 && w.s2n > 0) {
        i128 d2 = 2 * (i128)w.sn - w.s2n;
        if (d2 < 0) d2 = -d2;
        c2 = (i128)a.dden * d2 < (i128)a.dnum * w.s2n;
      }
      if (c1 && c2) mine = (uint64_t)q;
    }
    if (mine != ~0ull) atomicMin((unsigned long long*)&best, (unsigned long long)mine);
    __syncthreads();
    if (tid == 0 && best != ~0ull) atomicMin((unsigned long long*)&a.gfirst[g], (unsigned long long)best);
    __syncthreads();
  }
}

// ---- 5. outputs ----------------------------------------------------------------------------------------------
__global__ void k_finish(const uint64_t* key, const uint32_t* idx, const uint64_t* X, const uint64_t* Y,
                         const uint64_t* gstart, const uint32_t* G, const uint64_t* gfirst, const uint64_t* kro,
                         uint32_t bbits, uint32_t B, uint32_t n, int64_t* first_stable, uint64_t* dur) {
  uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  if (warp >= *G) return;
  uint64_t q = gfirst[warp];
  if (q == ~0ull) return;
  uint64_t k = key[q] >> bbits, b = key[q] & ((1ull << bbits) - 1);
  uint64_t s = 0;
  for (uint64_t i = q + 1 - n + lane; i <= q; i += 32) s += Y[i] - X[i];
  for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if (lane == 0) {
    first_stable[k * B + b] = (int64_t)(idx[q] - kro[k]);
    if (dur) dur[k * B + b] = s;
  }
}

// switch_at[k]: order stable BBs by position; first position where rate_den * acc > rate_num * total (L208)
__global__ void __launch_bounds__(256) k_switch(const uint64_t* key, const uint64_t* gstart, const uint32_t* G,
                                                const uint64_t* gfirst, const int64_t* first_stable,
                                                const uint64_t* kbb, uint32_t K, uint32_t B, uint32_t bbits,
                                                uint32_t rnum, uint32_t rden, int64_t* switch_at) {
  __shared__ uint64_t tot_lo[8], tot_hi[8];
  __shared__ int64_t best;
  const uint32_t ng = *G;
  for (uint32_t k = blockIdx.x; k < K; k += gridDim.x) {
    // total weight of the kernel's BB distribution (u128)
    u128 t = 0;
    for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) t += kbb[(uint64_t)k * B + b];
    uint64_t lo = (uint64_t)t, hi = (uint64_t)(t >> 64);
    for (int o = 16; o > 0; o >>= 1) {
      uint64_t lo2 = __shfl_xor_sync(0xffffffffu, lo, o), hi2 = __shfl_xor_sync(0xffffffffu, hi, o);
      uint64_t s = lo + lo2;
      hi = hi + hi2 + (s < lo);
      lo = s;
    }
    if ((threadIdx.x & 31) == 0) { tot_lo[threadIdx.x >> 5] = lo; tot_hi[threadIdx.x >> 5] = hi; }
    if (threadIdx.x == 0) best = -1;
    __syncthreads();
    u128 total = 0;
    for (int w = 0; w < 8; ++w) total += ((u128)tot_hi[w] << 64) | tot_lo[w];
    // groups of kernel k: keys in [k << bbits, (k+1) << bbits)
    uint32_t g_lo = 0, g_hi = 0;
    if (ng > 0) {
      uint64_t klo = (uint64_t)k << bbits, khi = (uint64_t)(k + 1) << bbits;
      uint32_t a = 0, b = ng;  // first g with key >= klo
      while (a < b) { uint32_t m = (a + b) >> 1; if (key[gstart[m]] < klo) a = m + 1; else b = m; }
      g_lo = a;
      b = ng;
      while (a < b) { uint32_t m = (a + b) >> 1; if (key[gstart[m]] < khi) a = m + 1; else b = m; }
      g_hi = a;
    }
    if (total > 0) {
      for (uint32_t gi = g_lo + threadIdx.x; gi < g_hi; gi += blockDim.x) {
        if (gfirst[gi] == ~0ull) continue;
        uint32_t bi = (uint32_t)(key[gstart[gi]] & ((1ull << bbits) - 1));
        int64_t ti = first_stable[(uint64_t)k * B + bi];
        u128 acc = 0;
        for (uint32_t gj = g_lo; gj < g_hi; ++gj) {
          if (gfirst[gj] == ~0ull) continue;
          uint32_t bj = (uint32_t)(key[gstart[gj]] & ((1ull << bbits) - 1));
          if (first_stable[(uint64_t)k * B + bj] <= ti) acc += kbb[(uint64_t)k * B + bj];
        }
        if ((u128)rden * acc > (u128)rnum * total) {
          // min over candidates
          unsigned long long cur = (unsigned long long)ti;
          atomicMin((unsigned long long*)&best, cur);  // best starts at -1 = 0xFF..: unsigned min works
        }
      }
    }
    __syncthreads();
    if (threadIdx.x == 0) switch_at[k] = best;
    __syncthreads();
  }
}

struct Layout {
  uint64_t* key0; uint64_t* key1;
  uint32_t* val0; uint32_t* val1;
  uint64_t* X; uint64_t* Y;
  uint32_t* hist; uint32_t* bsum; uint32_t* misc;  // misc[0] = G, misc[1] = total work
  uint32_t* flag;  // [R] heads -> group index (scan)
  uint64_t* gstart;  // [gcap+1]
  uint32_t* nwork;   // [gcap]
  uint64_t* gfirst;  // [gcap]
  uint64_t* coff;    // [K+1]
  uint64_t gcap, n_tiles;
  size_t bytes;
};

Layout make_layout(const photon_timing& t, void* base) {
  Carver c(base);
  Layout L;
  uint64_t R = t.n_records ? t.n_records : 1;
  L.n_tiles = ceil_div(R, RTILE);
  L.gcap = R;
  L.key0 = c.take<uint64_t>(R); L.key1 = c.take<uint64_t>(R);
  L.val0 = c.take<uint32_t>(R); L.val1 = c.take<uint32_t>(R);
  L.X = c.take<uint64_t>(R); L.Y = c.take<uint64_t>(R);
  uint64_t hn = (uint64_t)RNB * L.n_tiles;
  uint64_t scan_n = hn > R ? hn : R;
  L.hist = c.take<uint32_t>(hn);
  L.bsum = c.take<uint32_t>(ceil_div(scan_n, SB) + 1);
  L.misc = c.take<uint32_t>(16);
  L.flag = c.take<uint32_t>(R);
  L.gstart = c.take<uint64_t>(L.gcap + 1);
  L.nwork = c.take<uint32_t>(L.gcap);
  L.gfirst = c.take<uint64_t>(L.gcap);
  L.coff = c.take<uint64_t>((uint64_t)t.n_kernels + 1);
  L.bytes = c.off + 256;
  return L;
}

}  // namespace

size_t stable_ws_bytes(const photon_timing& t) { return make_layout(t, nullptr).bytes; }

cudaError_t launch_stable(const photon_timing& t, const uint64_t* kbb, photon_stable_params p, void* ws,
                          size_t ws_bytes, int64_t* first_stable, uint64_t* dur, int64_t* switch_at, DevErr* err,
                          int num_sms, cudaStream_t s) {
  (void)ws_bytes;
  Layout L = make_layout(t, ws);
  const uint64_t R = t.n_records;
  const uint32_t K = t.n_kernels, B = t.n_bb;
  uint32_t bbits = 1;
  while ((1u << bbits) < B) ++bbits;
  uint32_t kbits = 1;
  while ((1ull << kbits) < (uint64_t)K) ++kbits;
  cudaMemsetAsync(first_stable, 0xFF, sizeof(int64_t) * (size_t)K * B, s);
  if (dur) cudaMemsetAsync(dur, 0, sizeof(uint64_t) * (size_t)K * B, s);
  cudaMemsetAsync(L.misc, 0, 64, s);
  note_launch(), k_rec_chunks<<<1, 1024, 0, s>>>(t.kernel_rec_off, K, R, L.coff, err);
  if (R > 0) {
    uint64_t jobs_ub = ceil_div(R, REC_CHUNK) + K;
    unsigned grid = (unsigned)umin64(jobs_ub, (uint64_t)num_sms * 8);
    note_launch(), k_rec_prep<<<grid, 256, 0, s>>>(t, L.coff, bbits, L.key0, err);
    // radix passes over kbits + bbits bits
    uint32_t bits = kbits + bbits;
    uint64_t* kin = L.key0; uint64_t* kout = L.key1;
    uint32_t* vin = L.val0; uint32_t* vout = L.val1;
    int pass = 0;
    for (uint32_t sh = 0; sh < bits; sh += RBITS, ++pass) {
      note_launch(), k_radix_up<<<(unsigned)L.n_tiles, RT, 0, s>>>(kin, R, sh, L.hist, L.n_tiles);
      scan_u32(L.hist, L.hist, (uint64_t)RNB * L.n_tiles, L.bsum, L.misc + 4, s);
      note_launch(), k_radix_down<<<(unsigned)L.n_tiles, RT, 0, s>>>(kin, vin, R, sh, L.hist, L.n_tiles, kout, vout, pass == 0);
      uint64_t* tk = kin; kin = kout; kout = tk;
      uint32_t* tv = vin; vin = vout; vout = tv;
    }
    // sorted: kin / vin
    unsigned gR = (unsigned)ceil_div(R, 256);
    note_launch(), k_gather<<<gR, 256, 0, s>>>(vin, R, t.issue, t.retire, L.X, L.Y);
    note_launch(), k_heads<<<gR, 256, 0, s>>>(kin, R, L.flag);
    scan_u32(L.flag, L.flag, R, L.bsum, L.misc + 0, s);  // misc[0] = G
    note_launch(), k_group_start<<<gR, 256, 0, s>>>(kin, R, L.flag, L.gstart);
    note_launch(), k_group_end<<<1, 1, 0, s>>>(L.gstart, L.misc + 0, R);
    note_launch(), k_work_count<<<(unsigned)ceil_div(L.gcap, 256), 256, 0, s>>>(L.gstart, L.misc + 0, 2 * p.window_n, L.nwork,
                                                                 L.gfirst, L.gcap);
    scan_u32(L.nwork, L.nwork, L.gcap, L.bsum, L.misc + 1, s);  // misc[1] = work items
    WinArgs wa{};
    wa.X = L.X; wa.Y = L.Y; wa.gstart = L.gstart; wa.G = L.misc + 0; wa.work_off = L.nwork; wa.n_work = L.misc + 1;
    wa.gcap = L.gcap; wa.n = p.window_n; wa.dnum = p.delta_num; wa.dden = p.delta_den; wa.gfirst = L.gfirst;
    note_launch(), k_window<<<(unsigned)num_sms * 4, WT, 0, s>>>(wa);
    note_launch(), k_finish<<<(unsigned)ceil_div(L.gcap * 32, 256), 256, 0, s>>>(kin, vin, L.X, L.Y, L.gstart, L.misc + 0, L.gfirst,
                                                                 t.kernel_rec_off, bbits, B, p.window_n,
                                                                 first_stable, dur);
    unsigned gk = (unsigned)umin64(K, (uint64_t)num_sms * 8);
    note_launch(), k_switch<<<gk ? gk : 1, 256, 0, s>>>(kin, L.gstart, L.misc + 0, L.gfirst, first_stable, kbb, K, B, bbits,
                                         p.rate_num, p.rate_den, switch_at);
  } else {
    cudaMemsetAsync(switch_at, 0xFF, sizeof(int64_t) * K, s);
  }
  return cudaGetLastError();
}

}  // namespace photon
