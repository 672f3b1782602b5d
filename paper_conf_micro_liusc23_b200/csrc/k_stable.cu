// k_stable.cu — A5: per-BB stability test (Eq. 1 rolling slope + mean check) and the BB-sampling switch.
//
// PAPER.md L125 (BB executions indexed by retirement time), L229 ("rolling slope value a of the least-squares
// method for the last n basic blocks from the same type (we use 2048) ... |1-a| less than the threshold delta (we
// use 3%) ... also checking the average ... with the last 2n"), Eq. 1 (L222-225), L208 / Fig 7 (switch when the
// rate of stable basic blocks is larger than 95%).  Readings [P-11]..[P-18].
//
// Design:
//   1-3. bring every group g = (b, k) (dense id b*K + k) together in retirement order, with (issue, retire):
//      B <= 256: one pass -- one warp per (kernel, 2048-record) job histograms its bb ids, a bin-major scan of
//      the histograms gives every (bb, job) its output offset, and the warp scatters its records stably
//      (__match_any_sync rank + warp-private running counts), validating them on the way;
//      B > 256: composite keys b*K + k, stable LSD radix sort (8-bit digits, per-tile histograms -> device scan
//      -> scatter with a stable in-tile rank), gather (issue, retire), group starts by gap filling;
//      every group with >= 2n executions is split into runs of 4 x 2048 positions;
//   4. persistent CTAs take runs from a global ticket counter in run-major order (run 0 of every group first),
//      skipping runs that start past an already-latched position.  Per run: the window sums ending just before
//      it by a block reduction; per 2048-position item, per-thread deltas by a block scan, then each thread slides
//      over its 8 positions and evaluates cond1/cond2 exactly in i128; the first passing position per group is an
//      atomicMin; sums carry to the next item;
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
constexpr int JOB = 2048;       // records per warp job (one-pass multisplit)
// The grouped copy: per record the retire time relative to its kernel's first retire (u32) and the duration
// retire - issue (u32), 8 B/record; a relative retire or a duration >= kDurEsc is stored as kDurEsc with the exact
// relative value in a side array (Yw: relative retire; Xw: relative issue, may be negative), written only for
// those records.  Eq. 1's sums are shift-invariant over full windows and S_n, S_2n are durations, so the window
// test and S_n need no absolute time.  (The radix path, B > 8192, uses base 0: absolute times, escaped >= 2^32.)
constexpr uint32_t kDurEsc = 0xFFFFFFFFu;
struct GCopy {
  uint32_t* Y32;  // [R] relative retire, kDurEsc: in Yw
  uint32_t* D;    // [R] duration, kDurEsc: issue in Xw
  int64_t* Yw;    // [R] relative retire (escaped records only)
  int64_t* Xw;    // [R] relative issue (escaped durations only)
};
__device__ __forceinline__ void put_rec(const GCopy& G, uint64_t dest, uint64_t x, uint64_t y, uint64_t base) {
  const int64_t yr = (int64_t)(y - base);  // retire >= the kernel's first retire (validated order)
  if ((uint64_t)yr < kDurEsc) {
    G.Y32[dest] = (uint32_t)yr;
  } else {
    G.Y32[dest] = kDurEsc;
    G.Yw[dest] = yr;
  }
  const uint64_t d = y - x;
  if (d < kDurEsc) {
    G.D[dest] = (uint32_t)d;
  } else {
    G.D[dest] = kDurEsc;
    G.Xw[dest] = (int64_t)x - (int64_t)base;
  }
}
__device__ __forceinline__ int64_t g_y(const GCopy& G, uint64_t q) {
  const uint32_t v = __ldg(G.Y32 + q);
  return v != kDurEsc ? (int64_t)v : __ldg(G.Yw + q);
}
__device__ __forceinline__ int64_t g_x(const GCopy& G, uint64_t q, int64_t y) {
  const uint32_t d = __ldg(G.D + q);
  return d != kDurEsc ? y - (int64_t)d : __ldg(G.Xw + q);
}
constexpr int WT = 256;        // window threads
constexpr int WPT = 8;         // positions per thread
constexpr int WITEM = WT * WPT;
constexpr int NI = 4;          // items per run
constexpr int RUN = WITEM * NI;

// ---- generic device-wide exclusive scan of u32 (values and total < 2^32) --------------------------------------
constexpr int SB = 4096;
// ndev (optional): the live length on the device (n is then its capacity); cells past it are not touched
__device__ __forceinline__ uint64_t live_n(uint64_t n, const uint64_t* ndev) { return ndev ? umin64(n, *ndev) : n; }
__global__ void __launch_bounds__(256) k_scan_reduce(const uint32_t* in, uint64_t n, const uint64_t* ndev,
                                                     uint32_t* bsum) {
  __shared__ uint32_t ws[8];
  n = live_n(n, ndev);
  uint64_t base = (uint64_t)blockIdx.x * SB;
  if (base >= n) {
    if (threadIdx.x == 0) bsum[blockIdx.x] = 0;
    return;
  }
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
__global__ void __launch_bounds__(1024) k_scan_single(uint32_t* a, uint64_t n, const uint64_t* ndev, uint32_t* total) {
  __shared__ uint32_t ws[32];
  if (ndev) n = umin64(n, ceil_div(*ndev, (uint64_t)SB));
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
__global__ void __launch_bounds__(256) k_scan_apply(const uint32_t* in, uint64_t n, const uint64_t* ndev,
                                                    const uint32_t* bsum, uint32_t* out) {
  __shared__ uint32_t ws[8];
  __shared__ uint32_t carry;
  n = live_n(n, ndev);
  if ((uint64_t)blockIdx.x * SB >= n) return;
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
// out may alias in; bsum needs ceil(n/SB) entries; total (device) receives the sum; ndev (optional, device): scan
// only the first min(n, *ndev) cells
void scan_u32(const uint32_t* in, uint32_t* out, uint64_t n, uint32_t* bsum, uint32_t* total, cudaStream_t s,
              const uint64_t* ndev = nullptr) {
  uint64_t nb = ceil_div(n ? n : 1, SB);
  note_launch(), k_scan_reduce<<<(unsigned)nb, 256, 0, s>>>(in, n, ndev, bsum);
  note_launch(), k_scan_single<<<1, 1024, 0, s>>>(bsum, nb, ndev, total);
  note_launch(), k_scan_apply<<<(unsigned)nb, 256, 0, s>>>(in, n, ndev, bsum, out);
}
__global__ void k_zero_live(uint32_t* a, uint64_t n, const uint64_t* ndev) {
  n = live_n(n, ndev);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    a[i] = 0u;
}

// ---- 1. per-kernel record chunks + validation + keys -------------------------------------------------------
__global__ void __launch_bounds__(1024) k_rec_chunks(const uint64_t* kro, uint32_t K, uint64_t R, uint64_t chunk,
                                                     uint64_t* coff, DevErr* err) {
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
      uint64_t a = umin64(kro[k], R), b = umin64(kro[k + 1], R);
      if (kro[k + 1] < kro[k] || kro[k + 1] > R) latch(err, PHOTON_ERANGE, (int64_t)k);
      v = b > a ? ceil_div(b - a, chunk) : 0;
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

__global__ void __launch_bounds__(256) k_rec_prep(photon_timing t, const uint64_t* coff, uint64_t* key,
                                                  DevErr* err) {
  const uint64_t total = coff[t.n_kernels];
  for (uint64_t job = blockIdx.x; job < total; job += gridDim.x) {
    uint32_t k = upper_idx(coff, t.n_kernels, job);
    uint64_t c = job - coff[k];
    uint64_t a = umin64(t.kernel_rec_off[k], t.n_records), b = umin64(t.kernel_rec_off[k + 1], t.n_records);  // clamped: bad offsets are latched by k_rec_chunks
    uint64_t cs = a + c * REC_CHUNK, ce = umin64(cs + REC_CHUNK, b);
    for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
      uint32_t bb = t.bb[i];
      uint64_t x = t.issue[i], y = t.retire[i];
      if (bb >= t.n_bb || x >= kTimeLimit || y >= kTimeLimit || y < x || (i > a && t.retire[i - 1] > y)) {
        latch(err, PHOTON_ERANGE, (int64_t)i);
        bb = 0;
      }
      key[i] = (uint64_t)bb * t.n_kernels + k;  // group id g = b*K + k
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
__global__ void k_gather(const uint32_t* idx, uint64_t n, const uint64_t* issue, const uint64_t* retire, GCopy G) {
  uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p >= n) return;
  uint32_t i = idx[p];
  put_rec(G, p, issue[i], retire[i], 0);
}

__global__ void k_set_u32(uint32_t* p, uint32_t v) { *p = v; }

// gstart[g] = first sorted position with key >= g, for every g in [0, K*B] (empty groups have size 0)
__global__ void k_fill_gstart(const uint64_t* key, uint64_t n, uint64_t G, uint64_t* gstart) {
  uint64_t p = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (p > n) return;
  uint64_t lo = p == 0 ? 0 : key[p - 1] + 1, hi = p == n ? G : key[p];
  for (uint64_t g = lo; g <= hi && g <= G; ++g) gstart[g] = p;
}

constexpr uint32_t kNone = 0xFFFFFFFFu;  // padding lane (not a u16 id)

// ---- 2'. one-pass stable multisplit: one warp per job = (kernel, JOB records) --------------------------------
// Records of a job belong to one kernel, so a stable split by BB inside each job, with job offsets from a scan of
// the per-job histograms laid out kernel-major ((k, l, job) with l the kernel-local BB id), leaves every group
// (k, l) contiguous, in retirement order.  Local ids: B <= 256 -- the BB id itself (B_k = B, group g = k*B + b);
// 256 < B <= kCompactMaxB -- the rank of b among the BB ids present in kernel k's stream (a presence bitmap per
// kernel; C5 kernels use 16 of 4096 ids), groups g = goff[k] + l.  Kernels with more than 256 local ids keep their
// histogram / running offsets in global memory (atomics, still stable) instead of shared memory.
constexpr uint32_t kCompactMaxB = 8192;
constexpr uint32_t kSmemBins = 256;
struct JobMap {
  const uint64_t* coff;  // [K+1] jobs per kernel (scanned)
  const uint32_t* bits;  // compact: [K][nw] presence bitmap
  const uint32_t* lbase; // compact: [K][nw] local ids before each word
  const uint32_t* bk;    // compact: [K] local ids of kernel k
  const uint64_t* hb;    // compact: [K+1] first histogram entry of kernel k (scanned B_k * jobs_k)
  uint32_t nw;           // words per kernel bitmap
  bool compact;
  uint64_t hcap;         // histogram entries available (compact: the device total must fit, else ECAPACITY)
  __device__ __forceinline__ bool fits() const { return !compact || hb[nkern] <= hcap; }
  uint32_t nkern;
  __device__ __forceinline__ uint32_t nbins(uint32_t k, uint32_t B) const { return compact ? bk[k] : B; }
  __device__ __forceinline__ uint64_t hbase(uint32_t k, uint32_t B) const { return compact ? hb[k] : (uint64_t)B * coff[k]; }
  __device__ __forceinline__ uint32_t lid(uint32_t k, uint32_t b) const {
    if (!compact) return b;
    const uint64_t w = (uint64_t)k * nw + (b >> 5);
    return lbase[w] + __popc(bits[w] & ((1u << (b & 31)) - 1u));
  }
};

// The BB ids of one job [cs, ce) (at most JOB records), loaded up front as 16-byte vectors (9 per lane: enough
// memory parallelism for these order-free passes) and handed one per lane per step to f(id) -- kNone outside the
// job -- in warp-uniform steps (f may use warp collectives).  Vectors are aligned 8-id blocks; a block reaching
// past R (or an unaligned bb array) is read element by element.
template <class F>
__device__ __forceinline__ void job_ids(const uint16_t* bb, uint64_t R, uint64_t cs, uint64_t ce, int lane, F&& f) {
  constexpr int NV = JOB / 256 + 1;
  const uint64_t c0 = cs & ~7ull;
  const bool vec = ((uintptr_t)bb & 15) == 0;
  uint4 v[NV];
#pragma unroll
  for (int r = 0; r < NV; ++r) {
    const uint64_t i = c0 + (uint64_t)r * 256 + lane * 8;
    v[r] = make_uint4(~0u, ~0u, ~0u, ~0u);
    if (i < ce) {
      if (vec && i + 8 <= R) {
        v[r] = __ldg(reinterpret_cast<const uint4*>(bb + i));
      } else {
        uint32_t e[4];
#pragma unroll
        for (int h = 0; h < 4; ++h) {
          const uint32_t lo = i + 2 * h < R ? bb[i + 2 * h] : 0xFFFFu, hi = i + 2 * h + 1 < R ? bb[i + 2 * h + 1] : 0xFFFFu;
          e[h] = lo | hi << 16;
        }
        v[r] = make_uint4(e[0], e[1], e[2], e[3]);
      }
    }
  }
#pragma unroll
  for (int r = 0; r < NV; ++r) {
    const uint64_t i = c0 + (uint64_t)r * 256 + lane * 8;
    const uint32_t w[4] = {v[r].x, v[r].y, v[r].z, v[r].w};
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const uint64_t q = i + j;
      f(q >= cs && q < ce ? (w[j >> 1] >> ((j & 1) * 16)) & 0xFFFFu : kNone);
    }
  }
}

// presence bitmap per kernel (compact ids): one warp per job ORs its BB ids into a shared bitmap, then into global
__global__ void __launch_bounds__(256) k_presence(photon_timing t, const uint64_t* coff, uint64_t n_jobs, uint32_t nw,
                                                  uint32_t* bits) {
  extern __shared__ uint32_t pm[];  // [8][nw]
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t* m = pm + wid * nw;
  for (uint32_t w = lane; w < nw; w += 32) m[w] = 0u;
  __syncwarp();
  for (uint64_t job = (uint64_t)blockIdx.x * 8 + wid; job < n_jobs; job += (uint64_t)gridDim.x * 8) {
    const uint32_t k = upper_idx(coff, t.n_kernels, job);
    const uint64_t a = umin64(t.kernel_rec_off[k], t.n_records), e = umin64(t.kernel_rec_off[k + 1], t.n_records);
    const uint64_t cs = a + (job - coff[k]) * JOB, ce = umin64(cs + JOB, e);
    // each lane ORs the bits of its run of records into a register while they stay in one bitmap word (a kernel's
    // few BB ids share words) and flushes the word to shared memory when it changes: no warp collective per record;
    // the aligned middle of the job as 16-byte vectors of 8 ids, the unaligned head and tail id by id
    uint32_t cwd = kNone, cbits = 0;
    auto put = [&](uint32_t id) {
      if (id >= t.n_bb) id = 0;  // bad ids are latched by the scatter
      const uint32_t wd = id >> 5;
      if (wd != cwd) {
        if (cbits) atomicOr(&m[cwd], cbits);
        cwd = wd;
        cbits = 0;
      }
      cbits |= 1u << (id & 31);
    };
    const bool vec = ((uintptr_t)t.bb & 15) == 0;
    const uint64_t s8 = vec ? umin64((cs + 7) & ~7ull, ce) : ce, e8 = vec ? umax64(ce & ~7ull, s8) : ce;
    for (uint64_t i = cs + lane; i < s8; i += 32) put(t.bb[i]);
    for (uint64_t i = s8 + 8 * (uint64_t)lane; i < e8; i += 256) {
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(t.bb + i));
      const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
      for (int q = 0; q < 8; ++q) put((w4[q >> 1] >> ((q & 1) * 16)) & 0xFFFFu);
    }
    for (uint64_t i = e8 + lane; i < ce; i += 32) put(t.bb[i]);
    if (cbits) atomicOr(&m[cwd], cbits);
    __syncwarp();
    for (uint32_t w = lane; w < nw; w += 32) {
      const uint32_t v = m[w];
      if (v) {
        atomicOr(&bits[(uint64_t)k * nw + w], v);
        m[w] = 0u;
      }
    }
    __syncwarp();
  }
}
// per kernel (one warp): local ids before each bitmap word, and B_k
__global__ void k_lid_prep(uint32_t K, uint32_t nw, const uint32_t* bits, uint32_t* lbase, uint32_t* bk) {
  const uint32_t lane = threadIdx.x & 31, nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < K; k += nwarps) {
    uint32_t carry = 0;
    for (uint32_t w0 = 0; w0 < nw; w0 += 32) {
      const uint32_t w = w0 + lane;
      const uint32_t c = w < nw ? __popc(bits[(uint64_t)k * nw + w]) : 0u;
      uint32_t x = c;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      if (w < nw) lbase[(uint64_t)k * nw + w] = carry + x - c;
      carry += __shfl_sync(0xffffffffu, x, 31);
    }
    if (lane == 0) bk[k] = carry;
  }
}
// exclusive scans over kernels (one CTA): goff = groups before k, hb = histogram entries before k (B_k * jobs_k);
// misc[0] = total groups
__global__ void __launch_bounds__(1024) k_lid_scan(uint32_t K, const uint64_t* coff, const uint32_t* bk, uint64_t* goff,
                                                   uint64_t* hb, uint32_t* misc, uint64_t hcap, DevErr* err) {
  __shared__ uint64_t wa[32], wb[32];
  __shared__ uint64_t ca, cb;
  if (threadIdx.x == 0) ca = cb = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t base = 0; base < K; base += 1024) {
    const uint32_t k = base + threadIdx.x;
    const uint64_t va = k < K ? bk[k] : 0, vb = k < K ? (uint64_t)bk[k] * (coff[k + 1] - coff[k]) : 0;
    uint64_t xa = va, xb = vb;
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t ya = __shfl_up_sync(0xffffffffu, xa, o), yb = __shfl_up_sync(0xffffffffu, xb, o);
      if (lane >= o) { xa += ya; xb += yb; }
    }
    if (lane == 31) { wa[wid] = xa; wb[wid] = xb; }
    __syncthreads();
    uint64_t pa = ca, pb = cb;
    for (int w = 0; w < wid; ++w) { pa += wa[w]; pb += wb[w]; }
    if (k < K) { goff[k] = pa + xa - va; hb[k] = pb + xb - vb; }
    __syncthreads();
    if (threadIdx.x == 1023) { ca = pa + xa; cb = pb + xb; }
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    goff[K] = ca;
    hb[K] = cb;
    misc[0] = cb <= hcap ? (uint32_t)ca : 0u;  // no groups when the histogram does not fit
    if (cb > hcap) latch(err, PHOTON_ECAPACITY, (int64_t)cb);
  }
}
// per kernel (one warp): gkb[goff[k] + l] = k << 16 | b for its present BB ids
__global__ void k_lid_groups(uint32_t K, uint32_t nw, const uint32_t* bits, const uint32_t* lbase, const uint64_t* goff,
                             uint64_t* gkb) {
  const uint32_t lane = threadIdx.x & 31, nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < K; k += nwarps)
    for (uint32_t w = lane; w < nw; w += 32) {
      uint32_t v = bits[(uint64_t)k * nw + w];
      uint64_t g = goff[k] + lbase[(uint64_t)k * nw + w];
      while (v) {
        const uint32_t bit = __ffs(v) - 1;
        v &= v - 1;
        gkb[g++] = ((uint64_t)k << 16) | (w * 32 + bit);
      }
    }
}

// Per-job histograms.  Kernels with <= 256 (local) ids: lane-private byte counters in shared memory ([bin][lane],
// a lane counts at most JOB/32 = 64 ids of a job), no atomics and no warp collectives per id; the 32 columns of a
// bin are summed with dp4a at the end of the job.  More ids: __match_any_sync-aggregated global atomics.
constexpr int HW = 4;  // warps per k_job_hist block (4 x 8 KB of counters)
static_assert(JOB / 32 < 256, "byte counters");
__global__ void __launch_bounds__(HW * 32) k_job_hist(photon_timing t, JobMap jm, uint64_t n_jobs, uint32_t* hist) {
  __shared__ uint32_t h[HW][kSmemBins * 8];  // per warp: bin-major rows of 32 byte counters
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t B = t.n_bb;
  uint8_t* hb8 = reinterpret_cast<uint8_t*>(h[wid]);
  for (int d = lane; d < (int)kSmemBins * 8; d += 32) h[wid][d] = 0;
  __syncwarp();
  if (!jm.fits()) return;  // ECAPACITY latched by k_lid_scan
  n_jobs = umin64(n_jobs, jm.coff[t.n_kernels]);  // real jobs only: a job past the last would address the next
                                                  // group's cells in the kernel-major layout
  const bool vec = ((uintptr_t)t.bb & 15) == 0;
  for (uint64_t job = (uint64_t)blockIdx.x * HW + wid; job < n_jobs; job += (uint64_t)gridDim.x * HW) {
    const uint32_t k = upper_idx(jm.coff, t.n_kernels, job);
    const uint64_t jl = job - jm.coff[k], nj = jm.coff[k + 1] - jm.coff[k];
    const uint32_t nb = jm.nbins(k, B);
    const uint64_t hb = jm.hbase(k, B);
    uint64_t a = umin64(t.kernel_rec_off[k], t.n_records), e = umin64(t.kernel_rec_off[k + 1], t.n_records);  // clamped: bad offsets are latched by k_rec_chunks
    uint64_t cs = a + jl * JOB, ce = umin64(cs + JOB, e);
    if (nb > kSmemBins) {
      job_ids(t.bb, t.n_records, cs, ce, lane, [&](uint32_t d) {
        const uint32_t x = d == kNone ? kNone : jm.lid(k, d < B ? d : 0u);  // bad ids count as bb 0 (latched by the scatter)
        const unsigned peers = __match_any_sync(0xffffffffu, x);
        if (x != kNone && lane == __ffs(peers) - 1) atomicAdd(&hist[hb + (uint64_t)x * nj + jl], (uint32_t)__popc(peers));
      });
      continue;
    }
    // lane-contiguous 8-id blocks from the aligned start: a lane counts at most 8 ids per 256-id step
    const uint64_t c0 = cs & ~7ull;
    uint32_t cw_ = kNone, cb_ = 0, cl_ = 0;  // compact ids: the lane's cached bitmap word (index, bits, base)
    for (uint64_t i = c0 + lane * 8; i < ce; i += 256) {
      uint32_t w[4];
      if (vec && i + 8 <= t.n_records) {
        const uint4 v = __ldg(reinterpret_cast<const uint4*>(t.bb + i));
        w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
      } else {
#pragma unroll
        for (int hh = 0; hh < 4; ++hh)
          w[hh] = (i + 2 * hh < t.n_records ? t.bb[i + 2 * hh] : 0u) |
                  (i + 2 * hh + 1 < t.n_records ? (uint32_t)t.bb[i + 2 * hh + 1] : 0u) << 16;
      }
#pragma unroll
      for (int j = 0; j < 8; ++j) {
        const uint64_t q = i + j;
        uint32_t d = (w[j >> 1] >> ((j & 1) * 16)) & 0xFFFFu;
        if (q >= cs && q < ce) {
          d = d < B ? d : 0u;  // bad ids count as bb 0 (latched by the scatter)
          uint32_t x = d;
          if (jm.compact) {  // local id: the lane keeps the last bitmap word's base and bits (a kernel's ids share
                             // few words)
            if ((d >> 5) != cw_) {
              cw_ = d >> 5;
              cb_ = jm.bits[(uint64_t)k * jm.nw + cw_];
              cl_ = jm.lbase[(uint64_t)k * jm.nw + cw_];
            }
            x = cl_ + __popc(cb_ & ((1u << (d & 31)) - 1u));
          }
          hb8[x * 32 + lane] += 1;
        }
      }
    }
    __syncwarp();
    for (int dd = lane; dd < (int)nb; dd += 32) {
      uint32_t c = 0;
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        c = __dp4a(h[wid][dd * 8 + q], 0x01010101u, c);
        h[wid][dd * 8 + q] = 0;
      }
      hist[hb + (uint64_t)dd * nj + jl] = c;
    }
    __syncwarp();
  }
}

__global__ void __launch_bounds__(256, 3) k_job_scatter(photon_timing t, JobMap jm, uint64_t n_jobs, uint32_t* off,
                                                     GCopy G, DevErr* err) {
  __shared__ uint32_t run[8][kSmemBins];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint32_t B = t.n_bb;
  const unsigned lt = (1u << lane) - 1u;
  if (!jm.fits()) return;  // ECAPACITY latched by k_lid_scan
  n_jobs = umin64(n_jobs, jm.coff[t.n_kernels]);  // real jobs only: a job past the last would address the next
                                                  // group's cells in the kernel-major layout
  for (uint64_t job = (uint64_t)blockIdx.x * 8 + wid; job < n_jobs; job += (uint64_t)gridDim.x * 8) {
    const uint32_t k = upper_idx(jm.coff, t.n_kernels, job);
    const uint64_t jl = job - jm.coff[k], nj = jm.coff[k + 1] - jm.coff[k];
    const uint32_t nb = jm.nbins(k, B);
    const bool sm = nb <= kSmemBins;
    const uint64_t hb = jm.hbase(k, B);
    uint64_t a = umin64(t.kernel_rec_off[k], t.n_records), e = umin64(t.kernel_rec_off[k + 1], t.n_records);  // clamped: bad offsets are latched by k_rec_chunks
    uint64_t cs = a + jl * JOB, ce = umin64(cs + JOB, e);
    if (sm)
      for (int dd = lane; dd < (int)nb; dd += 32) run[wid][dd] = off[hb + (uint64_t)dd * nj + jl];
    __syncwarp();
    // tiles of TS x 32 records, the next tile's loads in flight while this one is ranked and written
    constexpr int TS = 4;
    uint32_t d[TS];
    uint64_t x[TS], y[TS];
    auto load = [&](uint64_t i0, uint32_t* dd, uint64_t* xx, uint64_t* yy) {
#pragma unroll
      for (int u = 0; u < TS; ++u) {
        const uint64_t i = i0 + u * 32 + lane;
        const bool v = i < ce;
        dd[u] = v ? (uint32_t)t.bb[i] : kNone;
        xx[u] = v ? t.issue[i] : 0;
        yy[u] = v ? t.retire[i] : 0;
      }
    };
    load(cs, d, x, y);
    const uint64_t kbase = a < e ? t.retire[a] : 0;  // the kernel's first retire: the copy's time base
    // retire[i - 1] of lane 0 in slot 0: the previous tile's last record (the job's first tile: one load)
    uint64_t carry = lane == 0 && cs > a && cs < ce ? t.retire[cs - 1] : 0;
    for (uint64_t i0 = cs; i0 < ce; i0 += 32 * TS) {
      uint32_t nd[TS];
      uint64_t nx[TS], ny[TS];
      load(i0 + 32 * TS, nd, nx, ny);
      uint64_t yp[TS];
#pragma unroll
      for (int u = 0; u < TS; ++u) {
        const uint64_t up = __shfl_up_sync(0xffffffffu, y[u], 1);
        const uint64_t wrap = u ? __shfl_sync(0xffffffffu, y[u ? u - 1 : 0], 31) : carry;
        yp[u] = lane ? up : wrap;
      }
      carry = __shfl_sync(0xffffffffu, y[TS - 1], 31);
#pragma unroll
      for (int u = 0; u < TS; ++u) {
        uint64_t i = i0 + u * 32 + lane;
        uint32_t dd = d[u];
        if (dd != kNone) {
          if (dd >= B || x[u] >= kTimeLimit || y[u] >= kTimeLimit || y[u] < x[u] || yp[u] > y[u]) {
            latch(err, PHOTON_ERANGE, (int64_t)i);
            if (dd >= B) dd = 0;
          }
          dd = jm.lid(k, dd);
        }
        unsigned peers = __match_any_sync(0xffffffffu, dd);
        const int lead = __ffs(peers) - 1;
        uint32_t base = 0;
        if (sm) {
          base = dd != kNone ? run[wid][dd] : 0;
          __syncwarp();
          if (dd != kNone && lane == lead) run[wid][dd] = base + __popc(peers);
        } else {
          if (dd != kNone && lane == lead) base = atomicAdd(&off[hb + (uint64_t)dd * nj + jl], (uint32_t)__popc(peers));
          base = __shfl_sync(0xffffffffu, base, lead);
        }
        if (dd != kNone) put_rec(G, base + __popc(peers & lt), x[u], y[u], kbase);
        __syncwarp();
      }
#pragma unroll
      for (int u = 0; u < TS; ++u) { d[u] = nd[u]; x[u] = nx[u]; y[u] = ny[u]; }
    }
  }
}

// gstart[g] = start of group g = (k, l) (g = k*B + b, or goff[k] + l): the scanned histogram entry (k, l, first
// job); groups of a kernel without records start where the next kernel's do; gstart[G] = R
__global__ void k_job_gstart(const uint32_t* off, JobMap jm, const uint64_t* goff, const uint64_t* gkb, uint32_t K,
                             uint32_t B, uint64_t R, uint64_t Htot_host, uint64_t* gstart, uint32_t* G) {
  if (!jm.fits()) return;
  const uint64_t n = jm.compact ? goff[K] : (uint64_t)K * B;
  const uint64_t Htot = jm.compact ? jm.hb[K] : Htot_host;
  for (uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; g <= n; g += (uint64_t)gridDim.x * blockDim.x) {
    if (g == n) { gstart[g] = R; if (!jm.compact) *G = (uint32_t)n; continue; }
    uint32_t k, l;
    if (jm.compact) { k = (uint32_t)(gkb[g] >> 16); l = (uint32_t)(g - goff[k]); }
    else { k = (uint32_t)(g / B); l = (uint32_t)(g % B); }
    const uint64_t nj = jm.coff[k + 1] - jm.coff[k];
    const uint64_t j = jm.hbase(k, B) + (uint64_t)l * nj;
    gstart[g] = j < Htot ? off[j] : R;
  }
}

// runs per group: a group of size sz tests positions [2n-1, sz) (L229: only once 2n executions exist), split
// into runs of RUN positions; maxr = the largest run count (the number of ticket rounds)
__global__ void k_work_count(const uint64_t* gstart, const uint32_t* G, uint32_t n2, uint32_t* nruns,
                             uint64_t* gfirst, uint32_t* maxr) {
  const uint32_t ng = *G;
  for (uint32_t g = blockIdx.x * blockDim.x + threadIdx.x; g < ng; g += gridDim.x * blockDim.x) {
    uint64_t sz = gstart[g + 1] - gstart[g];
    uint32_t r = sz >= n2 ? (uint32_t)ceil_div(sz - n2 + 1, RUN) : 0u;
    nruns[g] = r;
    gfirst[g] = ~0ull;
    if (r) atomicMax(maxr, r);
  }
}

// The compact run list, run-major (every group's run 0 before any group's run 1): count the groups per run index,
// scan, fill (the order of groups inside one run index is immaterial).  list[i] = g | (uint64)r << 32.
// one warp per group, lanes over its runs (a long group's runs are not a serial chain of atomics)
__global__ void k_runs_count(const uint32_t* G, const uint32_t* nruns, uint32_t* cnt) {
  const uint32_t ng = *G, lane = threadIdx.x & 31, nw = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t g = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; g < ng; g += nw)
    for (uint32_t r = lane; r < nruns[g]; r += 32) atomicAdd(&cnt[r], 1u);
}
__global__ void __launch_bounds__(1024) k_runs_scan(const uint32_t* maxr, uint32_t* cnt, uint32_t* total) {
  __shared__ uint32_t ws[32];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const uint32_t m = *maxr, lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t base = 0; base < m; base += 1024) {
    const uint32_t i = base + threadIdx.x;
    const uint32_t v = i < m ? cnt[i] : 0u;
    uint32_t x = v;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= (uint32_t)o) x += y;
    }
    if (lane == 31) ws[wid] = x;
    __syncthreads();
    uint32_t pre = carry;
    for (uint32_t k = 0; k < wid; ++k) pre += ws[k];
    if (i < m) cnt[i] = pre + x - v;  // exclusive
    __syncthreads();
    if (threadIdx.x == 1023) carry = pre + x;
    __syncthreads();
  }
  if (threadIdx.x == 0) *total = carry;
}
__global__ void k_runs_fill(const uint32_t* G, const uint32_t* nruns, const uint32_t* off, uint32_t* fill,
                            uint64_t* list) {
  const uint32_t ng = *G, lane = threadIdx.x & 31, nw = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t g = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; g < ng; g += nw)
    for (uint32_t r = lane; r < nruns[g]; r += 32)
      list[off[r] + atomicAdd(&fill[r], 1u)] = (uint64_t)g | ((uint64_t)r << 32);
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
  const uint64_t* X;  // raw streams (N1): issue times
  const uint64_t* Y;  // raw streams (N1): retire times
  const uint32_t* D;  // non-null: the positions are the grouped copy G (relative times), X / Y unused
  GCopy G;
  const uint64_t* gstart;
  const uint32_t* Gn;     // number of groups
  const uint64_t* list;   // compact run-major run list (k_runs_*)
  const uint32_t* total;  // its length
  uint32_t* ticket;       // global ticket counter (zeroed)
  uint32_t n;
  uint32_t dnum, dden;
  uint64_t* gfirst;
  uint32_t ring;   // fast path: shared positions per run (2n + RUN), 0 = off (n too large for shared memory)
  int64_t lim;     // fast path: shifted times must lie in (-lim, lim) (n * lim^2 < 2^61: int64 sums are exact)
};

// retire / issue time of position q (relative to the kernel's first retire for the grouped copy)
__device__ __forceinline__ int64_t win_y(const WinArgs& a, int64_t q) {
  return a.D ? g_y(a.G, q) : (int64_t)__ldg(a.Y + q);
}
__device__ __forceinline__ int64_t win_x(const WinArgs& a, int64_t q, int64_t y) {
  return a.D ? g_x(a.G, q, y) : (int64_t)__ldg(a.X + q);
}

__device__ __forceinline__ void sums_sub(Sums& a, const Sums& b) {
  a.sx -= b.sx; a.sy -= b.sy; a.sn -= b.sn; a.s2n -= b.s2n; a.sxy -= b.sxy; a.sxx -= b.sxx;
}

// ---- 4'. fast path of one run: shifted 32-bit times staged in shared memory, int64 sums ----------------------
// Eq. 1's numerator n*Sxy - Sx*Sy and denominator n*Sxx - Sx^2 are invariant under x -> x - c, y -> y - c over a
// full window of n positions, and S_n, S_2n are sums of durations (shift-free).  Every tested window lies inside
// its group (q >= gs + 2n - 1), so with c = the run's first retire time and every shifted time in (-lim, lim),
// all window sums fit int64 exactly; cond1 / cond2 are then evaluated exactly as on the
// unshifted values (in i128); n * lim^2 < 2^61 also bounds every difference of two window sums (the
// per-thread deltas and their block scan).  A run whose span has a time outside the range takes the general path below.
constexpr int WPT_F = 33;                 // positions per thread (odd: conflict-free 8-byte shared reads)
constexpr int WITEM_F = WT * WPT_F;       // one item covers a run
static_assert(RUN <= WITEM_F, "a fast-path run is one item");
struct FSums {
  int64_t sx, sy, s2n, sxy, sxx;
};
__device__ __forceinline__ void fs_add(FSums& a, const FSums& b) {
  a.sx += b.sx; a.sy += b.sy; a.s2n += b.s2n; a.sxy += b.sxy; a.sxx += b.sxx;
}
__device__ __forceinline__ void fs_zero(FSums& a) { a.sx = a.sy = a.s2n = a.sxy = a.sxx = 0; }
__device__ __forceinline__ FSums fs_shfl_up(const FSums& v, int d) {
  FSums r;
  r.sx = __shfl_up_sync(0xffffffffu, v.sx, d);
  r.sy = __shfl_up_sync(0xffffffffu, v.sy, d);
  r.s2n = __shfl_up_sync(0xffffffffu, v.s2n, d);
  r.sxy = __shfl_up_sync(0xffffffffu, v.sxy, d);
  r.sxx = __shfl_up_sync(0xffffffffu, v.sxx, d);
  return r;
}
__device__ __forceinline__ FSums fs_shfl_xor(const FSums& v, int m) {
  FSums r;
  r.sx = __shfl_xor_sync(0xffffffffu, v.sx, m);
  r.sy = __shfl_xor_sync(0xffffffffu, v.sy, m);
  r.s2n = __shfl_xor_sync(0xffffffffu, v.s2n, m);
  r.sxy = __shfl_xor_sync(0xffffffffu, v.sxy, m);
  r.sxx = __shfl_xor_sync(0xffffffffu, v.sxx, m);
  return r;
}
// cond2 (mean check, L229) then cond1 (Eq. 1 slope within delta, L222-225) on the fast path's int64 window sums.  cond2 in int64: S_2n < 4 n lim <= 2^39, delta_den <= 2^16.  cond1 by
// a filtered predicate: num, den and the two sides of the comparison in fp64 with a rigorous bound on their error
// (every int64 -> double conversion, product and difference rounds by at most 2^-53 relative; 2^-50 covers their
// sum); only a comparison within the bound (or den within its bound of 0) is re-done exactly in i128.
__device__ __forceinline__ bool window_pass_fast(int64_t n, int64_t sx, int64_t sy, int64_t s2n, int64_t sxy,
                                                 int64_t sxx, uint32_t dnum, uint32_t dden) {
  if (s2n <= 0) return false;
  int64_t d2 = 2 * (sy - sx) - s2n;
  if (d2 < 0) d2 = -d2;
  if (!((int64_t)dden * d2 < (int64_t)dnum * s2n)) return false;
  const double fn = (double)n, fx = (double)sx, fy = (double)sy;
  const double a1 = fn * (double)sxy, a2 = fx * fy, b1 = fn * (double)sxx, b2 = fx * fx;
  const double num = a1 - a2, den = b1 - b2;
  const double en = 0x1p-50 * (fabs(a1) + fabs(a2)), ed = 0x1p-50 * (b1 + b2);
  if (den < -ed) return false;
  if (den > ed) {
    const double L = (double)dden * fabs(den - num), R = (double)dnum * den;
    const double m = (double)dden * (en + ed) + (double)dnum * ed + 0x1p-50 * (L + R);
    if (L + m < R) return true;
    if (L - m > R) return false;
  }
  const i128 inum = (i128)n * sxy - (i128)sx * sy;
  const i128 iden = (i128)n * sxx - (i128)sx * sx;
  if (iden <= 0) return false;
  i128 diff = iden - inum;
  if (diff < 0) diff = -diff;
  return (i128)dden * diff < (i128)dnum * iden;
}
// returns false (nothing written but the shared buffer) when a time falls outside the range: caller goes general
__device__ bool window_run_fast(const WinArgs& a, uint32_t g, int64_t gs, int64_t P0, int64_t P1, int2* ring,
                                FSums* wpart, unsigned long long* best) {
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int64_t n = a.n, base0 = P0 - 2 * n, span = P1 - base0;
  const int64_t c = win_y(a, base0 > gs ? base0 : gs);
  bool ok = true;
  constexpr int FU = 8;  // loads in flight per thread (the fill is latency-bound otherwise)
  const uint32_t c32 = a.D ? __ldg(a.G.Y32 + (base0 > gs ? base0 : gs)) : kDurEsc;
  if (c32 != kDurEsc) {
    // the grouped copy without escapes (the usual case), in 32-bit arithmetic: retire times are non-decreasing
    // along the group, so y' = Y32[q] - c32 >= 0 is exact in u32; x' = y' - D[q] lies in (-lim, y'] exactly when
    // D[q] < y' + lim; an escaped record fails the test and the run takes the general path
    const uint32_t lim32 = (uint32_t)a.lim;
    for (int64_t i0 = 0; i0 < span; i0 += WT * FU) {
      uint32_t yv[FU], dv[FU];
#pragma unroll
      for (int u = 0; u < FU; ++u) {
        const int64_t i = i0 + u * WT + tid, q = base0 + i;
        const bool in = i < span && q >= gs;
        yv[u] = in ? __ldg(a.G.Y32 + q) : c32;
        dv[u] = in ? __ldg(a.G.D + q) : 0u;
      }
#pragma unroll
      for (int u = 0; u < FU; ++u) {
        const int64_t i = i0 + u * WT + tid;
        const uint32_t yr = yv[u] - c32;
        ok &= yv[u] != kDurEsc && dv[u] != kDurEsc && yr < lim32 && dv[u] < yr + lim32;
        if (i < span) ring[i] = make_int2((int)(yr - dv[u]), (int)yr);
      }
    }
    if (!__syncthreads_and(ok)) return false;
  } else {
  for (int64_t i0 = 0; i0 < span; i0 += WT * FU) {
    uint32_t yv[FU], dv[FU];
#pragma unroll
    for (int u = 0; u < FU; ++u) {
      const int64_t i = i0 + u * WT + tid, q = base0 + i;
      const bool in = i < span && q >= gs;
      if (a.D) {
        yv[u] = in ? __ldg(a.G.Y32 + q) : 0u;
        dv[u] = in ? __ldg(a.G.D + q) : 0u;
      } else {
        yv[u] = dv[u] = 0u;
      }
    }
#pragma unroll
    for (int u = 0; u < FU; ++u) {
      const int64_t i = i0 + u * WT + tid, q = base0 + i;
      int64_t x = c, y = c;  // positions < gs: (0, 0) after the shift
      if (i < span && q >= gs) {
        if (a.D) {
          y = yv[u] != kDurEsc ? (int64_t)yv[u] : __ldg(a.G.Yw + q);
          x = dv[u] != kDurEsc ? y - (int64_t)dv[u] : __ldg(a.G.Xw + q);
        } else {
          y = (int64_t)__ldg(a.Y + q);
          x = (int64_t)__ldg(a.X + q);
        }
      }
      x -= c;
      y -= c;
      ok &= x > -a.lim && y < a.lim;  // x <= y (validated), so both lie in (-lim, lim)
      if (i < span) ring[i] = make_int2((int)x, (int)y);
    }
  }
  if (!__syncthreads_and(ok)) return false;
  }
  // base: windows ending at P0 - 1 ([P0-n, P0-1] and [P0-2n, P0-1]); positions < gs are (0, 0)
  FSums s;
  fs_zero(s);
  for (int64_t i = tid; i < 2 * n; i += WT) {
    const int2 v = ring[i];
    s.s2n += (int64_t)v.y - v.x;
    if (i >= n) {
      s.sx += v.x; s.sy += v.y;
      s.sxy += (int64_t)v.x * v.y; s.sxx += (int64_t)v.x * v.x;
    }
  }
  for (int o = 16; o > 0; o >>= 1) fs_add(s, fs_shfl_xor(s, o));
  if (lane == 0) wpart[wid] = s;
  if (tid == 0) *best = ~0ull;
  __syncthreads();
  FSums base;
  fs_zero(base);
  for (int k = 0; k < WT / 32; ++k) fs_add(base, wpart[k]);
  __syncthreads();
  // pass 1: this thread's deltas over its WPT_F positions
  const int64_t r0 = 2 * n + (int64_t)tid * WPT_F, rend = P1 - base0;  // ring index of q = q - base0
  FSums dl;
  fs_zero(dl);
#pragma unroll 3
  for (int u = 0; u < WPT_F; ++u) {
    const int64_t i = r0 + u;
    if (i < rend) {
      const int2 vs = ring[i], vo = ring[i - n], v2 = ring[i - 2 * n];
      dl.sx += (int64_t)vs.x - vo.x; dl.sy += (int64_t)vs.y - vo.y;
      dl.s2n += ((int64_t)vs.y - vs.x) - ((int64_t)v2.y - v2.x);
      dl.sxy += (int64_t)vs.x * vs.y - (int64_t)vo.x * vo.y;
      dl.sxx += (int64_t)vs.x * vs.x - (int64_t)vo.x * vo.x;
    }
  }
  FSums incl = dl;
  for (int o = 1; o < 32; o <<= 1) {
    const FSums t = fs_shfl_up(incl, o);
    if (lane >= o) fs_add(incl, t);
  }
  if (lane == 31) wpart[wid] = incl;
  __syncthreads();
  FSums w = base;
  for (int k = 0; k < wid; ++k) fs_add(w, wpart[k]);
  fs_add(w, incl);
  w.sx -= dl.sx; w.sy -= dl.sy; w.s2n -= dl.s2n; w.sxy -= dl.sxy; w.sxx -= dl.sxx;  // exclusive
  // pass 2: slide and test
  uint64_t mine = ~0ull;
  for (int u = 0; u < WPT_F; ++u) {
    const int64_t i = r0 + u;
    if (i >= rend) break;
    const int2 vs = ring[i], vo = ring[i - n], v2 = ring[i - 2 * n];
    w.sx += (int64_t)vs.x - vo.x; w.sy += (int64_t)vs.y - vo.y;
    w.s2n += ((int64_t)vs.y - vs.x) - ((int64_t)v2.y - v2.x);
    w.sxy += (int64_t)vs.x * vs.y - (int64_t)vo.x * vo.y;
    w.sxx += (int64_t)vs.x * vs.x - (int64_t)vo.x * vo.x;
    if (window_pass_fast(n, w.sx, w.sy, w.s2n, w.sxy, w.sxx, a.dnum, a.dden)) {
      mine = (uint64_t)(base0 + i);
      break;
    }
  }
  if (mine != ~0ull) atomicMin(best, (unsigned long long)mine);
  __syncthreads();
  if (tid == 0 && *best != ~0ull) atomicMin((unsigned long long*)&a.gfirst[g], *best);
  __syncthreads();
  return true;
}

// Ticket t = r * G + g names run r of group g: every group's run 0 is handed out before any group's run 1, so a
// group whose first stable position was latched early skips its later runs (the test wants only the FIRST j).
// A run slides over up to NI items of WITEM positions, carrying the window sums from item to item, so the
// 2n-position base reduction is paid once per run.  Exactness: every run whose first position is <= the final
// answer is processed (a run is skipped only when gfirst[g] already holds a smaller position).
__global__ void __launch_bounds__(WT, 2) k_window(WinArgs a) {
  __shared__ Sums part[WT / 32];
  __shared__ Sums wtot[WT / 32];
  __shared__ uint64_t best, s_gf;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  __shared__ uint64_t s_item;
  __shared__ FSums fpart[WT / 32];
  __shared__ unsigned long long fbest;
  extern __shared__ int2 ring[];  // fast path: [2n + RUN] shifted (issue, retire) of the run's span
  const uint32_t total = *a.total;
  const int64_t n = a.n;
  for (;;) {
    // one run per claim: the next entry of the run-major list that no earlier latch has made pointless
    if (tid == 0) {
      uint64_t it = ~0ull;
      for (;;) {
        const uint32_t t = atomicAdd(a.ticket, 1u);
        if (t >= total) break;
        const uint64_t e = a.list[t];
        const uint32_t g = (uint32_t)e, r = (uint32_t)(e >> 32);
        const uint64_t P0 = a.gstart[g] + 2 * (uint64_t)n - 1 + (uint64_t)r * RUN;
        if (*(volatile const uint64_t*)&a.gfirst[g] > P0) { it = e; break; }
      }
      s_item = it;
    }
    __syncthreads();
    const uint64_t item = s_item;
    __syncthreads();
    if (item == ~0ull) break;
    {
      const uint32_t g = (uint32_t)item, r = (uint32_t)(item >> 32);
      const int64_t gs = (int64_t)a.gstart[g], ge = (int64_t)a.gstart[g + 1];
      const int64_t P0 = gs + 2 * n - 1 + (int64_t)r * RUN;
      const int64_t P1 = P0 + RUN < ge ? P0 + RUN : ge;
      if (a.ring && window_run_fast(a, g, gs, P0, P1, ring, fpart, &fbest)) continue;
      auto X = [&](int64_t q) -> int64_t { return q >= gs ? win_x(a, q, win_y(a, q)) : 0; };
      auto Yv = [&](int64_t q) -> int64_t { return q >= gs ? win_y(a, q) : 0; };
      // base: windows ending at P0-1 ([P0-n, P0-1] and [P0-2n, P0-1]); positions < gs contribute 0
      Sums s;
      sums_zero(s);
#pragma unroll 4
      for (int64_t q = P0 - 2 * n + tid; q < P0; q += WT) {
        int64_t x = X(q), y = Yv(q), d = y - x;
        s.s2n += d;
        if (q >= P0 - n) {
          s.sx += x; s.sy += y; s.sn += d;
          s.sxy += (i128)x * y; s.sxx += (i128)x * x;
        }
      }
      for (int o = 16; o > 0; o >>= 1) sums_add(s, shfl_xor_sums(s, o));
      if (lane == 0) part[wid] = s;
      if (tid == 0) best = ~0ull;
      __syncthreads();
      Sums base;
      sums_zero(base);
      for (int k = 0; k < WT / 32; ++k) sums_add(base, part[k]);
      for (int64_t Q0 = P0; Q0 < P1; Q0 += WITEM) {
        const int64_t Q1 = Q0 + WITEM < P1 ? Q0 + WITEM : P1;
        const int64_t q0 = Q0 + (int64_t)tid * WPT;
        // pass 1: this thread's deltas over its WPT positions
        Sums dl;
        sums_zero(dl);
#pragma unroll
        for (int u = 0; u < WPT; ++u) {
          int64_t q = q0 + u;
          if (q < Q1) {
            int64_t xs = X(q), ys = Yv(q), xo = X(q - n), yo = Yv(q - n);
            int64_t do2 = Yv(q - 2 * n) - X(q - 2 * n);
            dl.sx += xs - xo; dl.sy += ys - yo;
            dl.sn += (ys - xs) - (yo - xo);
            dl.s2n += (ys - xs) - do2;
            dl.sxy += (i128)xs * ys - (i128)xo * yo;
            dl.sxx += (i128)xs * xs - (i128)xo * xo;
          }
        }
        Sums incl = dl;
        for (int o = 1; o < 32; o <<= 1) {
          Sums tt = shfl_up_sums(incl, o);
          if (lane >= o) sums_add(incl, tt);
        }
        if (lane == 31) wtot[wid] = incl;
        __syncthreads();
        Sums w = base, tot;
        sums_zero(tot);
        for (int k = 0; k < WT / 32; ++k) {
          if (k < wid) sums_add(w, wtot[k]);
          sums_add(tot, wtot[k]);
        }
        sums_add(w, incl);
        sums_sub(w, dl);  // exclusive prefix: window sums ending at q0 - 1
        // pass 2: slide and test (values re-read through L1)
        uint64_t mine = ~0ull;
        for (int u = 0; u < WPT; ++u) {
          int64_t q = q0 + u;
          if (q >= Q1) break;
          int64_t xs = X(q), ys = Yv(q), xo = X(q - n), yo = Yv(q - n);
          int64_t do2 = Yv(q - 2 * n) - X(q - 2 * n);
          w.sx += xs - xo; w.sy += ys - yo;
          w.sn += (ys - xs) - (yo - xo);
          w.s2n += (ys - xs) - do2;
          w.sxy += (i128)xs * ys - (i128)xo * yo;
          w.sxx += (i128)xs * xs - (i128)xo * xo;
          // cond2 first (64-bit: |2 S_n - S_2n| < 2^41, times delta_den <= 2^16), then cond1 only where it holds
          bool c2 = false;
          if (w.s2n > 0) {
            int64_t d2 = 2 * w.sn - w.s2n;
            if (d2 < 0) d2 = -d2;
            c2 = (i128)a.dden * d2 < (i128)a.dnum * w.s2n;
          }
          if (c2) {
            // cond1: den > 0 and dden*|den - num| < dnum*den  (Eq. 1: a = num/den)
            i128 num = (i128)n * w.sxy - (i128)w.sx * w.sy;
            i128 den = (i128)n * w.sxx - (i128)w.sx * w.sx;
            bool c1 = false;
            if (den > 0) {
              i128 diff = den - num;
              if (diff < 0) diff = -diff;
              c1 = (i128)a.dden * diff < (i128)a.dnum * den;
            }
            if (c1) { mine = (uint64_t)q; break; }
          }
        }
        if (mine != ~0ull) atomicMin((unsigned long long*)&best, (unsigned long long)mine);
        if (tid == 0) s_gf = *(volatile const uint64_t*)&a.gfirst[g];
        sums_add(base, tot);
        __syncthreads();
        const uint64_t b = best;
        if (b != ~0ull) {
          if (tid == 0) atomicMin((unsigned long long*)&a.gfirst[g], (unsigned long long)b);
          break;
        }
        // another run of this group latched an earlier position: the rest of this run cannot matter
        if (s_gf < (uint64_t)Q1) break;
      }
      __syncthreads();
    }
  }
}

// ---- 5. outputs ----------------------------------------------------------------------------------------------
// Record index of the latched sorted position q of group (k, b) on the job paths (no index array is kept): the
// group's job cells give the job holding q (kernels with <= 256 local ids: cells = the jobs' start positions,
// unmodified; more ids: the scatter's atomics left the jobs' END positions), then one warp counts the job's
// records of b up to q's rank.
__device__ uint64_t locate_record(const photon_timing& t, const JobMap& jm, const uint32_t* cells, uint32_t k,
                                  uint32_t b, uint64_t q, uint64_t gs) {
  const uint32_t lane = threadIdx.x & 31, B = t.n_bb;
  const bool sm = jm.nbins(k, B) <= kSmemBins;
  const uint64_t nj = jm.coff[k + 1] - jm.coff[k];
  const uint32_t* c = cells + jm.hbase(k, B) + (uint64_t)jm.lid(k, b) * nj;
  // P = the number of cells <= q (monotone cells: a prefix), by a 32-ary search; sm: the job is P - 1 (its start
  // is <= q), else P (the first job ending after q)
  uint64_t lo = 0, hi = nj;  // c[j] <= q for j < lo, c[j] > q for j >= hi
  while (hi > lo) {
    const uint64_t step = (hi - lo + 31) / 32, j = lo + lane * step;
    const unsigned m = __ballot_sync(0xffffffffu, j < hi && c[j] <= q);
    const uint64_t n = __popc(m), lo0 = lo;
    if (n == 0) { hi = lo; break; }
    lo = lo0 + (n - 1) * step + 1;
    hi = umin64(hi, lo0 + n * step);
  }
  const uint64_t jl = sm ? (lo ? lo - 1 : 0) : lo;
  const uint64_t start = sm ? c[jl] : (jl ? c[jl - 1] : gs);
  const uint64_t rank = q - start;
  // the job's records: each lane counts b in its 64-record slice, a warp scan finds the slice, that lane the record
  const uint64_t a = umin64(t.kernel_rec_off[k], t.n_records), e = umin64(t.kernel_rec_off[k + 1], t.n_records);
  const uint64_t cs = a + jl * JOB, ce = umin64(cs + JOB, e);
  constexpr int PER = JOB / 32;
  const uint64_t l0 = cs + (uint64_t)lane * PER;
  uint32_t cnt = 0;
#pragma unroll 16
  for (int u = 0; u < PER; ++u) {  // independent loads: the compiler keeps many in flight
    const uint64_t i = l0 + u;
    uint32_t x = i < ce ? (uint32_t)t.bb[i] : kNone;
    if (x != kNone && x >= B) x = 0;  // as the scatter placed it (the error is latched)
    cnt += x == b;
  }
  uint32_t incl = cnt;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
    if ((int)lane >= o) incl += y;
  }
  const unsigned hit = __ballot_sync(0xffffffffu, rank < incl && rank >= incl - cnt);
  const int owner = __ffs(hit) - 1;
  if (owner < 0) return ~0ull;
  // the owner's 64-record slice, two records per lane (one round of loads, no serial walk): the r-th match
  const uint32_t r = (uint32_t)__shfl_sync(0xffffffffu, (uint32_t)(rank - (incl - cnt)), owner);
  static_assert(PER == 64, "two records per lane");
  const uint64_t i0 = cs + (uint64_t)owner * PER + 2 * lane;
  uint32_t x0 = i0 < ce ? (uint32_t)t.bb[i0] : kNone, x1 = i0 + 1 < ce ? (uint32_t)t.bb[i0 + 1] : kNone;
  if (x0 != kNone && x0 >= B) x0 = 0;
  if (x1 != kNone && x1 >= B) x1 = 0;
  const uint32_t m0 = x0 == b ? 1u : 0u, m1 = x1 == b ? 1u : 0u, c2 = m0 + m1;
  uint32_t in2 = c2;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, in2, o);
    if ((int)lane >= o) in2 += y;
  }
  const uint32_t ex2 = in2 - c2;  // matches before this lane's pair
  uint64_t pos = ~0ull;
  if (r >= ex2 && r < in2) pos = (r == ex2 && m0 ? i0 : i0 + 1) - a;
  const unsigned ph = __ballot_sync(0xffffffffu, pos != ~0ull);
  return __shfl_sync(0xffffffffu, pos, ph ? __ffs(ph) - 1 : 0);
}

// group g -> (k, b): mode 0 (radix path) g = b*K + k; 1 (job path, B <= 256) g = k*B + b; 2 (compact) gkb[g]
__global__ void k_finish(photon_timing t, JobMap jm, const uint32_t* cells, const uint32_t* idx, GCopy C,
                         const uint32_t* G, const uint64_t* gfirst,
                         const uint64_t* gstart, uint32_t n, int mode, const uint64_t* gkb, int64_t* first_stable,
                         uint64_t* dur) {
  const uint32_t lane = threadIdx.x & 31, ng = *G, K = t.n_kernels, B = t.n_bb;
  const uint32_t nw = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t g = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; g < ng; g += nw) {
    uint64_t q = gfirst[g];
    if (q == ~0ull) continue;
    uint64_t k, b;
    if (mode == 0) { k = g % K; b = g / K; }
    else if (mode == 1) { k = g / B; b = g % B; }
    else { k = gkb[g] >> 16; b = gkb[g] & 0xFFFFu; }
    uint64_t s = 0;
    for (uint64_t i = q + 1 - n + lane; i <= q; i += 32) {
      const uint32_t d = C.D[i];
      s += d != kDurEsc ? (uint64_t)d : (uint64_t)(g_y(C, i) - C.Xw[i]);
    }
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const uint64_t pos = mode == 0 ? idx[q] - t.kernel_rec_off[k]
                                   : locate_record(t, jm, cells, (uint32_t)k, (uint32_t)b, q, gstart[g]);
    if (lane == 0) {
      first_stable[k * B + b] = (int64_t)pos;
      if (dur) dur[k * B + b] = s;
    }
  }
}

// switch_at[k]: order stable BBs by t_b; the first t_b at which rate_den * acc > rate_num * total, where acc sums
// the weights of stable BBs with t <= t_b (L208, Fig 7) [P-14].  acc(t) is monotone and changes only at stable
// t_b values, so the answer is the least t with rate_den * acc(t) > rate_num * total: a binary search over t in
// [0, 2^32) with one block reduction per step (O(32 B) per kernel instead of sorting).
__device__ __forceinline__ u128 block_sum_u128(u128 v, uint64_t* slo, uint64_t* shi) {
  uint64_t lo = (uint64_t)v, hi = (uint64_t)(v >> 64);
  for (int o = 16; o > 0; o >>= 1) {
    uint64_t lo2 = __shfl_xor_sync(0xffffffffu, lo, o), hi2 = __shfl_xor_sync(0xffffffffu, hi, o);
    uint64_t s = lo + lo2;
    hi = hi + hi2 + (s < lo);
    lo = s;
  }
  __syncthreads();
  if ((threadIdx.x & 31) == 0) { slo[threadIdx.x >> 5] = lo; shi[threadIdx.x >> 5] = hi; }
  __syncthreads();
  u128 t = 0;
  for (int w = 0; w < 8; ++w) t += ((u128)shi[w] << 64) | slo[w];
  return t;
}

__global__ void __launch_bounds__(256) k_switch(const int64_t* first_stable, const uint64_t* kbb, uint32_t K,
                                                uint32_t B, uint32_t rnum, uint32_t rden, int64_t* switch_at) {
  __shared__ uint64_t slo[8], shi[8];
  __shared__ uint64_t s_t[256], s_w[256];
  __shared__ uint32_t s_n;
  __shared__ unsigned long long s_best;
  for (uint32_t k = blockIdx.x; k < K; k += gridDim.x) {
    if (threadIdx.x == 0) s_best = ~0ull;
    const int64_t* fs = first_stable + (uint64_t)k * B;
    const uint64_t* w = kbb + (uint64_t)k * B;
    u128 t = 0, a = 0;
    for (uint32_t b = threadIdx.x; b < B; b += blockDim.x) {
      t += w[b];
      if (fs[b] >= 0) a += w[b];
    }
    const u128 total = block_sum_u128(t, slo, shi);
    const u128 all = block_sum_u128(a, slo, shi);
    int64_t ans = -1;
    // the stable BBs compacted (their t_b are distinct: one record each); with at most 256 of them, each one's
    // acc(t_b) is summed over the compacted list in shared memory and the answer is the least qualifying t_b
    if (threadIdx.x == 0) s_n = 0;
    __syncthreads();
    for (uint32_t b = threadIdx.x; b < B; b += blockDim.x)
      if (fs[b] >= 0) {
        const uint32_t j = atomicAdd(&s_n, 1u);
        if (j < 256) { s_t[j] = (uint64_t)fs[b]; s_w[j] = w[b]; }
      }
    __syncthreads();
    const uint32_t ns = s_n;
    if (total > 0 && (u128)rden * all > (u128)rnum * total && ns <= 256) {
      unsigned long long best = ~0ull;
      if (threadIdx.x < ns) {
        const uint64_t ti = s_t[threadIdx.x];
        u128 acc = 0;
        for (uint32_t j = 0; j < ns; ++j)
          if (s_t[j] <= ti) acc += s_w[j];
        if ((u128)rden * acc > (u128)rnum * total) best = ti;
      }
      for (int o = 16; o > 0; o >>= 1) best = umin64(best, __shfl_xor_sync(0xffffffffu, best, o));
      if ((threadIdx.x & 31) == 0) atomicMin(&s_best, best);
      __syncthreads();
      ans = (int64_t)s_best;
    } else if (total > 0 && (u128)rden * all > (u128)rnum * total) {
      uint64_t lo = 0, hi = 0xFFFFFFFFull;  // invariant: acc(hi) passes
      while (lo < hi) {
        uint64_t mid = (lo + hi) >> 1;
        u128 m = 0;
        for (uint32_t b = threadIdx.x; b < B; b += blockDim.x)
          if (fs[b] >= 0 && (uint64_t)fs[b] <= mid) m += w[b];
        m = block_sum_u128(m, slo, shi);
        if ((u128)rden * m > (u128)rnum * total) hi = mid; else lo = mid + 1;
      }
      ans = (int64_t)lo;
    }
    if (threadIdx.x == 0) switch_at[k] = ans;
    __syncthreads();
  }
}

// ---- N1: warp-level stability (L249, L262, Fig 10) ------------------------------------------------------------
// The warp streams need no partition: a kernel's warp records are already one group in retirement order, so the
// groups are the kernels (gstart = kernel_rec_off) and k_window runs on issue / retire directly.
// Grid-stride over records: retire >= issue, times < 2^40, retire non-decreasing within a kernel [P-16][P-18] (a
// decrease is an error unless the record starts a kernel: binary search of kernel_rec_off, rare path); one thread
// per kernel checks the offsets.
__global__ void k_warp_validate(const uint64_t* kro, uint32_t K, uint64_t R, const uint64_t* issue,
                                const uint64_t* retire, DevErr* err) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x, nt = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t k = tid; k < K; k += nt) {
    const uint64_t a = kro[k], b = kro[k + 1];
    if ((k == 0 && a != 0) || b < a || b > R || (k + 1 == K && b != R)) latch(err, PHOTON_ERANGE, (int64_t)k);
  }
  for (uint64_t i = tid; i < R; i += nt) {
    const uint64_t x = issue[i], y = retire[i];
    bool bad = y < x || y >= kTimeLimit || x >= kTimeLimit;
    if (!bad && i > 0 && retire[i - 1] > y) {
      uint32_t lo = 0, hi = K;  // is i a kernel start? (largest k with kro[k] <= i)
      while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (kro[mid] <= i) lo = mid; else hi = mid - 1;
      }
      bad = kro[lo] != i;
    }
    if (bad) latch(err, PHOTON_ERANGE, (int64_t)i);
  }
}

// runs per kernel; kernels without a dominant warp type (ok[k] == 0) get none (warp sampling stays off, L249)
__global__ void k_warp_runs(const uint64_t* kro, uint32_t K, uint64_t R, const uint8_t* ok, uint32_t n2,
                            uint32_t* nruns, uint64_t* gfirst, uint32_t* misc) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x) {
    const uint64_t a = kro[k], b = kro[k + 1];
    const uint64_t sz = (b >= a && b <= R) ? b - a : 0;
    const uint32_t r = (sz >= n2 && (!ok || ok[k])) ? (uint32_t)ceil_div(sz - n2 + 1, RUN) : 0u;
    nruns[k] = r;
    gfirst[k] = ~0ull;
    if (r) atomicMax(misc + 1, r);
    if (k == 0) misc[0] = K;
  }
}

// switch position (0-based within the kernel's stream) and S_n = sum of the last n durations there
__global__ void k_warp_finish(const uint64_t* kro, uint32_t K, const uint64_t* issue, const uint64_t* retire,
                              const uint64_t* gfirst, uint32_t n, int64_t* switch_at, uint64_t* dur) {
  const uint32_t lane = threadIdx.x & 31, nw = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; k < K; k += nw) {
    const uint64_t q = gfirst[k];
    if (q == ~0ull) continue;
    uint64_t sum = 0;
    for (uint64_t i = q + 1 - n + lane; i <= q; i += 32) sum += retire[i] - issue[i];
    for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    if (lane == 0) {
      switch_at[k] = (int64_t)(q - kro[k]);
      if (dur) dur[k] = sum;
    }
  }
}

// run list workspace: runs per group <= R / RUN + 1; total runs <= R / RUN + R / (2n) + 1 (groups with >= 2n records)
struct RunList {
  uint32_t* cnt;   // [cap_r] groups per run index, then their exclusive prefix
  uint32_t* fill;  // [cap_r]
  uint64_t* list;  // [cap_l]
  uint64_t cap_r, cap_l;
};
inline void carve_runlist(Carver& c, uint64_t R, RunList& rl) {
  rl.cap_r = R / RUN + 2;
  rl.cap_l = R / RUN + R / 4 + 2;  // n >= 2
  rl.cnt = c.take<uint32_t>(rl.cap_r);
  rl.fill = c.take<uint32_t>(rl.cap_r);
  rl.list = c.take<uint64_t>(rl.cap_l);
}
// k_work_count / k_warp_runs have written nruns and misc[1] = max runs: build the list, set the window args
inline void build_runlist(const RunList& rl, const uint32_t* G, const uint32_t* nruns, uint32_t* misc, uint64_t gcap,
                          int num_sms, WinArgs& wa, cudaStream_t s) {
  cudaMemsetAsync(rl.cnt, 0, sizeof(uint32_t) * rl.cap_r, s);
  cudaMemsetAsync(rl.fill, 0, sizeof(uint32_t) * rl.cap_r, s);
  const unsigned gg = (unsigned)umin64(ceil_div(gcap * 32, 256), (uint64_t)num_sms * 8);
  note_launch(), k_runs_count<<<gg ? gg : 1, 256, 0, s>>>(G, nruns, rl.cnt);
  note_launch(), k_runs_scan<<<1, 1024, 0, s>>>(misc + 1, rl.cnt, misc + 3);
  note_launch(), k_runs_fill<<<gg ? gg : 1, 256, 0, s>>>(G, nruns, rl.cnt, rl.fill, rl.list);
  wa.list = rl.list;
  wa.total = misc + 3;
  wa.ticket = misc + 2;
}

// k_window launch: the fast path's shared span when it fits (n <= ~10K), and the shifted-time range
inline void window_launch(WinArgs& wa, int num_sms, cudaStream_t s) {
  const uint64_t span = 2 * (uint64_t)wa.n + RUN;
  const size_t smem = span * sizeof(int2);
  wa.ring = smem <= 200 * 1024 ? (uint32_t)span : 0u;
  int lg = 0;
  while ((1ull << lg) < (uint64_t)(wa.n ? wa.n : 1)) ++lg;  // ceil(log2 n)
  int L = (61 - lg) / 2;  // n * lim^2 < 2^61: window sums and their differences (deltas, scans) fit int64
  if (L > 31) L = 31;
  wa.lim = (int64_t)1 << L;
  const size_t dyn = wa.ring ? smem : 0;
  if (dyn) cudaFuncSetAttribute(k_window, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)dyn);
  note_launch(), k_window<<<(unsigned)num_sms * 2, WT, dyn, s>>>(wa);
}

struct Layout {
  int mode;          // 1: job multisplit on BB ids (B <= 256); 2: on per-kernel compacted ids (B <= 8192);
                     // 0: LSD radix sort of composite keys (larger B)
  uint64_t* key0; uint64_t* key1;  // radix path only
  uint32_t* val0; uint32_t* val1;  // val0 = original record index of each sorted position (all paths)
  GCopy G;  // the grouped copy (8 B/record + escape side arrays)
  uint32_t* hist; uint32_t* bsum; uint32_t* misc;  // misc[0] = G, [1] = max runs, [2] = ticket, [4] = scan total
  uint64_t* gstart;  // [gcap+1]
  uint32_t* nruns;   // [gcap]
  uint64_t* gfirst;  // [gcap]
  uint64_t* coff;    // [K+1] chunk (job) offsets per kernel
  // compact ids
  uint32_t nw;       // bitmap words per kernel
  uint32_t* bits; uint32_t* lbase; uint32_t* bk;  // [K*nw], [K*nw], [K]
  uint64_t* goff; uint64_t* hb; uint64_t* gkb;    // [K+1], [K+1], [gcap]
  RunList rl;
  uint64_t gcap, n_tiles, n_jobs, hn;
  size_t bytes;
};

Layout make_layout(const photon_timing& t, void* base) {
  Carver c(base);
  Layout L{};
  uint64_t R = t.n_records ? t.n_records : 1;
  const uint64_t KB = (uint64_t)t.n_kernels * t.n_bb;
  L.mode = t.n_bb <= kSmemBins ? 1 : (t.n_bb <= kCompactMaxB ? 2 : 0);
  L.gcap = L.mode == 2 ? (KB < R ? KB : R) : KB;  // dense group ids, or one per (kernel, BB present)
  if (L.gcap == 0) L.gcap = 1;
  L.n_tiles = ceil_div(R, RTILE);
  L.n_jobs = ceil_div(R, JOB) + t.n_kernels;
  if (L.mode == 0) {
    L.key0 = c.take<uint64_t>(R); L.key1 = c.take<uint64_t>(R);
    L.val0 = c.take<uint32_t>(R); L.val1 = c.take<uint32_t>(R);
  }
  L.G.Y32 = c.take<uint32_t>(R); L.G.D = c.take<uint32_t>(R); L.G.Yw = c.take<int64_t>(R);
  L.G.Xw = c.take<int64_t>(R);
  // histogram cells: B * jobs; compact: sum_k B_k * jobs_k <= 2R + ... whenever no kernel has more than 2048
  // distinct BB ids (ECAPACITY otherwise)
  L.hn = L.mode == 1 ? (uint64_t)t.n_bb * L.n_jobs : (L.mode == 2 ? 2 * R + 65536 : (uint64_t)RNB * L.n_tiles);
  L.hist = c.take<uint32_t>(L.hn);
  L.bsum = c.take<uint32_t>(ceil_div(L.hn, SB) + 1);
  L.misc = c.take<uint32_t>(16);
  L.gstart = c.take<uint64_t>(L.gcap + 1);
  L.nruns = c.take<uint32_t>(L.gcap);
  L.gfirst = c.take<uint64_t>(L.gcap);
  L.coff = c.take<uint64_t>((uint64_t)t.n_kernels + 1);
  if (L.mode == 2) {
    L.nw = (t.n_bb + 31) / 32;
    L.bits = c.take<uint32_t>((uint64_t)t.n_kernels * L.nw + 1);
    L.lbase = c.take<uint32_t>((uint64_t)t.n_kernels * L.nw + 1);
    L.bk = c.take<uint32_t>((uint64_t)t.n_kernels + 1);
    L.goff = c.take<uint64_t>((uint64_t)t.n_kernels + 1);
    L.hb = c.take<uint64_t>((uint64_t)t.n_kernels + 1);
    L.gkb = c.take<uint64_t>(L.gcap);
  }
  carve_runlist(c, R, L.rl);
  L.bytes = c.off + 256;
  return L;
}

}  // namespace

size_t stable_ws_bytes(const photon_timing& t) { return make_layout(t, nullptr).bytes; }

// ---- the stable LSD radix sort of (u64 key, u32 index) pairs, also used by the N2 ingest (k_full.cu) -----------
size_t radix_pairs_ws_bytes(uint64_t n) {
  Carver c(nullptr);
  const uint64_t N = n ? n : 1, nt = ceil_div(N, RTILE);
  c.take<uint64_t>(N);
  c.take<uint32_t>(N);
  c.take<uint32_t>(N);
  c.take<uint32_t>((uint64_t)RNB * nt);
  c.take<uint32_t>(ceil_div((uint64_t)RNB * nt, SB) + 1);
  c.take<uint32_t>(16);
  return c.off + 256;
}
// key[] (n keys < 2^bits, overwritten) sorted stably; *perm_out = the sorted position -> original index array
// (inside ws); keys end in *key_out (key or the workspace copy)
cudaError_t launch_radix_pairs(uint64_t* key, uint64_t n, uint32_t bits, void* ws, uint64_t** key_out,
                               uint32_t** perm_out, cudaStream_t s) {
  Carver c(ws);
  const uint64_t N = n ? n : 1, nt = ceil_div(N, RTILE);
  uint64_t* key1 = c.take<uint64_t>(N);
  uint32_t* val0 = c.take<uint32_t>(N);
  uint32_t* val1 = c.take<uint32_t>(N);
  uint32_t* hist = c.take<uint32_t>((uint64_t)RNB * nt);
  uint32_t* bsum = c.take<uint32_t>(ceil_div((uint64_t)RNB * nt, SB) + 1);
  uint32_t* misc = c.take<uint32_t>(16);
  uint64_t* kin = key; uint64_t* kout = key1;
  uint32_t* vin = val0; uint32_t* vout = val1;
  int pass = 0;
  for (uint32_t sh = 0; sh < (bits ? bits : 1); sh += RBITS, ++pass) {
    if (n == 0) break;
    note_launch(), k_radix_up<<<(unsigned)nt, RT, 0, s>>>(kin, n, sh, hist, nt);
    scan_u32(hist, hist, (uint64_t)RNB * nt, bsum, misc, s);
    note_launch(), k_radix_down<<<(unsigned)nt, RT, 0, s>>>(kin, vin, n, sh, hist, nt, kout, vout, pass == 0);
    uint64_t* tk = kin; kin = kout; kout = tk;
    uint32_t* tv = vin; vin = vout; vout = tv;
  }
  *key_out = kin;
  *perm_out = vin;
  return cudaGetLastError();
}

cudaError_t launch_stable(const photon_timing& t, const uint64_t* kbb, photon_stable_params p, void* ws,
                          size_t ws_bytes, int64_t* first_stable, uint64_t* dur, int64_t* switch_at, DevErr* err,
                          int num_sms, cudaStream_t s) {
  (void)ws_bytes;
  Layout L = make_layout(t, ws);
  const uint64_t R = t.n_records;
  const uint32_t K = t.n_kernels, B = t.n_bb;
  cudaMemsetAsync(first_stable, 0xFF, sizeof(int64_t) * (size_t)K * B, s);
  if (dur) cudaMemsetAsync(dur, 0, sizeof(uint64_t) * (size_t)K * B, s);
  cudaMemsetAsync(L.misc, 0, 64, s);
  const uint64_t chunk = L.mode != 0 ? JOB : REC_CHUNK;
  note_launch(), k_rec_chunks<<<1, 1024, 0, s>>>(t.kernel_rec_off, K, R, chunk, L.coff, err);
  if (R > 0) {
    uint32_t* idx;
    JobMap jmf{};  // the job map (job paths), for k_finish
    if (L.mode != 0) {
      // 1-2. per-job histograms of (kernel-local) BB ids -> kernel-major scan -> stable scatter of (issue, retire,
      // index) into group order
      unsigned gj = (unsigned)umin64(ceil_div(L.n_jobs, 8), (uint64_t)num_sms * 8);
      JobMap jm{};
      jm.coff = L.coff;
      jm.compact = L.mode == 2;
      jm.nkern = K;
      jm.hcap = L.hn;
      if (jm.compact) {
        jm.bits = L.bits; jm.lbase = L.lbase; jm.bk = L.bk; jm.hb = L.hb; jm.nw = L.nw;
        cudaMemsetAsync(L.bits, 0, sizeof(uint32_t) * (size_t)K * L.nw, s);
        const size_t psm = (size_t)8 * L.nw * 4;
        cudaFuncSetAttribute(k_presence, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)psm);
        note_launch(), k_presence<<<gj, 256, psm, s>>>(t, L.coff, L.n_jobs, L.nw, L.bits);
        const unsigned gk = (unsigned)umin64(ceil_div((uint64_t)K * 32, 256), (uint64_t)num_sms * 8);
        note_launch(), k_lid_prep<<<gk, 256, 0, s>>>(K, L.nw, L.bits, L.lbase, L.bk);
        note_launch(), k_lid_scan<<<1, 1024, 0, s>>>(K, L.coff, L.bk, L.goff, L.hb, L.misc + 0, L.hn, err);
        note_launch(), k_lid_groups<<<gk, 256, 0, s>>>(K, L.nw, L.bits, L.lbase, L.goff, L.gkb);
      }
      // compact: only hb[K] cells are live (C5: ~R/128 of the 2R + 65536 reserved)
      const uint64_t* hlive = jm.compact ? L.hb + K : nullptr;
      if (jm.compact) note_launch(), k_zero_live<<<(unsigned)num_sms * 4, 256, 0, s>>>(L.hist, L.hn, hlive);
      else cudaMemsetAsync(L.hist, 0, sizeof(uint32_t) * L.hn, s);
      const unsigned gh = (unsigned)umin64(ceil_div(L.n_jobs, HW), (uint64_t)num_sms * 12);
      note_launch(), k_job_hist<<<gh, HW * 32, 0, s>>>(t, jm, L.n_jobs, L.hist);
      scan_u32(L.hist, L.hist, L.hn, L.bsum, L.misc + 4, s, hlive);
      // group starts first: kernels with > 256 local ids use the scanned cells as running offsets in the scatter
      note_launch(), k_job_gstart<<<(unsigned)umin64(ceil_div(L.gcap + 1, 256), (uint64_t)num_sms * 8), 256, 0, s>>>(
          L.hist, jm, L.goff, L.gkb, K, B, R, (uint64_t)B * L.n_jobs, L.gstart, L.misc + 0);
      note_launch(), k_job_scatter<<<gj, 256, 0, s>>>(t, jm, L.n_jobs, L.hist, L.G, err);
      idx = nullptr;
      jmf = jm;
    } else {
      uint64_t jobs_ub = ceil_div(R, REC_CHUNK) + K;
      unsigned grid = (unsigned)umin64(jobs_ub, (uint64_t)num_sms * 8);
      cudaMemsetAsync(L.key0, 0, sizeof(uint64_t) * R, s);  // keys stay < K*B even if offsets are malformed
      note_launch(), k_rec_prep<<<grid, 256, 0, s>>>(t, L.coff, L.key0, err);
      // radix passes over the bits of the composite key b*K + k
      uint32_t bits = 1;
      while ((1ull << bits) < L.gcap) ++bits;
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
      unsigned gR = (unsigned)ceil_div(R + 1, 256);
      note_launch(), k_gather<<<gR, 256, 0, s>>>(vin, R, t.issue, t.retire, L.G);
      note_launch(), k_fill_gstart<<<gR, 256, 0, s>>>(kin, R, L.gcap, L.gstart);
      note_launch(), k_set_u32<<<1, 1, 0, s>>>(L.misc + 0, (uint32_t)L.gcap);
      idx = vin;
    }
    // 3-4. runs per group, windowed exact test
    note_launch(), k_work_count<<<(unsigned)umin64(ceil_div(L.gcap, 256), (uint64_t)num_sms * 4), 256, 0, s>>>(
        L.gstart, L.misc + 0, 2 * p.window_n, L.nruns, L.gfirst, L.misc + 1);
    WinArgs wa{};
    wa.X = nullptr; wa.Y = nullptr; wa.D = L.G.D; wa.G = L.G; wa.gstart = L.gstart; wa.Gn = L.misc + 0;
    wa.n = p.window_n; wa.dnum = p.delta_num; wa.dden = p.delta_den; wa.gfirst = L.gfirst;
    build_runlist(L.rl, L.misc + 0, L.nruns, L.misc, L.gcap, num_sms, wa, s);
    window_launch(wa, num_sms, s);
    // 5. outputs
    note_launch(), k_finish<<<(unsigned)umin64(ceil_div(L.gcap * 32, 256), (uint64_t)num_sms * 8), 256, 0, s>>>(
        t, jmf, L.hist, idx, L.G, L.misc + 0, L.gfirst, L.gstart, p.window_n, L.mode, L.gkb, first_stable,
        dur);
    unsigned gk = (unsigned)umin64(K, (uint64_t)num_sms * 8);
    note_launch(), k_switch<<<gk ? gk : 1, 256, 0, s>>>(first_stable, kbb, K, B, p.rate_num, p.rate_den, switch_at);
  } else {
    cudaMemsetAsync(switch_at, 0xFF, sizeof(int64_t) * K, s);
  }
  return cudaGetLastError();
}

size_t warp_stable_ws_bytes(uint32_t K, uint64_t R) {
  Carver c(nullptr);
  c.take<uint32_t>(16);
  c.take<uint32_t>((uint64_t)K + 1);
  c.take<uint64_t>((uint64_t)K + 1);
  RunList rl;
  carve_runlist(c, R, rl);
  return c.off + 256;
}

cudaError_t launch_warp_stable(const photon_timing& t, const uint8_t* ok, uint32_t n, uint32_t dnum, uint32_t dden,
                               void* ws, int64_t* switch_at, uint64_t* dur, DevErr* err, int num_sms,
                               cudaStream_t s) {
  Carver c(ws);
  uint32_t* misc = c.take<uint32_t>(16);
  uint32_t* nruns = c.take<uint32_t>((uint64_t)t.n_kernels + 1);
  uint64_t* gfirst = c.take<uint64_t>((uint64_t)t.n_kernels + 1);
  RunList rl;
  carve_runlist(c, t.n_records, rl);
  const uint32_t K = t.n_kernels;
  cudaMemsetAsync(switch_at, 0xFF, sizeof(int64_t) * K, s);
  if (dur) cudaMemsetAsync(dur, 0, sizeof(uint64_t) * K, s);
  cudaMemsetAsync(misc, 0, 64, s);
  const unsigned gk = (unsigned)umin64(ceil_div((uint64_t)K * 32, 256), (uint64_t)num_sms * 8);
  const unsigned gv = (unsigned)umin64(ceil_div(umax64(t.n_records, K), 256), (uint64_t)num_sms * 8);
  note_launch(), k_warp_validate<<<gv ? gv : 1, 256, 0, s>>>(t.kernel_rec_off, K, t.n_records, t.issue, t.retire,
                                                             err);
  if (t.n_records == 0) return cudaGetLastError();
  note_launch(), k_warp_runs<<<(unsigned)ceil_div(K, 256), 256, 0, s>>>(t.kernel_rec_off, K, t.n_records, ok, 2 * n,
                                                                       nruns, gfirst, misc);
  WinArgs wa{};
  wa.X = t.issue; wa.Y = t.retire; wa.D = nullptr; wa.gstart = t.kernel_rec_off; wa.Gn = misc + 0;
  wa.n = n; wa.dnum = dnum; wa.dden = dden; wa.gfirst = gfirst;
  build_runlist(rl, misc + 0, nruns, misc, K, num_sms, wa, s);
  window_launch(wa, num_sms, s);
  note_launch(), k_warp_finish<<<gk, 256, 0, s>>>(t.kernel_rec_off, K, t.issue, t.retire, gfirst, n, switch_at, dur);
  return cudaGetLastError();
}

}  // namespace photon
