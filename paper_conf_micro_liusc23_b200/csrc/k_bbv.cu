// k_bbv.cu — A1 (per-warp BBV projected to 16 bins) fused with A2's insertion step (K1 + K2a).
//
// PAPER.md: L161 (a BBV lists the basic blocks a warp executed, identified by start PC), L154 (same instruction
// sequence => same BBV => same warp type), L178 ("project these BBVs into fixed-size BBVs (We use 16) to improve
// online clustering performance ... we can easily cluster the warps if they have the same BBV").  Readings [P-1]
// (entry = executions x length) and [P-2] (sum-preserving fold into 16 bins).
//
// Design: one persistent CTA per SM slot.  A CTA owns "tiles" of 256 consecutive analysed warps
// (one warp segment per thread) and streams each tile's contiguous event range from HBM into a 4-stage ring of
// 8 KB shared-memory chunks with cp.async.bulk (the TMA copy engine) completing on mbarriers; thread 0 keeps the
// ring full across tile boundaries.  Each thread folds its own segment's events into a private column of a
// 16 x 256 shared-memory histogram (conflict-free: column = thread), reading 8 events per 128-bit LDS and one
// packed (len, bin) word per event from a shared-memory BB table.  At the end of a tile each thread holds its
// warp's 16-bin key: warps of a CUDA warp are de-duplicated with __match_any_sync on a 64-bit hash, then across
// the CTA in a shared-memory table, and each distinct (kernel, key) is inserted once into the global
// open-addressing table (exact key verification).  The warp's slot id is written to warp_slot[w]; the
// canonical type id replaces it later (k_types.cu).
#include "internal.h"

namespace photon {

namespace {

constexpr int TPB = 256;            // threads per CTA = warp segments per tile
constexpr int CH = 4096;            // events per ring chunk (8 KB)
constexpr int NST = 4;              // ring stages
constexpr int SMEM_TBL_MAX = 8192;  // BB table entries kept in shared memory
constexpr int LSLOTS = 256;         // CTA-local de-dup slots (>= distinct keys per tile)

struct BbvArgs {
  const uint64_t* kwo;
  const uint64_t* weo;
  const uint16_t* bb;
  const uint32_t* tbl;
  const uint32_t* max_len;
  uint32_t K, B, P2;
  uint64_t W, E;
  uint32_t* warp_bbv16;
  uint64_t* warp_insts;
  HashTable ht;
  uint32_t* warp_slot;
  int fused;
  DevErr* err;
  uint64_t n_tiles;
};

constexpr size_t kHistBytes = 16 * TPB * 4;
constexpr size_t kStageBytes = (size_t)NST * CH * 2;
constexpr size_t kLocalBytes = LSLOTS * (8 + 4 + 4 + 4);
constexpr size_t kMiscBytes = 128;
constexpr size_t kKidBytes = TPB * 4;

__host__ __device__ constexpr size_t bbv_smem_bytes(uint32_t tbl_entries) {
  return kHistBytes + kStageBytes + NST * 8 + kLocalBytes + kMiscBytes + kKidBytes + (size_t)tbl_entries * 4;
}

struct Smem {
  uint32_t* hist;
  uint16_t* stage;
  uint64_t* mbar;
  uint64_t* lhash;
  uint32_t* lowner;
  uint32_t* lcount;
  uint32_t* lgslot;
  uint32_t* misc;
  uint32_t* kid;
  uint32_t* tbl;
};

__device__ __forceinline__ Smem carve(uint8_t* s) {
  Smem m;
  m.hist = (uint32_t*)s;
  m.stage = (uint16_t*)(s + kHistBytes);
  m.mbar = (uint64_t*)(s + kHistBytes + kStageBytes);
  m.lhash = m.mbar + NST;
  m.lowner = (uint32_t*)(m.lhash + LSLOTS);
  m.lcount = m.lowner + LSLOTS;
  m.lgslot = m.lcount + LSLOTS;
  m.misc = m.lgslot + LSLOTS;
  m.kid = m.misc + kMiscBytes / 4;
  m.tbl = m.kid + TPB;
  return m;
}

__device__ __forceinline__ uint32_t kernel_of(const uint64_t* kwo, uint32_t K, uint64_t w) {
  // last k with kwo[k] <= w (upper_bound - 1): skips empty kernels
  uint32_t lo = 0, hi = K;  // answer in [0, K-1]
  while (lo < hi) {
    uint32_t mid = (lo + hi + 1) >> 1;
    if (kwo[mid] <= w) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// ---- tile finalisation: grouping (K2a) -------------------------------------------------------------------
// Keys live in the hist columns (hist[j*TPB + tid]).  Three CTA barriers: claim local slots, count + verify,
// global insert; then every thread writes its warp's slot.
__device__ void tile_group(const BbvArgs& a, const Smem& m, uint64_t w0, bool valid, uint32_t k, const uint32_t* p) {
  const int tid = threadIdx.x, lane = tid & 31;
  uint64_t h = valid ? hash_key(k, p) : 0;
  // warp-level de-dup on the hash, then exact verification against the leader's key
  unsigned active = __ballot_sync(0xffffffffu, valid);
  unsigned peers = __match_any_sync(0xffffffffu, (unsigned long long)h);
  int leader = __ffs(peers) - 1;
  bool eq = true;
  uint32_t lk = __shfl_sync(0xffffffffu, k, leader);
  eq = eq && (lk == k);
#pragma unroll
  for (int j = 0; j < 16; ++j) {
    uint32_t v = __shfl_sync(0xffffffffu, p[j], leader);
    eq = eq && (v == p[j]);
  }
  unsigned eqm = __ballot_sync(0xffffffffu, eq);
  bool is_leader = valid && (lane == leader || !eq);
  uint32_t cnt = (lane == leader) ? (uint32_t)__popc(peers & eqm & active) : 1u;
  // claim a local slot (by hash); a different key with the same hash is resolved by exact compare below
  int slot = -1;
  bool pending = false;
  if (is_leader) {
    uint32_t i = (uint32_t)(h & (LSLOTS - 1));
    for (int probe = 0; probe < LSLOTS; ++probe) {
      unsigned long long cur = atomicCAS((unsigned long long*)&m.lhash[i], 0ull, (unsigned long long)h);
      if (cur == 0ull) { m.lowner[i] = (uint32_t)tid; slot = (int)i; break; }
      if (cur == h) { slot = (int)i; pending = true; break; }
      i = (i + 1) & (LSLOTS - 1);
    }
  }
  __syncthreads();
  bool bypass = false;  // hash collision inside the tile: insert globally on our own
  if (slot >= 0) {
    if (pending) {
      uint32_t o = m.lowner[slot];
      bool same = (m.kid[o] == k);
#pragma unroll
      for (int j = 0; j < 16; ++j) same = same && (m.hist[j * TPB + o] == p[j]);
      if (!same) bypass = true;
    }
    if (!bypass) {
      atomicAdd(&m.lcount[slot], cnt);
      atomicMin(&m.lgslot[slot], (uint32_t)tid);  // group leaders are the lowest tid of their group
    }
  }
  __syncthreads();
  // global insert: one thread per occupied local slot (owner's key) + bypassing leaders
  for (int i = tid; i < LSLOTS; i += TPB) {
    uint64_t hh = m.lhash[i];
    if (hh != 0ull) {
      uint32_t o = m.lowner[i];
      uint32_t key[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) key[j] = m.hist[j * TPB + o];
      m.lgslot[i] = ht_insert(a.ht, a.err, m.kid[o], key, hh, m.lcount[i], w0 + m.lgslot[i]);
    }
  }
  uint32_t gslot = UINT32_MAX;
  if (bypass) gslot = ht_insert(a.ht, a.err, k, p, h, cnt, w0 + tid);
  __syncthreads();
  if (!bypass && slot >= 0) gslot = m.lgslot[slot];
  // members of a warp group take the leader's slot
  uint32_t from_leader = __shfl_sync(0xffffffffu, gslot, leader);
  if (valid) {
    uint32_t mine = (lane == leader || !eq) ? gslot : from_leader;
    a.warp_slot[w0 + tid] = mine;
  }
  __syncthreads();
  for (int i = tid; i < LSLOTS; i += TPB) { m.lhash[i] = 0ull; m.lcount[i] = 0u; m.lgslot[i] = UINT32_MAX; }
}

// Slow path (bad input only): locate the first event of [s, e) whose id is >= B.
__device__ void report_bad_event(const BbvArgs& a, uint64_t s, uint64_t e) {
  for (uint64_t i = s; i < e; ++i)
    if (a.bb[i] >= a.B) { latch(a.err, PHOTON_ERANGE, (int64_t)i); return; }
}

template <bool SMEM_TBL, bool CHECK_MARK>
__global__ void __launch_bounds__(TPB, 3) k_bbv(BbvArgs a) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  Smem m = carve(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t bmask = a.P2 - 1;
  const uint32_t* tblp = SMEM_TBL ? m.tbl : a.tbl;

  if (SMEM_TBL)
    for (uint32_t i = tid; i < a.P2; i += TPB) m.tbl[i] = a.tbl[i];
#pragma unroll
  for (int j = 0; j < 16; ++j) m.hist[j * TPB + tid] = 0u;
  for (int i = tid; i < LSLOTS; i += TPB) { m.lhash[i] = 0ull; m.lcount[i] = 0u; m.lgslot[i] = UINT32_MAX; }
  if (tid == 0) {
    for (int s = 0; s < NST; ++s) mbar_init(&m.mbar[s], 1);
    fence_mbar_init();
  }
  const uint32_t max_len = *a.max_len;
  const uint64_t E8 = a.E & ~7ull;
  __syncthreads();

  // ---- producer (thread 0): walks the same (tile, chunk) sequence as the consumers ----
  uint64_t p_tile = blockIdx.x, p_A = 0, p_te = 0;
  uint32_t p_c = 0, p_n = 0;
  auto p_load = [&]() {
    if (p_tile < a.n_tiles) {
      uint64_t w0 = p_tile * TPB, w1 = umin64(a.W, w0 + TPB);
      uint64_t ts = a.weo[w0], te = a.weo[w1];
      p_A = ts & ~7ull;
      p_te = te;
      p_n = te > p_A ? (uint32_t)ceil_div(te - p_A, CH) : 0u;
      p_c = 0;
    }
  };
  auto p_issue = [&](uint32_t slot) {
    while (p_tile < a.n_tiles && p_c >= p_n) { p_tile += gridDim.x; p_load(); }
    if (p_tile >= a.n_tiles) return;
    uint64_t cs = p_A + (uint64_t)p_c * CH, ce = umin64(cs + CH, p_te);
    uint64_t ae = umin64((ce + 7) & ~7ull, E8);  // bulk part [cs, ae)
    uint16_t* dst = m.stage + (size_t)slot * CH;
    uint32_t bytes = ae > cs ? (uint32_t)((ae - cs) * 2) : 0u;
    for (uint64_t i = umax64(cs, E8); i < ce; ++i) dst[i - cs] = a.bb[i];  // < 8 tail events of the trace
    mbar_arrive_expect_tx(&m.mbar[slot], bytes);
    if (bytes) bulk_g2s(dst, a.bb + cs, bytes, &m.mbar[slot]);
    ++p_c;
  };
  if (tid == 0) {
    p_load();
    for (int s = 0; s < NST; ++s) p_issue((uint32_t)s);
  }

  uint32_t q = 0;  // chunks consumed by this CTA
  uint32_t* col = m.hist + tid;
  for (uint64_t t = blockIdx.x; t < a.n_tiles; t += gridDim.x) {
    const uint64_t w0 = t * TPB, w1 = umin64(a.W, w0 + TPB);
    const uint64_t w = w0 + tid;
    const bool valid = w < w1;
    uint64_t s = 0, e = 0;
    if (valid) { s = a.weo[w]; e = a.weo[w + 1]; }
    const uint64_t ts = a.weo[w0], te = a.weo[w1];
    const uint64_t A = ts & ~7ull;
    const uint32_t nch = te > A ? (uint32_t)ceil_div(te - A, CH) : 0u;
    uint32_t raw = 0, orr = 0;
    for (uint32_t c = 0; c < nch; ++c, ++q) {
      const uint32_t slot = q % NST;
      const uint64_t cs = A + (uint64_t)c * CH, ce = umin64(cs + CH, te);
      mbar_wait(&m.mbar[slot], (q / NST) & 1u);
      const uint16_t* sb = m.stage + (size_t)slot * CH;
      uint64_t lo = umax64(s, cs), hi = umin64(e, ce);
      if (lo < hi) {
        uint32_t i = (uint32_t)(lo - cs), end = (uint32_t)(hi - cs);
        auto acc1 = [&](uint32_t b) {
          raw |= b;
          uint32_t tv = tblp[b & bmask];
          if (CHECK_MARK) orr |= tv;
          uint32_t* cell = (uint32_t*)((uint8_t*)col + (tv & 0x3C00u));
          *cell += tv >> 14;
        };
        for (; i < end && (i & 7u); ++i) acc1(sb[i]);
        for (; i + 8 <= end; i += 8) {
          uint4 v = *(const uint4*)(sb + i);
          raw |= v.x | v.y | v.z | v.w;
          uint32_t ws[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
          for (int h = 0; h < 4; ++h) {
            uint32_t t0 = tblp[ws[h] & bmask];
            uint32_t t1 = tblp[(ws[h] >> 16) & bmask];
            if (CHECK_MARK) orr |= t0 | t1;
            uint32_t* c0 = (uint32_t*)((uint8_t*)col + (t0 & 0x3C00u));
            *c0 += t0 >> 14;
            uint32_t* c1 = (uint32_t*)((uint8_t*)col + (t1 & 0x3C00u));
            *c1 += t1 >> 14;
          }
        }
        for (; i < end; ++i) acc1(sb[i]);
      }
      __syncthreads();  // everyone is done with this slot
      if (tid == 0) p_issue(slot);
    }
    // ---- finalise the tile ----
    if (tid == 0) m.misc[0] = kernel_of(a.kwo, a.K, w0);
    uint32_t p[16];
    uint64_t I = 0;
#pragma unroll
    for (int j = 0; j < 16; ++j) { p[j] = col[j * TPB]; I += p[j]; }
    if (valid) {
      if (e < s) latch(a.err, PHOTON_ERANGE, (int64_t)w);
      uint32_t hi_ids = (raw | (raw >> 16)) & 0xFFFFu;
      if ((hi_ids & ~bmask) != 0u || (CHECK_MARK && (orr & 1u))) report_bad_event(a, s, e);
      if (e > s && (uint64_t)(e - s) * max_len >= kInstsLimit) {
        // bins may have wrapped: recompute the exact total (rare, long warps only)
        uint64_t exact = 0;
        for (uint64_t i = s; i < e; ++i) exact += a.tbl[a.bb[i] & bmask] >> 14;
        I = exact;
      }
      if (I >= kInstsLimit) latch(a.err, PHOTON_ERANGE, (int64_t)w);
      if (a.warp_bbv16) {
        uint4* dst = (uint4*)(a.warp_bbv16 + w * 16);
        dst[0] = make_uint4(p[0], p[1], p[2], p[3]);
        dst[1] = make_uint4(p[4], p[5], p[6], p[7]);
        dst[2] = make_uint4(p[8], p[9], p[10], p[11]);
        dst[3] = make_uint4(p[12], p[13], p[14], p[15]);
      }
      if (a.warp_insts) a.warp_insts[w] = I;
    }
    if (a.fused) {
      __syncthreads();
      uint32_t k = m.misc[0];
      if (valid)
        while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
      m.kid[tid] = k;  // kernel of each thread's warp, read by tile_group for owners' keys
      __syncthreads();
      tile_group(a, m, w0, valid, k, p);
    }
#pragma unroll
    for (int j = 0; j < 16; ++j) col[j * TPB] = 0u;
  }
}

// K2a over materialised BBVs (the unfused API path): one CTA per tile, keys loaded from warp_bbv16.
__global__ void __launch_bounds__(TPB) k_group_from_bbv(BbvArgs a, const uint32_t* __restrict__ bbv) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  Smem m = carve(smem_raw);
  const int tid = threadIdx.x;
  const uint64_t w0 = (uint64_t)blockIdx.x * TPB, w1 = umin64(a.W, w0 + TPB), w = w0 + tid;
  const bool valid = w < w1;
  for (int i = tid; i < LSLOTS; i += TPB) { m.lhash[i] = 0ull; m.lcount[i] = 0u; m.lgslot[i] = UINT32_MAX; }
  uint32_t p[16];
  if (valid) {
    const uint4* src = (const uint4*)(bbv + w * 16);
#pragma unroll
    for (int v = 0; v < 4; ++v) {
      uint4 x = src[v];
      p[4 * v] = x.x; p[4 * v + 1] = x.y; p[4 * v + 2] = x.z; p[4 * v + 3] = x.w;
    }
  } else {
#pragma unroll
    for (int j = 0; j < 16; ++j) p[j] = 0u;
  }
#pragma unroll
  for (int j = 0; j < 16; ++j) m.hist[j * TPB + tid] = p[j];
  if (tid == 0) m.misc[0] = kernel_of(a.kwo, a.K, w0);
  __syncthreads();
  uint32_t k = m.misc[0];
  if (valid)
    while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
  m.kid[tid] = k;
  __syncthreads();
  tile_group(a, m, w0, valid, k, p);
}

// ---- per-BB table and input validation -----------------------------------------------------------------
__global__ void k_table_prep(const uint32_t* __restrict__ bb_len, const uint8_t* __restrict__ bb_bin, uint32_t B,
                             uint32_t P2, uint32_t* __restrict__ tbl, uint32_t* max_len, DevErr* err) {
  uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= P2) return;
  if (b >= B) { tbl[b] = 1u; return; }  // marker: id in [B, P2) is out of range
  uint32_t len = bb_len[b];
  uint32_t bin = bb_bin ? bb_bin[b] : (b & 15u);
  if (len == 0 || len > kMaxLen || bin > 15) {
    latch(err, PHOTON_EINVAL, (int64_t)b);
    len = 0;
    bin = 0;
  }
  tbl[b] = (len << 14) | (bin << 10);
  atomicMax(max_len, len);
}

__global__ void k_validate_offsets(const uint64_t* __restrict__ kwo, uint32_t K, const uint64_t* __restrict__ weo,
                                   uint64_t W, uint64_t E, DevErr* err) {
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i == 0) {
    if (kwo[0] != 0 || kwo[K] != W) latch(err, PHOTON_ERANGE, 0);
    if (weo[0] != 0 || weo[W] != E) latch(err, PHOTON_ERANGE, 0);
  }
  if (i < K && kwo[i + 1] < kwo[i]) latch(err, PHOTON_ERANGE, (int64_t)i);
}

// ---- optional BB distribution kernel_bb_insts[k][b] (L208-210) ------------------------------------------------
// One CTA per (kernel, event chunk); shared-memory counters for B <= 8192 else global atomics.
constexpr int KBB_CHUNK = 16384;
__global__ void __launch_bounds__(256) k_kbb(const uint64_t* __restrict__ kwo, const uint64_t* __restrict__ weo,
                                             const uint16_t* __restrict__ bb, const uint32_t* __restrict__ tbl,
                                             uint32_t K, uint32_t B, uint32_t P2, uint64_t* __restrict__ kbb,
                                             uint64_t chunks_total, const uint64_t* __restrict__ kchunk_off) {
  extern __shared__ __align__(16) uint32_t cnt[];
  const uint64_t total = kchunk_off[K];
  for (uint64_t job = blockIdx.x; job < total && job < chunks_total; job += gridDim.x) {
    // job -> (kernel, chunk) via binary search over per-kernel chunk prefix
    uint32_t lo = 0, hi = K - 1;
    while (lo < hi) {
      uint32_t mid = (lo + hi + 1) >> 1;
      if (kchunk_off[mid] <= job) lo = mid; else hi = mid - 1;
    }
    uint32_t k = lo;
    uint64_t c = job - kchunk_off[k];
    uint64_t es = weo[kwo[k]], ee = weo[kwo[k + 1]];
    uint64_t cs = es + c * KBB_CHUNK, ce = umin64(cs + KBB_CHUNK, ee);
    bool smem = B <= 8192;
    if (smem) {
      for (uint32_t i = threadIdx.x; i < B; i += blockDim.x) cnt[i] = 0u;
      __syncthreads();
      for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
        uint32_t b = bb[i];
        if (b < B) atomicAdd(&cnt[b], 1u);
      }
      __syncthreads();
      for (uint32_t b = threadIdx.x; b < B; b += blockDim.x)
        if (cnt[b]) atomicAdd((unsigned long long*)&kbb[(uint64_t)k * B + b],
                              (unsigned long long)cnt[b] * (tbl[b] >> 14));
      __syncthreads();
    } else {
      for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
        uint32_t b = bb[i];
        if (b < B) atomicAdd((unsigned long long*)&kbb[(uint64_t)k * B + b], (unsigned long long)(tbl[b] >> 14));
      }
    }
  }
}

__global__ void k_kchunks(const uint64_t* __restrict__ kwo, const uint64_t* __restrict__ weo, uint32_t K,
                          uint64_t* kchunk_off) {
  // single-thread prefix over K (K is small relative to events; launched <<<1,1>>>)
  uint64_t acc = 0;
  for (uint32_t k = 0; k < K; ++k) {
    kchunk_off[k] = acc;
    uint64_t es = weo[kwo[k]], ee = weo[kwo[k + 1]];
    acc += ee > es ? ceil_div(ee - es, KBB_CHUNK) : 0;
  }
  kchunk_off[K] = acc;
}

}  // namespace

size_t bbv_table_bytes(uint32_t B) { return (size_t)next_pow2_u32(B < 16 ? 16 : B) * 4 + 64; }

cudaError_t launch_table_prep(const TraceDev& t, uint32_t* tbl, uint32_t* max_len, DevErr* err, cudaStream_t s) {
  uint32_t P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  cudaMemsetAsync(max_len, 0, 4, s);
  note_launch(), k_table_prep<<<(P2 + 255) / 256, 256, 0, s>>>(t.bb_len, t.bb_bin, t.B, P2, tbl, max_len, err);
  return cudaGetLastError();
}

cudaError_t launch_validate_offsets(const TraceDev& t, DevErr* err, cudaStream_t s) {
  uint64_t n = t.K > 0 ? t.K : 1;
  note_launch(), k_validate_offsets<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(t.kwo, t.K, t.weo, t.W, t.E, err);
  return cudaGetLastError();
}

template <bool SMEM_TBL, bool CHECK_MARK>
static cudaError_t launch_bbv_t(const BbvArgs& a, size_t smem, int num_sms, cudaStream_t s) {
  auto fn = k_bbv<SMEM_TBL, CHECK_MARK>;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, TPB, smem);
  if (e != cudaSuccess) return e;
  if (per_sm < 1) per_sm = 1;
  uint64_t grid = (uint64_t)num_sms * per_sm;
  if (grid > a.n_tiles) grid = a.n_tiles;
  if (grid == 0) return cudaSuccess;
  note_launch(), fn<<<(unsigned)grid, TPB, smem, s>>>(a);
  return cudaGetLastError();
}

cudaError_t launch_bbv(const TraceDev& t, const uint32_t* tbl, const uint32_t* max_len, uint32_t* warp_bbv16,
                       uint64_t* warp_insts, const HashTable* ht, uint32_t* warp_slot, DevErr* err, int num_sms,
                       cudaStream_t s) {
  BbvArgs a{};
  a.kwo = t.kwo; a.weo = t.weo; a.bb = t.bb; a.tbl = tbl; a.max_len = max_len;
  a.K = t.K; a.B = t.B; a.P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  a.W = t.W; a.E = t.E;
  a.warp_bbv16 = warp_bbv16; a.warp_insts = warp_insts;
  if (ht) { a.ht = *ht; a.fused = 1; }
  a.warp_slot = warp_slot;
  a.err = err;
  a.n_tiles = ceil_div(t.W, TPB);
  if (a.n_tiles == 0) return cudaSuccess;
  bool smem_tbl = a.P2 <= SMEM_TBL_MAX;
  bool mark = a.P2 != t.B;
  size_t smem = bbv_smem_bytes(smem_tbl ? a.P2 : 0);
  if (smem_tbl) return mark ? launch_bbv_t<true, true>(a, smem, num_sms, s) : launch_bbv_t<true, false>(a, smem, num_sms, s);
  return mark ? launch_bbv_t<false, true>(a, smem, num_sms, s) : launch_bbv_t<false, false>(a, smem, num_sms, s);
}

cudaError_t launch_group_from_bbv(const TraceDev& t, const uint32_t* warp_bbv16, const HashTable& ht,
                                  uint32_t* warp_slot, DevErr* err, cudaStream_t s) {
  BbvArgs a{};
  a.kwo = t.kwo; a.K = t.K; a.W = t.W; a.ht = ht; a.fused = 1; a.warp_slot = warp_slot; a.err = err;
  uint64_t tiles = ceil_div(t.W, TPB);
  if (tiles == 0) return cudaSuccess;
  size_t smem = bbv_smem_bytes(0);
  cudaError_t e = cudaFuncSetAttribute(k_group_from_bbv, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  note_launch(), k_group_from_bbv<<<(unsigned)tiles, TPB, smem, s>>>(a, warp_bbv16);
  return cudaGetLastError();
}

cudaError_t launch_kernel_bb_insts(const TraceDev& t, const uint32_t* tbl, uint64_t* kbb, DevErr* err, int num_sms,
                                   cudaStream_t s) {
  (void)err;
  cudaMemsetAsync(kbb, 0, sizeof(uint64_t) * (size_t)t.K * t.B, s);
  // chunk prefix lives right after the table in the caller's table area? use a small separate allocation in tbl
  // area: the caller reserves K+1 u64 after the table (see abi.cu).
  uint32_t P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  uint64_t* kchunk_off = (uint64_t*)(((uintptr_t)(tbl + P2) + 255) & ~(uintptr_t)255);
  note_launch(), k_kchunks<<<1, 1, 0, s>>>(t.kwo, t.weo, t.K, kchunk_off);
  // upper bound on jobs: E/KBB_CHUNK + K
  uint64_t jobs_ub = ceil_div(t.E, KBB_CHUNK) + t.K;
  uint64_t grid = jobs_ub < (uint64_t)num_sms * 4 ? jobs_ub : (uint64_t)num_sms * 4;
  if (grid == 0) grid = 1;
  size_t smem = t.B <= 8192 ? (size_t)t.B * 4 : 0;
  cudaFuncSetAttribute(k_kbb, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(smem < 1024 ? 1024 : smem));
  // exact job count is on the device (kchunk_off[K]); CTAs loop over [0, chunks_total) with chunks_total read
  // from the upper bound and a guard in the kernel via kchunk_off[K].
  note_launch(), k_kbb<<<(unsigned)grid, 256, smem < 1024 ? 1024 : smem, s>>>(t.kwo, t.weo, t.bb, tbl, t.K, t.B, P2, kbb, jobs_ub,
                                                              kchunk_off);
  return cudaGetLastError();
}

}  // namespace photon
