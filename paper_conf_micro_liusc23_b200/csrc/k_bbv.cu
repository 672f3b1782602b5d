// k_bbv.cu — A1 (per-warp BBV projected to 16 bins) fused with A2's de-duplication step (K1 + K2a).
//
// PAPER.md: L161 (a BBV lists the basic blocks a warp executed, identified by start PC), L154 (same instruction
// sequence => same BBV => same warp type), L178 ("project these BBVs into fixed-size BBVs (We use 16) to improve
// online clustering performance ... we can easily cluster the warps if they have the same BBV").  Readings [P-1]
// (entry = executions x length) and [P-2] (sum-preserving fold into 16 bins).
//
// Design.  Persistent CTAs of 256 threads; a "tile" is 256 consecutive analysed warps, tile t is
// handled by CTA t mod grid.  The tile's events, widened to whole 16-byte words, are streamed through shared
// memory in chunks of up to 24K events (48 KB), each staged with cp.async.bulk (TMA copy engine, mbarrier
// completion) while the previous chunk is combined / the previous tile finalised.  Each chunk's words are split
// into 256 equal runs, one per thread (merge-path balance: independent of how long the warps are), so every lane
// executes the same word loop: 8 events per 128-bit LDS, two events per dependent step (both bins read before
// either is written; equal cells merged), one packed (len, bin-offset) word per event from a shared-memory BB
// table.  A word may contain one warp boundary (events before it go to the current column, after it to the next
// warp's); words with more boundaries (warps shorter than 8 events) take a per-event path.  A thread adds events
// of a warp that STARTS in its run straight into that warp's result column R[w] (its only writer); events of the
// warp already open at its run start go to its private HEAD column.  After a barrier, warp w's owner adds the HEAD
// columns of the threads its events spilled into.  Events of neighbouring tiles in the first / last word belong to
// virtual warps whose column is a scratch column.  Finalise: each thread holds warp w's 16-bin key in R[w]; warps
// are de-duplicated with __match_any_sync on a 64-bit hash (exact key check), then across the CTA in a shared-
// memory table; the tile's distinct (kernel, key, count, first warp) entries go to a per-tile slot area and each
// warp gets its local entry id (u16).  No global atomics on the streaming path: k_entries_insert (k_types.cu)
// inserts the entries into the global type table.
#include "internal.h"

namespace photon {

namespace {

constexpr int TPB = 256;            // threads per CTA = warps per tile
constexpr int COLS = 288;           // column stride (u32) of the 16 x COLS arrays: a multiple of 32 banks, so a
                                    // cell's bank is its column's (lanes on distinct columns never conflict)
constexpr int COLB = COLS * 4;      // bin stride in bytes; table entry = len << LSH | bin * COLB
constexpr int LSH = 15;             // length field shift (lengths < 2^17)
constexpr uint32_t AMASK = 0x7FFCu; // cell byte offset bits of a table entry
constexpr int DUMMY = 256;          // scratch column (events of neighbouring tiles)
constexpr int CAPE = 24576;         // staging chunk (events, multiple of 8), 48 KB
constexpr int SMEM_TBL_MAX = 4096;  // BB table entries kept in shared memory
constexpr int LSLOTS = 256;         // CTA-local de-dup slots
static_assert(15 * COLB < (1 << LSH) && (COLS % 32) == 0, "bin offset must fit below the length field");

struct BbvArgs {
  const uint64_t* kwo;
  const uint64_t* weo;
  const uint16_t* bb;
  const uint32_t* tbl;
  const uint32_t* max_len;
  const uint32_t* tile_k0;  // [n_tiles] kernel of each tile's first warp
  uint32_t K, B, P2;
  uint64_t W, E;
  uint32_t* warp_bbv16;
  uint64_t* warp_insts;
  TileEntries te;           // fused grouping outputs (te.tile_n == nullptr => not fused)
  DevErr* err;
  uint64_t n_tiles;
};

constexpr size_t kColBytes = (size_t)16 * COLB;
constexpr size_t kStageBytes = (size_t)CAPE * 2;
constexpr size_t kOffsBytes = (TPB + 4) * 8;
constexpr size_t kLocalBytes = LSLOTS * (8 + 4 + 4 + 4 + 4);
constexpr size_t kMiscBytes = 256;
constexpr size_t kKidBytes = TPB * 4 + (TPB + 8) * 2;

__host__ __device__ constexpr size_t bbv_smem_bytes(uint32_t tbl_entries) {
  return 2 * kColBytes + kStageBytes + kOffsBytes + 16 + kLocalBytes + kMiscBytes + kKidBytes +
         (size_t)tbl_entries * 4;
}

struct Smem {
  uint32_t* hist;    // R: [16][COLS] result column of each warp of the tile (the key at finalise) + DUMMY
  uint32_t* head;    // A: [16][COLS] HEAD partial of each thread
  uint16_t* stage;   // [CAPE]
  uint64_t* offs;    // [TPB+3] o[0] = aligned tile start, o[1+v] = start of warp v, o[nw+1] = end, o[nw+2] = Z
  uint64_t* mbar;    // [1]
  uint64_t* lhash;   // [LSLOTS]
  uint32_t* lowner;  // [LSLOTS] thread whose column holds the key
  uint32_t* lcount;  // [LSLOTS]
  uint32_t* lminw;   // [LSLOTS] lowest thread (warp) of the entry
  uint32_t* lent;    // [LSLOTS] dense local entry id
  uint32_t* misc;    // [64]: 0 n_entries; [2..3] u64 overflow base
  uint32_t* kid;     // [TPB] kernel of each thread's warp
  uint16_t* nxt;     // [TPB+8] next non-empty warp after each (virtual) warp of the tile
  uint32_t* tbl;     // [P2]
};

__device__ __forceinline__ Smem carve(uint8_t* s) {
  Smem m;
  m.hist = (uint32_t*)s;
  m.head = (uint32_t*)(s + kColBytes);
  m.stage = (uint16_t*)(s + 2 * kColBytes);
  m.offs = (uint64_t*)(s + 2 * kColBytes + kStageBytes);
  m.mbar = (uint64_t*)(s + 2 * kColBytes + kStageBytes + kOffsBytes);
  m.lhash = m.mbar + 2;
  m.lowner = (uint32_t*)(m.lhash + LSLOTS);
  m.lcount = m.lowner + LSLOTS;
  m.lminw = m.lcount + LSLOTS;
  m.lent = m.lminw + LSLOTS;
  m.misc = m.lent + LSLOTS;
  m.kid = m.misc + kMiscBytes / 4;
  m.nxt = (uint16_t*)(m.kid + TPB);
  m.tbl = (uint32_t*)(m.nxt + TPB + 8);
  return m;
}

// ---- per-event accumulation --------------------------------------------------------------------------------
// Table entry t: len << LSH | bin * COLB (bit 0 = id in [B, P2)); cell address = column + (t & AMASK).
struct Acc {
  const uint32_t* tbl;
  uint32_t bmask;
  uint32_t raw, orr;
  __device__ __forceinline__ void one(uint32_t* col, uint32_t b) {
    uint32_t t = tbl[b & bmask];
    orr |= t;
    *(uint32_t*)((uint8_t*)col + (t & AMASK)) += t >> LSH;
  }
  // two events whose table entries are already loaded; `same` = both go to the same column
  __device__ __forceinline__ void pair(uint32_t t0, uint32_t t1, uint32_t* c0, uint32_t* c1, bool same) {
    const uint32_t a0 = t0 & AMASK, a1 = t1 & AMASK;
    uint32_t* p0 = (uint32_t*)((uint8_t*)c0 + a0);
    uint32_t* p1 = (uint32_t*)((uint8_t*)c1 + a1);
    const uint32_t l1 = t1 >> LSH;
    uint32_t h0 = *p0, h1 = *p1;
    *p1 = h1 + l1;
    *p0 = h0 + (t0 >> LSH) + ((same && a0 == a1) ? l1 : 0u);
  }
  // one 16-byte word: events j < bo into ca, j >= bo into cb.  All 8 table entries are loaded before any
  // histogram cell is written (the compiler cannot hoist them past the stores itself), so the word costs four
  // short load->add->store chains instead of four chains that each also wait for their table reads.
  __device__ __forceinline__ void word(uint4 v, uint32_t bo, uint32_t* ca, uint32_t* cb) {
    raw |= v.x | v.y | v.z | v.w;
    const uint32_t t0 = tbl[v.x & bmask], t1 = tbl[(v.x >> 16) & bmask];
    const uint32_t t2 = tbl[v.y & bmask], t3 = tbl[(v.y >> 16) & bmask];
    const uint32_t t4 = tbl[v.z & bmask], t5 = tbl[(v.z >> 16) & bmask];
    const uint32_t t6 = tbl[v.w & bmask], t7 = tbl[(v.w >> 16) & bmask];
    orr |= (t0 | t1 | t2 | t3) | (t4 | t5 | t6 | t7);
    pair(t0, t1, bo > 0 ? ca : cb, bo > 1 ? ca : cb, bo != 1);
    pair(t2, t3, bo > 2 ? ca : cb, bo > 3 ? ca : cb, bo != 3);
    pair(t4, t5, bo > 4 ? ca : cb, bo > 5 ? ca : cb, bo != 5);
    pair(t6, t7, bo > 6 ? ca : cb, bo > 7 ? ca : cb, bo != 7);
  }
};

// Slow path (bad input only): first event of [s, e) whose id is >= B.
__device__ void report_bad_event(const BbvArgs& a, uint64_t s, uint64_t e) {
  for (uint64_t i = s; i < e; ++i)
    if (a.bb[i] >= a.B) { latch(a.err, PHOTON_ERANGE, (int64_t)i); return; }
}

// ---- tile finalisation: CTA de-duplication and per-tile entries -----------------------------------------------
// Keys are in the result columns (hist[j*COLS + tid]); kid[] holds each thread's kernel.
__device__ void tile_group(const BbvArgs& a, const Smem& m, uint64_t t, uint64_t w0, bool valid, uint32_t k,
                           const uint32_t* p) {
  const int tid = threadIdx.x, lane = tid & 31;
  const uint64_t h = valid ? hash_key(k, p) : 0;
  const unsigned active = __ballot_sync(0xffffffffu, valid);
  const unsigned peers = __match_any_sync(0xffffffffu, (unsigned long long)h);
  const int leader = __ffs(peers) - 1;
  bool eq = (__shfl_sync(0xffffffffu, k, leader) == k);
#pragma unroll
  for (int j = 0; j < 16; ++j) eq = eq && (__shfl_sync(0xffffffffu, p[j], leader) == p[j]);
  const unsigned eqm = __ballot_sync(0xffffffffu, eq);
  const bool is_leader = valid && (lane == leader || !eq);
  const uint32_t cnt = (lane == leader) ? (uint32_t)__popc(peers & eqm & active) : 1u;
  // claim a local slot by hash; the first claimer owns it and takes a dense entry id
  int slot = -1;
  bool pending = false;
  if (is_leader) {
    uint32_t i = (uint32_t)(h & (LSLOTS - 1));
    for (int probe = 0; probe < LSLOTS; ++probe) {
      unsigned long long cur = atomicCAS((unsigned long long*)&m.lhash[i], 0ull, (unsigned long long)h);
      if (cur == 0ull) {
        m.lowner[i] = (uint32_t)tid;
        m.lent[i] = atomicAdd(&m.misc[0], 1u);
        slot = (int)i;
        break;
      }
      if (cur == h) { slot = (int)i; pending = true; break; }
      i = (i + 1) & (LSLOTS - 1);
    }
  }
  __syncthreads();
  // verify pending claims (equal hash, maybe different key); a mismatch gets its own entry (bypass)
  uint32_t my_ent = UINT32_MAX;
  if (slot >= 0) {
    bool own = true;
    if (pending) {
      uint32_t o = m.lowner[slot];
      bool same = (m.kid[o] == k);
#pragma unroll
      for (int j = 0; j < 16; ++j) same = same && (m.hist[j * COLS + o] == p[j]);
      own = same;
    }
    if (own) {
      atomicAdd(&m.lcount[slot], cnt);
      atomicMin(&m.lminw[slot], (uint32_t)tid);  // leaders are the lowest thread of their warp group
      my_ent = m.lent[slot];
    } else {
      my_ent = atomicAdd(&m.misc[0], 1u) | 0x80000000u;
    }
  }
  __syncthreads();
  const uint32_t n_ent = m.misc[0];
  const uint32_t M = a.te.per_tile;
  uint64_t* ovf_base = (uint64_t*)(m.misc + 2);
  if (n_ent > M) {  // rare: more distinct keys than the tile's fixed entry slots
    if (tid == 0) {
      unsigned long long pos = atomicAdd((unsigned long long*)a.te.ovf_count, (unsigned long long)(n_ent - M));
      if (pos + (n_ent - M) > a.te.ovf_cap) latch(a.err, PHOTON_ECAPACITY, (int64_t)pos);
      a.te.tile_ovf[t] = pos;
      *ovf_base = pos;
    }
    __syncthreads();
  }
  if (tid == 0) a.te.tile_n[t] = n_ent;
  auto put = [&](uint32_t e, uint32_t kern, const uint32_t* key, uint32_t count, uint32_t minw, uint64_t hh) {
    TileEntry* dst;
    if (e < M) {
      dst = a.te.ent + t * M + e;
    } else {
      uint64_t pos = *ovf_base + (e - M);
      if (pos >= a.te.ovf_cap) return;
      dst = a.te.ovf + pos;
    }
    dst->hash = hh;
    dst->first = w0 + minw;
    dst->kernel = kern;
    dst->count = count;
    uint4* kd = (uint4*)dst->key;
    kd[0] = make_uint4(key[0], key[1], key[2], key[3]);
    kd[1] = make_uint4(key[4], key[5], key[6], key[7]);
    kd[2] = make_uint4(key[8], key[9], key[10], key[11]);
    kd[3] = make_uint4(key[12], key[13], key[14], key[15]);
  };
  for (int i = tid; i < LSLOTS; i += TPB) {
    uint64_t hh = m.lhash[i];
    if (hh != 0ull) {
      uint32_t o = m.lowner[i];
      uint32_t key[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) key[j] = m.hist[j * COLS + o];
      put(m.lent[i], m.kid[o], key, m.lcount[i], m.lminw[i], hh);
    }
  }
  if (my_ent != UINT32_MAX && (my_ent & 0x80000000u)) put(my_ent & 0x7FFFFFFFu, k, p, cnt, (uint32_t)tid, h);
  // members of a warp group take the leader's entry
  const uint32_t from_leader = __shfl_sync(0xffffffffu, my_ent, leader);
  if (valid) {
    uint32_t e = (lane == leader || !eq) ? my_ent : from_leader;
    a.te.lid[w0 + tid] = (uint16_t)(e & 0xFFFFu);
  }
  __syncthreads();
  for (int i = tid; i < LSLOTS; i += TPB) {
    m.lhash[i] = 0ull;
    m.lcount[i] = 0u;
    m.lminw[i] = UINT32_MAX;
  }
  if (tid == 0) m.misc[0] = 0u;
}

// thread 0: stage the word-aligned events [cs, ce) into shared memory (bulk part on the TMA copy engine; events
// at or past E8 with plain loads, positions past E zero-filled), completing on the mbarrier
__device__ __forceinline__ void stage_chunk(const BbvArgs& a, const Smem& m, uint64_t cs, uint64_t ce, uint64_t E8) {
  uint64_t ae = umin64(ce, E8);
  uint32_t bytes = ae > cs ? (uint32_t)((ae - cs) * 2) : 0u;
  for (uint64_t i = umax64(cs, E8); i < ce; ++i) m.stage[i - cs] = i < a.E ? a.bb[i] : (uint16_t)0;
  mbar_arrive_expect_tx(m.mbar, bytes);
  for (uint32_t off = 0; off < bytes; off += 16384) {
    uint32_t n = bytes - off < 16384 ? bytes - off : 16384;
    bulk_g2s((uint8_t*)m.stage + off, (const uint8_t*)(a.bb + cs) + off, n, m.mbar);
  }
}

// Chunk sequence of the CTA: tiles blockIdx.x, +gridDim.x, ...; tile events widened to words [A, Z), split into
// CAPE chunks; tiles without events have no chunk.
struct Cursor {
  uint64_t t, A, Z, c, nch;
  bool valid;
};
__device__ __forceinline__ void cursor_tile(const BbvArgs& a, Cursor& u, uint64_t t) {
  u.t = t;
  u.valid = t < a.n_tiles;
  u.c = 0;
  u.nch = 0;
  u.A = u.Z = 0;
  if (!u.valid) return;
  uint64_t w0 = t * TPB, w1 = umin64(a.W, w0 + TPB);
  uint64_t te = umin64(a.weo[w1], a.E), ts = umin64(a.weo[w0], te);  // clamped: bad offsets stay memory-safe
  if (te <= ts) return;
  u.A = ts & ~7ull;
  u.Z = (te + 7) & ~7ull;
  u.nch = ceil_div(u.Z - u.A, CAPE);
}

template <bool SMEM_TBL, bool CHECK_MARK>
__global__ void __launch_bounds__(TPB, 2) k_bbv(BbvArgs a) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  Smem m = carve(smem_raw);
  const int tid = threadIdx.x;
  const uint32_t bmask = a.P2 - 1;
  const bool fused = a.te.tile_n != nullptr;

  if (SMEM_TBL)
    for (uint32_t i = tid; i < a.P2; i += TPB) m.tbl[i] = a.tbl[i];
  for (int i = tid; i < 16 * COLS; i += TPB) { m.hist[i] = 0u; m.head[i] = 0u; }
  for (int i = tid; i < LSLOTS; i += TPB) { m.lhash[i] = 0ull; m.lcount[i] = 0u; m.lminw[i] = UINT32_MAX; }
  if (tid < 64) m.misc[tid] = 0u;
  if (tid == 0) {
    mbar_init(m.mbar, 1);
    fence_mbar_init();
  }
  const uint32_t max_len = *a.max_len;
  const uint64_t E8 = a.E & ~7ull;

  // producer cursor (thread 0): one chunk ahead of the consumers
  Cursor pc;
  if (tid == 0) {
    cursor_tile(a, pc, blockIdx.x);
    while (pc.valid && pc.nch == 0) cursor_tile(a, pc, pc.t + gridDim.x);
    if (pc.valid) stage_chunk(a, m, pc.A, umin64(pc.A + CAPE, pc.Z), E8);
  }
  uint32_t phase = 0;

  Acc acc;
  acc.tbl = SMEM_TBL ? m.tbl : a.tbl;
  acc.bmask = bmask;

  uint64_t t = blockIdx.x;
  uint64_t my_off = 0, last_off = 0;  // weo[w0 + tid] (clamped) and weo[w1] of the current tile
  if (t < a.n_tiles) {
    uint64_t w0 = t * TPB, nw = umin64(a.W, w0 + TPB) - w0;
    my_off = a.weo[w0 + umin64((uint64_t)tid, nw)];
    if (tid == 0) last_off = a.weo[w0 + nw];
  }
  __syncthreads();

  while (t < a.n_tiles) {
    const uint64_t w0 = t * TPB, w1 = umin64(a.W, w0 + TPB);
    const uint32_t nw = (uint32_t)(w1 - w0);
    const uint64_t w = w0 + tid;
    const bool valid = w < w1;
    // o[1 + v] = start of warp v, o[nw + 1] = tile end; o[0] / o[nw + 2] = word-aligned bounds (virtual warps)
    if ((uint32_t)tid <= nw) m.offs[1 + tid] = my_off;
    if (tid == 0) {
      m.offs[1 + nw] = last_off;
    }
    const uint64_t tn = t + gridDim.x;
    uint64_t nx_off = 0, nx_last = 0;
    if (tn < a.n_tiles) {
      uint64_t n0 = tn * TPB, nn = umin64(a.W, n0 + TPB) - n0;
      nx_off = a.weo[n0 + umin64((uint64_t)tid, nn)];
      if (tid == 0) nx_last = a.weo[n0 + nn];
    }
    __syncthreads();
    // same clamping as cursor_tile (monotone offsets are validated per warp below: e < s latches ERANGE)
    const uint64_t te = umin64(m.offs[1 + nw], a.E), ts = umin64(m.offs[1], te);
    const uint64_t At = ts & ~7ull, Zt = (te + 7) & ~7ull;
    if (tid == 0) {
      m.offs[0] = At;
      m.offs[nw + 2] = Zt;
    }
    const uint64_t s = valid ? m.offs[1 + tid] : te, e = valid ? m.offs[2 + tid] : te;
    const uint64_t nch = te > ts ? ceil_div(Zt - At, CAPE) : 0;
    const uint32_t last = nw + 1;  // index of the virtual tail warp
    {
      // nxt[s'] = next non-empty (virtual) warp after s' (last = sentinel); o[0] / o[nw+2] taken from registers
      auto O = [&](uint32_t i) -> uint64_t { return i == 0 ? At : (i == nw + 2 ? Zt : m.offs[i]); };
      for (uint32_t sp = tid; sp <= last; sp += TPB) {
        uint32_t x = sp + 1;
        while (x < last && O(x + 1) == O(x)) ++x;
        m.nxt[sp] = (uint16_t)(x < last ? x : last);
      }
    }
    __syncthreads();
    uint32_t* const headcol = m.head + tid;
    uint32_t* const dummy = m.hist + DUMMY;
    auto colof = [&](uint32_t sp) -> uint32_t* { return (sp == 0 || sp == last) ? dummy : m.hist + (sp - 1); };
    acc.raw = 0;
    acc.orr = 0;
    for (uint64_t c = 0; c < nch; ++c) {
      const uint64_t cs = At + c * CAPE, ce = umin64(cs + CAPE, Zt);
      const uint64_t nwc = (ce - cs) >> 3;
      mbar_wait(m.mbar, phase);
      phase ^= 1u;
      // my run of words [r0, r1) of the chunk
      const uint64_t r0 = cs + 8 * (((uint64_t)tid * nwc) / TPB), r1 = cs + 8 * (((uint64_t)(tid + 1) * nwc) / TPB);
      if (r0 < r1) {
        // warp (with virtual ones) containing r0: last s' with o[s'] <= r0.  Start from the proportional guess
        // and narrow a +-8 window around it when it brackets r0 (it usually does), else search everything.
        uint32_t lo = 0, hi = last;
        {
          const float fr = (float)(r0 - At) / (float)(Zt - At);
          int g = (int)(fr * (float)(nw + 2));
          int glo = g - 8 < 0 ? 0 : g - 8, ghi = g + 8 > (int)last ? (int)last : g + 8;
          if (m.offs[glo] <= r0 && m.offs[ghi + 1] > r0) { lo = (uint32_t)glo; hi = (uint32_t)ghi; }
        }
        while (lo < hi) {
          uint32_t mid = (lo + hi + 1) >> 1;
          if (m.offs[mid] <= r0) lo = mid; else hi = mid - 1;
        }
        // all positions below are u32 offsets from the chunk start, clamped to [0, LIM]
        const uint32_t LIM = (uint32_t)(ce - cs) + 8u;
        auto rel = [&](uint64_t x) -> uint32_t {
          return x <= cs ? 0u : (x - cs >= LIM ? LIM : (uint32_t)(x - cs));
        };
        uint32_t sg = lo;
        uint32_t* col = (m.offs[sg] < r0) ? headcol : colof(sg);  // warp open at my run start -> HEAD
        uint32_t nb = rel(m.offs[sg + 1]);
        uint32_t sgn = m.nxt[sg];
        uint32_t* coln = colof(sgn);
        uint32_t nb2 = sgn != sg ? rel(m.offs[sgn + 1]) : LIM + 8u;
        const uint4* sb4 = (const uint4*)m.stage;
        const uint32_t q0 = (uint32_t)(r0 - cs), qe = (uint32_t)(r1 - cs);
        uint4 vnext = sb4[q0 >> 3];
        for (uint32_t q = q0; q < qe; q += 8) {
          const uint4 v = vnext;
          if (q + 8 < qe) vnext = sb4[(q + 8) >> 3];  // next word read before this word's stores
          if (nb2 < q + 8) {
            // several warp boundaries inside this word (warps shorter than 8 events): event by event
            acc.raw |= v.x | v.y | v.z | v.w;
            const uint32_t wv[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              while (q + j >= nb) {
                sg = m.nxt[sg];
                col = colof(sg);
                nb = rel(m.offs[sg + 1]);
              }
              acc.one(col, (j & 1) ? (wv[j >> 1] >> 16) : (wv[j >> 1] & 0xFFFFu));
            }
            while (q + 8 >= nb && sg < last) {  // move to the warp open after this word
              sg = m.nxt[sg];
              col = colof(sg);
              nb = rel(m.offs[sg + 1]);
            }
            sgn = m.nxt[sg];
            coln = colof(sgn);
            nb2 = sgn != sg ? rel(m.offs[sgn + 1]) : LIM + 8u;
            continue;
          }
          const uint32_t bo = nb < q + 8 ? nb - q : 8u;  // first event of the next warp
          acc.word(v, bo, col, coln);
          // advance past a crossed boundary without branching (lanes cross at different words; a divergent
          // update would serialise): when bo == 8 the same values are recomputed
          const bool cross = bo < 8u;
          sg = cross ? sgn : sg;
          col = cross ? coln : col;
          nb = cross ? nb2 : nb;
          sgn = m.nxt[sg];
          coln = colof(sgn);
          nb2 = sgn != sg ? rel(m.offs[sgn + 1]) : LIM + 8u;
        }
      }
      __syncthreads();  // accumulation done; the stage is free
      if (tid == 0) {   // stage the next chunk (this tile's next, or the next tile's first) during the combine
        ++pc.c;
        if (pc.c >= pc.nch) {
          do { cursor_tile(a, pc, pc.t + gridDim.x); } while (pc.valid && pc.nch == 0);
        }
        if (pc.valid) {
          uint64_t ncs = pc.A + pc.c * CAPE;
          stage_chunk(a, m, ncs, umin64(ncs + CAPE, pc.Z), E8);
        }
      }
      // combine: warp tid (if it has events in this chunk) adds the HEAD partials of the threads it spilled into
      if (valid && e > s && e > cs && s < ce) {
        const uint64_t lo_e = umax64(s, cs), hi_e = umin64(e, ce) - 1;
        const uint32_t ta = (uint32_t)((((lo_e - cs) >> 3) * TPB + TPB - 1) / nwc);
        const uint32_t tb = (uint32_t)((((hi_e - cs) >> 3) * TPB + TPB - 1) / nwc);
        const uint32_t from = ta + (s >= cs ? 1u : 0u);  // a warp starting in ta's run went straight into R
        if (from <= tb) {
          uint32_t sum[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) sum[j] = 0u;
          for (uint32_t u = from; u <= tb; ++u) {
#pragma unroll
            for (int j = 0; j < 16; ++j) sum[j] += m.head[j * COLS + u];
          }
#pragma unroll
          for (int j = 0; j < 16; ++j) m.hist[j * COLS + tid] += sum[j];
        }
      }
      __syncthreads();  // HEAD columns consumed
#pragma unroll
      for (int j = 0; j < 16; ++j) headcol[j * COLS] = 0u;
    }
    // ---- finalise the tile ----
    uint32_t p[16];
    uint64_t I = 0;
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      p[j] = m.hist[j * COLS + tid];
      I += p[j];
    }
    // bad ids anywhere in the tile (runs != warps): every warp re-scans its own events (bad input only)
    const uint32_t raw = acc.raw, orr = acc.orr;
    const int bad_here = ((((raw | (raw >> 16)) & 0xFFFFu) & ~bmask) != 0u || (CHECK_MARK && (orr & 1u))) ? 1 : 0;
    if (__syncthreads_or(bad_here) && valid) report_bad_event(a, umin64(s, a.E), umin64(e, a.E));
    uint32_t k = a.tile_k0 ? a.tile_k0[t] : 0u;
    if (valid) {
      if (e < s) latch(a.err, PHOTON_ERANGE, (int64_t)w);
      if (e > s && (uint64_t)(e - s) * max_len >= kInstsLimit) {
        // bins may have wrapped: recompute the exact total (rare, long warps only)
        uint64_t exact = 0;
        for (uint64_t i = s; i < umin64(e, a.E); ++i) exact += a.tbl[a.bb[i] & bmask] >> LSH;
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
      if (fused)
        while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
    }
    if (fused) {
      m.kid[tid] = k;
      __syncthreads();
      tile_group(a, m, t, w0, valid, k, p);
    } else {
      __syncthreads();
    }
#pragma unroll
    for (int j = 0; j < 16; ++j) m.hist[j * COLS + tid] = 0u;
    my_off = nx_off;
    last_off = nx_last;
    t = tn;
    __syncthreads();  // result columns cleared and offs free before the next tile
  }
}

// K2a over materialised BBVs (the unfused API path): one CTA per tile, keys loaded from warp_bbv16.
__global__ void __launch_bounds__(TPB) k_group_from_bbv(BbvArgs a, const uint32_t* __restrict__ bbv) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  Smem m = carve(smem_raw);
  const int tid = threadIdx.x;
  const uint64_t t = blockIdx.x;
  const uint64_t w0 = t * TPB, w1 = umin64(a.W, w0 + TPB), w = w0 + tid;
  const bool valid = w < w1;
  for (int i = tid; i < LSLOTS; i += TPB) { m.lhash[i] = 0ull; m.lcount[i] = 0u; m.lminw[i] = UINT32_MAX; }
  if (tid < 64) m.misc[tid] = 0u;
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
  for (int j = 0; j < 16; ++j) m.hist[j * COLS + tid] = p[j];
  uint32_t k = a.tile_k0[t];
  if (valid)
    while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
  m.kid[tid] = k;
  __syncthreads();
  tile_group(a, m, t, w0, valid, k, p);
}

// ---- per-BB table, tile kernels, input validation ----------------------------------------------------------
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
  tbl[b] = (len << LSH) | (bin * (uint32_t)COLB);
  atomicMax(max_len, len);
}

__global__ void k_tile_k0(const uint64_t* __restrict__ kwo, uint32_t K, uint64_t n_tiles, uint32_t* tile_k0) {
  uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (t >= n_tiles) return;
  uint64_t w = t * TPB;
  uint32_t lo = 0, hi = K - 1;  // last k with kwo[k] <= w
  while (lo < hi) {
    uint32_t mid = (lo + hi + 1) >> 1;
    if (kwo[mid] <= w) lo = mid; else hi = mid - 1;
  }
  tile_k0[t] = lo;
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
                                             uint32_t K, uint32_t B, uint64_t* __restrict__ kbb, uint64_t jobs_ub,
                                             const uint64_t* __restrict__ kchunk_off) {
  extern __shared__ __align__(16) uint32_t cnt[];
  const uint64_t total = kchunk_off[K];
  for (uint64_t job = blockIdx.x; job < total && job < jobs_ub; job += gridDim.x) {
    uint32_t lo = 0, hi = K - 1;
    while (lo < hi) {
      uint32_t mid = (lo + hi + 1) >> 1;
      if (kchunk_off[mid] <= job) lo = mid; else hi = mid - 1;
    }
    uint32_t k = lo;
    uint64_t c = job - kchunk_off[k];
    uint64_t es = weo[kwo[k]], ee = weo[kwo[k + 1]];
    uint64_t cs = es + c * KBB_CHUNK, ce = umin64(cs + KBB_CHUNK, ee);
    if (B <= 8192) {
      for (uint32_t i = threadIdx.x; i < B; i += blockDim.x) cnt[i] = 0u;
      __syncthreads();
      for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
        uint32_t b = bb[i];
        if (b < B) atomicAdd(&cnt[b], 1u);
      }
      __syncthreads();
      for (uint32_t b = threadIdx.x; b < B; b += blockDim.x)
        if (cnt[b])
          atomicAdd((unsigned long long*)&kbb[(uint64_t)k * B + b], (unsigned long long)cnt[b] * (tbl[b] >> LSH));
      __syncthreads();
    } else {
      for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
        uint32_t b = bb[i];
        if (b < B) atomicAdd((unsigned long long*)&kbb[(uint64_t)k * B + b], (unsigned long long)(tbl[b] >> LSH));
      }
    }
  }
}

// per-kernel chunk prefix (one CTA, block scan over K)
__global__ void __launch_bounds__(1024) k_kchunks(const uint64_t* __restrict__ kwo, const uint64_t* __restrict__ weo,
                                                  uint32_t K, uint64_t* kchunk_off) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint32_t base = 0; base < K; base += 1024) {
    uint32_t k = base + threadIdx.x;
    uint64_t v = 0;
    if (k < K) {
      uint64_t es = weo[kwo[k]], ee = weo[kwo[k + 1]];
      v = ee > es ? ceil_div(ee - es, KBB_CHUNK) : 0;
    }
    uint64_t x = v;
    for (int o = 1; o < 32; o <<= 1) {
      uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= o) x += y;
    }
    if (lane == 31) ws[wid] = x;
    __syncthreads();
    if (wid == 0) {
      uint64_t sacc = ws[lane];
      for (int o = 1; o < 32; o <<= 1) {
        uint64_t y = __shfl_up_sync(0xffffffffu, sacc, o);
        if (lane >= o) sacc += y;
      }
      ws[lane] = sacc;
    }
    __syncthreads();
    uint64_t ex = carry + (wid ? ws[wid - 1] : 0) + x - v;
    if (k < K) kchunk_off[k] = ex;
    __syncthreads();
    if (threadIdx.x == 1023) carry = ex + v;
    __syncthreads();
  }
  if (threadIdx.x == 0) kchunk_off[K] = carry;
}

}  // namespace

size_t bbv_table_bytes(uint32_t B) { return (size_t)next_pow2_u32(B < 16 ? 16 : B) * 4 + 64; }
uint64_t bbv_n_tiles(uint64_t W) { return ceil_div(W, TPB); }

cudaError_t launch_table_prep(const TraceDev& t, uint32_t* tbl, uint32_t* max_len, uint32_t* tile_k0, DevErr* err,
                              cudaStream_t s) {
  uint32_t P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  cudaMemsetAsync(max_len, 0, 4, s);
  note_launch(), k_table_prep<<<(P2 + 255) / 256, 256, 0, s>>>(t.bb_len, t.bb_bin, t.B, P2, tbl, max_len, err);
  uint64_t nt = bbv_n_tiles(t.W);
  if (tile_k0 && nt) note_launch(), k_tile_k0<<<(unsigned)ceil_div(nt, 256), 256, 0, s>>>(t.kwo, t.K, nt, tile_k0);
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

cudaError_t launch_bbv(const TraceDev& t, const uint32_t* tbl, const uint32_t* max_len, const uint32_t* tile_k0,
                       uint32_t* warp_bbv16, uint64_t* warp_insts, const TileEntries* te, DevErr* err, int num_sms,
                       cudaStream_t s) {
  BbvArgs a{};
  a.kwo = t.kwo; a.weo = t.weo; a.bb = t.bb; a.tbl = tbl; a.max_len = max_len; a.tile_k0 = tile_k0;
  a.K = t.K; a.B = t.B; a.P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  a.W = t.W; a.E = t.E;
  a.warp_bbv16 = warp_bbv16; a.warp_insts = warp_insts;
  if (te) a.te = *te;
  a.err = err;
  a.n_tiles = bbv_n_tiles(t.W);
  if (a.n_tiles == 0) return cudaSuccess;
  bool smem_tbl = a.P2 <= SMEM_TBL_MAX;
  bool mark = a.P2 != t.B;
  size_t smem = bbv_smem_bytes(smem_tbl ? a.P2 : 0);
  if (smem_tbl) return mark ? launch_bbv_t<true, true>(a, smem, num_sms, s) : launch_bbv_t<true, false>(a, smem, num_sms, s);
  return mark ? launch_bbv_t<false, true>(a, smem, num_sms, s) : launch_bbv_t<false, false>(a, smem, num_sms, s);
}

cudaError_t launch_group_from_bbv(const TraceDev& t, const uint32_t* warp_bbv16, const uint32_t* tile_k0,
                                  const TileEntries& te, DevErr* err, cudaStream_t s) {
  BbvArgs a{};
  a.kwo = t.kwo; a.K = t.K; a.W = t.W; a.te = te; a.err = err; a.tile_k0 = tile_k0;
  uint64_t tiles = bbv_n_tiles(t.W);
  a.n_tiles = tiles;
  if (tiles == 0) return cudaSuccess;
  size_t smem = bbv_smem_bytes(0);
  cudaError_t e = cudaFuncSetAttribute(k_group_from_bbv, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  note_launch(), k_group_from_bbv<<<(unsigned)tiles, TPB, smem, s>>>(a, warp_bbv16);
  return cudaGetLastError();
}

cudaError_t launch_kernel_bb_insts(const TraceDev& t, const uint32_t* tbl, uint64_t* kbb, uint64_t* kchunk_off,
                                   DevErr* err, int num_sms, cudaStream_t s) {
  (void)err;
  cudaMemsetAsync(kbb, 0, sizeof(uint64_t) * (size_t)t.K * t.B, s);
  note_launch(), k_kchunks<<<1, 1024, 0, s>>>(t.kwo, t.weo, t.K, kchunk_off);
  uint64_t jobs_ub = ceil_div(t.E, KBB_CHUNK) + t.K;
  uint64_t grid = jobs_ub < (uint64_t)num_sms * 4 ? jobs_ub : (uint64_t)num_sms * 4;
  if (grid == 0) grid = 1;
  size_t smem = t.B <= 8192 ? (size_t)t.B * 4 : 0;
  if (smem < 1024) smem = 1024;
  cudaFuncSetAttribute(k_kbb, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  note_launch(), k_kbb<<<(unsigned)grid, 256, smem, s>>>(t.kwo, t.weo, t.bb, tbl, t.K, t.B, kbb, jobs_ub,
                                                           kchunk_off);
  return cudaGetLastError();
}

}  // namespace photon
