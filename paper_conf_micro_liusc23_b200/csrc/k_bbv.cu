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
#include <stdlib.h>

#include "internal.h"

#ifndef PHOTON_EXP
#define PHOTON_EXP 0  // profiling experiments only (1: no accumulation, 2: no tile de-dup); never set in builds
#endif

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
  const uint32_t* tile_k0;  // [cap] kernel of each item's first warp
  const uint64_t* item_w0;  // [cap + 1] first warp of each item
  const uint32_t* n_items;  // device item count
  uint32_t* counter;        // dynamic item counter (zeroed before the launch)
  uint32_t K, B, P2;
  uint64_t W, E;
  uint32_t* warp_bbv16;
  uint64_t* warp_insts;
  TileEntries te;           // fused grouping outputs (te.tile_n == nullptr => not fused)
  DevErr* err;
  uint64_t n_tiles;         // item capacity
};

// warps [w0, w1) of item it (clamped: malformed offsets stay memory-safe; they are latched by k_items_fill)
__device__ __forceinline__ void item_range(const BbvArgs& a, uint64_t it, uint64_t& w0, uint64_t& w1) {
  w0 = umin64(a.item_w0[it], a.W);
  const uint64_t x = umax64(a.item_w0[it + 1], w0);
  w1 = umin64(umin64(x, w0 + TPB), a.W);
}

constexpr size_t kColBytes = (size_t)16 * COLB;
constexpr size_t kStageBytes = (size_t)CAPE * 2;
constexpr size_t kOffsBytes = (TPB + 4) * 8;
constexpr size_t kLocalBytes = LSLOTS * (8 + 4 + 4 + 4 + 4);
constexpr size_t kMiscBytes = 256;
constexpr size_t kKidBytes = TPB * 4 + (TPB + 4) * 8;

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
  uint2* info;       // [TPB+4] per (virtual) warp sp of the tile, for the current chunk: x = column (smem byte
                     // offset) of nxt(sp) | end of nxt(sp) << 16, y = nxt(sp) | start of sp << 16 (chunk-relative
                     // event offsets clamped to [0, LIM]; nxt = next non-empty warp, the tail sentinel maps to itself)
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
  m.info = (uint2*)(m.kid + TPB);
  m.tbl = (uint32_t*)(m.info + TPB + 4);
  return m;
}

// ---- per-event accumulation --------------------------------------------------------------------------------
// Table entry t: len << LSH | bin * COLB (bit 0 = id in [B, P2)); cell address = column + (t & AMASK).
struct Acc {
  const uint32_t* tbl;
  uint32_t bmask;
  uint32_t raw, orr;
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
  // a word whose events go to eight given columns (byte offsets from sbase)
  __device__ __forceinline__ void word8(uint4 v, const uint32_t (&t)[8], const uint32_t (&c)[8], uint8_t* sbase) {
    raw |= v.x | v.y | v.z | v.w;
    orr |= (t[0] | t[1] | t[2] | t[3]) | (t[4] | t[5] | t[6] | t[7]);
#pragma unroll
    for (int j = 0; j < 8; j += 2)
      pair(t[j], t[j + 1], (uint32_t*)(sbase + c[j]), (uint32_t*)(sbase + c[j + 1]), c[j] == c[j + 1]);
  }
  // the 8 table entries of a 16-byte word (loaded one word ahead of its accumulation: the table is read-only, so
  // issuing these before the previous word's cell stores is safe, and hides their latency)
  __device__ __forceinline__ void lookup(uint4 v, uint32_t (&t)[8]) const {
    t[0] = tbl[v.x & bmask]; t[1] = tbl[(v.x >> 16) & bmask];
    t[2] = tbl[v.y & bmask]; t[3] = tbl[(v.y >> 16) & bmask];
    t[4] = tbl[v.z & bmask]; t[5] = tbl[(v.z >> 16) & bmask];
    t[6] = tbl[v.w & bmask]; t[7] = tbl[(v.w >> 16) & bmask];
  }
  // one 16-byte word with its table entries: events j < bo into ca, j >= bo into cb (four load->add->store
  // steps of two events each)
  __device__ __forceinline__ void word(uint4 v, const uint32_t (&t)[8], uint32_t bo, uint32_t* ca, uint32_t* cb) {
    raw |= v.x | v.y | v.z | v.w;
    orr |= (t[0] | t[1] | t[2] | t[3]) | (t[4] | t[5] | t[6] | t[7]);
    pair(t[0], t[1], bo > 0 ? ca : cb, bo > 1 ? ca : cb, bo != 1);
    pair(t[2], t[3], bo > 2 ? ca : cb, bo > 3 ? ca : cb, bo != 3);
    pair(t[4], t[5], bo > 4 ? ca : cb, bo > 5 ? ca : cb, bo != 5);
    pair(t[6], t[7], bo > 6 ? ca : cb, bo > 7 ? ca : cb, bo != 7);
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
    const uint32_t e = ((lane == leader || !eq) ? my_ent : from_leader) & 0x7FFFFFFFu;
    a.te.gid[w0 + tid] = e < M ? (uint32_t)(t * M + e) : (0x80000000u | (uint32_t)(*ovf_base + (e - M)));
  }
  __syncthreads();
  for (int i = tid; i < LSLOTS; i += TPB) {
    m.lhash[i] = 0ull;
    m.lcount[i] = 0u;
    m.lminw[i] = UINT32_MAX;
  }
  if (tid == 0) m.misc[0] = 0u;
}

// Runs: thread t takes words [run_start(t), run_start(t+1)) of an nwc-word chunk (an equal split; moving starts
// to put each quarter-warp's LDS.128 in distinct bank groups was measured slower overall)
__device__ __forceinline__ uint32_t run_start(uint32_t t, uint32_t nwc) { return (t * nwc) / TPB; }
// the thread whose run holds word x (x < nwc): the largest t with run_start(t) <= x
__device__ __forceinline__ uint32_t run_holder(uint32_t x, uint32_t nwc) { return (x * TPB + TPB - 1) / nwc; }

// thread 0: stage the word-aligned events [cs, ce) into shared memory (bulk part on the TMA copy engine; events
// at or past E8 with plain loads, positions past E zero-filled), completing on the mbarrier
__device__ __forceinline__ void stage_chunk(const BbvArgs& a, const Smem& m, uint64_t cs, uint64_t ce, uint64_t E8) {
  uint64_t ae = umin64(ce, E8);
  uint32_t bytes = ae > cs ? (uint32_t)((ae - cs) * 2) : 0u;
  for (uint64_t i = umax64(cs, E8); i < ce; ++i) m.stage[i - cs] = i < a.E ? a.bb[i] : (uint16_t)0;
  mbar_arrive_expect_tx(m.mbar, bytes);
  for (uint32_t off = 0; off < bytes; off += 16384) {
    uint32_t n = bytes - off < 16384 ? bytes - off : 16384;
    const uint64_t src = PHOTON_EXP == 3 ? (cs & 0x7FFF8ull) : cs;  // experiment 3: L2-resident source
    bulk_g2s((uint8_t*)m.stage + off, (const uint8_t*)(a.bb + src) + off, n, m.mbar);
  }
}

// An item's events widened to words [A, Z), split into CAPE chunks; items without events have no chunk.
struct Cursor {
  uint64_t t, A, Z, c, nch;
  bool valid;
};
__device__ __forceinline__ void cursor_tile(const BbvArgs& a, Cursor& u, uint64_t t) {
  u.t = t;
  u.valid = true;
  u.c = 0;
  u.nch = 0;
  u.A = u.Z = 0;
  uint64_t w0, w1;
  item_range(a, t, w0, w1);
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

  // dynamic schedule: thread 0 takes items from the counter (skipping warp-less ones) one item ahead of the
  // consumers; sched[0] / sched[1] publish the first / next item
  const uint64_t NI = umin64(*a.n_items, a.n_tiles);
  uint32_t* const sched = m.misc + 8;
  __syncthreads();  // misc zeroed before thread 0 publishes the schedule
  auto grab = [&]() -> uint64_t { return umin64(atomicAdd(a.counter, 1u), NI); };  // items may be warp-less
  // producer (thread 0): the chunk in flight on the mbarrier, if any
  uint64_t fl_t = ~0ull, fl_c = 0;
  if (tid == 0) {
    const uint64_t x = grab();
    sched[0] = (uint32_t)x;
    sched[1] = (uint32_t)(x < NI ? grab() : NI);
    if (x < NI) {
      Cursor pc;
      cursor_tile(a, pc, x);
      if (pc.nch) {
        stage_chunk(a, m, pc.A, umin64(pc.A + CAPE, pc.Z), E8);
        fl_t = x;
        fl_c = 0;
      }
    }
  }
  uint32_t phase = 0;

  Acc acc;
  acc.tbl = SMEM_TBL ? m.tbl : a.tbl;
  acc.bmask = bmask;
  __syncthreads();

  uint64_t t = sched[0], tn = sched[1];
  uint64_t my_off = 0, last_off = 0;  // weo[w0 + tid] (clamped) and weo[w1] of the current item
  uint32_t my_k = 0;                  // kernel of the item's first warp (fused path), prefetched an item ahead
  uint64_t my_kb = ~0ull;             // start of the kernel after it
  if (t < NI) {
    uint64_t w0, w1;
    item_range(a, t, w0, w1);
    const uint64_t nw = w1 - w0;
    my_off = a.weo[w0 + umin64((uint64_t)tid, nw)];
    if (tid == 0) last_off = a.weo[w0 + nw];
    if (fused) {
      my_k = a.tile_k0[t];
      my_kb = my_k + 1 < a.K ? a.kwo[my_k + 1] : ~0ull;
    }
  }
  __syncthreads();

  while (t < NI) {
    uint64_t w0, w1;
    item_range(a, t, w0, w1);
    const uint32_t nw = (uint32_t)(w1 - w0);
    const uint64_t w = w0 + tid;
    const bool valid = w < w1;
    // o[1 + v] = start of warp v, o[nw + 1] = item end; o[0] / o[nw + 2] = word-aligned bounds (virtual warps)
    if ((uint32_t)tid <= nw) m.offs[1 + tid] = my_off;
    if (tid == 0) {
      m.offs[1 + nw] = last_off;
    }
    uint64_t nx_off = 0, nx_last = 0;
    uint32_t nx_k = 0;
    // the item after next: issued now, its value is only read at this item's end (latency hidden)
    uint32_t x_after = 0;
    if (tid == 0 && tn < NI) x_after = atomicAdd(a.counter, 1u);
    if (tn < NI) {
      uint64_t n0, n1;
      item_range(a, tn, n0, n1);
      const uint64_t nn = n1 - n0;
      nx_off = a.weo[n0 + umin64((uint64_t)tid, nn)];
      if (tid == 0) nx_last = a.weo[n0 + nn];
      if (fused) nx_k = a.tile_k0[tn];
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
    uint8_t* const sbase = smem_raw;
    const uint32_t dummy_off = (uint32_t)((uint8_t*)(m.hist + DUMMY) - sbase);
    uint32_t* const headcol = m.head + tid;
    const uint32_t head_off = (uint32_t)((uint8_t*)headcol - sbase);
    acc.raw = 0;
    acc.orr = 0;
    auto colof = [&](uint32_t sp) -> uint32_t {
      return (sp == 0 || sp == last) ? dummy_off : (uint32_t)((uint8_t*)(m.hist + (sp - 1)) - sbase);
    };
    // nxt(sp) = next non-empty (virtual) warp after sp (last = sentinel); o[0] / o[nw+2] taken from registers
    auto O = [&](uint32_t i) -> uint64_t { return i == 0 ? At : (i == nw + 2 ? Zt : m.offs[i]); };
    uint32_t nx[2] = {0u, 0u};
#pragma unroll
    for (int r = 0; r < 2; ++r) {
      const uint32_t sp = tid + r * TPB;
      if (sp <= last) {
        uint32_t x = sp + 1;
        while (x < last && O(x + 1) == O(x)) ++x;
        nx[r] = x < last ? x : last;
      }
    }
    for (uint64_t c = 0; c < nch; ++c) {
      const uint64_t cs = At + c * CAPE, ce = umin64(cs + CAPE, Zt);
      const uint32_t nwc = (uint32_t)((ce - cs) >> 3);
      // all positions in the loop are u32 offsets from the chunk start, clamped to [0, LIM]
      const uint32_t LIM = (uint32_t)(ce - cs) + 8u;
      auto rel = [&](uint64_t x) -> uint32_t {
        return x <= cs ? 0u : (x - cs >= LIM ? LIM : (uint32_t)(x - cs));
      };
      // this chunk's warp table (the previous chunk's readers finished at its trailing barrier)
#pragma unroll
      for (int r = 0; r < 2; ++r) {
        const uint32_t sp = tid + r * TPB;
        if (sp <= last) {
          const uint32_t n = nx[r];
          const uint32_t endn = n != sp ? rel(O(n + 1)) : LIM + 8u;
          m.info[sp] = make_uint2(colof(n) | (endn << 16), n | (rel(O(sp)) << 16));
        }
      }
      __syncthreads();
      if (tid == 0 && !(fl_t == t && fl_c == c)) {  // not prefetched (the previous item had no events)
        stage_chunk(a, m, cs, ce, E8);
        fl_t = t;
        fl_c = c;
      }
      mbar_wait(m.mbar, phase);
      phase ^= 1u;
      // my run of words [r0, r1) of the chunk
      const uint32_t q0 = 8u * run_start(tid, nwc), qe = 8u * run_start(tid + 1, nwc);
      if (q0 < qe) {
        // warp (with virtual ones) containing q0: last sp with start(sp) <= q0.  Start from the proportional guess
        // and narrow a +-8 window around it when it brackets q0 (it usually does), else search everything.
        auto start = [&](uint32_t sp) -> uint32_t { return m.info[sp].y >> 16; };
        uint32_t lo = 0, hi = last;
        {
          const uint64_t r0 = cs + q0;
          const float fr = (float)(r0 - At) / (float)(Zt - At);
          int g = (int)(fr * (float)(nw + 2));
          int glo = g - 8 < 0 ? 0 : g - 8, ghi = g + 8 > (int)last ? (int)last : g + 8;
          if (start(glo) <= q0 && (ghi == (int)last || start(ghi + 1) > q0)) { lo = (uint32_t)glo; hi = (uint32_t)ghi; }
        }
        while (lo < hi) {
          uint32_t mid = (lo + hi + 1) >> 1;
          if (start(mid) <= q0) lo = mid; else hi = mid - 1;
        }
        uint32_t sg = lo;
        uint32_t col = (O(sg) < cs + q0) ? head_off : colof(sg);  // warp open at my run start -> HEAD
        uint32_t nb = rel(O(sg + 1));
        uint2 f = m.info[sg];
        uint32_t sgn = f.y & 0xFFFFu, coln = f.x & 0xFFFFu, nb2 = f.x >> 16;
        const uint4* sb4 = (const uint4*)m.stage;
        // one word: v / t = this word and its table entries; vn / tn receive the next word's (software pipeline,
        // unrolled by two below so the buffers swap roles without register moves)
        auto step = [&](uint32_t q, const uint4& v, const uint32_t (&t)[8], uint4& vn, uint32_t (&tn)[8]) {
          vn = sb4[(q + 8 < qe ? q + 8 : q) >> 3];
          acc.lookup(vn, tn);
          if (nb2 < q + 8) {
            // several warp boundaries inside this word (warps shorter than 8 events): each event's column by
            // stepping (empty warps are skipped by nxt, so an event crosses at most one boundary), then the same
            // paired accumulation as a one-boundary word
            uint32_t c[8];
#pragma unroll
            for (int j = 0; j < 8; ++j) {
              if (q + j >= nb) {
                sg = sgn;
                col = coln;
                nb = nb2;
                f = m.info[sg];
                sgn = f.y & 0xFFFFu;
                coln = f.x & 0xFFFFu;
                nb2 = f.x >> 16;
              }
              c[j] = col;
            }
            acc.word8(v, t, c, sbase);
            if (q + 8 >= nb) {  // the next word starts in the next warp
              sg = sgn;
              col = coln;
              nb = nb2;
            }
          } else {
            const uint32_t bo = nb < q + 8 ? nb - q : 8u;  // first event of the next warp
            acc.word(v, t, bo, (uint32_t*)(sbase + col), (uint32_t*)(sbase + coln));
            // advance past a crossed boundary without branching (lanes cross at different words; a divergent
            // update would serialise): when bo == 8 the same values are reloaded
            const bool cross = bo < 8u;
            sg = cross ? sgn : sg;
            col = cross ? coln : col;
            nb = cross ? nb2 : nb;
          }
          f = m.info[sg];
          sgn = f.y & 0xFFFFu;
          coln = f.x & 0xFFFFu;
          nb2 = f.x >> 16;
        };
        uint4 va = sb4[q0 >> 3], vb;
        uint32_t ta[8], tb[8];
        acc.lookup(va, ta);
        if (PHOTON_EXP == 1) {  // profiling experiment: no accumulation
          acc.raw |= va.x;
          goto chunk_done;
        }
        for (uint32_t q = q0;;) {
          step(q, va, ta, vb, tb);
          q += 8;
          if (q >= qe) break;
          step(q, vb, tb, va, ta);
          q += 8;
          if (q >= qe) break;
        }
      }
    chunk_done:
      __syncthreads();  // accumulation done; the stage is free
      if (tid == 0) {   // stage the next chunk (this item's next, or the next item's first) during the combine
        fl_t = ~0ull;
        if (c + 1 < nch) {
          const uint64_t ncs = At + (c + 1) * CAPE;
          stage_chunk(a, m, ncs, umin64(ncs + CAPE, Zt), E8);
          fl_t = t;
          fl_c = c + 1;
        } else if (tn < NI) {  // thread 0 holds the next item's bounds (nx_off / nx_last), same clamping as cursor_tile
          const uint64_t nte = umin64(nx_last, a.E), nts = umin64(nx_off, nte);
          if (nte > nts) {
            const uint64_t nA = nts & ~7ull, nZ = (nte + 7) & ~7ull;
            stage_chunk(a, m, nA, umin64(nA + CAPE, nZ), E8);
            fl_t = tn;
            fl_c = 0;
          }
        }
      }
      // combine: warp tid (if it has events in this chunk) adds the HEAD partials of the threads it spilled into
      if (valid && e > s && e > cs && s < ce) {
        const uint32_t lo_w = (uint32_t)((umax64(s, cs) - cs) >> 3), hi_w = (uint32_t)((umin64(e, ce) - 1 - cs) >> 3);
        const uint32_t ta = run_holder(lo_w, nwc);  // thread whose run holds word lo_w
        const uint32_t tb = run_holder(hi_w, nwc);
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
    uint32_t k = my_k;
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
      if (fused && w >= my_kb) {  // the tile crosses into later kernels
        ++k;
        while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
      }
    }
    if (fused && PHOTON_EXP != 2) {
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
    if (fused && tn < NI) {
      my_k = nx_k;
      my_kb = my_k + 1 < a.K ? a.kwo[my_k + 1] : ~0ull;
    }
    if (tid == 0) sched[1] = (uint32_t)(tn < NI ? umin64(x_after, NI) : NI);
    __syncthreads();  // result columns cleared and offs free before the next item
    t = tn;
    tn = sched[1];
  }
}

// K2a over materialised BBVs (the unfused API path): one CTA per item, keys loaded from warp_bbv16.
__global__ void __launch_bounds__(TPB) k_group_from_bbv(BbvArgs a, const uint32_t* __restrict__ bbv) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  Smem m = carve(smem_raw);
  const int tid = threadIdx.x;
  const uint64_t t = blockIdx.x;
  if (t >= umin64(*a.n_items, a.n_tiles)) return;
  uint64_t w0, w1;
  item_range(a, t, w0, w1);
  if (w1 <= w0) {
    if (tid == 0) a.te.tile_n[t] = 0u;
    return;
  }
  const uint64_t w = w0 + tid;
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

// ---- work items -----------------------------------------------------------------------------------------------
// Items of block b: nsub(b) = windows spanned by the starts of its warps (sub(w) = (start(w) - start(b0)) >> xs).
// Two-level exclusive scan: k_items_count writes nsub, the CTA-local exclusive prefix (into boff) and each CTA's
// total; k_items_scan scans the CTA totals; k_items_fill adds them.  n[0] = item count (clamped to cap), n[1] = work
// counter, n[2] = split-block count.
__global__ void __launch_bounds__(256) k_items_count(const uint64_t* __restrict__ weo, uint64_t W, uint64_t E,
                                                     uint32_t xs, uint64_t n_blocks, uint32_t* nsub, uint32_t* boff,
                                                     uint32_t* part) {
  __shared__ uint32_t wsum[8];
  const uint64_t b = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  uint32_t v = 0;
  if (b < n_blocks) {
    const uint64_t b0 = b * TPB, bl = umin64(W, b0 + TPB) - 1;
    const uint64_t s0 = umin64(weo[b0], E), sl = umin64(weo[bl], E);
    v = (uint32_t)umin64(((sl > s0 ? sl - s0 : 0) >> xs) + 1, (uint64_t)TPB);
    nsub[b] = v;
  }
  uint32_t x = v;
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) wsum[wid] = x;
  __syncthreads();
  uint32_t pre = 0, tot = 0;
  for (int k = 0; k < 8; ++k) {
    pre += k < wid ? wsum[k] : 0u;
    tot += wsum[k];
  }
  if (b < n_blocks) boff[b] = pre + x - v;
  if (threadIdx.x == 0) part[blockIdx.x] = tot;
}

// exclusive scan of the CTA totals (one CTA, 16 per thread per pass)
constexpr int ISCAN_PT = 16;
__global__ void __launch_bounds__(1024) k_items_scan(uint32_t* part, uint64_t n_parts, uint64_t n_blocks, uint64_t cap,
                                                     uint32_t* boff, uint32_t* n, DevErr* err) {
  __shared__ uint64_t ws[32];
  __shared__ uint64_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  for (uint64_t base = 0; base < n_parts; base += 1024 * ISCAN_PT) {
    const uint64_t b0 = base + (uint64_t)threadIdx.x * ISCAN_PT;
    uint32_t v[ISCAN_PT];
    uint64_t tot = 0;
#pragma unroll
    for (int i = 0; i < ISCAN_PT; ++i) {
      v[i] = b0 + i < n_parts ? part[b0 + i] : 0u;
      tot += v[i];
    }
    uint64_t x = tot;
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
    uint64_t ex = carry + (wid ? ws[wid - 1] : 0) + x - tot;
#pragma unroll
    for (int i = 0; i < ISCAN_PT; ++i) {
      if (b0 + i < n_parts) part[b0 + i] = (uint32_t)umin64(ex, 0xFFFFFFFFull);
      ex += v[i];
    }
    __syncthreads();
    if (threadIdx.x == 1023) carry = ex;
    __syncthreads();
  }
  if (threadIdx.x == 0) {
    boff[n_blocks] = (uint32_t)umin64(carry, cap);
    if (carry > cap) latch(err, PHOTON_ERANGE, 0);  // only with non-monotone warp_event_off
    n[0] = (uint32_t)umin64(carry, cap);
    n[1] = 0;
    n[2] = 0;
  }
}

// one thread per block: final first item; a one-item block starts at its first warp; split blocks are queued
__global__ void k_items_fill(uint64_t W, uint32_t* boff, const uint32_t* __restrict__ nsub,
                             const uint32_t* __restrict__ part, uint64_t n_blocks, uint64_t cap, uint32_t* n,
                             uint64_t* item_w0, uint32_t* split) {
  const uint64_t b = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (b == 0) item_w0[n[0]] = W;
  if (b >= n_blocks) return;
  const uint64_t it0 = umin64((uint64_t)boff[b] + part[blockIdx.x], cap);
  const uint32_t nb = (uint32_t)umin64(nsub[b], cap - it0);
  boff[b] = (uint32_t)it0;
  if (nb == 1) item_w0[it0] = b * TPB;
  else if (nb > 1) split[atomicAdd(&n[2], 1u)] = (uint32_t)b;
}

// one warp per split block: each warp opens the windows between the previous warp's and its own (windows holding no
// start become empty items); non-monotone warp_event_off is latched
__global__ void k_items_split(const uint64_t* __restrict__ weo, uint64_t W, uint64_t E, uint32_t xs,
                              const uint32_t* __restrict__ boff, const uint32_t* __restrict__ nsub, uint64_t cap,
                              const uint32_t* __restrict__ n, const uint32_t* __restrict__ split, uint64_t* item_w0,
                              DevErr* err) {
  const int lane = threadIdx.x & 31;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t q = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; q < n[2]; q += nwarps) {
    const uint64_t b = split[q], b0 = b * TPB, b1 = umin64(W, b0 + TPB);
    const uint32_t it0 = boff[b], nb = nsub[b];
    const uint64_t base = umin64(weo[b0], E);
    for (uint64_t w = b0 + lane; w < b1; w += 32) {
      const uint64_t sw = umin64(weo[w], E);
      const uint64_t s = (sw > base ? sw - base : 0) >> xs;
      int64_t sp = -1;
      if (w > b0) {
        if (weo[w - 1] > weo[w]) latch(err, PHOTON_ERANGE, (int64_t)(w - 1));
        const uint64_t sv = umin64(weo[w - 1], E);
        sp = (int64_t)((sv > base ? sv - base : 0) >> xs);
      }
      for (int64_t i = sp + 1; i <= (int64_t)s && (uint64_t)i < nb && it0 + (uint64_t)i < cap; ++i) item_w0[it0 + i] = w;
    }
  }
}

// kernel of each item's first warp (one thread per item)
__global__ void k_items_k0(const uint64_t* __restrict__ kwo, uint32_t K, const uint32_t* __restrict__ n,
                           const uint64_t* __restrict__ item_w0, uint64_t cap, uint32_t* item_k0) {
  const uint64_t it = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (it >= cap || it >= n[0]) return;
  const uint64_t w = item_w0[it];
  uint32_t lo = 0, hi = K - 1;  // last k with kwo[k] <= w
  while (lo < hi) {
    uint32_t mid = (lo + hi + 1) >> 1;
    if (kwo[mid] <= w) lo = mid; else hi = mid - 1;
  }
  item_k0[it] = lo;
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
uint64_t bbv_n_blocks(uint64_t W) { return ceil_div(W, TPB); }
uint64_t bbv_item_cap(uint64_t W, uint64_t E, uint32_t xs) {
  return bbv_n_blocks(W) + (xs < 63 ? (E >> xs) : 0) + 1;
}

cudaError_t launch_table_prep(const TraceDev& t, uint32_t* tbl, uint32_t* max_len, const ItemTable& it,
                              const TileEntries* te, DevErr* err, cudaStream_t s) {
  uint32_t P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  cudaMemsetAsync(max_len, 0, 4, s);
  note_launch(), k_table_prep<<<(P2 + 255) / 256, 256, 0, s>>>(t.bb_len, t.bb_bin, t.B, P2, tbl, max_len, err);
  const uint64_t nb = bbv_n_blocks(t.W);
  if (nb == 0) return cudaGetLastError();
  (void)te;
  const uint64_t gb = ceil_div(nb, 256);
  note_launch(), k_items_count<<<(unsigned)gb, 256, 0, s>>>(t.weo, t.W, t.E, it.xs, nb, it.nsub, it.boff, it.part);
  note_launch(), k_items_scan<<<1, 1024, 0, s>>>(it.part, gb, nb, it.cap, it.boff, it.n, err);
  note_launch(), k_items_fill<<<(unsigned)gb, 256, 0, s>>>(t.W, it.boff, it.nsub, it.part, nb, it.cap, it.n, it.w0,
                                                           it.split);
  note_launch(), k_items_split<<<(unsigned)umin64(ceil_div(nb * 32, 256), 1184), 256, 0, s>>>(
      t.weo, t.W, t.E, it.xs, it.boff, it.nsub, it.cap, it.n, it.split, it.w0, err);
  note_launch(), k_items_k0<<<(unsigned)ceil_div(it.cap, 256), 256, 0, s>>>(t.kwo, t.K, it.n, it.w0, it.cap, it.k0);
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

cudaError_t launch_bbv(const TraceDev& t, const uint32_t* tbl, const uint32_t* max_len, const ItemTable& it,
                       uint32_t* warp_bbv16, uint64_t* warp_insts, const TileEntries* te, DevErr* err, int num_sms,
                       cudaStream_t s) {
  if (bbv2_supported(t.B) && !getenv("PHOTON_K1_V1"))
    return launch_bbv2(t, tbl, it, warp_bbv16, warp_insts, te, err, num_sms, s);
  BbvArgs a{};
  a.kwo = t.kwo; a.weo = t.weo; a.bb = t.bb; a.tbl = tbl; a.max_len = max_len; a.tile_k0 = it.k0;
  a.item_w0 = it.w0; a.n_items = it.n; a.counter = it.n + 1;
  a.K = t.K; a.B = t.B; a.P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  a.W = t.W; a.E = t.E;
  a.warp_bbv16 = warp_bbv16; a.warp_insts = warp_insts;
  if (te) a.te = *te;
  a.err = err;
  a.n_tiles = it.cap;
  if (t.W == 0) return cudaSuccess;
  cudaMemsetAsync(a.counter, 0, 4, s);
  bool smem_tbl = a.P2 <= SMEM_TBL_MAX;
  bool mark = a.P2 != t.B;
  size_t smem = bbv_smem_bytes(smem_tbl ? a.P2 : 0);
  if (smem_tbl) return mark ? launch_bbv_t<true, true>(a, smem, num_sms, s) : launch_bbv_t<true, false>(a, smem, num_sms, s);
  return mark ? launch_bbv_t<false, true>(a, smem, num_sms, s) : launch_bbv_t<false, false>(a, smem, num_sms, s);
}

cudaError_t launch_group_from_bbv(const TraceDev& t, const uint32_t* warp_bbv16, const ItemTable& it,
                                  const TileEntries& te, DevErr* err, cudaStream_t s) {
  BbvArgs a{};
  a.kwo = t.kwo; a.K = t.K; a.W = t.W; a.te = te; a.err = err; a.tile_k0 = it.k0;
  a.item_w0 = it.w0; a.n_items = it.n;
  const uint64_t tiles = it.cap;
  a.n_tiles = tiles;
  if (t.W == 0) return cudaSuccess;
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
