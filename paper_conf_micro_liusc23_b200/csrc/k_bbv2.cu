// k_bbv2.cu — A1 (per-warp BBV projected to 16 bins) fused with A2's de-duplication step: the streaming pass K1.
//
// PAPER.md: L161 (a BBV lists the basic blocks a warp executed), L154 (same instruction sequence => same BBV => same
// warp type), L178 ("project these BBVs into fixed-size BBVs (We use 16) to improve online clustering performance
// ... we can easily cluster the warps if they have the same BBV").  Readings [P-1] (entry = executions x length)
// and [P-2] (sum-preserving fold into 16 bins).  DESIGN.md §5.1.
//
// Design.  The per-event work is one table lookup and one shared-memory add; what bounds the pass is the number of
// shared-memory wavefronts per event, so everything is laid out to keep that at its minimum:
//  * Persistent CTAs of 256 threads (two per SM) take work items (<= 256 consecutive analysed warps, ~32K events)
//    from a counter.  Thread u owns warp u of the item: its 16-bin key lives in thread u's registers for the whole
//    item and is finalised (hash, CTA de-duplication, entry output) once at the item's end.
//  * An item's events are staged in chunks of <= 18432 events (cp.async.bulk on the TMA engine; the next chunk is
//    issued as soon as the lanes are done with the stage, and lands while the pieces are collected and the next
//    chunk's lane tables are built).  Each chunk is split into 256 equal lane ranges of Q <= 9 words (Q odd, so the 32 lanes' 16-byte LDS hit distinct
//    bank groups).  Lane t walks its range in order; the piece of each analysed warp it meets is accumulated in a
//    column private to the lane with red.shared.add (no read-modify-write latency chain): the first piece in the
//    lane's slot-0 column (bank = lane, conflict-free); a warp starting inside the lane's range goes to the pool
//    column of its own index (an item holds <= 256 warps, so pool columns are unique).  Per event: one LDS of
//    the packed (len, bin) entry, one RED.
//  * Thread u then sums its warp's pieces (the owner column in the lane holding the warp's first event of the
//    chunk, then slot 0 of every later lane the warp spans) into its key registers.  The cells are cleared with
//    16-byte stores (conflict-free) while the next chunk's lane tables are built.
//  * Bin cells are u32: a chunk holds <= 18432 events of length < 2^17, so a chunk piece cannot wrap; the per-warp
//    totals are carried in u64 and checked against 2^32 (PHOTON_ERANGE).
#include "internal.h"

namespace photon {

namespace {

constexpr int NT = 256;              // threads per CTA = warps per item (ItemTable blocks)
constexpr int QMAX = 9;              // words per lane per chunk (odd)
constexpr int CHW = NT * QMAX;       // words per chunk
constexpr int CHE = CHW * 8;         // events per chunk (10240)
constexpr int ROW = 2 * NT;          // u32 per bin row: slot-0 column of each lane [0, NT), pool columns [NT, 2NT)
constexpr int ROWB = ROW * 4;        // bin stride in bytes; local table entry = len << 15 | bin << 11 | mark
constexpr uint32_t TOFF = 0x7800u;   // bin * ROWB bits of an entry
constexpr int TSH = 15;              // length shift
constexpr int LSLOTS = 256;          // CTA-local de-dup slots
constexpr int LPROBE = 16;           // probes before a leader takes an entry of its own (the global insert merges)
constexpr int SMEM_TBL_MAX = 4096;   // BB table entries kept in shared memory
static_assert(ROWB == 2048 && 15 * ROWB <= (int)TOFF, "bin offset layout");

struct Args {
  const uint64_t* kwo;
  const uint64_t* weo;
  const uint16_t* bb;
  const uint32_t* tbl;       // global packed table (len << 15 | bin * 1152 | mark), see k_table_prep
  const uint32_t* tile_k0;   // [cap] kernel of each item's first warp
  const uint64_t* item_w0;   // [cap + 1] first warp of each item
  const uint32_t* n_items;   // device item count
  uint32_t* counter;         // dynamic item counter (zeroed before the launch)
  uint32_t K, B, P2;
  uint64_t W, E;
  uint32_t* warp_bbv16;
  uint64_t* warp_insts;
  TileEntries te;            // fused grouping outputs (te.tile_n == nullptr => not fused)
  DevErr* err;
  uint64_t n_tiles;          // item capacity
  uint32_t pre;              // bytes in front of the cells (see smem_bytes)
};

constexpr size_t kCellBytes = (size_t)16 * ROWB;     // 32 KB
constexpr size_t kStageBytes = (size_t)CHE * 2;      // 36 KB
constexpr size_t kOffBytes = (size_t)(NT + 4) * 8;   // item warp offsets (u64)
constexpr size_t kRelBytes = (size_t)(NT + 4) * 4;   // chunk-relative warp starts (u32)
constexpr size_t kLocalBytes = (size_t)LSLOTS * (8 + 4 + 4 + 4 + 4);
constexpr size_t kMiscBytes = 256;
constexpr size_t kKidBytes = (size_t)NT * 4;

// everything but the cells and the stage
__host__ __device__ constexpr size_t small_bytes(uint32_t tbl_entries) {
  return kOffBytes + kRelBytes + 16 + kLocalBytes + kMiscBytes + kKidBytes +
         (size_t)tbl_entries * 4;
}
// Layout: the cells must start on a 32 KB boundary of the shared window (cell address = column | bin offset).  The
// dynamic window starts `pre` bytes before such a boundary (the reserved shared memory): the small arrays go in
// front when they fit there, else behind the stage.
__host__ __device__ constexpr size_t smem_bytes(uint32_t tbl_entries, uint32_t pre) {
  return pre + kCellBytes + kStageBytes + (small_bytes(tbl_entries) <= pre ? 0 : small_bytes(tbl_entries));
}

struct Smem {
  uint32_t* cells;   // [16][ROW]
  uint16_t* stage;   // [CHE]
  uint64_t* off;     // [NT+4] weo of the item's warps (monotone), off[nw] = item end, padded
  uint32_t* rel;     // [NT+4] chunk-relative starts (clamped to [0, LIM])
  uint64_t* mbar;    // [1]
  uint64_t* lhash;   // [LSLOTS]
  uint32_t* lowner;  // [LSLOTS]
  uint32_t* lcount;  // [LSLOTS]
  uint32_t* lminw;   // [LSLOTS]
  uint32_t* lent;    // [LSLOTS]
  uint32_t* misc;    // [64]: 0 n_entries, [2..3] next free overflow entry of the CTA's block, [4..5] its end,
                     // [6..7] the current item's overflow base, [8..9] schedule
  uint32_t* kid;     // [NT]
  uint32_t* tbl;     // [P2]
};

__device__ __forceinline__ Smem carve(uint8_t* s, uint32_t pre, uint32_t P2) {
  Smem m;
  m.cells = (uint32_t*)(s + pre);
  m.stage = (uint16_t*)(s + pre + kCellBytes);
  size_t o = small_bytes(P2) <= pre ? 0 : pre + kCellBytes + kStageBytes;
  m.off = (uint64_t*)(s + o); o += kOffBytes;
  m.rel = (uint32_t*)(s + o); o += kRelBytes;
  m.mbar = (uint64_t*)(s + o); o += 16;
  m.lhash = (uint64_t*)(s + o);
  m.lowner = (uint32_t*)(m.lhash + LSLOTS);
  m.lcount = m.lowner + LSLOTS;
  m.lminw = m.lcount + LSLOTS;
  m.lent = m.lminw + LSLOTS;
  o += kLocalBytes;
  m.misc = (uint32_t*)(s + o); o += kMiscBytes;
  m.kid = (uint32_t*)(s + o); o += kKidBytes;
  m.tbl = (uint32_t*)(s + o);
  return m;
}

// No "memory" clobber: the cells are only written by these adds and only read after a __syncthreads(), so the
// compiler may move the (read-only) stage and table loads across them, which the event loop relies on.
__device__ __forceinline__ void red_add(uint32_t saddr, uint32_t v) {
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v));
}

// warps [w0, w1) of item it (clamped: malformed offsets stay memory-safe; they are latched by k_items_fill)
__device__ __forceinline__ void item_range(const Args& a, uint64_t it, uint64_t& w0, uint64_t& w1) {
  w0 = umin64(a.item_w0[it], a.W);
  const uint64_t x = umax64(a.item_w0[it + 1], w0);
  w1 = umin64(umin64(x, w0 + NT), a.W);
}

// A chunk: events [cs, ce) (absolute) staged as the words from a8 = cs & ~7; chunk-relative range [lo, hi).
struct Chunk {
  uint64_t a8;
  uint32_t lo, hi;
};
__device__ __forceinline__ Chunk plan(uint64_t cs, uint64_t te) {
  Chunk c;
  c.a8 = cs & ~7ull;
  c.lo = (uint32_t)(cs - c.a8);
  c.hi = (uint32_t)(umin64(te, c.a8 + CHE) - c.a8);
  return c;
}

// thread 0: stage the words of chunk c (bulk part on the TMA copy engine; words at or past E8
// with plain loads, positions past E zero-filled), completing on the mbarrier
__device__ __forceinline__ void stage_chunk(const Args& a, const Smem& m, const Chunk& c, uint64_t E8) {
  uint16_t* dst = m.stage;
  const uint64_t ce = c.a8 + (((uint64_t)c.hi + 7) & ~7ull);
  const uint64_t ae = umin64(ce, E8);
  const uint32_t bytes = ae > c.a8 ? (uint32_t)((ae - c.a8) * 2) : 0u;
  for (uint64_t i = umax64(c.a8, E8); i < ce; ++i) dst[i - c.a8] = i < a.E ? a.bb[i] : (uint16_t)0;
  mbar_arrive_expect_tx(m.mbar, bytes);
  for (uint32_t off = 0; off < bytes; off += 16384)
    bulk_g2s((uint8_t*)dst + off, (const uint8_t*)(a.bb + c.a8) + off, umin(bytes - off, 16384u), m.mbar);
}

// Slow path (bad input only): first event of [s, e) whose id is >= B.
__device__ void report_bad_event(const Args& a, uint64_t s, uint64_t e) {
  for (uint64_t i = s; i < e; ++i)
    if (a.bb[i] >= a.B) { latch(a.err, PHOTON_ERANGE, (int64_t)i); return; }
}

// ---- item finalisation: CTA de-duplication and per-item entries ------------------------------------------------
// Each thread holds its warp's key p (registers).  A slot owner publishes its key in its slot-0 column of `cells`
// (overwritten; the next chunk's bulk clear resets the cells) so pending claimers can verify it.
__device__ void item_group(const Args& a, const Smem& m, uint64_t t, uint64_t w0, bool valid, uint32_t k,
                           const uint32_t* p) {
  const int tid = threadIdx.x, lane = tid & 31;
  const uint64_t h = valid ? hash_key(k, p) : 0;
  const unsigned active = __ballot_sync(0xffffffffu, valid);
  const unsigned peers = __match_any_sync(0xffffffffu, (unsigned long long)h);
  const int leader = __ffs(peers) - 1;
  bool eq = (__shfl_sync(0xffffffffu, k, leader) == k);
#pragma unroll
  for (int j = 0; j < 16; ++j) eq &= (__shfl_sync(0xffffffffu, p[j], leader) == p[j]);  // no short circuit
  const unsigned eqm = __ballot_sync(0xffffffffu, eq);
  const bool is_leader = valid && (lane == leader || !eq);
  const uint32_t cnt = (lane == leader) ? (uint32_t)__popc(peers & eqm & active) : 1u;
  int slot = -1;
  bool pending = false;
  if (is_leader) {
    uint32_t i = (uint32_t)(h & (LSLOTS - 1));
    for (int probe = 0; probe < LPROBE; ++probe) {
      unsigned long long cur = atomicCAS((unsigned long long*)&m.lhash[i], 0ull, (unsigned long long)h);
      if (cur == 0ull) {
        m.lowner[i] = (uint32_t)tid;
        m.lent[i] = atomicAdd(&m.misc[0], 1u);
        slot = (int)i;
#pragma unroll
        for (int j = 0; j < 16; ++j) m.cells[j * ROW + tid] = p[j];
        m.kid[tid] = k;
        break;
      }
      if (cur == h) { slot = (int)i; pending = true; break; }
      i = (i + 1) & (LSLOTS - 1);
    }
  }
  __syncthreads();
  uint32_t my_ent = UINT32_MAX;
  if (slot >= 0) {
    bool own = true;
    if (pending) {
      const uint32_t o = m.lowner[slot];
      bool same = (m.kid[o] == k);
#pragma unroll
      for (int j = 0; j < 16; ++j) same &= (m.cells[j * ROW + o] == p[j]);  // independent loads
      own = same;
    }
    if (own) {
      atomicAdd(&m.lcount[slot], cnt);
      atomicMin(&m.lminw[slot], (uint32_t)tid);  // leaders are the lowest thread of their warp group
      my_ent = m.lent[slot];
    } else {
      my_ent = atomicAdd(&m.misc[0], 1u) | 0x80000000u;  // equal hash, different key: an entry of its own
    }
  } else if (is_leader) {
    my_ent = atomicAdd(&m.misc[0], 1u) | 0x80000000u;  // no free slot within LPROBE probes: an entry of its own
  }
  __syncthreads();
  const uint32_t n_ent = m.misc[0];
  const uint32_t M = a.te.per_tile;
  uint64_t* ovf_base = (uint64_t*)(m.misc + 2);
  if (n_ent > M) {  // more distinct keys than the item's fixed entry slots: overflow entries from the CTA's block
    if (tid == 0) {
      uint64_t* ovf_end = (uint64_t*)(m.misc + 4);
      const uint64_t need = n_ent - M;
      uint64_t pos = *ovf_base;
      if (pos + need > *ovf_end) {  // refill (rare): a block of at least 256 entries; the old block's unused tail
                                     // is marked empty (count 0, skipped by the insertion)
        for (uint64_t j = pos; j < umin64(*ovf_end, a.te.ovf_cap); ++j) a.te.ovf[j].count = 0u;
        const uint64_t blk = need > 256 ? need : 256;
        pos = atomicAdd((unsigned long long*)a.te.ovf_count, (unsigned long long)blk);
        if (pos + need > a.te.ovf_cap) latch(a.err, PHOTON_ECAPACITY, (int64_t)pos);
        *ovf_end = pos + blk;
      }
      a.te.tile_ovf[t] = pos;
      m.misc[6] = (uint32_t)pos;  // this item's base (low word; the high word below)
      m.misc[7] = (uint32_t)(pos >> 32);
      *ovf_base = pos + need;
    }
    __syncthreads();
  }
  const uint64_t obase = ((uint64_t)m.misc[7] << 32) | m.misc[6];
  if (tid == 0) a.te.tile_n[t] = n_ent;
  auto put = [&](uint32_t e, uint32_t kern, const uint32_t* key, uint32_t count, uint32_t minw, uint64_t hh) {
    TileEntry* dst;
    if (e < M) {
      dst = a.te.ent + t * M + e;
    } else {
      uint64_t pos = obase + (e - M);
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
  for (int i = tid; i < LSLOTS; i += NT) {
    uint64_t hh = m.lhash[i];
    if (hh != 0ull) {
      uint32_t o = m.lowner[i];
      uint32_t key[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) key[j] = m.cells[j * ROW + o];
      put(m.lent[i], m.kid[o], key, m.lcount[i], m.lminw[i], hh);
    }
  }
  if (my_ent != UINT32_MAX && (my_ent & 0x80000000u)) put(my_ent & 0x7FFFFFFFu, k, p, cnt, (uint32_t)tid, h);
  const uint32_t from_leader = __shfl_sync(0xffffffffu, my_ent, leader);
  if (valid) {
    const uint32_t e = ((lane == leader || !eq) ? my_ent : from_leader) & 0x7FFFFFFFu;
    a.te.gid[w0 + tid] = e < M ? (uint32_t)(t * M + e) : (0x80000000u | (uint32_t)(obase + (e - M)));
  }
  __syncthreads();
  for (int i = tid; i < LSLOTS; i += NT) {
    m.lhash[i] = 0ull;
    m.lcount[i] = 0u;
    m.lminw[i] = UINT32_MAX;
  }
  if (tid == 0) m.misc[0] = 0u;
}

// column (byte offset in cells) of warp u's piece in lane t: the lane's first warp fw goes to the lane's own
// slot-0 column, a warp starting inside the lane's range to the pool column of its index (<= 256 warps per item)
__device__ __forceinline__ uint32_t colof(uint32_t t, uint32_t fw, uint32_t u) {
  return u == fw ? t * 4u : (uint32_t)(NT + u) * 4u;
}

template <bool CHECK_MARK>
__global__ void __launch_bounds__(NT, 2) k_bbv2(Args a) {
  extern __shared__ __align__(128) uint8_t smem_raw[];
  Smem m = carve(smem_raw, a.pre, a.P2);
  const int tid = threadIdx.x;
  const uint32_t bmask = a.P2 - 1, mask4 = bmask << 2;
  const bool fused = a.te.tile_n != nullptr;
  const uint32_t cbase = smem_u32(m.cells);
  // a cell address is (entry & TOFF) | column: the cell array must sit on a 32 KB boundary of the shared window
  if ((cbase & 0x7FFFu) != 0u) {
    if (tid == 0) latch(a.err, PHOTON_ECUDA, -2);
    return;
  }

  // shared table in the cell layout: bin * 1152 -> bin << 11
  for (uint32_t i = tid; i < a.P2; i += NT) {
    const uint32_t x = a.tbl[i];
    const uint32_t bin = (x & 0x7FFEu) / 1152u;
    m.tbl[i] = (x & 0xFFFF8001u) | (bin << 11);
  }
  const uint8_t* const tb8 = (const uint8_t*)m.tbl;
  for (int i = tid; i < 16 * ROW; i += NT) m.cells[i] = 0u;
  for (int i = tid; i < LSLOTS; i += NT) { m.lhash[i] = 0ull; m.lcount[i] = 0u; m.lminw[i] = UINT32_MAX; }
  if (tid < 64) m.misc[tid] = 0u;
  if (tid == 0) {
    mbar_init(m.mbar, 1);
    fence_mbar_init();
  }
  const uint64_t E8 = a.E & ~7ull;
  const uint64_t NI = umin64(*a.n_items, a.n_tiles);
  uint32_t* const sched = m.misc + 8;
  __syncthreads();
  auto grab = [&]() -> uint64_t { return umin64(atomicAdd(a.counter, 1u), NI); };
  uint32_t phase = 0u;
  bool staged = false;  // thread 0: the next chunk to process is already in flight
  if (tid == 0) {
    const uint64_t x = grab();
    sched[0] = (uint32_t)x;
    sched[1] = (uint32_t)(x < NI ? grab() : NI);
    if (x < NI) {
      uint64_t w0, w1;
      item_range(a, x, w0, w1);
      const uint64_t te = umin64(a.weo[w1], a.E), ts = umin64(a.weo[w0], te);
      if (te > ts) {
        stage_chunk(a, m, plan(ts, te), E8);
        staged = true;
      }
    }
  }
  __syncthreads();
  uint64_t t = sched[0], tn = sched[1];
  uint64_t my_off = 0;      // weo[w0 + tid] of the current item
  uint64_t my_last = 0;     // thread 0: weo[w1] of the current item
  uint32_t my_k = 0;        // kernel of the item's first warp
  uint64_t my_kb = ~0ull;   // start of the kernel after it
  if (t < NI) {
    uint64_t w0, w1;
    item_range(a, t, w0, w1);
    my_off = a.weo[w0 + umin64((uint64_t)tid, w1 - w0)];
    if (tid == 0) my_last = a.weo[w1];
    if (fused) {
      my_k = a.tile_k0[t];
      my_kb = my_k + 1 < a.K ? a.kwo[my_k + 1] : ~0ull;
    }
  }
  uint32_t raw = 0, orr = 0;

  while (t < NI) {
    uint64_t w0, w1;
    item_range(a, t, w0, w1);
    const uint32_t nw = (uint32_t)(w1 - w0);
    const uint64_t w = w0 + tid;
    const bool valid = w < w1;
    if ((uint32_t)tid < nw) m.off[tid] = my_off;
    if (tid == 0) m.off[nw] = my_last;
    // the next item's offsets (read at this item's end) and the item after next (claimed now, read at the end)
    uint64_t nx_off = 0, nx_last = 0;
    uint32_t nx_k = 0;
    uint32_t x_after = 0;
    if (tid == 0 && tn < NI) x_after = atomicAdd(a.counter, 1u);
    // the next item's warp range is loaded now; the dependent offset loads are issued once it has surely arrived
    // (before the first chunk's event loop), so no warp waits on the two-step chain
    uint64_t nr0 = 0, nr1 = 0;
    bool nx_issued = !(tn < NI);
    if (tn < NI) {
      nr0 = a.item_w0[tn];
      nr1 = a.item_w0[tn + 1];
      if (fused) nx_k = a.tile_k0[tn];
    }
    auto issue_next = [&]() {
      if (nx_issued) return;
      nx_issued = true;
      const uint64_t n0 = umin64(nr0, a.W), n1 = umin64(umin64(umax64(nr1, n0), n0 + NT), a.W);
      nx_off = a.weo[n0 + umin64((uint64_t)tid, n1 - n0)];
      if (tid == 0) nx_last = a.weo[n1];
    };
    __syncthreads();
    // item bounds; non-monotone offsets are latched and made monotone (memory safety of the lane walks)
    const uint64_t te = umin64(m.off[nw], a.E), ts = umin64(m.off[0], te);
    bool bad = false;
    if ((uint32_t)tid < nw) bad = m.off[tid + 1] < m.off[tid];
    if (__syncthreads_or(bad)) {
      if (tid == 0) {
        latch(a.err, PHOTON_ERANGE, (int64_t)w0);
        uint64_t mx = ts;
        for (uint32_t u = 0; u <= nw; ++u) { mx = umax64(mx, umin64(m.off[u], te)); m.off[u] = mx; }
      }
      __syncthreads();
    }
    for (uint32_t u = tid; u <= nw; u += NT) m.off[u] = umin64(umax64(m.off[u], ts), te);
    if (tid < 3) m.off[nw + 1 + tid] = te;
    // this warp's key (thread tid <-> warp w0 + tid for the whole item); I = its instruction total (u64)
    uint32_t p[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) p[j] = 0u;
    uint64_t I = 0;
    __syncthreads();

    for (uint64_t cs = ts; cs < te;) {
      const Chunk c = plan(cs, te);
      const uint64_t ce = c.a8 + c.hi;
      const uint32_t nwd = (c.hi + 7) >> 3;
      const uint32_t Q = (((nwd + NT - 1) / NT) | 1u);
      const uint32_t L = Q * 8u;
      // x / L == umulhi(x >> 3, ceil(2^32 / Q)) for x < 2^20
      const uint32_t qinv = Q == 3u ? 0x55555556u : Q == 5u ? 0x33333334u : Q == 7u ? 0x24924925u : 0x1C71C71Du;
      auto divL = [&](uint32_t x) -> uint32_t { return Q == 1u ? (x >> 3) : __umulhi(x >> 3, qinv); };
      const uint32_t LIM = CHE + 16u;
      auto relx = [&](uint64_t x) -> uint32_t { return x <= c.a8 ? 0u : (x - c.a8 >= LIM ? LIM : (uint32_t)(x - c.a8)); };
      // [A] chunk-relative warp starts; the previous chunk's (or item's) cells cleared with 16-byte stores
      for (uint32_t u = tid; u < nw + 4; u += NT) m.rel[u] = relx(m.off[u]);
#pragma unroll
      for (int i = 0; i < (int)(kCellBytes / 16 / NT); ++i) ((uint4*)m.cells)[i * NT + tid] = make_uint4(0u, 0u, 0u, 0u);
      __syncthreads();
      const uint32_t nact = divL(c.hi + L - 1);  // lanes with events
      // [B] my lane's first warp: the last warp starting at or before my first event (empty warps start where the
      // next one does, so the search lands on the non-empty one); a proportional guess, then a search
      const bool act = (uint32_t)tid < nact;
      uint32_t myfw = 0;
      if (act) {
        const uint32_t r = umax((uint32_t)tid * L, c.lo);
        uint32_t lo = 0, hi = nw - 1;
        uint32_t g = umin((uint32_t)((float)r * ((float)nw / (float)c.hi)), nw - 1);
#pragma unroll
        for (int step = 0; step < 3; ++step) {
          if (m.rel[g] > r && g > 0) --g;
          else if (g + 1 < nw && m.rel[g + 1] <= r) ++g;
        }
        if (m.rel[g] <= r && (g + 1 == nw || m.rel[g + 1] > r)) {
          lo = g;
        } else {
          while (lo < hi) {
            const uint32_t mid = (lo + hi + 1) >> 1;
            if (m.rel[mid] <= r) lo = mid; else hi = mid - 1;
          }
        }
        myfw = lo;
      }
      if (tid == 0 && !staged) stage_chunk(a, m, c, E8);  // not prefetched (the previous item had no events)
      issue_next();
      // [C] accumulate my lane range
      mbar_wait(m.mbar, phase);
      phase ^= 1u;
      if (act) {
        const uint32_t t0 = (uint32_t)tid;
        const uint32_t r = umax(t0 * L, c.lo), e = umin((t0 + 1) * L, c.hi);
        const uint4* sb4 = (const uint4*)m.stage + t0 * Q;
        uint32_t u = myfw;
        uint32_t nb = m.rel[u + 1], nb2 = m.rel[u + 2];
        uint32_t col = cbase + t0 * 4u, coln = cbase + (NT + u + 1) * 4u;
        const uint32_t kn = umin(Q, (e - t0 * L + 7u) >> 3);  // words holding my events
        auto lookup = [&](const uint4& v, uint32_t (&tv)[8]) {
          tv[0] = *(const uint32_t*)(tb8 + ((v.x << 2) & mask4));
          tv[1] = *(const uint32_t*)(tb8 + ((v.x >> 14) & mask4));
          tv[2] = *(const uint32_t*)(tb8 + ((v.y << 2) & mask4));
          tv[3] = *(const uint32_t*)(tb8 + ((v.y >> 14) & mask4));
          tv[4] = *(const uint32_t*)(tb8 + ((v.z << 2) & mask4));
          tv[5] = *(const uint32_t*)(tb8 + ((v.z >> 14) & mask4));
          tv[6] = *(const uint32_t*)(tb8 + ((v.w << 2) & mask4));
          tv[7] = *(const uint32_t*)(tb8 + ((v.w >> 14) & mask4));
        };
        // software pipeline: word k+1 is loaded (stage, then table) while word k's adds are issued
        uint4 vnx = sb4[0];
        uint32_t tv[8];
        lookup(vnx, tv);
        for (uint32_t k = 0; k < kn; ++k) {
          const uint32_t p0 = (t0 * Q + k) * 8u;
          raw |= (vnx.x | vnx.y) | (vnx.z | vnx.w);
          vnx = sb4[k + 1 < kn ? k + 1 : k];
          if (CHECK_MARK) orr |= (tv[0] | tv[1] | tv[2] | tv[3]) | (tv[4] | tv[5] | tv[6] | tv[7]);
          const bool fast = p0 >= r && p0 + 8u <= e && nb2 >= p0 + 8u;  // nb2 >= nb: at most one boundary
          if (fast) {
            const uint32_t mcut = nb - p0;  // events j >= mcut belong to the next warp
#pragma unroll
            for (int j = 0; j < 8; ++j) red_add(((uint32_t)j < mcut ? col : coln) | (tv[j] & TOFF), tv[j] >> TSH);
            if (nb <= p0 + 8u) {  // crossed into the next warp
              ++u;
              col = coln;
              coln += 4u;
              nb = nb2;
              nb2 = m.rel[u + 2];
            }
          } else {
            // partial word (chunk edge) or several warp boundaries in the word: event by event
#pragma unroll
            for (uint32_t j = 0; j < 8; ++j) {
              const uint32_t pos = p0 + j;
              if (pos < r || pos >= e) continue;
              while (pos >= nb && u < nw) {
                ++u;
                nb = m.rel[u + 1];
              }
              red_add((cbase + colof(t0, myfw, u)) | (tv[j] & TOFF), tv[j] >> TSH);
            }
            while (p0 + 8u < e && nb <= p0 + 8u && u < nw) {  // the next word starts in a later warp
              ++u;
              nb = m.rel[u + 1];
            }
            col = cbase + colof(t0, myfw, u);
            coln = cbase + (NT + u + 1) * 4u;
            nb2 = m.rel[u + 2];
          }
          lookup(vnx, tv);
        }
      }
      __syncthreads();  // pieces complete; the stage is free
      // stage the next chunk (this item's next, else the next item's first) while the pieces are collected
      if (tid == 0) {
        staged = false;
        const uint64_t nte = umin64(nx_last, a.E), nts = umin64(nx_off, nte);
        if (ce < te) {
          stage_chunk(a, m, plan(ce, te), E8);
          staged = true;
        } else if (tn < NI && nte > nts) {
          stage_chunk(a, m, plan(nts, nte), E8);
          staged = true;
        }
      }
      // [D] each warp with events in this chunk sums its pieces (its owner column in the lane holding its first
      // event here, then slot 0 of each later lane it spans) into its key registers
      if (valid) {
        const uint32_t x0 = umax(m.rel[tid], c.lo), x1 = umin(m.rel[tid + 1], c.hi);
        if (x0 < x1) {
          const uint32_t ta = divL(x0), tb = divL(x1 - 1);
          // owner column: slot 0 of lane ta when the warp is that lane's first piece, else the warp's pool column
          uint32_t oc = x0 == umax(ta * L, c.lo) ? ta : NT + (uint32_t)tid;
          for (uint32_t tt = ta;;) {
#pragma unroll
            for (int j = 0; j < 16; ++j) p[j] += m.cells[j * ROW + oc];
            if (++tt > tb) break;
            oc = tt;
          }
          // the chunk added < 2^31 (<= CHE events of length < 2^17): the exact u64 total follows from the u32 sum
          uint32_t sum = 0;
#pragma unroll
          for (int j = 0; j < 16; ++j) sum += p[j];
          I += (uint32_t)(sum - (uint32_t)I);
        }
      }
      cs = ce;
      __syncthreads();  // pieces read; rel / fw / pb free for the next chunk
    }

    // ---- finalise the item ----
    issue_next();  // items without events
    const uint64_t s = m.off[tid <= (int)nw ? tid : nw], e = m.off[tid < (int)nw ? tid + 1 : nw];
    const int bad_here = ((((raw | (raw >> 16)) & 0xFFFFu) & ~bmask) != 0u || (CHECK_MARK && (orr & 1u))) ? 1 : 0;
    if (__syncthreads_or(bad_here)) {
      if (valid) report_bad_event(a, s, e);
      raw = 0;
      orr = 0;
    }
    uint32_t k = my_k;
    if (valid) {
      if (I >= kInstsLimit) latch(a.err, PHOTON_ERANGE, (int64_t)w);
      if (a.warp_bbv16) {
        uint4* dst = (uint4*)(a.warp_bbv16 + w * 16);
        dst[0] = make_uint4(p[0], p[1], p[2], p[3]);
        dst[1] = make_uint4(p[4], p[5], p[6], p[7]);
        dst[2] = make_uint4(p[8], p[9], p[10], p[11]);
        dst[3] = make_uint4(p[12], p[13], p[14], p[15]);
      }
      if (a.warp_insts) a.warp_insts[w] = I;
      if (fused && w >= my_kb) {  // the item crosses into later kernels
        ++k;
        while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
      }
    }
    if (fused) item_group(a, m, t, w0, valid, k, p);
    my_off = nx_off;
    my_last = nx_last;
    if (fused && tn < NI) {
      my_k = nx_k;
      my_kb = my_k + 1 < a.K ? a.kwo[my_k + 1] : ~0ull;
    }
    if (tid == 0) sched[1] = (uint32_t)(tn < NI ? umin64(x_after, NI) : NI);
    __syncthreads();
    t = tn;
    tn = sched[1];
  }
  // the unused rest of the CTA's overflow block: count 0 marks an entry the insertion skips
  if (fused) {
    const uint64_t nxt = *(const uint64_t*)(m.misc + 2), end = umin64(*(const uint64_t*)(m.misc + 4), a.te.ovf_cap);
    for (uint64_t j = nxt + tid; j < end; j += NT) a.te.ovf[j].count = 0u;
  }
}

}  // namespace

bool bbv2_supported(uint32_t B) { return next_pow2_u32(B < 16 ? 16 : B) <= (uint32_t)SMEM_TBL_MAX; }

cudaError_t launch_bbv2(const TraceDev& t, const uint32_t* tbl, const ItemTable& it, uint32_t* warp_bbv16,
                        uint64_t* warp_insts, const TileEntries* te, DevErr* err, int num_sms, cudaStream_t s) {
  Args a{};
  a.kwo = t.kwo; a.weo = t.weo; a.bb = t.bb; a.tbl = tbl; a.tile_k0 = it.k0;
  a.item_w0 = it.w0; a.n_items = it.n; a.counter = it.n + 1;
  a.K = t.K; a.B = t.B; a.P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  a.W = t.W; a.E = t.E;
  a.warp_bbv16 = warp_bbv16; a.warp_insts = warp_insts;
  if (te) a.te = *te;
  a.err = err;
  a.n_tiles = it.cap;
  if (t.W == 0) return cudaSuccess;
  if (a.P2 > (uint32_t)SMEM_TBL_MAX) return cudaErrorNotSupported;
  cudaMemsetAsync(a.counter, 0, 4, s);
  const bool mark = a.P2 != t.B;
  int dev = 0, reserved = 0;
  cudaGetDevice(&dev);
  if (cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev) != cudaSuccess) reserved = 0;
  a.pre = (uint32_t)((32768 - reserved % 32768) % 32768);
  const size_t smem = smem_bytes(a.P2, a.pre);
  auto fn = mark ? k_bbv2<true> : k_bbv2<false>;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  int per_sm = 0;
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, NT, smem);
  if (e != cudaSuccess) return e;
  if (per_sm < 1) per_sm = 1;
  uint64_t grid = (uint64_t)num_sms * per_sm;
  if (grid > a.n_tiles) grid = a.n_tiles;
  if (grid == 0) return cudaSuccess;
  note_launch(), fn<<<(unsigned)grid, NT, smem, s>>>(a);
  return cudaGetLastError();
}

}  // namespace photon
