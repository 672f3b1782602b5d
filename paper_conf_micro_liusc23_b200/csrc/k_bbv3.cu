// k_bbv3.cu — A1 (per-warp BBV projected to 16 bins) fused with A2's de-duplication step: the streaming pass K1,
// plus the per-BB table, input validation, the unfused A2 de-duplication and the BB distribution (L208-210).
//
// PAPER.md: L161 (a BBV lists the basic blocks a warp executed), L154 (same instruction sequence => same BBV => same
// warp type), L178 ("project these BBVs into fixed-size BBVs (We use 16) to improve online clustering performance
// ... we can easily cluster the warps if they have the same BBV").  Readings [P-1] (entry = executions x length)
// and [P-2] (sum-preserving fold into 16 bins).  DESIGN.md §5.1.
//
// Design.  Per event the work is one BB-table lookup and one shared-memory add, so the pass is bound by
// shared-memory wavefronts and everything else is kept off that pipe and off CTA-wide barriers:
//  * Workers are hardware warps, independent of each other (no __syncthreads after the table load).  The analysed
//    warps are cut into blocks of 32 consecutive warps; worker g takes the blocks whose first event lies in its
//    1/G share of the trace (event-balanced contiguous ranges, found by a 32-ary search), so a worker sees few
//    kernels and few warp types.  Lane u owns warp u of the current block.
//  * A block's events are staged in chunks of <= 32*Q 16-byte words with cp.async.bulk (TMA copy engine) into a
//    per-worker buffer (K1_NBUF = 1, the default: chunk i+1 is issued right after chunk i's event loop and lands
//    during its collect / finalisation; K1_NBUF = 2 double-buffers at the cost of occupancy).
//  * A chunk is cut into 32 equal lane ranges (Q' words, Q' odd so the quarter-warp 16-byte loads hit distinct
//    bank groups).  Lane t walks its range; the piece of each analysed warp it meets is accumulated with
//    red.shared.add into a column private to the lane: the first piece into the lane's slot-0 column, a warp
//    starting inside the range into that warp's pool column (32 + u).  Columns of one worker lie side by side in
//    row arrays shared by GRP workers, so a cell address is column | (entry & row bits) — one LOP3 per event.
//  * Narrow mode (every BB length * 8Q < 2^16): cells are u16 pairs (row i holds bins 2i and 2i+1), halving the
//    cells to collect and clear.  Wide mode (longer BBs) uses u32 cells (one row per bin) and smaller chunks.
//  * After the loop each lane sums its warp's pieces (owner column, then slot 0 of every later lane it spans) into
//    16 key registers, carried across the chunks of a block; the worker's cells are cleared with 16-byte stores.
//  * Fused: at the block's end the keys are hashed, grouped with __match_any_sync plus an exact 17-word check, and
//    each distinct (kernel, key) of the block is looked up in the worker's 2-way set-associative cache of its recent
//    entries (hash -> entry id): a hit that matches the entry's own key exactly adds the block's count to it,
//    otherwise the key becomes a new 80-byte entry (key, first warp, kernel, count) from the worker's run of the
//    global entry pool (one atomic per ENT_BLK entries).  Each warp records its entry index (u32).  The entries
//    are inserted into the global type table afterwards (k_types.cu).
#include "internal.h"

namespace photon {

namespace {

#ifndef K1_WPC
#define K1_WPC 20
#endif
#ifndef K1_NBUF
#define K1_NBUF 1
#endif
constexpr int WPC = K1_WPC;         // workers (hardware warps) per CTA, one CTA per SM
constexpr int NBUF = K1_NBUF;       // staging buffers per worker (2: chunk i+1 in flight during chunk i; 1: issued
                                    // after chunk i's event loop, landing during its collect / finalisation)
constexpr int NCOL = 64;            // columns per worker: [0, 32) lane slot-0 columns, [32, 64) block-warp pool columns
constexpr int GRP = 4;              // workers sharing a row array (row stride GRP * NCOL * 4 = 1 KB)
constexpr uint32_t ROWB = GRP * NCOL * 4;
constexpr uint32_t ENT_BLK = 64;    // entries taken from the global pool at a time
constexpr int SMEM_TBL_MAX = 4096;  // BB table entries kept in shared memory (else read through L1)
#ifndef K1_PIN
#define K1_PIN 1
#endif
#ifndef K1_VNX
#define K1_VNX 1
#endif
#ifndef K1_QMAX
#define K1_QMAX 11
#endif
constexpr uint32_t NARROW_QMAX = K1_QMAX;  // odd, <= 17 (divL)
constexpr uint32_t kMarkN = 0x80000000u;  // neutral table: id in [B, P2)

// Narrow: u16 cells, entry = (bin odd ? len << 16 : len) | (bin >> 1) << 10 (len < 1024); mark = bit 31.
// Wide:   u32 cells, entry = len << 15 | bin << 10 (len < 2^17); mark = bit 14.
template <bool WIDE>
struct Mode;
template <>
struct Mode<false> {
  static constexpr uint32_t Q = NARROW_QMAX;
  static constexpr int ROWS = 8;
  static constexpr uint32_t ROFF = 0x1C00u;
  static constexpr uint32_t MARKB = 0x80000000u;
  __host__ __device__ static constexpr uint32_t entry(uint32_t len, uint32_t bin) {
    return ((bin & 1u) ? (len << 16) : len) | ((bin >> 1) << 10);
  }
  __device__ static __forceinline__ uint32_t val(uint32_t e) { return e & 0x03FF03FFu; }
};
template <>
struct Mode<true> {
  static constexpr uint32_t Q = 7;
  static constexpr int ROWS = 16;
  static constexpr uint32_t ROFF = 0x3C00u;
  static constexpr uint32_t MARKB = 0x4000u;
  __host__ __device__ static constexpr uint32_t entry(uint32_t len, uint32_t bin) { return (len << 15) | (bin << 10); }
  __device__ static __forceinline__ uint32_t val(uint32_t e) { return e >> 15; }
};
static_assert(Mode<false>::entry(1023, 15) == ((1023u << 16) | (7u << 10)), "narrow entry layout");
// a narrow lane range holds <= 8Q events; their per-bin sum must stay below 2^16 in a u16 cell
__host__ __device__ constexpr bool narrow_ok(uint32_t max_len) { return max_len * (NARROW_QMAX * 8) < 65536u; }

struct Args3 {
  const uint64_t* kwo;
  const uint64_t* weo;
  const uint16_t* bb;
  const uint32_t* tbl_mode;  // [P2] entries in this mode's format (GTBL lookups; copied to shared memory otherwise)
  const uint32_t* max_len;   // device: max bb_len (selects narrow / wide)
  uint32_t K, B, P2;
  uint64_t W, E;
  uint32_t* warp_bbv16;
  uint64_t* warp_insts;
  EntryPool ep;              // fused outputs (ep.ent == nullptr => not fused)
  DevErr* err;
  uint32_t off_tbl, off_misc, off_stage, off_cells;  // shared-memory layout (bytes)
};

// per-worker scratch in shared memory
#ifndef K1_NRANGE
#define K1_NRANGE 1  // ranges per worker: worker g takes parts g, g + G, ... of a cost partition into G * K1_NRANGE
#endif
#ifndef K1_CWAYS
#define K1_CWAYS 2  // entry-cache associativity (1, 2 or 4)
#endif
#ifndef K1_ENTCACHE
#define K1_ENTCACHE 128
#endif
constexpr int kEntCache = K1_ENTCACHE;
struct WMisc {
  uint32_t rel[40];             // chunk-relative starts of the block's warps (rel[nw..] = block end), clamped
  uint32_t fwt[32];             // first-warp scatter table of the lane ranges
  uint64_t mbar[2];
  // chunk issuer (lane 0)
  uint64_t i_b, i_cs, i_te, i_pf;
  uint32_t i_live, i_n, i_ri;
  uint64_t rlo[K1_NRANGE], rhi[K1_NRANGE];  // the worker's warp ranges (round-robin over the cost partition)
  // the worker's current block of pool entries (fused)
  uint64_t e_next, e_end;
  // K1_CWAYS-way set-associative cache of the worker's recent entries (hash -> entry id): a type seen again in a
  // later block of the worker adds to its entry after an exact key check instead of opening a new one
  uint64_t ch[kEntCache];
  uint32_t ce[kEntCache];
};
constexpr uint32_t kWMiscBytes = (sizeof(WMisc) + 127) & ~127u;

__device__ __forceinline__ void red_add(uint32_t saddr, uint32_t v) {
  // no "memory" clobber: cells are written only by these adds and read only after __syncwarp
  asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(saddr), "r"(v));
}
__device__ __forceinline__ uint32_t lds_u32(uint32_t saddr) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr) : "memory");
  return v;
}
// BB-table lookup: read-only while the kernel runs, so no volatile / memory clobber (free scheduling)
__device__ __forceinline__ uint32_t lds_tbl(uint32_t saddr) {
  uint32_t v;
  asm("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(saddr));
  return v;
}
__device__ __forceinline__ void sts_v4_zero(uint32_t saddr) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %1, %1, %1};" ::"r"(saddr), "r"(0u) : "memory");
}

// first index b in [lo, hi] with b == hi or f(b) >= T (f monotone); 32-ary search, all lanes participate
template <class F>
__device__ __forceinline__ uint64_t search32(uint64_t lo, uint64_t hi, F f, uint64_t T) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t end = hi;
  while (lo < hi) {
    const uint64_t span = hi - lo;
    const uint64_t q = span <= 32 ? lo + lane : lo + (uint64_t)((double)span * (lane + 1) / 33.0);
    const uint64_t qq = q < hi ? q : hi;
    const bool pred = q <= hi && (qq == end || f(qq) >= T);
    const unsigned m = __ballot_sync(0xffffffffu, pred);
    if (m) {
      const int i = __ffs(m) - 1;
      const uint64_t qi = __shfl_sync(0xffffffffu, qq, i);
      const uint64_t qp = i ? __shfl_sync(0xffffffffu, qq, i - 1) + 1 : lo;
      hi = qi;
      lo = span <= 32 ? qi : umin64(qp, qi);
    } else {
      lo = umin64(__shfl_sync(0xffffffffu, qq, 31) + 1, hi);
    }
  }
  return hi;
}

// Slow path (bad input only): first event of [s, e) whose id is >= B.
__device__ void report_bad_event(const Args3& a, uint64_t s, uint64_t e) {
  for (uint64_t i = s; i < e; ++i)
    if (a.bb[i] >= a.B) { latch(a.err, PHOTON_ERANGE, (int64_t)i); return; }
}

// Grouping hash (bucketing only; equality is always verified on the full key): 32x32->64-bit multiply-adds with
// distinct odd multipliers, then a 64-bit finaliser.
__device__ __forceinline__ uint64_t hash16(uint32_t k, const uint32_t* p) {
  constexpr uint32_t M[17] = {0x9E3779B1u, 0x85EBCA77u, 0xC2B2AE3Du, 0x27D4EB2Fu, 0x165667B1u, 0xD3A2646Du,
                              0xFD7046C5u, 0xB55A4F09u, 0x7FEB352Du, 0x846CA68Bu, 0x6C8E9CF5u, 0xCC9E2D51u,
                              0x1B873593u, 0xE6546B65u, 0x85EBCA6Bu, 0xC2B2AE35u, 0x2545F491u};
  uint64_t h = (uint64_t)k * M[16] + 0x632BE59BD9B4E019ull;
#pragma unroll
  for (int j = 0; j < 16; ++j) h += (uint64_t)p[j] * M[j];
  h = mix64(h ^ (h >> 29));
  return h ? h : 1;
}

__device__ __forceinline__ void pool_init(WMisc* wm) {
  if ((threadIdx.x & 31) == 0) { wm->e_next = 0; wm->e_end = 0; }
  for (int i = threadIdx.x & 31; i < kEntCache; i += 32) wm->ch[i] = 0;
  __syncwarp();
}
__device__ __forceinline__ void pool_flush(const Args3& a, WMisc* wm) {
  const uint32_t lane = threadIdx.x & 31;
  __syncwarp();
  for (uint64_t j = wm->e_next + lane; j < wm->e_end; j += 32)  // the unused rest of the worker's entry block
    if (j < a.ep.cap) a.ep.ent[j].count = 0u;
}

// Fused finalisation of one block: lanes < nw hold warp (w0 + lane)'s key p and kernel k.  Distinct keys are found
// with __match_any_sync on a hash plus an exact 17-word check; each distinct key's leader writes one pool entry
// (key, kernel, count, first warp) at a consecutive index of the worker's entry block, and every warp records its
// leader's entry.  k_entries_insert merges the entries of all blocks into the global type table.
__device__ void finalize_fused(const Args3& a, WMisc* wm, uint64_t w0, bool valid, uint32_t k, const uint32_t* p) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t h = valid ? hash16(k, p) : 0ull;
  const unsigned vmask = __ballot_sync(0xffffffffu, valid);
  const unsigned peers = __match_any_sync(0xffffffffu, (unsigned long long)h);
  const int leader = __ffs(peers) - 1;
  bool eq = __shfl_sync(0xffffffffu, k, leader) == k;
#pragma unroll
  for (int j = 0; j < 16; ++j) eq &= (__shfl_sync(0xffffffffu, p[j], leader) == p[j]);  // no short circuit
  const unsigned eqm = __ballot_sync(0xffffffffu, eq);
  const bool is_l = valid && ((int)lane == leader || !eq);
  const uint32_t cnt = ((int)lane == leader) ? (uint32_t)__popc(peers & eqm & vmask) : 1u;
  // the worker's entry cache: an exact (kernel, key) match adds this block's count to the existing entry
  uint32_t hit = UINT32_MAX;
  // K1_CWAYS-way set-associative: set (h mod kEntCache / ways) at cslot, most recent way first
  constexpr uint32_t NWAY = K1_CWAYS;
  const uint32_t cslot = ((uint32_t)h & (kEntCache / NWAY - 1)) * NWAY;
  uint32_t cway = cslot;
#pragma unroll
  for (uint32_t q = NWAY - 1; q > 0; --q)
    if (wm->ch[cslot + q] == h) cway = cslot + q;
  if (is_l && wm->ch[cway] == h) {
    const uint32_t e = wm->ce[cway];
    if (e < a.ep.cap) {  // the exact check against the entry itself (written by this warp earlier)
      TileEntry* d = a.ep.ent + e;
      const uint4* kd = (const uint4*)d->key;
      bool same = d->kernel == k;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint4 v = kd[q];
        same &= v.x == p[4 * q] && v.y == p[4 * q + 1] && v.z == p[4 * q + 2] && v.w == p[4 * q + 3];
      }
      if (same) {
        atomicAdd(&d->count, cnt);
        hit = e;
      }
    }
  }
  const bool alloc = is_l && hit == UINT32_MAX;
  const unsigned lm = __ballot_sync(0xffffffffu, alloc);
  const uint32_t nl = __popc(lm), rank = __popc(lm & ((1u << lane) - 1u));
  // entry ids: the rest of the worker's block, then a new block of ENT_BLK (one atomic per ENT_BLK entries)
  uint64_t e_next = wm->e_next, e_end = wm->e_end;
  const uint32_t room = (uint32_t)(e_end - e_next);
  uint64_t id;
  if (nl > room) {
    uint64_t pos = 0;
    if (lane == 0) {
      pos = atomicAdd((unsigned long long*)a.ep.count, (unsigned long long)ENT_BLK);
      if (pos + ENT_BLK > a.ep.cap) latch(a.err, PHOTON_ECAPACITY, (int64_t)pos);
    }
    pos = __shfl_sync(0xffffffffu, pos, 0);
    id = rank < room ? e_next + rank : pos + (rank - room);
    e_next = pos + (nl - room);
    e_end = pos + ENT_BLK;
  } else {
    id = e_next + rank;
    e_next += nl;
  }
  if (alloc && id < a.ep.cap) {
    TileEntry* d = a.ep.ent + id;
    uint4* kd = (uint4*)d->key;
    kd[0] = make_uint4(p[0], p[1], p[2], p[3]);
    kd[1] = make_uint4(p[4], p[5], p[6], p[7]);
    kd[2] = make_uint4(p[8], p[9], p[10], p[11]);
    kd[3] = make_uint4(p[12], p[13], p[14], p[15]);
    const uint64_t w = w0 + lane;
    kd[4] = make_uint4((uint32_t)w, (uint32_t)(w >> 32), k, cnt);  // first warp, kernel, count
  }
  __syncwarp();
  // remember the new entries: one writer per slot (the lowest allocating lane mapping to it; every hit is checked
  // against the entry's own key anyway)
  const unsigned same_slot = __match_any_sync(0xffffffffu, alloc ? cslot : 0xFFFFFFFFu);
  if (alloc && (int)lane == __ffs(same_slot) - 1) {
#pragma unroll
    for (uint32_t q = NWAY - 1; q > 0; --q) {  // the set's entries move one way down
      wm->ch[cslot + q] = wm->ch[cslot + q - 1];
      wm->ce[cslot + q] = wm->ce[cslot + q - 1];
    }
    wm->ch[cslot] = h;
    wm->ce[cslot] = (uint32_t)umin64(id, 0xFFFFFFFFull);
  }
  if (lane == 0) { wm->e_next = e_next; wm->e_end = e_end; }
  __syncwarp();
  const uint32_t ent = alloc ? (uint32_t)umin64(id, 0xFFFFFFFFull) : hit;
  const uint32_t le = __shfl_sync(0xffffffffu, ent, leader);
  if (valid) a.ep.gid[w0 + lane] = (eq && (int)lane != leader) ? le : ent;
}

// cells: byte address of (row 0, column 0) of this worker
template <bool WIDE>
__device__ __forceinline__ void clear_cells(uint32_t cw) {
  constexpr int ROWS = Mode<WIDE>::ROWS;
  const uint32_t lane = threadIdx.x & 31;
  // a worker's 64 columns of one row are 256 contiguous bytes = 16 uint4: two rows per pass
#pragma unroll
  for (int i = 0; i < ROWS / 2; ++i) {
    const uint32_t r = 2 * i + (lane >> 4);
    sts_v4_zero(cw + r * ROWB + (lane & 15) * 16);
  }
}

// x / L for L = 8 Qe, Qe odd <= 17, x < 2^20: umulhi(x >> 3, ceil(2^32 / Qe))
__constant__ uint32_t kQinv[9] = {0u,          0x55555556u, 0x33333334u, 0x24924925u, 0x1C71C71Du,
                                  0x1745D175u, 0x13B13B14u, 0x11111112u, 0x0F0F0F10u};  // Qe = 1, 3, ..., 17
__device__ __forceinline__ uint32_t qinv_of(uint32_t Qe) { return kQinv[Qe >> 1]; }  // ceil(2^32 / Qe), odd Qe
__device__ __forceinline__ uint32_t divL(uint32_t x, uint32_t Qe, uint32_t qinv) {
  return Qe == 1u ? (x >> 3) : __umulhi(x >> 3, qinv);
}

#ifndef K1_ALPHA
#define K1_ALPHA 48
#endif
constexpr uint64_t kAlpha = K1_ALPHA;  // per-warp cost of a block in event units (worker balance: events + kAlpha * warps)

template <bool WIDE, bool GTBL, bool MARK, bool FUSED>
__global__ void __launch_bounds__(WPC * 32, 1) k_bbv3(Args3 a) {
  using M = Mode<WIDE>;
  constexpr uint32_t Q = M::Q, CW = 32 * Q, CE = CW * 8;
  static_assert((uint64_t)CE * kMaxLen < (1ull << 32), "a chunk adds < 2^32 to a warp's bins (u32 delta of I)");
  constexpr int ROWS = M::ROWS;
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (narrow_ok(*a.max_len) == WIDE) return;  // the other variant's launch handles this trace
  uint32_t* tbl_s = (uint32_t*)(smem + a.off_tbl);
  if (!GTBL) {
    for (uint32_t i = threadIdx.x; i < a.P2; i += blockDim.x) tbl_s[i] = a.tbl_mode[i];
    __syncthreads();
  }
  const uint32_t* __restrict__ tbl_g = a.tbl_mode;
  const uint32_t tbase = smem_u32(tbl_s);
  if (!GTBL && (tbase & (a.P2 * 4u - 1u)) != 0u) {  // the OR addressing of the table needs it aligned to its size
    if (threadIdx.x == 0) latch(a.err, PHOTON_ECUDA, -3);
    return;
  }
  const uint32_t bmask = a.P2 - 1, mask4 = bmask << 2;
  WMisc* wm = (WMisc*)(smem + a.off_misc + wid * kWMiscBytes);
  uint4* stage0 = (uint4*)(smem + a.off_stage + wid * NBUF * CW * 16);
  const uint32_t cw = smem_u32(smem + a.off_cells + (wid / GRP) * ROWS * ROWB) + (wid % GRP) * NCOL * 4;
  // the OR addressing needs the row array aligned to its size
  if (((cw - (wid % GRP) * NCOL * 4) & (ROWS * ROWB - 1)) != 0u) {
    if (lane == 0) latch(a.err, PHOTON_ECUDA, -2);
    return;
  }
  clear_cells<WIDE>(cw);
  // every RED lands in this worker's 64 columns of its row array (debug build: checked)
  auto red = [&](uint32_t ad, uint32_t v) {
    PHOTON_DCHECK((ad - (cw - (wid % GRP) * NCOL * 4)) < ROWS * ROWB &&
                      (((ad - (cw - (wid % GRP) * NCOL * 4)) & (ROWB - 1)) - (wid % GRP) * NCOL * 4) < NCOL * 4,
                  "K1 cell address outside the worker's columns", ad);
    red_add(ad, v);
  };
  if (FUSED) pool_init(wm);
  if (lane == 0) {
    mbar_init(&wm->mbar[0], 1);
    mbar_init(&wm->mbar[1], 1);
    fence_mbar_init();
  }

  const uint64_t W = a.W, E = a.E, E8 = E & ~7ull;
  const uint32_t NWK = gridDim.x * WPC, gw = blockIdx.x * WPC + wid;
  // worker gw takes the warps whose cost(w) = start(w) + kAlpha * w lies in parts gw, gw + G, ... of a partition of
  // the cost into G * K1_NRANGE equal parts (G workers; the last part: all remaining warps, trailing empty warps
  // included), each in blocks of up to 32 consecutive warps from its first warp.  Warp-granular parts (not whole
  // 32-warp blocks) let a group of long warps -- VGG's fully connected layers, ~150K events per 32 warps -- spread
  // over several workers; several parts per worker average out regional cost differences.
  const uint64_t C = E + kAlpha * W;
  const uint64_t NP = (uint64_t)NWK * K1_NRANGE;
  auto wcost = [&](uint64_t w) -> uint64_t { return a.weo[w] + kAlpha * w; };
  auto part_lo = [&](uint64_t j) -> uint64_t {
    if (j == 0) return 0;
    if (j >= NP) return W;
    return search32(0, W, wcost, (uint64_t)(((unsigned __int128)C * j) / NP));
  };
#pragma unroll 1
  for (int ri = 0; ri < K1_NRANGE; ++ri) {
    const uint64_t j = (uint64_t)ri * NWK + gw;
    const uint64_t lo = part_lo(j), hi = part_lo(j + 1);
    if (lane == 0) { wm->rlo[ri] = lo; wm->rhi[ri] = hi; }
  }
  __syncwarp();
  auto clampE = [&](uint64_t x) -> uint64_t { return x < E ? x : E; };

  // ---- chunk issuer (lane 0): stages the worker's chunk sequence one chunk ahead.  State in shared memory except
  // the prefetched raw end of the block after the issuer's (a register, so its load is not waited on early).
  uint64_t i_pf = 0;
  auto i_enter = [&](uint32_t ri) {  // lane 0: the first non-empty range from ri on (i_live = 0: none)
    while (ri < K1_NRANGE && wm->rlo[ri] >= wm->rhi[ri]) ++ri;
    wm->i_ri = ri;
    wm->i_live = ri < K1_NRANGE ? 1u : 0u;
    if (ri >= K1_NRANGE) return;
    const uint64_t lo = wm->rlo[ri], hi = wm->rhi[ri];
    const uint64_t s0 = clampE(a.weo[lo]);
    const uint64_t e_raw = a.weo[umin64(lo + 32, hi)];
    wm->i_b = lo;  // first warp of the issuer's block
    wm->i_cs = s0;
    wm->i_te = umax64(clampE(e_raw), s0);
    wm->i_pf = e_raw;  // raw end of the block (= raw start of the next block)
    i_pf = a.weo[umin64(lo + 64, hi)];
  };
  if (lane == 0) {
    wm->i_n = 0;
    i_enter(0);
  }
  auto issue = [&]() {  // lane 0 only
    if (!wm->i_live) return;
    const uint32_t n = wm->i_n;
    const uint32_t buf = NBUF == 2 ? (n & 1u) : 0u;
    uint4* dst = stage0 + buf * CW;
    const uint64_t cs = wm->i_cs, te = wm->i_te;
    const uint64_t a8 = cs & ~7ull;
    const uint64_t ce = umin64(te, a8 + CE);
    const uint64_t w_a = a8 >> 3, wend = (ce + 7) >> 3;  // words [w_a, wend)
    const uint64_t bulk_end = umin64(wend, E8 >> 3);
    const uint32_t bytes = bulk_end > w_a ? (uint32_t)((bulk_end - w_a) * 16) : 0u;
    if (wend > (E8 >> 3) && wend > w_a) {  // the last partial word of the trace: zero-filled
      const uint64_t wd = wend - 1;
      uint16_t* d16 = (uint16_t*)(dst + (wd - w_a));
      for (int j = 0; j < 8; ++j) d16[j] = (wd * 8 + j) < E ? a.bb[wd * 8 + j] : (uint16_t)0;
    }
    mbar_arrive_expect_tx(&wm->mbar[buf], bytes);
    if (bytes) bulk_g2s(dst, a.bb + a8, bytes, &wm->mbar[buf]);
    wm->i_n = n + 1;
    if (ce < te) {
      wm->i_cs = ce;
    } else {  // the next block starts where this one ends
      const uint64_t nw0 = wm->i_b + 32;
      const uint64_t rhi = wm->rhi[wm->i_ri];
      if (nw0 < rhi) {
        wm->i_b = nw0;
        wm->i_cs = te;
        wm->i_te = umax64(clampE(i_pf), te);
        wm->i_pf = i_pf;
        i_pf = a.weo[umin64(nw0 + 64, rhi)];
      } else {
        i_enter(wm->i_ri + 1);
      }
    }
  };
  if (lane == 0) issue();
  __syncwarp();

  uint32_t n_done = 0;  // chunks consumed
  uint64_t prev_te = 0;
  uint32_t raw = 0, orr = 0;
#pragma unroll 1
  for (int ri = 0; ri < K1_NRANGE; ++ri) {
  const uint64_t r_lo = wm->rlo[ri], r_hi = wm->rhi[ri];
  // ---- per-block state (all lanes) ----
  uint64_t w0 = r_lo;              // first warp of the current block
  uint64_t my_s = 0, blk_end = 0;  // weo[w0 + lane], weo[min(w0 + 32, r_hi)] (raw)
  if (w0 < r_hi) {
    my_s = a.weo[umin64(w0 + lane, r_hi)];
    blk_end = a.weo[umin64(w0 + 32, r_hi)];
  }
  // kernel of the block's first warp: last k with kwo[k] <= w0
  uint32_t kb = 0;
  if (w0 < r_hi && a.K > 1) {
    auto kf = [&](uint64_t kk) -> uint64_t { return a.kwo[kk]; };
    kb = (uint32_t)(search32(1, a.K, kf, w0 + 1) - 1);
  }
  uint64_t kb1 = kb + 1 < a.K ? a.kwo[kb + 1] : ~0ull;  // first warp of the next kernel (prefetched)

  while (w0 < r_hi) {
    const uint64_t start_b = __shfl_sync(0xffffffffu, my_s, 0);
    const uint32_t nw = (uint32_t)umin64(32, r_hi - w0);
    // prefetch the next block's starts (used at its start)
    uint64_t nx_s = 0, nx_end = 0;
    if (w0 + 32 < r_hi) {
      nx_s = a.weo[umin64(w0 + 32 + lane, r_hi)];
      nx_end = a.weo[umin64(w0 + 64, r_hi)];
    }
    // warp starts: lane u <= nw holds s_u; non-monotone offsets are latched and made monotone (memory safety)
    const uint64_t s_raw = lane < nw ? my_s : blk_end;
    const uint64_t s_next_raw = __shfl_down_sync(0xffffffffu, s_raw, 1);
    const bool bad = lane < nw && (lane + 1 < nw ? s_next_raw : blk_end) < s_raw;
    // the block's event range, exactly as the chunk issuer computes it: it starts where the previous block ended
    const uint64_t ts = w0 == r_lo ? clampE(start_b) : prev_te;
    const uint64_t te = umax64(clampE(blk_end), ts);
    uint64_t s = umin64(umax64(clampE(s_raw), ts), te);
    if (__any_sync(0xffffffffu, bad)) {
      const unsigned bm = __ballot_sync(0xffffffffu, bad);
      if (lane == 0) latch(a.err, PHOTON_ERANGE, (int64_t)(w0 + __ffs(bm) - 1));
      for (int o = 1; o < 32; o <<= 1) {  // inclusive max-scan over lanes: monotone starts (memory safety)
        const uint64_t y = __shfl_up_sync(0xffffffffu, s, o);
        if ((int)lane >= o) s = umax64(s, y);
      }
    }
    if (lane >= nw) s = te;
    prev_te = te;
    const uint64_t s_nx = __shfl_down_sync(0xffffffffu, s, 1);
    const uint64_t s_end = lane + 1 < nw ? s_nx : te;  // my warp's events: [s, s_end)
    // this warp's key (lane u <-> warp w0 + u for the whole block)
    uint32_t p[16];
#pragma unroll
    for (int j = 0; j < 16; ++j) p[j] = 0u;
    uint64_t I = 0;
    uint64_t cs = ts;
    do {  // chunks of the block (one empty chunk for a block without events)
      const uint64_t a8 = cs & ~7ull;
      const uint64_t ce = umin64(te, a8 + CE);
      const uint32_t lo = (uint32_t)(cs - a8), hi = (uint32_t)(ce - a8);
      const uint32_t LIM = CE + 16;
      auto relx = [&](uint64_t x) -> uint32_t {
        return x <= a8 ? 0u : (x - a8 >= LIM ? LIM : (uint32_t)(x - a8));
      };
      const uint32_t my_rel = relx(s), rel_te = relx(te);
      const uint32_t rel_nx = __shfl_down_sync(0xffffffffu, my_rel, 1);
      const uint32_t my_rel_end = lane + 1 < nw ? rel_nx : rel_te;
      // rel[u] = start of warp u (u < nw), rel[nw] = block end, beyond: "never" (the virtual warp after the block)
      wm->rel[lane] = lane <= nw ? my_rel : LIM;
      if (lane < 8) wm->rel[32 + lane] = lane + 32 == nw ? rel_te : LIM;
      const uint32_t buf = NBUF == 2 ? (n_done & 1u) : 0u, par = NBUF == 2 ? ((n_done >> 1) & 1u) : (n_done & 1u);
      ++n_done;
      if (NBUF == 2 && lane == 0) issue();  // the next chunk (this block's or the next block's) into the other buffer
      const uint32_t nwd = (hi + 7) >> 3;
      const uint32_t Qe = ((nwd + 31) >> 5) | 1u;
      const uint32_t L = Qe * 8u, qinv = qinv_of(Qe);
      // lane ranges: lane t covers chunk positions [max(tL, lo), min((t+1)L, hi)); its first warp fw(t) = the
      // last warp u with rel[u] <= max(tL, lo).  d_u = the first lane whose range start is >= rel[u]; the last
      // warp of each run of equal d writes itself at fwt[d]; fw = max-scan over lanes.
      const uint32_t d = my_rel <= lo ? 0u : divL(my_rel + L - 1u, Qe, qinv);
      const uint32_t d_nx = __shfl_down_sync(0xffffffffu, d, 1);
      wm->fwt[lane] = 0u;
      __syncwarp();
      if (lane < nw && d < 32u && (lane + 1 == nw || d_nx != d)) wm->fwt[d] = lane;
      __syncwarp();
      uint32_t myfw = wm->fwt[lane];
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, myfw, o);
        if ((int)lane >= o) myfw = umax(myfw, y);
      }
      mbar_wait(&wm->mbar[buf], par);
      const uint32_t t0 = lane;
      const uint32_t r = umax(t0 * L, lo), e = umin((t0 + 1) * L, hi);
      if (r < e) {
        // Pieces: the lane's first warp fw goes to its slot-0 column t0, a warp u starting inside the range to its
        // pool column 32 + u.  Pool column 32 is never a real piece (warp 0 is always lane 0's first warp), so it
        // is the scratch column for events outside the chunk: lane 0's first word before lo (a virtual warp
        // ending at lo) and the events past the block end in the last word (the virtual warp after nw - 1).
        const uint32_t scr = cw + 32u * 4u;
        // pool column of warp uu (1 <= uu <= 32); uu = 32 (after the block's last warp) wraps to the scratch
        // column 32, and a column 32 + uu with nw <= uu < 32 belongs to no warp: also scratch
        auto pcol = [&](uint32_t uu) -> uint32_t { return scr + ((uu & 31u) << 2); };
        const uint4* sb4 = stage0 + buf * CW + t0 * Qe;
        uint32_t u = myfw;
        uint32_t col, coln, nb, nb2;
        if (t0 == 0 && lo > 0) {  // virtual warp [0, lo) in the scratch column, then warp fw in slot 0
          col = scr;
          coln = cw;
          nb = lo;
          nb2 = wm->rel[u + 1];
          --u;  // (wraps for u = 0; only ever compared after the increment that follows the crossing)
        } else {
          col = cw + t0 * 4u;
          coln = pcol(u + 1);
          nb = wm->rel[u + 1];
          nb2 = wm->rel[u + 2];
        }
        const uint32_t kn = (e - t0 * L + 7u) >> 3;
        uint32_t tbr = tbase, m4r = mask4;
        auto look = [&](uint32_t x4) -> uint32_t {  // x4 = id * 4 (in the low bits, masked here)
          if (GTBL) return __ldg(tbl_g + ((x4 & m4r) >> 2));
          return lds_tbl((x4 & m4r) | tbr);  // the table is aligned to its size: one LOP3
        };
        // low halves: rotate left by 2 (one SHF; the wrapped bits fall outside mask4), high halves: shift right by 14
        auto lookup = [&](const uint4& v, uint32_t (&tv)[8]) {
          tv[0] = look(__funnelshift_l(v.x, v.x, 2));
          tv[1] = look(v.x >> 14);
          tv[2] = look(__funnelshift_l(v.y, v.y, 2));
          tv[3] = look(v.y >> 14);
          tv[4] = look(__funnelshift_l(v.z, v.z, 2));
          tv[5] = look(v.z >> 14);
          tv[6] = look(__funnelshift_l(v.w, v.w, 2));
          tv[7] = look(v.w >> 14);
        };
        uint4 vnx = sb4[0];
        uint32_t tv[8];
        lookup(vnx, tv);
        for (uint32_t kk = 0; kk < kn; ++kk) {
#if K1_PIN
          asm volatile("" : "+r"(tbr), "+r"(m4r));  // keep the table base and mask live (no per-word remat)
#endif
          const uint32_t p0 = (t0 * Qe + kk) * 8u;
          raw |= (vnx.x | vnx.y) | (vnx.z | vnx.w);
          PHOTON_DCHECK(t0 * Qe + kk + 1u <= CW, "K1 stage read past the worker's buffer", t0 * Qe + kk + 1u);
#if K1_VNX
          vnx = sb4[kk + 1];  // one word past the lane's range: always inside the allocation (unused at the end)
#else
          vnx = sb4[kk + 1 < kn ? kk + 1 : kk];
#endif
          if (MARK) orr |= (tv[0] | tv[1] | tv[2] | tv[3]) | (tv[4] | tv[5] | tv[6] | tv[7]);
          if (nb2 >= p0 + 8u) {  // at most one boundary (at nb) in the word: events j >= nb - p0 go to coln
            const uint32_t mcut = nb - p0;
#pragma unroll
            for (int j = 0; j < 8; ++j) red(((uint32_t)j < mcut ? col : coln) | (tv[j] & M::ROFF), M::val(tv[j]));
            if (nb <= p0 + 8u) {
              ++u;
              col = coln;
              coln = pcol(u + 1);
              nb = nb2;
              PHOTON_DCHECK(u + 2u < 40u, "K1 warp index past rel[]", u);
              nb2 = wm->rel[u + 2];
            }
          } else {
            // several warp boundaries in the word (warps shorter than 8 events): event by event
            if (col == scr && t0 == 0 && p0 == 0) {  // still in the leading virtual warp: enter warp fw
              ++u;
              col = cw;
            }
#pragma unroll
            for (uint32_t j = 0; j < 8; ++j) {
              const uint32_t pos = p0 + j;
              const bool in = pos >= r && pos < e;
              while (in && pos >= wm->rel[u + 1] && u + 1 < nw) ++u;
              red((in ? (u == myfw ? cw + t0 * 4u : pcol(u)) : scr) | (tv[j] & M::ROFF), M::val(tv[j]));
            }
            while (p0 + 8u < e && wm->rel[u + 1] <= p0 + 8u && u + 1 < nw) ++u;  // the next word's warp
            col = u == myfw ? cw + t0 * 4u : pcol(u);
            coln = pcol(u + 1);
            nb = wm->rel[u + 1];
            nb2 = wm->rel[u + 2];
          }
          lookup(vnx, tv);
        }
      }
      __syncwarp();
      if (NBUF == 1 && lane == 0) issue();  // the stage is free: the next chunk lands during collect / finalise
      // collect: lane u sums its warp's pieces (owner column, then slot 0 of each later lane it spans)
      {
        const uint32_t x0 = umax(my_rel, lo), x1 = umin(my_rel_end, hi);
        if (lane < nw && x0 < x1) {
          const uint32_t ta = divL(x0, Qe, qinv), tb = divL(x1 - 1u, Qe, qinv);
          uint32_t ca = cw + (x0 == umax(ta * L, lo) ? ta : 32u + lane) * 4u;
          if (WIDE) {
            for (uint32_t tt = ta;;) {
#pragma unroll
              for (int j = 0; j < 16; ++j) p[j] += lds_u32(ca + j * ROWB);
              if (++tt > tb) break;
              ca = cw + tt * 4u;
            }
          } else {
            // carry-save sum of the packed pieces: pk = sum of the words (mod 2^32), hs = sum of the high halves;
            // the low-half sum is pk - (hs << 16) (mod 2^32), exact since a chunk adds < 2^32 per bin
            uint32_t pk[8], hs[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) { pk[i] = 0u; hs[i] = 0u; }
            for (uint32_t tt = ta;;) {
#pragma unroll
              for (int i = 0; i < 8; ++i) {
                const uint32_t v = lds_u32(ca + i * ROWB);
                pk[i] += v;
                hs[i] += v >> 16;
              }
              if (++tt > tb) break;
              ca = cw + tt * 4u;
            }
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              p[2 * i] += pk[i] - (hs[i] << 16);
              p[2 * i + 1] += hs[i];
            }
          }
        }
      }
      // a chunk adds < 2^32 to a warp (<= CE events of length < 2^17): the u64 total follows from the u32 sum
      {
        uint32_t sum = 0;
#pragma unroll
        for (int j = 0; j < 16; ++j) sum += p[j];
        I += (uint32_t)(sum - (uint32_t)I);
      }
      __syncwarp();
      clear_cells<WIDE>(cw);
      __syncwarp();
      cs = ce;
    } while (cs < te);

    // ---- finalise the block ----
    const bool valid = lane < nw;
    const uint64_t w = w0 + lane;
    const int bad_here = ((((raw | (raw >> 16)) & 0xFFFFu) & ~bmask) != 0u || (MARK && (orr & M::MARKB))) ? 1 : 0;
    if (__any_sync(0xffffffffu, bad_here)) {
      if (valid) report_bad_event(a, s, s_end);
      raw = 0;
      orr = 0;
    }
    uint32_t k = kb;
    if (valid) {
      if (I >= kInstsLimit) latch(a.err, PHOTON_ERANGE, (int64_t)w);
      if (w >= kb1) {  // a later kernel (rare inside a block)
        ++k;
        while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
      }
      if (a.warp_bbv16) {
        uint4* dst = (uint4*)(a.warp_bbv16 + w * 16);
        dst[0] = make_uint4(p[0], p[1], p[2], p[3]);
        dst[1] = make_uint4(p[4], p[5], p[6], p[7]);
        dst[2] = make_uint4(p[8], p[9], p[10], p[11]);
        dst[3] = make_uint4(p[12], p[13], p[14], p[15]);
      }
      if (a.warp_insts) a.warp_insts[w] = I;
    }
    if (FUSED) finalize_fused(a, wm, w0, valid, k, p);
    // next block
    kb = __shfl_sync(0xffffffffu, k, nw - 1);
    kb1 = kb + 1 < a.K ? a.kwo[kb + 1] : ~0ull;  // consumed at the next block's end
    w0 += 32;
    my_s = nx_s;
    blk_end = nx_end;
  }
  }  // ranges
  if (FUSED) pool_flush(a, wm);
}

// ---- unfused A2 de-duplication from materialised BBVs: the same finalisation over 32-warp blocks ---------------
__global__ void __launch_bounds__(WPC * 32, 1) k_group3_from_bbv(Args3 a, const uint32_t* __restrict__ bbv) {
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  WMisc* wm = (WMisc*)(smem + wid * kWMiscBytes);
  const uint64_t NB = (a.W + 31) >> 5;
  const uint64_t NWK = (uint64_t)gridDim.x * WPC, gw = (uint64_t)blockIdx.x * WPC + wid;
  const uint64_t b0 = NB * gw / NWK, b1 = NB * (gw + 1) / NWK;
  pool_init(wm);
  uint32_t kb = 0;
  if (b0 < b1 && a.K > 1) {
    auto kf = [&](uint64_t kk) -> uint64_t { return a.kwo[kk]; };
    kb = (uint32_t)(search32(1, a.K, kf, (b0 << 5) + 1) - 1);
  }
  for (uint64_t b = b0; b < b1; ++b) {
    const uint64_t w0 = b << 5, w = w0 + lane;
    const uint32_t nw = (uint32_t)umin64(32, a.W - w0);
    const bool valid = lane < nw;
    uint32_t p[16];
    if (valid) {
      const uint4* src = (const uint4*)(bbv + w * 16);
#pragma unroll
      for (int v = 0; v < 4; ++v) {
        const uint4 x = src[v];
        p[4 * v] = x.x; p[4 * v + 1] = x.y; p[4 * v + 2] = x.z; p[4 * v + 3] = x.w;
      }
    } else {
#pragma unroll
      for (int j = 0; j < 16; ++j) p[j] = 0u;
    }
    while (kb + 1 < a.K && a.kwo[kb + 1] <= w0) ++kb;
    uint32_t k = kb;
    if (valid)
      while (k + 1 < a.K && a.kwo[k + 1] <= w) ++k;
    finalize_fused(a, wm, w0, valid, k, p);
    kb = __shfl_sync(0xffffffffu, k, nw - 1);
  }
  pool_flush(a, wm);
}

// ---- per-BB tables, input validation ---------------------------------------------------------------------------
// tbl_n[b] = len << 4 | bin (neutral, BB distribution), tbl_w / tbl_x = the narrow / wide K1 entries; ids in
// [B, P2) are marked.  max_len = max bb_len.
__global__ void k_table_prep3(const uint32_t* __restrict__ bb_len, const uint8_t* __restrict__ bb_bin, uint32_t B,
                              uint32_t P2, uint32_t* __restrict__ tbl_n, uint32_t* __restrict__ tbl_w,
                              uint32_t* __restrict__ tbl_x, uint32_t* max_len, DevErr* err, uint64_t* zero) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (zero && b == 0) *zero = 0;  // the K1 entry pool's count (photon_analyse: one memset node fewer before K1)
  if (b >= P2) return;
  if (b >= B) {
    tbl_n[b] = kMarkN;
    tbl_w[b] = Mode<false>::MARKB;
    tbl_x[b] = Mode<true>::MARKB;
    return;
  }
  uint32_t len = bb_len[b];
  uint32_t bin = bb_bin ? bb_bin[b] : (b & 15u);
  if (len == 0 || len > kMaxLen || bin > 15) {
    latch(err, PHOTON_EINVAL, (int64_t)b);
    len = 0;
    bin = 0;
  }
  tbl_n[b] = (len << 4) | bin;
  tbl_w[b] = Mode<false>::entry(len & 0x3FFu, bin);  // used only when every length passes narrow_ok
  tbl_x[b] = Mode<true>::entry(len, bin);
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
                                             const uint16_t* __restrict__ bb, const uint32_t* __restrict__ tbl_n,
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
          atomicAdd((unsigned long long*)&kbb[(uint64_t)k * B + b],
                    (unsigned long long)cnt[b] * ((tbl_n[b] >> 4) & kMaxLen));
      __syncthreads();
    } else {
      for (uint64_t i = cs + threadIdx.x; i < ce; i += blockDim.x) {
        uint32_t b = bb[i];
        if (b < B)
          atomicAdd((unsigned long long*)&kbb[(uint64_t)k * B + b], (unsigned long long)((tbl_n[b] >> 4) & kMaxLen));
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

// ---- host side ------------------------------------------------------------------------------------------------
struct Layout3 {
  uint32_t off_tbl, off_misc, off_stage, off_cells, bytes;
};
// [misc][table, aligned to its size][cells, row arrays aligned to their size][stage]; alignment is of the shared
// window address (dynamic shared memory starts `reserved` bytes into the window)
template <bool WIDE>
Layout3 layout3(uint32_t P2, bool gtbl, int reserved) {
  using M = Mode<WIDE>;
  auto up = [&](uint64_t off, uint64_t A) -> uint32_t {
    return (uint32_t)((((uint64_t)reserved + off + A - 1) / A) * A - (uint64_t)reserved);
  };
  Layout3 L;
  L.off_misc = 0;
  const uint32_t tbl = gtbl ? 0u : P2 * 4u;
  L.off_tbl = gtbl ? WPC * kWMiscBytes : up(WPC * kWMiscBytes, tbl);
  const uint32_t A = M::ROWS * ROWB;  // row arrays aligned to their size (OR addressing)
  L.off_cells = up(L.off_tbl + tbl, A);
  L.off_stage = L.off_cells + (WPC / GRP) * A;
  L.bytes = L.off_stage + WPC * NBUF * 32 * M::Q * 16 + 16;  // + one word: the event loop reads a word ahead
  return L;
}

int reserved_smem() {
  int dev = 0, reserved = 0;
  cudaGetDevice(&dev);
  if (cudaDeviceGetAttribute(&reserved, cudaDevAttrReservedSharedMemoryPerBlock, dev) != cudaSuccess) reserved = 0;
  return reserved;
}

template <bool WIDE, bool GTBL, bool MARK, bool FUSED>
cudaError_t launch3_t(Args3 a, int num_sms, cudaStream_t s) {
  const Layout3 L = layout3<WIDE>(a.P2, GTBL, reserved_smem());
  a.off_tbl = L.off_tbl;
  a.off_misc = L.off_misc;
  a.off_stage = L.off_stage;
  a.off_cells = L.off_cells;
  auto fn = k_bbv3<WIDE, GTBL, MARK, FUSED>;
  cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)L.bytes);
  if (e != cudaSuccess) return e;
  note_launch(), fn<<<(unsigned)num_sms, WPC * 32, L.bytes, s>>>(a);
  return cudaGetLastError();
}

template <bool GTBL, bool MARK, bool FUSED>
cudaError_t launch3_both(Args3 a, const BbvTables& tb, int num_sms, cudaStream_t s) {
  a.tbl_mode = tb.narrow;
  cudaError_t e = launch3_t<false, GTBL, MARK, FUSED>(a, num_sms, s);
  if (e != cudaSuccess) return e;
  a.tbl_mode = tb.wide;
  return launch3_t<true, GTBL, MARK, FUSED>(a, num_sms, s);
}

}  // namespace

size_t bbv_table_bytes(uint32_t B) { return (size_t)next_pow2_u32(B < 16 ? 16 : B) * 4 + 64; }

cudaError_t launch_table_prep(const TraceDev& t, const BbvTables& tb, DevErr* err, cudaStream_t s, uint64_t* zero) {
  const uint32_t P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  cudaMemsetAsync(tb.max_len, 0, 4, s);
  note_launch(), k_table_prep3<<<(P2 + 255) / 256, 256, 0, s>>>(t.bb_len, t.bb_bin, t.B, P2, tb.neutral, tb.narrow,
                                                               tb.wide, tb.max_len, err, zero);
  return cudaGetLastError();
}

cudaError_t launch_validate_offsets(const TraceDev& t, DevErr* err, cudaStream_t s) {
  uint64_t n = t.K > 0 ? t.K : 1;
  note_launch(), k_validate_offsets<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(t.kwo, t.K, t.weo, t.W, t.E, err);
  return cudaGetLastError();
}

cudaError_t launch_bbv3(const TraceDev& t, const BbvTables& tb, uint32_t* warp_bbv16, uint64_t* warp_insts,
                        const EntryPool* ep, DevErr* err, int num_sms, cudaStream_t s) {
  if (t.W == 0) return cudaSuccess;
  Args3 a{};
  a.kwo = t.kwo; a.weo = t.weo; a.bb = t.bb; a.max_len = tb.max_len;
  a.K = t.K; a.B = t.B; a.P2 = next_pow2_u32(t.B < 16 ? 16 : t.B);
  a.W = t.W; a.E = t.E;
  a.warp_bbv16 = warp_bbv16; a.warp_insts = warp_insts;
  if (ep) a.ep = *ep;
  a.err = err;
  const bool gtbl = a.P2 > (uint32_t)SMEM_TBL_MAX;
  const bool mark = a.P2 != t.B || gtbl;
  const bool fused = ep != nullptr;
  if (gtbl) return fused ? launch3_both<true, true, true>(a, tb, num_sms, s) : launch3_both<true, true, false>(a, tb, num_sms, s);
  if (mark) return fused ? launch3_both<false, true, true>(a, tb, num_sms, s) : launch3_both<false, true, false>(a, tb, num_sms, s);
  return fused ? launch3_both<false, false, true>(a, tb, num_sms, s) : launch3_both<false, false, false>(a, tb, num_sms, s);
}

cudaError_t launch_group_from_bbv(const TraceDev& t, const uint32_t* warp_bbv16, const EntryPool& ep, DevErr* err,
                                  int num_sms, cudaStream_t s) {
  if (t.W == 0) return cudaSuccess;
  Args3 a{};
  a.kwo = t.kwo; a.K = t.K; a.W = t.W; a.ep = ep; a.err = err;
  const size_t smem = WPC * kWMiscBytes;
  cudaError_t e = cudaFuncSetAttribute(k_group3_from_bbv, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  note_launch(), k_group3_from_bbv<<<(unsigned)num_sms, WPC * 32, smem, s>>>(a, warp_bbv16);
  return cudaGetLastError();
}

cudaError_t launch_kernel_bb_insts(const TraceDev& t, const BbvTables& tb, uint64_t* kbb, uint64_t* kchunk_off,
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
  note_launch(), k_kbb<<<(unsigned)grid, 256, smem, s>>>(t.kwo, t.weo, t.bb, tb.neutral, t.K, t.B, kbb, jobs_ub,
                                                           kchunk_off);
  return cudaGetLastError();
}

}  // namespace photon
