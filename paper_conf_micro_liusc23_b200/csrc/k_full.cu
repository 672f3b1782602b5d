// k_full.cu — N2: full-BBV exact warp grouping and tagged-stream ingest.
//
// PAPER.md L154 ("warps that execute the same instruction sequence ... have the same BBV", one warp type) and L161
// (a BBV lists the basic blocks a warp executed).  A2 groups on the 16-bin projection of L178 [P-3]; this mode keys
// on the full BBV — the execution count of every BB id — so two warps share a type iff their event multisets are
// equal.  Reading [N2-a]: the type's key row is the 16-bin projection of its members (equal full
// BBVs project equally); rows are ordered by (count desc, key asc, lowest warp asc).
//
// Steps (one stream, every step on the device; no library sort):
//  1. k_full_hash_short / _long: one thread per analysed warp of <= 16 events, longer warps from a work list with
//     one hardware warp each; two 64-bit mixes of each event's BB id are summed (an order-independent 128-bit
//     hash, = sum over b of count(b) * H(b) mod 2^64 per half).
//  2. k_full_insert: (kernel, 128-bit hash) inserted into the A2 hash table (warp-aggregated: runs of equal
//     consecutive warps insert once), each warp's slot recorded; a slot's first warp = its lowest member.
//  3. k_full_project: every slot's key row <- the 16-bin projection of its first warp (reading [N2-a]).
//  4. exact verification of every member against its slot's first warp: warps of <= 16 events in registers
//     (multiset counts), longer ones by one hardware warp with a shared-memory histogram of count differences
//     over 4096-id chunks of the BB id space; a difference (a 128-bit hash collision) is latched exactly
//     (PHOTON_ERANGE, index = the warp).
//  5. the A2 canonicalisation (k_types.cu) over the table; k_full_remap writes warp_type.
// Ingest: a stream of (warp, bb) tagged events in arbitrary interleaving -> CSR by warp with a stable LSD radix sort
// of the warp ids (k_stable.cu's, 8-bit digits over ceil(log2 W) bits: each warp keeps its events' stream order)
// and boundary-filled offsets.

#include "internal.h"

namespace photon {

namespace {

__device__ __forceinline__ uint64_t hmix(uint64_t x) {
  x ^= x >> 33;
  x *= 0xFF51AFD7ED558CCDull;
  x ^= x >> 33;
  x *= 0xC4CEB9FE1A85EC53ull;
  x ^= x >> 33;
  return x;
}

constexpr uint64_t FULL_LONG = 16;  // events above which a warp is handled by a whole hardware warp (work list; 16 measured best on C3)

__device__ __forceinline__ void full_mix(uint32_t x, uint64_t& a, uint64_t& b) {
  a += hmix(0x9E3779B97F4A7C15ull * (x + 1));
  b += hmix(0xC2B2AE3D27D4EB4Full * (x + 1) + 0x165667B19E3779F9ull);
}

// the two 64-bit mixes of every BB id, tabulated once (a lookup per event instead of two mixes)
__global__ void k_full_htab(uint32_t B, ulonglong2* htab) {
  const uint32_t x = blockIdx.x * blockDim.x + threadIdx.x;
  if (x >= B) return;
  uint64_t a = 0, b = 0;
  full_mix(x, a, b);
  htab[x] = make_ulonglong2(a, b);
}
__device__ __forceinline__ void tab_mix(const ulonglong2* __restrict__ htab, uint32_t x, uint32_t B, uint64_t& a,
                                        uint64_t& b) {
  const ulonglong2 v = __ldg(htab + (x < B ? x : 0));
  a += v.x;
  b += v.y;
}

// one thread per analysed warp, 256 consecutive warps per CTA step (the step's first kernel by one binary search,
// then each thread steps forward): short warps are hashed here, longer ones go to the work list
__global__ void __launch_bounds__(256) k_full_hash_short(const uint64_t* __restrict__ kwo, uint32_t K,
                                                         const uint64_t* __restrict__ weo, uint64_t W, uint64_t E,
                                                         const uint16_t* __restrict__ bb, uint32_t B, uint64_t* h_lo,
                                                         uint64_t* h_hi, uint32_t* kid, uint64_t* list, uint32_t* nlist,
                                                         const ulonglong2* __restrict__ htab, DevErr* err) {
  __shared__ uint32_t s_k0;
  for (uint64_t w0 = (uint64_t)blockIdx.x * 256; w0 < W; w0 += (uint64_t)gridDim.x * 256) {
    if (threadIdx.x == 0) {
      uint32_t lo = 0, hi = K - 1;
      while (lo < hi) {
        const uint32_t mid = (lo + hi + 1) >> 1;
        if (kwo[mid] <= w0) lo = mid; else hi = mid - 1;
      }
      s_k0 = lo;
    }
    __syncthreads();
    const uint64_t w = w0 + threadIdx.x;
    uint32_t k = s_k0;
    __syncthreads();
    if (w >= W) continue;
    while (k + 1 < K && kwo[k + 1] <= w) ++k;
    kid[w] = k;
    if (weo[w + 1] < weo[w]) latch(err, PHOTON_ERANGE, (int64_t)w);
    const uint64_t s = umin64(weo[w], E), e = umin64(umax64(weo[w + 1], s), E);
    if (e - s > FULL_LONG) {
      list[atomicAdd(nlist, 1u)] = w;
      continue;
    }
    uint64_t a = 0, b = 0;
    for (uint64_t i = s; i < e; ++i) {
      const uint32_t x = bb[i];
      if (x >= B) latch(err, PHOTON_ERANGE, (int64_t)i);
      tab_mix(htab, x, B, a, b);
    }
    h_lo[w] = a;
    h_hi[w] = b;
  }
}

// one hardware warp per listed long warp: lanes read its events coalesced
__global__ void k_full_hash_long(const uint64_t* __restrict__ weo, uint64_t E, const uint16_t* __restrict__ bb,
                                 uint32_t B, uint64_t* h_lo, uint64_t* h_hi, const uint64_t* __restrict__ list,
                                 const uint32_t* nlist, const ulonglong2* __restrict__ htab, DevErr* err) {
  const int lane = threadIdx.x & 31;
  const uint32_t nl = *nlist;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nl; j += nw) {
    const uint64_t w = list[j];
    const uint64_t s = umin64(weo[w], E), e = umin64(umax64(weo[w + 1], s), E);
    uint64_t a = 0, b = 0;
    // head (to a 16-byte boundary) and tail element-wise; the body as 8-event vectors, two per lane in flight
    const bool vec = ((uintptr_t)bb & 15) == 0;
    const uint64_t s8 = vec ? umin64((s + 7) & ~7ull, e) : e, e8 = vec ? umax64(e & ~7ull, s8) : e;
    for (uint64_t i = s + lane; i < s8; i += 32) {
      const uint32_t x = bb[i];
      if (x >= B) latch(err, PHOTON_ERANGE, (int64_t)i);
      tab_mix(htab, x, B, a, b);
    }
    for (uint64_t i0 = s8 + 8 * lane; i0 < e8; i0 += 512) {
      uint4 v[2];
#pragma unroll
      for (int u = 0; u < 2; ++u)
        v[u] = i0 + 256 * u < e8 ? __ldg(reinterpret_cast<const uint4*>(bb + i0 + 256 * u)) : make_uint4(0, 0, 0, 0);
#pragma unroll
      for (int u = 0; u < 2; ++u) {
        if (i0 + 256 * u >= e8) continue;
        const uint32_t wv[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
#pragma unroll
        for (int q = 0; q < 8; ++q) {
          const uint32_t x = (wv[q >> 1] >> ((q & 1) * 16)) & 0xFFFFu;
          if (x >= B) latch(err, PHOTON_ERANGE, (int64_t)(i0 + 256 * u + q));
          tab_mix(htab, x, B, a, b);
        }
      }
    }
    for (uint64_t i = e8 + lane; i < e; i += 32) {
      const uint32_t x = bb[i];
      if (x >= B) latch(err, PHOTON_ERANGE, (int64_t)i);
      tab_mix(htab, x, B, a, b);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      a += __shfl_xor_sync(0xffffffffu, a, o);
      b += __shfl_xor_sync(0xffffffffu, b, o);
    }
    if (lane == 0) {
      h_lo[w] = a;
      h_hi[w] = b;
    }
  }
}

// (kernel, h_lo, h_hi) -> slot of the A2 hash table; lanes of equal consecutive warps insert once (count = the
// run, first = its lowest warp = the leader)
__global__ void __launch_bounds__(256) k_full_insert(uint64_t W, const uint32_t* __restrict__ kid,
                                                     const uint64_t* __restrict__ h_lo,
                                                     const uint64_t* __restrict__ h_hi, HashTable ht,
                                                     uint32_t* wslot, DevErr* err) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t base = (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) << 5; base < W; base += nw << 5) {
    const uint64_t w = base + lane;
    const bool valid = w < W;
    uint32_t key[16];
#pragma unroll
    for (int q = 0; q < 16; ++q) key[q] = 0u;
    uint32_t k = 0;
    if (valid) {
      const uint64_t a = h_lo[w], b = h_hi[w];
      key[0] = (uint32_t)a; key[1] = (uint32_t)(a >> 32); key[2] = (uint32_t)b; key[3] = (uint32_t)(b >> 32);
      k = kid[w];
    }
    const uint64_t h = valid ? hash_key(k, key) : 0ull;
    const unsigned peers = __match_any_sync(0xffffffffu, (unsigned long long)h);
    const int leader = __ffs(peers) - 1;
    bool eq = __shfl_sync(0xffffffffu, k, leader) == k;
#pragma unroll
    for (int q = 0; q < 4; ++q) eq &= __shfl_sync(0xffffffffu, key[q], leader) == key[q];
    const unsigned grp = __ballot_sync(0xffffffffu, valid && eq) & peers;  // my leader's exact group
    const bool lead = valid && (!eq || lane == (uint32_t)leader);
    uint32_t slot = UINT32_MAX;
    if (lead) slot = ht_insert(ht, err, k, key, h, eq ? __popc(grp) : 1u, w);
    const uint32_t ls = __shfl_sync(0xffffffffu, slot, leader);
    if (valid) wslot[w] = eq ? ls : slot;
  }
}

// key row of every occupied slot <- the 16-bin projection of its first (lowest) warp
__global__ void k_full_project(HashTable ht, const uint32_t* __restrict__ bbv16) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > ht.mask || ht.hkey[i] == 0ull) return;
  const uint4* src = (const uint4*)(bbv16 + ht.first[i] * 16);
  uint4* dst = (uint4*)(ht.key + i * 16);
  dst[0] = src[0]; dst[1] = src[1]; dst[2] = src[2]; dst[3] = src[3];
}

// exact verification, one thread per warp: equal event counts for all; warps of <= 16 events compared with their
// slot's first warp in registers (each event's multiplicity in both lists); longer ones by k_full_verify_long
__global__ void k_full_verify_short(uint64_t W, const uint32_t* __restrict__ wslot, HashTable ht,
                                    const uint64_t* __restrict__ weo, uint64_t E, const uint16_t* __restrict__ bb,
                                    DevErr* err) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < W; w += stride) {
    const uint32_t sl = wslot[w];
    if (sl > ht.mask) continue;  // ECAPACITY latched by the insert
    const uint64_t r = ht.first[sl];
    if (r == w) continue;
    const uint64_t ws = umin64(weo[w], E), we = umin64(umax64(weo[w + 1], ws), E);
    const uint64_t rs = umin64(weo[r], E), re = umin64(umax64(weo[r + 1], rs), E);
    const uint64_t n = we - ws;
    if (n != re - rs) {
      latch(err, PHOTON_ERANGE, (int64_t)w);  // a 128-bit hash collision, detected exactly
      continue;
    }
    if (n > FULL_LONG) continue;
    uint32_t a[FULL_LONG], b[FULL_LONG];
#pragma unroll
    for (int j = 0; j < (int)FULL_LONG; ++j) {
      a[j] = (uint64_t)j < n ? bb[ws + j] : 0x10000u;
      b[j] = (uint64_t)j < n ? bb[rs + j] : 0x10000u;
    }
    bool same = true, seq = true;
#pragma unroll
    for (int j = 0; j < (int)FULL_LONG; ++j) seq &= a[j] == b[j];
    if (seq) continue;  // the same sequence (the usual case: same instruction stream, L154)
#pragma unroll
    for (int j = 0; j < (int)FULL_LONG; ++j) {
      int ca = 0, cb = 0;
#pragma unroll
      for (int q = 0; q < (int)FULL_LONG; ++q) {
        ca += a[q] == a[j];
        cb += b[q] == a[j];
      }
      same &= ca == cb;
    }
    if (!same) latch(err, PHOTON_ERANGE, (int64_t)w);
  }
}

// one hardware warp per listed long warp that is not its slot's first: an equal SEQUENCE (the usual case: the same
// instruction stream, L154) passes; the others are listed for k_full_verify_long
__global__ void __launch_bounds__(256) k_full_verify_seq(const uint32_t* __restrict__ wslot, HashTable ht,
                                                         const uint64_t* __restrict__ weo, uint64_t E,
                                                         const uint16_t* __restrict__ bb,
                                                         const uint64_t* __restrict__ list, const uint32_t* nlist,
                                                         uint64_t* list2, uint32_t* nlist2) {
  const int lane = threadIdx.x & 31;
  const uint32_t nl = *nlist;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nl; j += nw) {
    const uint64_t w = list[j];
    const uint32_t sl = wslot[w];
    if (sl > ht.mask) continue;
    const uint64_t r = ht.first[sl];
    if (r == w) continue;
    const uint64_t ws = umin64(weo[w], E), we = umin64(umax64(weo[w + 1], ws), E);
    const uint64_t rs = umin64(weo[r], E), re = umin64(umax64(weo[r + 1], rs), E);
    if (we - ws != re - rs) continue;  // latched by k_full_verify_short
    const uint64_t n = we - ws;
    bool seq = true;
    uint64_t i = lane;
    for (; i + 224 < n; i += 256) {  // eight load pairs in flight per lane
      uint32_t x[8], y[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) { x[u] = bb[ws + i + 32 * u]; y[u] = bb[rs + i + 32 * u]; }
#pragma unroll
      for (int u = 0; u < 8; ++u) seq &= x[u] == y[u];
    }
    for (; i + 96 < n; i += 128) {
      uint32_t x[4], y[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) { x[u] = bb[ws + i + 32 * u]; y[u] = bb[rs + i + 32 * u]; }
#pragma unroll
      for (int u = 0; u < 4; ++u) seq &= x[u] == y[u];
    }
    for (; i < n; i += 32) seq &= bb[ws + i] == bb[rs + i];
    if (!__all_sync(0xffffffffu, seq) && lane == 0) list2[atomicAdd(nlist2, 1u)] = w;
  }
}

// one hardware warp per long warp whose sequence differs from its slot's first: count differences (member +1,
// first -1, warp-aggregated) in a shared-memory histogram, one 4096-id chunk of the BB id space at a time; all
// zero at the member's ids (with equal lengths) <=> equal multisets
constexpr int VCHUNK = 4096;
constexpr int VWARPS = 4;  // hardware warps per block (4 x 16 KB of counters)
__global__ void __launch_bounds__(VWARPS * 32) k_full_verify_long(const uint32_t* __restrict__ wslot, HashTable ht,
                                                                 const uint64_t* __restrict__ weo, uint64_t E,
                                                                 const uint16_t* __restrict__ bb, uint32_t B,
                                                                 const uint64_t* __restrict__ list,
                                                                 const uint32_t* nlist, DevErr* err) {
  extern __shared__ int32_t hist[];  // (list, nlist: the sequence mismatches of k_full_verify_seq)  // [VWARPS][VCHUNK]
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  int32_t* h = hist + wid * VCHUNK;
  for (int i = lane; i < VCHUNK; i += 32) h[i] = 0;
  __syncwarp();
  const uint32_t nl = *nlist;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nl; j += nw) {
    const uint64_t w = list[j];
    const uint32_t sl = wslot[w];
    if (sl > ht.mask) continue;
    const uint64_t r = ht.first[sl];
    if (r == w) continue;
    const uint64_t ws = umin64(weo[w], E), we = umin64(umax64(weo[w + 1], ws), E);
    const uint64_t rs = umin64(weo[r], E), re = umin64(umax64(weo[r + 1], rs), E);
    if (we - ws != re - rs) continue;  // latched by k_full_verify_short
    const uint64_t n = we - ws;
    bool bad = false;
    for (uint32_t c0 = 0; c0 < B && !bad; c0 += VCHUNK) {
      for (uint64_t i0 = 0; i0 < n; i0 += 32) {  // warp-uniform steps: equal ids aggregate before the atomic
        const uint64_t i = i0 + lane;
        const uint32_t x = i < n ? (uint32_t)bb[ws + i] - c0 : ~0u, y = i < n ? (uint32_t)bb[rs + i] - c0 : ~0u;
        const unsigned px = __match_any_sync(0xffffffffu, x), py = __match_any_sync(0xffffffffu, y);
        if (x < (uint32_t)VCHUNK && lane == __ffs(px) - 1) atomicAdd(&h[x], __popc(px));
        if (y < (uint32_t)VCHUNK && lane == __ffs(py) - 1) atomicSub(&h[y], __popc(py));
      }
      __syncwarp();
      for (uint64_t i = lane; i < n; i += 32) {
        const uint32_t x = (uint32_t)bb[ws + i] - c0;
        if (x < (uint32_t)VCHUNK && h[x] != 0) bad = true;
      }
      __syncwarp();
      for (uint64_t i = lane; i < n; i += 32) {
        const uint32_t x = (uint32_t)bb[ws + i] - c0, y = (uint32_t)bb[rs + i] - c0;
        if (x < (uint32_t)VCHUNK) h[x] = 0;
        if (y < (uint32_t)VCHUNK) h[y] = 0;
      }
      __syncwarp();
      bad = __any_sync(0xffffffffu, bad);
    }
    if (bad && lane == 0) latch(err, PHOTON_ERANGE, (int64_t)w);  // a 128-bit hash collision, detected exactly
  }
}

__global__ void k_full_remap(uint64_t W, const uint32_t* __restrict__ wslot, const uint32_t* __restrict__ canon,
                             uint64_t mask, uint32_t* warp_type) {
  const uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (w < W) {
    const uint32_t sl = wslot[w];
    warp_type[w] = sl <= mask ? canon[sl] : UINT32_MAX;
  }
}

// ---- ingest ----------------------------------------------------------------------------------------------------
// key[i] = warp[i] (the radix key), range-checked
__global__ void k_ingest_keys(uint64_t n, const uint32_t* __restrict__ warp, uint64_t W, uint64_t* key, DevErr* err) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const uint32_t w = warp[i];
  if (w >= W) latch(err, PHOTON_ERANGE, (int64_t)i);
  key[i] = w < W ? w : 0;
}
// bb_out[j] = bb[perm[j]]
__global__ void k_ingest_gather(uint64_t n, const uint32_t* __restrict__ perm, const uint16_t* __restrict__ bb,
                                uint16_t* bb_out) {
  const uint64_t j = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (j < n) bb_out[j] = bb[perm[j]];
}
// off[w] = first sorted position with warp >= w (boundary fill: each key change writes the offsets it spans)
__global__ void k_ingest_offsets(uint64_t n, const uint64_t* __restrict__ key, uint64_t W, uint64_t* off) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > n) return;
  const uint64_t lo = i == 0 ? 0 : umin64(key[i - 1] + 1, W + 1);
  const uint64_t hi = i == n ? W : umin64(key[i], W);
  for (uint64_t w = lo; w <= hi && w <= W; ++w) off[w] = i;
}

unsigned grid_for(uint64_t n, int threads) { return (unsigned)(n ? ceil_div(n, (uint64_t)threads) : 1); }

}  // namespace

cudaError_t launch_group_full(const TraceDev& t, const uint32_t* bbv16, const FullWs& f, const HashTable& ht,
                              const CanonWs& cw, const photon_types& out, DevErr* err, int num_sms, cudaStream_t s) {
  const uint64_t W = t.W;
  if (W == 0) return cudaSuccess;
  const unsigned hg = (unsigned)umin64(ceil_div(W * 32, 256), (uint64_t)num_sms * 16);
  const unsigned tg = (unsigned)umin64(ceil_div(W, 256), (uint64_t)num_sms * 8);
  cudaMemsetAsync(f.nlist, 0, 8, s);
  note_launch(), k_full_htab<<<grid_for(t.B, 256), 256, 0, s>>>(t.B, f.htab);
  note_launch(), k_full_hash_short<<<tg, 256, 0, s>>>(t.kwo, t.K, t.weo, W, t.E, t.bb, t.B, f.h_lo, f.h_hi, f.kid,
                                                     f.list, f.nlist, f.htab, err);
  note_launch(), k_full_hash_long<<<hg, 256, 0, s>>>(t.weo, t.E, t.bb, t.B, f.h_lo, f.h_hi, f.list, f.nlist, f.htab,
                                                     err);
  cudaError_t e;
  if ((e = launch_ht_clear(ht, s))) return e;
  const unsigned ig = (unsigned)umin64(ceil_div(W, 256), (uint64_t)num_sms * 8);
  note_launch(), k_full_insert<<<ig, 256, 0, s>>>(W, f.kid, f.h_lo, f.h_hi, ht, f.wslot, err);
  note_launch(), k_full_project<<<grid_for(ht.mask + 1, 256), 256, 0, s>>>(ht, bbv16);
  note_launch(), k_full_verify_short<<<tg, 256, 0, s>>>(W, f.wslot, ht, t.weo, t.E, t.bb, err);
  const unsigned vg = (unsigned)umin64(ceil_div(W, VWARPS), (uint64_t)num_sms * 8);
  note_launch(), k_full_verify_seq<<<hg, 256, 0, s>>>(f.wslot, ht, t.weo, t.E, t.bb, f.list, f.nlist, f.list2,
                                                     f.nlist + 1);
  const int vsm = VWARPS * VCHUNK * (int)sizeof(int32_t);
  cudaFuncSetAttribute(k_full_verify_long, cudaFuncAttributeMaxDynamicSharedMemorySize, vsm);
  note_launch(), k_full_verify_long<<<vg, VWARPS * 32, vsm, s>>>(f.wslot, ht, t.weo, t.E, t.bb, t.B, f.list2,
                                                              f.nlist + 1, err);
  if ((e = launch_canonicalise(ht, t.K, t.kwo, nullptr, out, cw, err, num_sms, s))) return e;
  if (out.warp_type)
    note_launch(), k_full_remap<<<grid_for(W, 256), 256, 0, s>>>(W, f.wslot, cw.canon, ht.mask, out.warp_type);
  return cudaGetLastError();
}

cudaError_t launch_ingest(uint64_t n, uint64_t W, const uint32_t* warp, const uint16_t* bb, uint64_t* key,
                          void* sort_ws, uint16_t* bb_out, uint64_t* off, DevErr* err, cudaStream_t s) {
  uint64_t* skey = key;
  uint32_t* perm = nullptr;
  if (n) {
    note_launch(), k_ingest_keys<<<grid_for(n, 256), 256, 0, s>>>(n, warp, W, key, err);
    uint32_t bits = 1;
    while (bits < 32 && (1ull << bits) < W) ++bits;
    cudaError_t e = launch_radix_pairs(key, n, bits, sort_ws, &skey, &perm, s);
    if (e) return e;
    note_launch(), k_ingest_gather<<<grid_for(n, 256), 256, 0, s>>>(n, perm, bb, bb_out);
  }
  note_launch(), k_ingest_offsets<<<grid_for(n + 1, 256), 256, 0, s>>>(n, skey, W, off);
  return cudaGetLastError();
}

}  // namespace photon
