// k_full.cu — N2: full-BBV exact warp grouping and tagged-stream ingest.
//
// PAPER.md L154 ("warps that execute the same instruction sequence ... have the same BBV", one warp type) and L161
// (a BBV lists the basic blocks a warp executed).  A2 groups on the 16-bin projection of L178 [P-3]; this mode keys
// on the full BBV — the execution count of every BB id — so two warps share a type iff their event multisets are
// equal.  Reading [N2-a]: the type's key row is the 16-bin projection of its members (equal full
// BBVs project equally); rows are ordered by (count desc, key asc, lowest warp asc).
//
// Steps (one stream, every step on the device):
//  1. k_full_hash_short / _long: one thread per analysed warp of <= 16 events, longer warps from a work list with
//     one hardware warp each; two 64-bit mixes of each event's BB id are summed (an order-independent 128-bit
//     hash, = sum over b of count(b) * H(b) mod 2^64 per half), each event's (warp << 16 | bb) key is written.
//  2. three stable radix sorts (CUB) of the warp indices by h_lo, h_hi, kernel: groups of equal (kernel, hash) are
//     contiguous, members in ascending warp order.
//  3. k_full_groups: group ids (CUB scan of the boundary flags), one slot per group in a type table (kernel,
//     projected key of the first member, count, first warp) and each warp's group.
//  4. k_full_verify_short / k_full_verify (long members from the work list): every member is compared with its
//     group's first warp on the per-warp SORTED event lists (one
//     CUB radix sort of the (warp << 16 | bb) keys written in step 1): a hash collision is detected exactly and
//     latched (PHOTON_ERANGE, index = the warp).
//  5. the A2 canonicalisation (k_types.cu) over the group table; k_full_remap writes warp_type.
// Ingest: a stream of (warp, bb) tagged events in arbitrary interleaving -> CSR by warp with a stable radix sort
// (each warp keeps its events' stream order) and boundary-filled offsets.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

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

// one thread per analysed warp, 256 consecutive warps per CTA step (the step's first kernel by one binary search,
// then each thread steps forward): short warps are hashed here, longer ones go to the work list
__global__ void __launch_bounds__(256) k_full_hash_short(const uint64_t* __restrict__ kwo, uint32_t K,
                                                         const uint64_t* __restrict__ weo, uint64_t W, uint64_t E,
                                                         const uint16_t* __restrict__ bb, uint32_t B, uint64_t* h_lo,
                                                         uint64_t* h_hi, uint32_t* kid, uint32_t* perm, uint64_t* ekey,
                                                         uint64_t* list, uint32_t* nlist, DevErr* err) {
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
    perm[w] = (uint32_t)w;
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
      full_mix(x, a, b);
      ekey[i] = (w << 16) | x;
    }
    h_lo[w] = a;
    h_hi[w] = b;
  }
}

// one hardware warp per listed long warp: lanes read its events coalesced
__global__ void k_full_hash_long(const uint64_t* __restrict__ weo, uint64_t E, const uint16_t* __restrict__ bb,
                                 uint32_t B, uint64_t* h_lo, uint64_t* h_hi, uint64_t* ekey,
                                 const uint64_t* __restrict__ list, const uint32_t* nlist, DevErr* err) {
  const int lane = threadIdx.x & 31;
  const uint32_t nl = *nlist;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nl; j += nw) {
    const uint64_t w = list[j];
    const uint64_t s = umin64(weo[w], E), e = umin64(umax64(weo[w + 1], s), E);
    uint64_t a = 0, b = 0;
    for (uint64_t i = s + lane; i < e; i += 32) {
      const uint32_t x = bb[i];
      if (x >= B) latch(err, PHOTON_ERANGE, (int64_t)i);
      full_mix(x, a, b);
      ekey[i] = (w << 16) | x;
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

// exact verification, one thread per sorted position that is not a group start (short warps), longer ones listed
__global__ void k_full_verify_short(uint64_t W, const uint32_t* __restrict__ perm, const uint32_t* __restrict__ flag,
                                    const uint32_t* __restrict__ gid, const uint64_t* __restrict__ gstart,
                                    const uint64_t* __restrict__ weo, uint64_t E, const uint64_t* __restrict__ sorted,
                                    uint64_t* list, uint32_t* nlist, DevErr* err) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < W; i += stride) {
    if (flag[i]) continue;
    const uint32_t w = perm[i], r = perm[gstart[gid[i] - 1]];
    const uint64_t ws = umin64(weo[w], E), we = umin64(umax64(weo[w + 1], ws), E);
    const uint64_t rs = umin64(weo[r], E), re = umin64(umax64(weo[r + 1], rs), E);
    if (we - ws != re - rs) {
      latch(err, PHOTON_ERANGE, (int64_t)w);  // a 128-bit hash collision, detected exactly
      continue;
    }
    if (we - ws > FULL_LONG) {
      list[atomicAdd(nlist, 1u)] = i;
      continue;
    }
    bool same = true;
    for (uint64_t j = 0; same && j < we - ws; ++j) same = (sorted[ws + j] & 0xFFFFu) == (sorted[rs + j] & 0xFFFFu);
    if (!same) latch(err, PHOTON_ERANGE, (int64_t)w);
  }
}

__global__ void k_gather_u64(uint64_t n, const uint32_t* __restrict__ perm, const uint64_t* __restrict__ src,
                             uint64_t* dst) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = src[perm[i]];
}
__global__ void k_gather_u32(uint64_t n, const uint32_t* __restrict__ perm, const uint32_t* __restrict__ src,
                             uint32_t* dst) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) dst[i] = src[perm[i]];
}

// flag[i] = sorted position i starts a new (kernel, hash) group
__global__ void k_full_flags(uint64_t W, const uint32_t* __restrict__ perm, const uint32_t* __restrict__ kid,
                             const uint64_t* __restrict__ h_lo, const uint64_t* __restrict__ h_hi, uint32_t* flag) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= W) return;
  const uint32_t w = perm[i];
  bool start = i == 0;
  if (!start) {
    const uint32_t v = perm[i - 1];
    start = kid[w] != kid[v] || h_lo[w] != h_lo[v] || h_hi[w] != h_hi[v];
  }
  flag[i] = start ? 1u : 0u;
}

// gid[i] = inclusive count of group starts (1-based group id); the group's slot g = gid - 1
__global__ void k_full_groups(uint64_t W, const uint32_t* __restrict__ perm, const uint32_t* __restrict__ flag,
                              const uint32_t* __restrict__ gid, const uint32_t* __restrict__ kid,
                              const uint32_t* __restrict__ bbv16, HashTable ht, uint64_t* gstart, uint32_t* wgroup) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= W) return;
  const uint32_t w = perm[i], g = gid[i] - 1;
  wgroup[w] = g;
  if (flag[i]) {
    gstart[g] = i;
    ht.hkey[g] = 1ull;  // occupied
    ht.kern[g] = kid[w];
    ht.first[g] = w;    // the lowest member: the sorts are stable over ascending warp indices
    const uint4* src = (const uint4*)(bbv16 + (uint64_t)w * 16);
    uint4* dst = (uint4*)(ht.key + (uint64_t)g * 16);
    dst[0] = src[0]; dst[1] = src[1]; dst[2] = src[2]; dst[3] = src[3];
  }
}

// count of group g = next group's start - its start (G = gid[W-1] groups)
__global__ void k_full_counts(uint64_t W, const uint32_t* __restrict__ gid, const uint64_t* __restrict__ gstart,
                              HashTable ht) {
  const uint64_t g = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const uint64_t G = W ? gid[W - 1] : 0;
  if (g >= G) return;
  ht.count[g] = (uint32_t)((g + 1 < G ? gstart[g + 1] : W) - gstart[g]);
}

// one hardware warp per listed long member: its sorted event list equals the group's first
__global__ void k_full_verify(uint64_t W, const uint32_t* __restrict__ perm, const uint32_t* __restrict__ flag,
                              const uint32_t* __restrict__ gid, const uint64_t* __restrict__ gstart,
                              const uint64_t* __restrict__ weo, uint64_t E, const uint64_t* __restrict__ sorted,
                              const uint64_t* __restrict__ list, const uint32_t* nlist, DevErr* err) {
  const int lane = threadIdx.x & 31;
  const uint32_t nl = *nlist;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j0 = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j0 < nl; j0 += nw) {
    const uint64_t i = list[j0];
    const uint32_t w = perm[i], r = perm[gstart[gid[i] - 1]];
    const uint64_t ws = umin64(weo[w], E), we = umin64(umax64(weo[w + 1], ws), E);
    const uint64_t rs = umin64(weo[r], E), re = umin64(umax64(weo[r + 1], rs), E);
    bool same = (we - ws) == (re - rs);
    for (uint64_t j = lane; same && j < we - ws; j += 32)
      same = (sorted[ws + j] & 0xFFFFu) == (sorted[rs + j] & 0xFFFFu);
    same = __all_sync(0xffffffffu, same);
    if (!same && lane == 0) latch(err, PHOTON_ERANGE, (int64_t)w);  // a 128-bit hash collision, detected exactly
  }
}

__global__ void k_full_remap(uint64_t W, const uint32_t* __restrict__ wgroup, const uint32_t* __restrict__ canon,
                             uint32_t* warp_type) {
  const uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (w < W) warp_type[w] = canon[wgroup[w]];
}

// ---- ingest ----------------------------------------------------------------------------------------------------
__global__ void k_ingest_check(uint64_t n, const uint32_t* __restrict__ warp, uint64_t W, DevErr* err) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n && warp[i] >= W) latch(err, PHOTON_ERANGE, (int64_t)i);
}
// off[w] = first sorted position with warp >= w (boundary fill: each key change writes the offsets it spans)
__global__ void k_ingest_offsets(uint64_t n, const uint32_t* __restrict__ key, uint64_t W, uint64_t* off) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > n) return;
  const uint64_t lo = i == 0 ? 0 : umin64((uint64_t)key[i - 1] + 1, W + 1);
  const uint64_t hi = i == n ? W : umin64((uint64_t)key[i], W);
  for (uint64_t w = lo; w <= hi && w <= W; ++w) off[w] = i;
}

unsigned grid_for(uint64_t n, int threads) { return (unsigned)(n ? ceil_div(n, (uint64_t)threads) : 1); }

}  // namespace

// CUB temp-storage sizes (host queries; no launch)
size_t full_cub_bytes(uint64_t W, uint64_t E) {
  size_t a = 0, b = 0, c = 0, d = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, a, (const uint64_t*)nullptr, (uint64_t*)nullptr,
                                  (const uint32_t*)nullptr, (uint32_t*)nullptr, (int64_t)W);
  cub::DeviceRadixSort::SortPairs(nullptr, b, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                  (const uint32_t*)nullptr, (uint32_t*)nullptr, (int64_t)W);
  cub::DeviceScan::InclusiveSum(nullptr, c, (const uint32_t*)nullptr, (uint32_t*)nullptr, (int64_t)W);
  cub::DeviceRadixSort::SortKeys(nullptr, d, (const uint64_t*)nullptr, (uint64_t*)nullptr, (int64_t)E);
  size_t m = a > b ? a : b;
  m = m > c ? m : c;
  return m > d ? m : d;
}
size_t ingest_cub_bytes(uint64_t n) {
  size_t a = 0;
  cub::DeviceRadixSort::SortPairs(nullptr, a, (const uint32_t*)nullptr, (uint32_t*)nullptr,
                                  (const uint16_t*)nullptr, (uint16_t*)nullptr, (int64_t)n);
  return a;
}

cudaError_t launch_group_full(const TraceDev& t, const uint32_t* bbv16, const FullWs& f, const HashTable& ht,
                              const CanonWs& cw, const photon_types& out, DevErr* err, int num_sms, cudaStream_t s) {
  const uint64_t W = t.W;
  if (W == 0) return cudaSuccess;
  cudaError_t e;
  const unsigned hg = (unsigned)umin64(ceil_div(W * 32, 256), (uint64_t)num_sms * 16);
  const unsigned tg = (unsigned)umin64(ceil_div(W, 256), (uint64_t)num_sms * 8);
  cudaMemsetAsync(f.nlist, 0, 8, s);
  note_launch(), k_full_hash_short<<<tg, 256, 0, s>>>(t.kwo, t.K, t.weo, W, t.E, t.bb, t.B, f.h_lo, f.h_hi, f.kid,
                                                     f.perm_a, f.ekey, f.list, f.nlist, err);
  note_launch(), k_full_hash_long<<<hg, 256, 0, s>>>(t.weo, t.E, t.bb, t.B, f.h_lo, f.h_hi, f.ekey, f.list, f.nlist,
                                                     err);
  size_t tb = f.cub_bytes;
  // stable passes: h_lo, then h_hi, then kernel (each carries the warp permutation)
  if ((e = cub::DeviceRadixSort::SortPairs(f.cub, tb, f.h_lo, f.k64, f.perm_a, f.perm_b, (int64_t)W, 0, 64, s)))
    return e;
  note_launch(), k_gather_u64<<<grid_for(W, 256), 256, 0, s>>>(W, f.perm_b, f.h_hi, f.g64);
  tb = f.cub_bytes;
  if ((e = cub::DeviceRadixSort::SortPairs(f.cub, tb, f.g64, f.k64, f.perm_b, f.perm_a, (int64_t)W, 0, 64, s)))
    return e;
  note_launch(), k_gather_u32<<<grid_for(W, 256), 256, 0, s>>>(W, f.perm_a, f.kid, f.g32);
  tb = f.cub_bytes;
  if ((e = cub::DeviceRadixSort::SortPairs(f.cub, tb, f.g32, f.k32, f.perm_a, f.perm_b, (int64_t)W, 0, 32, s)))
    return e;
  const uint32_t* perm = f.perm_b;
  note_launch(), k_full_flags<<<grid_for(W, 256), 256, 0, s>>>(W, perm, f.kid, f.h_lo, f.h_hi, f.flag);
  tb = f.cub_bytes;
  if ((e = cub::DeviceScan::InclusiveSum(f.cub, tb, f.flag, f.gid, (int64_t)W, s))) return e;
  cudaMemsetAsync(ht.hkey, 0, sizeof(uint64_t) * (ht.mask + 1), s);
  note_launch(), k_full_groups<<<grid_for(W, 256), 256, 0, s>>>(W, perm, f.flag, f.gid, f.kid, bbv16, ht, f.gstart,
                                                               f.wgroup);
  note_launch(), k_full_counts<<<grid_for(W, 256), 256, 0, s>>>(W, f.gid, f.gstart, ht);
  // every warp's events sorted (by warp, then BB id): one radix sort of (warp << 16 | bb) over the bits in use
  int wbits = 1;
  while (wbits < 48 && (1ull << wbits) < W) ++wbits;
  tb = f.cub_bytes;
  if (t.E && (e = cub::DeviceRadixSort::SortKeys(f.cub, tb, f.ekey, f.sorted, (int64_t)t.E, 0, 16 + wbits, s)))
    return e;
  note_launch(), k_full_verify_short<<<tg, 256, 0, s>>>(W, perm, f.flag, f.gid, f.gstart, t.weo, t.E, f.sorted,
                                                       f.list, f.nlist + 1, err);
  note_launch(), k_full_verify<<<hg, 256, 0, s>>>(W, perm, f.flag, f.gid, f.gstart, t.weo, t.E, f.sorted, f.list,
                                                  f.nlist + 1, err);
  if ((e = launch_canonicalise(ht, t.K, t.kwo, nullptr, out, cw, err, num_sms, s))) return e;
  if (out.warp_type)
    note_launch(), k_full_remap<<<grid_for(W, 256), 256, 0, s>>>(W, f.wgroup, cw.canon, out.warp_type);
  return cudaGetLastError();
}

cudaError_t launch_ingest(uint64_t n, uint64_t W, const uint32_t* warp, const uint16_t* bb, void* cub, size_t cub_bytes,
                          uint32_t* key_out, uint16_t* bb_out, uint64_t* off, DevErr* err, cudaStream_t s) {
  note_launch(), k_ingest_check<<<grid_for(n, 256), 256, 0, s>>>(n, warp, W, err);
  cudaError_t e;
  if (n) {
    size_t tb = cub_bytes;
    if ((e = cub::DeviceRadixSort::SortPairs(cub, tb, warp, key_out, bb, bb_out, (int64_t)n, 0, 32, s))) return e;
  }
  note_launch(), k_ingest_offsets<<<grid_for(n + 1, 256), 256, 0, s>>>(n, key_out, W, off);
  return cudaGetLastError();
}

}  // namespace photon
