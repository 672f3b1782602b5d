// k_types.cu — A2 canonicalisation (K2b, K2c) and the multi-GPU type-row export / merge / remap.
//
// weight_t = portion of the kernel's warps in type t; "the weighted BBVs are ordered according to a
// descending order based on the weights" -> canonical order (count desc, key asc) [P-4].  L249: warp-sampling is
// possible when the dominant type holds more than 95% of the warps [P-15].
//
// The hash table filled by K1/K2a (or by the row merge) is turned into CSR tables by: count types per kernel ->
// exclusive scan -> scatter slot ids per kernel -> per-kernel sort (shared-memory bitonic for T_k <= 4096,
// global-memory bitonic by one CTA beyond) -> emit rows and the slot -> canonical id map.  Insertion order into
// the hash table is nondeterministic; the sort key is total (keys are unique per kernel), so the result is not.
#include "internal.h"

namespace photon {

namespace {

constexpr int SORT_SMEM_MAX = 4096;
constexpr uint32_t WARP_SORT_MAX = 128;

__global__ void k_ht_clear(HashTable ht) {
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > ht.mask) return;
  ht.hkey[i] = 0ull;
  ht.ready[i] = 0u;
  ht.count[i] = 0u;
  ht.first[i] = ~0ull;
}

__global__ void k_count_types(HashTable ht, uint32_t K, uint32_t* tcount, DevErr* err) {
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > ht.mask || ht.hkey[i] == 0ull) return;
  uint32_t k = ht.kern[i];
  if (k >= K) { latch(err, PHOTON_ERANGE, (int64_t)k); return; }
  atomicAdd(&tcount[k], 1u);
}

// single CTA exclusive scan of tcount[K] -> kto[K+1]; also zeroes cursor and checks capacity
__global__ void __launch_bounds__(1024) k_scan_types(const uint32_t* tcount, uint32_t K, uint64_t* kto,
                                                      uint32_t* cursor, uint64_t capacity, DevErr* err) {
  const uint64_t total = cta_scan_counts(tcount, K, kto, cursor);
  if (threadIdx.x == 0 && total > capacity) latch(err, PHOTON_ECAPACITY, (int64_t)total);
}

__global__ void k_scatter_types(HashTable ht, uint32_t K, const uint64_t* kto, uint32_t* cursor, uint32_t* list,
                                uint64_t capacity) {
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i > ht.mask || ht.hkey[i] == 0ull) return;
  uint32_t k = ht.kern[i];
  if (k >= K) return;
  uint64_t pos = kto[k] + atomicAdd(&cursor[k], 1u);
  PHOTON_DCHECK(pos < kto[k + 1], "type slot past its kernel's list", k);
  if (pos < capacity) list[pos] = (uint32_t)i;
}

// canonical order: count descending, then key lexicographically ascending [P-4], then the lowest warp [N2-a] (the
// projected grouping has unique keys per kernel, so only full-BBV types reach it); UINT32_MAX = padding (last)
__device__ __forceinline__ bool type_before(const HashTable& ht, uint32_t a, uint32_t b) {
  if (b == UINT32_MAX) return a != UINT32_MAX;
  if (a == UINT32_MAX) return false;
  uint32_t ca = ht.count[a], cb = ht.count[b];
  if (ca != cb) return ca > cb;
  const uint32_t* ka = ht.key + (uint64_t)a * 16;
  const uint32_t* kb = ht.key + (uint64_t)b * 16;
#pragma unroll 1
  for (int j = 0; j < 16; ++j)
    if (ka[j] != kb[j]) return ka[j] < kb[j];
  return ht.first[a] < ht.first[b];
}

// A3 of one row (Fig 5, L178 [P-5]): g = count * key word (u64), and g / N_k in fp32 through 1/N_k in fp64 (the
// same arithmetic as k_sigf)
__device__ __forceinline__ uint64_t key_sum(const uint4* kp) {
  uint64_t t = 0;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint4 v = kp[q];
    t += (uint64_t)v.x + v.y + v.z + v.w;
  }
  return t;
}
__device__ __forceinline__ void emit_sig_row(const SigOut& so, uint64_t row, uint64_t cnt, const uint4* kp,
                                             double inv) {
  ulonglong2* g2 = (ulonglong2*)(so.sig + row * 16);
  float4* f4 = (float4*)(so.sigf + row * 16);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint4 v = kp[q];
    const uint64_t a = cnt * v.x, b = cnt * v.y, c = cnt * v.z, d = cnt * v.w;
    g2[2 * q] = make_ulonglong2(a, b);
    g2[2 * q + 1] = make_ulonglong2(c, d);
    f4[q] = make_float4((float)((double)a * inv), (float)((double)b * inv), (float)((double)c * inv),
                        (float)((double)d * inv));
  }
}
__device__ __forceinline__ uint64_t warp_sum_u64(uint64_t x) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
  return x;
}

__device__ void emit_rows(const HashTable& ht, uint32_t k, const uint32_t* sorted, uint64_t n, uint64_t off,
                          const photon_types& out, uint32_t* canon, uint64_t Wk, const SigOut& so) {
  __shared__ unsigned long long s_mass;
  if (threadIdx.x == 0) s_mass = 0;
  __syncthreads();
  uint64_t part = 0;
  for (uint64_t r = threadIdx.x; r < n && off + r < out.capacity; r += blockDim.x) {
    uint32_t s = sorted[r];
    const uint4* src = (const uint4*)(ht.key + (uint64_t)s * 16);
    uint4* dst = (uint4*)(out.type_key + (off + r) * 16);
    dst[0] = src[0]; dst[1] = src[1]; dst[2] = src[2]; dst[3] = src[3];
    out.type_count[off + r] = ht.count[s];
    out.type_first_warp[off + r] = ht.first[s];
    canon[s] = (uint32_t)r;
    if (so.sig) part += (uint64_t)ht.count[s] * key_sum(src);
  }
  if (threadIdx.x == 0) {
    uint64_t c0 = n ? ht.count[sorted[0]] : 0;
    out.warp_sampling_ok[k] = (Wk > 0 && 100ull * c0 > 95ull * Wk) ? 1 : 0;  // L249, strict [P-15]
  }
  if (so.sig) {
    part = warp_sum_u64(part);
    if ((threadIdx.x & 31) == 0) atomicAdd(&s_mass, (unsigned long long)part);
    __syncthreads();
    const uint64_t N = s_mass;
    const double inv = N ? 1.0 / (double)N : 0.0;
    for (uint64_t r = threadIdx.x; r < n && off + r < out.capacity; r += blockDim.x) {
      const uint32_t s = sorted[r];
      emit_sig_row(so, off + r, ht.count[s], (const uint4*)(ht.key + (uint64_t)s * 16), inv);
    }
  }
}

// 32 < T_k <= 128: a register bitonic sort of 32E elements (E per lane, element i = lane * E + e) on a packed key
// (~count) << 32 | key word 0 -- count desc, then key asc -- with the full-key compare (type_before) on ties.
template <int E>
__device__ __forceinline__ void warp_sort_reg(const HashTable& ht, uint64_t (&sk)[E], uint32_t (&sl)[E]) {
  const uint32_t lane = threadIdx.x & 31;
  auto before = [&](uint64_t ka, uint32_t sa, uint64_t kb, uint32_t sb) -> bool {  // a before b, padding last
    if (sa == UINT32_MAX) return false;
    if (sb == UINT32_MAX) return true;
    if (ka != kb) return ka < kb;
    return type_before(ht, sa, sb);
  };
  auto cswap = [&](int e, int f, uint32_t size) {  // in-lane pair (e < f)
    const bool up = ((lane * E + e) & size) == 0;
    const bool sw = up ? before(sk[f], sl[f], sk[e], sl[e]) : before(sk[e], sl[e], sk[f], sl[f]);
    if (sw) {
      const uint64_t tk = sk[e]; sk[e] = sk[f]; sk[f] = tk;
      const uint32_t ts = sl[e]; sl[e] = sl[f]; sl[f] = ts;
    }
  };
  for (uint32_t size = 2; size <= 32u * E; size <<= 1) {
    for (uint32_t st = size >> 1; st > 0; st >>= 1) {
      if (st >= (uint32_t)E) {
        const uint32_t ls = st / E;
        const bool lower = (lane & ls) == 0;
#pragma unroll
        for (int e = 0; e < E; ++e) {
          const uint64_t ok = __shfl_xor_sync(0xffffffffu, sk[e], ls);
          const uint32_t os = __shfl_xor_sync(0xffffffffu, sl[e], ls);
          const bool up = ((lane * E + e) & size) == 0;
          const bool mb = before(sk[e], sl[e], ok, os);
          const bool keep = (lower == up) ? mb : !mb;
          if (!keep && os != sl[e]) { sk[e] = ok; sl[e] = os; }
        }
      } else if (st == 1) {
#pragma unroll
        for (int e = 0; e < E; e += 2) cswap(e, e + 1, size);
      } else {  // st == 2 (E == 4)
        if (E == 4) { cswap(0, 2, size); cswap(1, 3, size); }
      }
    }
  }
}
template <int E>
__device__ __forceinline__ void sort_mid_reg(const HashTable& ht, uint64_t off, uint64_t n, const uint32_t* list,
                                             const photon_types& out, uint32_t* canon, uint64_t Wk, uint32_t k,
                                             const SigOut& so) {
  const uint32_t lane = threadIdx.x & 31;
  uint64_t sk[E];
  uint32_t sl[E];
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const uint32_t i = lane * E + e;
    sl[e] = i < n ? list[off + i] : UINT32_MAX;
    sk[e] = sl[e] != UINT32_MAX ? ((uint64_t)(~ht.count[sl[e]]) << 32) | ht.key[(uint64_t)sl[e] * 16] : ~0ull;
  }
  warp_sort_reg<E>(ht, sk, sl);
#pragma unroll
  for (int e = 0; e < E; ++e) {
    const uint32_t r = lane * E + e, sl_ = sl[e];
    if (r < n && off + r < out.capacity) {
      const uint4* src = (const uint4*)(ht.key + (uint64_t)sl_ * 16);
      uint4* dst = (uint4*)(out.type_key + (off + r) * 16);
      dst[0] = src[0]; dst[1] = src[1]; dst[2] = src[2]; dst[3] = src[3];
      out.type_count[off + r] = ht.count[sl_];
      out.type_first_warp[off + r] = ht.first[sl_];
      canon[sl_] = r;
    }
  }
  if (so.sig) {
    uint64_t part = 0;
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const uint32_t r = lane * E + e;
      if (r < n && off + r < out.capacity)
        part += (uint64_t)ht.count[sl[e]] * key_sum((const uint4*)(ht.key + (uint64_t)sl[e] * 16));
    }
    const uint64_t N = warp_sum_u64(part);
    const double inv = N ? 1.0 / (double)N : 0.0;
#pragma unroll
    for (int e = 0; e < E; ++e) {
      const uint32_t r = lane * E + e;
      if (r < n && off + r < out.capacity)
        emit_sig_row(so, off + r, ht.count[sl[e]], (const uint4*)(ht.key + (uint64_t)sl[e] * 16), inv);
    }
  }
  const uint32_t first = __shfl_sync(0xffffffffu, sl[0], 0);
  if (lane == 0) {
    const uint64_t c0 = ht.count[first];
    out.warp_sampling_ok[k] = (Wk > 0 && 100ull * c0 > 95ull * Wk) ? 1 : 0;  // L249 [P-15]
  }
}

// Kernels with T_k <= 32 (almost all): one warp each, bitonic network over the first P = next_pow2(T_k) lanes with
// shuffles; 32 < T_k <= 128: the same warp, a register bitonic sort of 2 or 4 elements per lane.  Larger kernels are queued:
// T_k <= SORT_SMEM_MAX at the front of cw.big (k_sort_mid, one CTA each), larger ones at the back (k_sort_large).
__global__ void __launch_bounds__(256) k_sort_warp(HashTable ht, uint32_t K, const uint64_t* kto,
                                                   const uint32_t* list, const uint64_t* kwo,
                                                   const uint64_t* kernel_warps, photon_types out, uint32_t* canon,
                                                   uint32_t* big, uint32_t* nbig, SigOut so) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t k = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  if (k >= K) return;
  const uint64_t off = kto[k], n = kto[k + 1] - off;
  const uint64_t Wk = kernel_warps ? kernel_warps[k] : (kwo[k + 1] - kwo[k]);
  if (n > 32 && n <= 64) {
    sort_mid_reg<2>(ht, off, n, list, out, canon, Wk, k, so);
    return;
  }
  if (n > 64 && n <= WARP_SORT_MAX) {
    sort_mid_reg<4>(ht, off, n, list, out, canon, Wk, k, so);
    return;
  }
  if (n > 32) {
    if (lane == 0) {
      if (n <= SORT_SMEM_MAX) big[atomicAdd(&nbig[0], 1u)] = k;
      else big[K - 1 - atomicAdd(&nbig[1], 1u)] = k;
    }
    return;
  }
  // register bitonic over (count, key words 0-3, slot): values travel with the slot; full-key compare only on ties
  uint32_t mine = lane < n ? list[off + lane] : UINT32_MAX;
  uint32_t mc = 0;
  uint4 mk = make_uint4(0, 0, 0, 0);
  if (mine != UINT32_MAX) {
    mc = ht.count[mine];
    mk = *(const uint4*)(ht.key + (uint64_t)mine * 16);
  }
  uint32_t P = 1;  // the network over the first P >= n lanes only (xor partners stay inside aligned P-blocks)
  while (P < n) P <<= 1;
  for (uint32_t size = 2; size <= P; size <<= 1) {
    for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
      const uint32_t other = __shfl_xor_sync(0xffffffffu, mine, stride);
      const uint32_t oc = __shfl_xor_sync(0xffffffffu, mc, stride);
      uint4 ok;
      ok.x = __shfl_xor_sync(0xffffffffu, mk.x, stride);
      ok.y = __shfl_xor_sync(0xffffffffu, mk.y, stride);
      ok.z = __shfl_xor_sync(0xffffffffu, mk.z, stride);
      ok.w = __shfl_xor_sync(0xffffffffu, mk.w, stride);
      const bool up = (lane & size) == 0;
      const bool lower = (lane & stride) == 0;
      bool mb;  // mine before other (padding last)
      if (other == UINT32_MAX) mb = mine != UINT32_MAX;
      else if (mine == UINT32_MAX) mb = false;
      else if (mc != oc) mb = mc > oc;
      else if (mk.x != ok.x) mb = mk.x < ok.x;
      else if (mk.y != ok.y) mb = mk.y < ok.y;
      else if (mk.z != ok.z) mb = mk.z < ok.z;
      else if (mk.w != ok.w) mb = mk.w < ok.w;
      else mb = type_before(ht, mine, other);  // words 4.. (rare)
      bool keep = (lower == up) ? mb : !mb;
      if (mine == other) keep = true;
      if (!keep) { mine = other; mc = oc; mk = ok; }
    }
  }
  const bool row = lane < n && off + lane < out.capacity;
  if (row) {
    const uint4* src = (const uint4*)(ht.key + (uint64_t)mine * 16);
    uint4* dst = (uint4*)(out.type_key + (off + lane) * 16);
    dst[0] = src[0]; dst[1] = src[1]; dst[2] = src[2]; dst[3] = src[3];
    out.type_count[off + lane] = ht.count[mine];
    out.type_first_warp[off + lane] = ht.first[mine];
    canon[mine] = lane;
  }
  if (so.sig) {
    const uint4* kp = (const uint4*)(ht.key + (uint64_t)(row ? mine : 0u) * 16);
    const uint64_t N = warp_sum_u64(row ? (uint64_t)mc * key_sum(kp) : 0ull);
    const double inv = N ? 1.0 / (double)N : 0.0;
    if (row) emit_sig_row(so, off + lane, mc, kp, inv);
  }
  uint32_t c0 = __shfl_sync(0xffffffffu, mine != UINT32_MAX ? mc : 0u, 0);
  if (lane == 0) out.warp_sampling_ok[k] = (Wk > 0 && 100ull * c0 > 95ull * Wk) ? 1 : 0;  // L249 [P-15]
}

// 32 < T_k <= SORT_SMEM_MAX: one CTA per queued kernel, shared-memory bitonic sort
__global__ void __launch_bounds__(512) k_sort_mid(HashTable ht, uint32_t K, const uint64_t* kto,
                                                  const uint32_t* list, const uint64_t* kwo,
                                                  const uint64_t* kernel_warps, photon_types out, uint32_t* canon,
                                                  const uint32_t* big, const uint32_t* nbig, SigOut so) {
  __shared__ uint32_t sh[SORT_SMEM_MAX];
  const uint32_t nmid = nbig[0];
  for (uint32_t q = blockIdx.x; q < nmid; q += gridDim.x) {
    const uint32_t k = big[q];
    uint64_t off = kto[k], n = kto[k + 1] - off;
    uint64_t Wk = kernel_warps ? kernel_warps[k] : (kwo[k + 1] - kwo[k]);
    uint32_t P = 1;
    while (P < n) P <<= 1;
    for (uint32_t i = threadIdx.x; i < P; i += blockDim.x) sh[i] = i < n ? list[off + i] : UINT32_MAX;
    __syncthreads();
    for (uint32_t size = 2; size <= P; size <<= 1) {
      for (uint32_t stride = size >> 1; stride > 0; stride >>= 1) {
        for (uint32_t t = threadIdx.x; t < P / 2; t += blockDim.x) {
          uint32_t i = 2 * stride * (t / stride) + (t % stride);
          uint32_t j = i + stride;
          bool up = ((i & size) == 0);
          uint32_t a = sh[i], b = sh[j];
          bool sw = up ? type_before(ht, b, a) : type_before(ht, a, b);
          if (sw) { sh[i] = b; sh[j] = a; }
        }
        __syncthreads();
      }
    }
    emit_rows(ht, k, sh, n, off, out, canon, Wk, so);
    __syncthreads();
  }
}

// T_k > SORT_SMEM_MAX (rare: highly irregular kernels): one CTA, global-memory bitonic sort in scratch
__global__ void __launch_bounds__(1024) k_sort_large(HashTable ht, uint32_t K, const uint64_t* kto,
                                                     const uint32_t* list, const uint64_t* kwo,
                                                     const uint64_t* kernel_warps, photon_types out, uint32_t* canon,
                                                     uint32_t* scratch, const uint32_t* big, const uint32_t* nbig,
                                                     SigOut so) {
  const uint32_t nlarge = nbig[1];
  for (uint32_t q = 0; q < nlarge; ++q) {
    const uint32_t k = big[K - 1 - q];
    uint64_t off = kto[k], n = kto[k + 1] - off;
    uint64_t Wk = kernel_warps ? kernel_warps[k] : (kwo[k + 1] - kwo[k]);
    uint64_t P = 1;
    while (P < n) P <<= 1;
    for (uint64_t i = threadIdx.x; i < P; i += blockDim.x) scratch[i] = i < n ? list[off + i] : UINT32_MAX;
    __syncthreads();
    for (uint64_t size = 2; size <= P; size <<= 1) {
      for (uint64_t stride = size >> 1; stride > 0; stride >>= 1) {
        for (uint64_t t = threadIdx.x; t < P / 2; t += blockDim.x) {
          uint64_t i = 2 * stride * (t / stride) + (t % stride);
          uint64_t j = i + stride;
          bool up = ((i & size) == 0);
          uint32_t a = scratch[i], b = scratch[j];
          bool sw = up ? type_before(ht, b, a) : type_before(ht, a, b);
          if (sw) { scratch[i] = b; scratch[j] = a; }
        }
        __syncthreads();
      }
    }
    emit_rows(ht, k, scratch, n, off, out, canon, Wk, so);
    __syncthreads();
  }
}

// K2a: insert every used pool entry into the global table.  One hardware warp takes 32 consecutive entries (a K1
// worker's entries are consecutive, so neighbours often share a key): equal (kernel, key) entries are grouped with
// __match_any_sync on the hash plus an exact key check, their counts / first warps combined in shared memory, and
// only each group's leader probes the table.  Unused entries (count 0) get no slot.
#ifndef PHOTON_IMINB
#define PHOTON_IMINB 5  // > 0: __launch_bounds__(256, PHOTON_IMINB) (5: an 8-byte spill, measured -4 us on C5)
#endif
#if PHOTON_IMINB > 0
#define PHOTON_IMINB_LB __launch_bounds__(256, PHOTON_IMINB)
#else
#define PHOTON_IMINB_LB __launch_bounds__(256)
#endif
__global__ void PHOTON_IMINB_LB k_entries_insert(EntryPool ep, HashTable ht, DevErr* err) {
  __shared__ uint32_t s_cnt[256];
  __shared__ unsigned long long s_first[256];
  const uint64_t n = umin64(*ep.count, ep.cap);
  const uint32_t lane = threadIdx.x & 31, wb = threadIdx.x & ~31u;
  const uint64_t nwarps = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t base = (((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5) << 5; base < n; base += nwarps << 5) {
    const uint64_t j = base + lane;
    uint32_t key[16], k = 0, cnt = 0;
    uint64_t first = ~0ull;
    if (j < n) {
      const TileEntry* x = ep.ent + j;
      const uint4* kp = (const uint4*)x->key;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const uint4 v = kp[q];
        key[4 * q] = v.x; key[4 * q + 1] = v.y; key[4 * q + 2] = v.z; key[4 * q + 3] = v.w;
      }
      const uint4 m = kp[4];  // first (u64), kernel, count
      first = ((uint64_t)m.y << 32) | m.x;
      k = m.z;
      cnt = m.w;
    } else {
#pragma unroll
      for (int q = 0; q < 16; ++q) key[q] = 0u;
    }
    const bool valid = cnt != 0u;
    const uint64_t h = valid ? hash_key(k, key) : 0ull;
    const unsigned peers = __match_any_sync(0xffffffffu, (unsigned long long)h);
    const int leader = __ffs(peers) - 1;
    bool eq = __shfl_sync(0xffffffffu, k, leader) == k;
#pragma unroll
    for (int q = 0; q < 16; ++q) eq &= (__shfl_sync(0xffffffffu, key[q], leader) == key[q]);
    const int g = (valid && eq) ? leader : (int)lane;  // my group's representative lane
    s_cnt[threadIdx.x] = 0u;
    s_first[threadIdx.x] = ~0ull;
    __syncwarp();
    if (valid) {
      atomicAdd(&s_cnt[wb + g], cnt);
      atomicMin(&s_first[wb + g], (unsigned long long)first);
    }
    __syncwarp();
    uint32_t slot = UINT32_MAX;
    if (valid && g == (int)lane) slot = ht_insert(ht, err, k, key, h, s_cnt[threadIdx.x], s_first[threadIdx.x]);
    const uint32_t gs = __shfl_sync(0xffffffffu, slot, g);
    if (j < n) ep.slot[j] = valid ? gs : UINT32_MAX;
  }
}

// K2c: warp_type[w] = canonical id of the warp's entry.  Eight warps per thread (strided by the grid) so each
// thread keeps eight independent gid -> slot -> canon chains in flight.
constexpr int REMAP_ILP = 8;
__device__ __forceinline__ uint32_t entry_slot(const EntryPool& ep, uint32_t g) {
  return g < ep.cap ? ep.slot[g] : UINT32_MAX;  // beyond cap only after ECAPACITY was latched
}
__global__ void __launch_bounds__(256) k_remap_entries(EntryPool ep, uint64_t W, const uint32_t* canon,
                                                       uint32_t* warp_type) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t w0 = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint32_t g[REMAP_ILP], sl[REMAP_ILP];
#pragma unroll
  for (int u = 0; u < REMAP_ILP; ++u) {
    const uint64_t w = w0 + u * stride;
    g[u] = w < W ? ep.gid[w] : 0u;
  }
#pragma unroll
  for (int u = 0; u < REMAP_ILP; ++u) sl[u] = w0 + u * stride < W ? entry_slot(ep, g[u]) : UINT32_MAX;
#pragma unroll
  for (int u = 0; u < REMAP_ILP; ++u) {
    const uint64_t w = w0 + u * stride;
    if (w < W) warp_type[w] = sl[u] == UINT32_MAX ? UINT32_MAX : canon[sl[u]];
  }
}

__device__ __forceinline__ uint32_t row_kernel(const uint64_t* kto, uint32_t K, uint64_t row) {
  uint32_t lo = 0, hi = K - 1;
  while (lo < hi) {
    uint32_t mid = (lo + hi + 1) >> 1;
    if (kto[mid] <= row) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// rows [0, min(T, cap)) = the local types; [T, cap) = padding rows (kernel PHOTON_ROW_PAD, skipped by the merge);
// n_rows (device, optional) = T, so a caller with a fixed capacity can detect T > cap
__global__ void k_export(uint32_t K, photon_types local, uint32_t kernel_base, uint64_t warp_base,
                         photon_type_row* rows, uint64_t cap, uint64_t* n_rows) {
  uint64_t T = local.kernel_type_off[K];
  uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (r == 0 && n_rows) *n_rows = T;
  if (r >= cap) return;
  photon_type_row x;
  if (r >= T) {
    x.kernel = PHOTON_ROW_PAD;
    x.pad = 0;
    for (int j = 0; j < 16; ++j) x.key[j] = 0;
    x.count = 0;
    x.first_warp = 0;
    rows[r] = x;
    return;
  }
  x.kernel = kernel_base + row_kernel(local.kernel_type_off, K, r);
  x.pad = 0;
  for (int j = 0; j < 16; ++j) x.key[j] = local.type_key[r * 16 + j];
  x.count = local.type_count[r];
  x.first_warp = local.type_first_warp[r] + warp_base;
  rows[r] = x;
}

__global__ void k_rows_insert(const photon_type_row* rows, uint64_t n, uint32_t K, HashTable ht, DevErr* err) {
  uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= n) return;
  const photon_type_row x = rows[r];
  if (x.kernel == PHOTON_ROW_PAD) return;  // padding of a fixed-capacity exchange
  if (x.kernel >= K || x.count >= (1ull << 32)) { latch(err, PHOTON_ERANGE, (int64_t)r); return; }
  uint64_t h = hash_key(x.kernel, x.key);
  ht_insert(ht, err, x.kernel, x.key, h, (uint32_t)x.count, x.first_warp);
}

__device__ uint32_t ht_find(const HashTable& ht, uint32_t k, const uint32_t* p, uint64_t h) {
  uint64_t i = h & ht.mask;
  for (uint64_t probe = 0; probe <= ht.mask; ++probe) {
    uint64_t cur = ht.hkey[i];
    if (cur == 0ull) return UINT32_MAX;
    if (cur == h && ht.kern[i] == k) {
      bool same = true;
      for (int j = 0; j < 16; ++j) same = same && (ht.key[i * 16 + j] == p[j]);
      if (same) return (uint32_t)i;
    }
    i = (i + 1) & ht.mask;
  }
  return UINT32_MAX;
}

__global__ void k_remap_direct(const uint64_t* kwo, uint32_t K, uint64_t W, photon_types local,
                               uint32_t kernel_base, HashTable ht, const uint32_t* canon, uint32_t* out, DevErr* err) {
  uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v >= W) return;
  uint32_t lo = 0, hi = K - 1;
  while (lo < hi) {
    uint32_t mid = (lo + hi + 1) >> 1;
    if (kwo[mid] <= v) lo = mid; else hi = mid - 1;
  }
  uint32_t t = local.warp_type[v];
  uint64_t row = local.kernel_type_off[lo] + t;
  uint32_t kg = kernel_base + lo;
  uint32_t key[16];
  const uint4* src = (const uint4*)(local.type_key + row * 16);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint4 x = src[q];
    key[4 * q] = x.x; key[4 * q + 1] = x.y; key[4 * q + 2] = x.z; key[4 * q + 3] = x.w;
  }
  uint32_t s = ht_find(ht, kg, key, hash_key(kg, key));
  if (s == UINT32_MAX) { latch(err, PHOTON_ERANGE, (int64_t)v); out[v] = UINT32_MAX; return; }
  out[v] = canon[s];
}

}  // namespace

cudaError_t launch_ht_clear(const HashTable& ht, cudaStream_t s) {
  uint64_t cap = ht.mask + 1;
  note_launch(), k_ht_clear<<<(unsigned)ceil_div(cap, 256), 256, 0, s>>>(ht);
  return cudaGetLastError();
}

cudaError_t launch_canon_lists(const HashTable& ht, uint32_t K, const photon_types& out, const CanonWs& cw,
                               DevErr* err, cudaStream_t s, bool zeroed) {
  uint64_t cap = ht.mask + 1;
  if (!zeroed) cudaMemsetAsync(cw.tcount, 0, sizeof(uint32_t) * (K ? K : 1), s);
  note_launch(), k_count_types<<<(unsigned)ceil_div(cap, 256), 256, 0, s>>>(ht, K, cw.tcount, err);
  note_launch(), k_scan_types<<<1, 1024, 0, s>>>(cw.tcount, K, out.kernel_type_off, cw.cursor, out.capacity, err);
  note_launch(), k_scatter_types<<<(unsigned)ceil_div(cap, 256), 256, 0, s>>>(ht, K, out.kernel_type_off, cw.cursor, cw.list,
                                                               out.capacity);
  return cudaGetLastError();
}
cudaError_t launch_canon_sort(const HashTable& ht, uint32_t K, const uint64_t* kwo, const uint64_t* kernel_warps,
                              const photon_types& out, const CanonWs& cw, int num_sms, cudaStream_t s, SigOut so,
                              bool zeroed) {
  if (!zeroed) cudaMemsetAsync(cw.nbig, 0, 8, s);
  note_launch(), k_sort_warp<<<(unsigned)ceil_div((uint64_t)K * 32, 256), 256, 0, s>>>(
      ht, K, out.kernel_type_off, cw.list, kwo, kernel_warps, out, cw.canon, cw.big, cw.nbig, so);
  note_launch(), k_sort_mid<<<(unsigned)num_sms, 512, 0, s>>>(ht, K, out.kernel_type_off, cw.list, kwo, kernel_warps,
                                                             out, cw.canon, cw.big, cw.nbig, so);
  note_launch(), k_sort_large<<<1, 1024, 0, s>>>(ht, K, out.kernel_type_off, cw.list, kwo, kernel_warps, out, cw.canon,
                                                cw.scratch, cw.big, cw.nbig, so);
  return cudaGetLastError();
}
cudaError_t launch_canonicalise(const HashTable& ht, uint32_t K, const uint64_t* kwo, const uint64_t* kernel_warps,
                                const photon_types& out, const CanonWs& cw, DevErr* err, int num_sms,
                                cudaStream_t s) {
  cudaError_t e = launch_canon_lists(ht, K, out, cw, err, s);
  if (e) return e;
  return launch_canon_sort(ht, K, kwo, kernel_warps, out, cw, num_sms, s);
}

cudaError_t launch_entries_insert(const EntryPool& ep, const HashTable& ht, DevErr* err, int num_sms,
                                  cudaStream_t s) {
  // grid-stride over the device entry count (unknown here): enough threads for the pool, at most 16 CTAs per SM
  uint64_t g = ceil_div(ep.cap, 256);
  const uint64_t gmax = (uint64_t)num_sms * 16;
  if (g > gmax) g = gmax;
  if (g == 0) return cudaSuccess;
  note_launch(), k_entries_insert<<<(unsigned)g, 256, 0, s>>>(ep, ht, err);
  return cudaGetLastError();
}

cudaError_t launch_remap_entries(const EntryPool& ep, uint64_t W, const uint32_t* canon, uint32_t* warp_type,
                                 cudaStream_t s) {
  if (W == 0) return cudaSuccess;
  note_launch(), k_remap_entries<<<(unsigned)ceil_div(ceil_div(W, REMAP_ILP), 256), 256, 0, s>>>(ep, W, canon,
                                                                                                 warp_type);
  return cudaGetLastError();
}

cudaError_t launch_types_export(uint32_t K, const photon_types& local, uint32_t kernel_base, uint64_t warp_base,
                                photon_type_row* rows, uint64_t row_cap, uint64_t* n_rows, cudaStream_t s) {
  // T is on the device: launch for the row capacity and guard inside
  const uint64_t cap = row_cap ? row_cap : 1;
  note_launch(), k_export<<<(unsigned)ceil_div(cap, 256), 256, 0, s>>>(K, local, kernel_base, warp_base, rows,
                                                                         row_cap, n_rows);
  return cudaGetLastError();
}

cudaError_t launch_rows_insert(const photon_type_row* rows, uint64_t n, uint32_t K, const HashTable& ht,
                               DevErr* err, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  note_launch(), k_rows_insert<<<(unsigned)ceil_div(n, 256), 256, 0, s>>>(rows, n, K, ht, err);
  return cudaGetLastError();
}

cudaError_t launch_remap_direct(const uint64_t* kwo_local, uint32_t K_local, uint64_t W_local,
                                const photon_types& local, uint32_t kernel_base, const HashTable& ht,
                                const uint32_t* canon, uint32_t* warp_type_global, DevErr* err, cudaStream_t s) {
  if (W_local == 0) return cudaSuccess;
  note_launch(), k_remap_direct<<<(unsigned)ceil_div(W_local, 256), 256, 0, s>>>(kwo_local, K_local, W_local, local, kernel_base, ht,
                                                                   canon, warp_type_global, err);
  return cudaGetLastError();
}

}  // namespace photon
