// common.cuh — device helpers shared by the libphoton kernels (sm_100a only).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <cstdio>

#include <atomic>

#include "../../include/photon.h"

#if defined(__CUDA_ARCH__) && (__CUDA_ARCH__ < 1000)
#error "libphoton is written for sm_100a (B200) only"
#endif

namespace photon {

// launches of libphoton kernels since load (one counter per process; bench.py reports it as gpu_launches)
inline std::atomic<uint64_t>& launch_counter() {
  static std::atomic<uint64_t> n{0};
  return n;
}
inline void note_launch() { launch_counter().fetch_add(1, std::memory_order_relaxed); }

// ---- debug build (PHOTON_DEBUG=1, libphoton_debug.so): device-side bounds checks ------------------------------
// compute-sanitizer is disabled on the GPU pool, so the debug library checks the accesses whose bounds are not
// evident from the code (computed shared-memory cell / table / stage addresses, bucket cursors, scatter positions):
// a failed check prints its site and traps, which the tests see as a CUDA error.  Compiled out otherwise.
#ifndef PHOTON_DEBUG
#define PHOTON_DEBUG 0
#endif
#if PHOTON_DEBUG
#define PHOTON_DCHECK(cond, what, v)                                                                       \
  do {                                                                                                     \
    if (!(cond)) {                                                                                         \
      printf("PHOTON_DCHECK failed: %s (%s:%d) value %llu\n", what, __FILE__, __LINE__,                    \
             (unsigned long long)(v));                                                                     \
      __trap();                                                                                            \
    }                                                                                                      \
  } while (0)
#else
#define PHOTON_DCHECK(cond, what, v) \
  do {                               \
  } while (0)
#endif

typedef unsigned __int128 u128;
typedef __int128 i128;

constexpr uint64_t kTimeLimit = 1ull << 40;  // [P-16] ticks < 2^40
constexpr uint64_t kMassLimit = 1ull << 50;  // N_k < 2^50 (u128 cross products stay exact)
constexpr uint64_t kInstsLimit = 1ull << 32; // per-warp instructions < 2^32 (u32 bins)
constexpr uint32_t kMaxLen = (1u << 17) - 1; // bb_len < 2^17 (packed table entry)

// ---- device error latch: first error wins (code, index) -----------------------------------------------------
struct DevErr {
  int32_t code;
  int32_t pad;
  int64_t index;
};

__device__ __forceinline__ void latch(DevErr* e, int code, int64_t index) {
  if (*(volatile int32_t*)&e->code != 0) return;  // already latched: skip the contended CAS
  if (atomicCAS(&e->code, 0, code) == 0) {
    e->index = index;
  }
}

// ---- workspace carving ------------------------------------------------------------------------------------
struct Carver {
  size_t off = 0;
  uint8_t* base = nullptr;
  explicit Carver(void* b) : base((uint8_t*)b) {}
  template <class T>
  T* take(size_t n) {
    off = (off + 255) & ~(size_t)255;
    T* p = base ? (T*)(base + off) : nullptr;
    off += n * sizeof(T);
    return p;
  }
};

// ---- single-CTA exclusive scan of u32 counts into u64 offsets (any multiple of 32 threads) -------------------
// off[i] = sum of cnt[0..i), off[n] = the total; zero[i] = 0 when zero != nullptr.  Tiles of 1024 x 8 counts: each
// thread sums 8 consecutive counts in registers, one block scan of the thread sums per tile (two barriers), so a
// K of 10^4 takes two tiles.  Returns the total (thread 0 only).
__device__ __forceinline__ uint64_t cta_scan_counts(const uint32_t* __restrict__ cnt, uint32_t n, uint64_t* off,
                                                    uint32_t* zero) {
  constexpr int IT = 8;
  __shared__ uint64_t s_ws[32];
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  uint64_t carry = 0;  // identical in every thread
  for (uint32_t base = 0; base < n; base += blockDim.x * IT) {
    uint32_t v[IT];
    const uint32_t i0 = base + tid * IT;
    uint64_t sum = 0;
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      v[j] = i0 + j < n ? cnt[i0 + j] : 0u;
      sum += v[j];
    }
    if (zero) {
#pragma unroll
      for (int j = 0; j < IT; ++j)
        if (i0 + j < n) zero[i0 + j] = 0u;
    }
    uint64_t x = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(0xffffffffu, x, o);
      if ((int)lane >= o) x += y;
    }
    if (lane == 31) s_ws[wid] = x;
    __syncthreads();
    uint64_t w = lane < (blockDim.x >> 5) ? s_ws[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint64_t y = __shfl_up_sync(0xffffffffu, w, o);
      if ((int)lane >= o) w += y;
    }
    const uint64_t wex = __shfl_sync(0xffffffffu, w, wid) - s_ws[wid];  // warps before this one
    const uint64_t tot = __shfl_sync(0xffffffffu, w, 31);
    __syncthreads();  // s_ws is rewritten by the next tile
    uint64_t run = carry + wex + x - sum;
#pragma unroll
    for (int j = 0; j < IT; ++j) {
      if (i0 + j < n) off[i0 + j] = run;
      run += v[j];
    }
    carry += tot;
  }
  if (tid == 0) off[n] = carry;
  return carry;
}

__host__ __device__ __forceinline__ uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }
__host__ __device__ __forceinline__ uint64_t umax64(uint64_t a, uint64_t b) { return a > b ? a : b; }
__host__ __device__ __forceinline__ uint64_t ceil_div(uint64_t a, uint64_t b) { return (a + b - 1) / b; }
__host__ __device__ __forceinline__ uint32_t next_pow2_u32(uint32_t v) {
  uint32_t p = 1;
  while (p < v) p <<= 1;
  return p;
}

// ---- hashing of (kernel, 16-bin key) ----------------------------------------------------------------------
__device__ __forceinline__ uint64_t mix64(uint64_t x) {
  x ^= x >> 31;
  x *= 0x7FB5D329728EA185ull;
  x ^= x >> 27;
  x *= 0x81DADEF4BC2DD44Dull;
  x ^= x >> 33;
  return x;
}
// Bucketing hash only (equality is always verified on the full key): a sum of products with distinct odd 64-bit
// multipliers (two IMADs each, mod 2^64) followed by a 64-bit finaliser.
__device__ __forceinline__ uint64_t hash_key(uint32_t k, const uint32_t* p) {
  constexpr uint64_t M[17] = {0x9E3779B97F4A7C15ull, 0xC2B2AE3D27D4EB4Full, 0x165667B19E3779F9ull,
                              0xD6E8FEB86659FD93ull, 0xFF51AFD7ED558CCDull, 0xC4CEB9FE1A85EC53ull,
                              0x94D049BB133111EBull, 0xBF58476D1CE4E5B9ull, 0x2545F4914F6CDD1Dull,
                              0x5851F42D4C957F2Dull, 0x14057B7EF767814Full, 0x7FB5D329728EA185ull,
                              0x81DADEF4BC2DD44Dull, 0xA0761D6478BD642Full, 0xE7037ED1A0B428DBull,
                              0x8EBC6AF09C88C6E3ull, 0x589965CC75374CC3ull};
  uint64_t h = (uint64_t)k * M[16] + 0x632BE59BD9B4E019ull;
#pragma unroll
  for (int j = 0; j < 16; ++j) h += (uint64_t)p[j] * M[j];
  h = mix64(h);
  return h ? h : 1;
}

// ---- PTX wrappers: mbarrier + 1-D bulk copy (TMA engine) ------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.release.cta.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.acquire.cta.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
      : "=r"(ok)
      : "r"(smem_u32(bar)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  while (!mbar_try_wait(bar, parity)) {
  }
}
// global -> shared bulk copy, completion counted on `bar` (bytes multiple of 16, addresses 16-byte aligned)
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__device__ __forceinline__ uint32_t ld_acquire_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(uint32_t* p, uint32_t v) {
  asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint4 ld_relaxed_v4(const uint32_t* p) {
  uint4 v;
  asm volatile("ld.relaxed.gpu.global.v4.u32 {%0, %1, %2, %3}, [%4];"
               : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
               : "l"(p)
               : "memory");
  return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_u32(const uint32_t* p) {
  uint32_t v;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// ---- 128-bit helpers ---------------------------------------------------------------------------------------
__device__ __forceinline__ u128 mul64x64(uint64_t a, uint64_t b) {
  return (u128)a * b;
}

// ---- global warp-type hash table (workspace) ------------------------------------------------------------------
struct HashTable {
  uint64_t* hkey;   // [cap] 0 = empty, else hash (nonzero)
  uint32_t* ready;  // [cap] 1 once kern/key are published
  uint32_t* kern;   // [cap]
  uint32_t* key;    // [cap][16]
  uint32_t* count;  // [cap]
  uint64_t* first;  // [cap] min warp index (init ~0)
  uint64_t mask;    // cap - 1 (cap power of two)
};

// Insert-or-find (k, p) with hash h.  Returns the slot, or UINT32_MAX (after latching ECAPACITY) when full.
// Adds `cnt` to the slot's count and lowers its first warp to `wmin`.  Readers spin only on slots whose writer
// already won the CAS (it runs to completion without waiting), so there is no deadlock.
__device__ __forceinline__ uint32_t ht_insert(const HashTable& ht, DevErr* err, uint32_t k, const uint32_t* p,
                                              uint64_t h, uint32_t cnt, uint64_t wmin) {
  uint64_t i = h & ht.mask;
  for (uint64_t probe = 0; probe <= ht.mask; ++probe) {
    // a plain read first: most insertions find their key already published (no CAS round trip)
    unsigned long long cur = *(volatile unsigned long long*)&ht.hkey[i];
    if (cur == 0ull) cur = atomicCAS((unsigned long long*)&ht.hkey[i], 0ull, (unsigned long long)h);
    bool mine = false;
    if (cur == 0ull) {
      ht.kern[i] = k;
      uint4* dst = (uint4*)&ht.key[i * 16];
      dst[0] = make_uint4(p[0], p[1], p[2], p[3]);
      dst[1] = make_uint4(p[4], p[5], p[6], p[7]);
      dst[2] = make_uint4(p[8], p[9], p[10], p[11]);
      dst[3] = make_uint4(p[12], p[13], p[14], p[15]);
      st_release_u32(&ht.ready[i], 1u);  // release: the key and kernel writes above are visible first
      mine = true;
    } else if (cur == h) {
      while (ld_acquire_u32(&ht.ready[i]) == 0u) {
      }
      mine = ld_relaxed_u32(&ht.kern[i]) == k;
#pragma unroll
      for (int q = 0; q < 4; ++q) {  // 16-byte loads (the key row is 64-byte aligned)
        const uint4 v = ld_relaxed_v4(&ht.key[i * 16 + 4 * q]);
        mine = mine && v.x == p[4 * q] && v.y == p[4 * q + 1] && v.z == p[4 * q + 2] && v.w == p[4 * q + 3];
      }
    }
    if (mine) {
      atomicAdd(&ht.count[i], cnt);
      atomicMin((unsigned long long*)&ht.first[i], (unsigned long long)wmin);
      return (uint32_t)i;
    }
    i = (i + 1) & ht.mask;
  }
  latch(err, PHOTON_ECAPACITY, (int64_t)h);
  return UINT32_MAX;
}

}  // namespace photon
