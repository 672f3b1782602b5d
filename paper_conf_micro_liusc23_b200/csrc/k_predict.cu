// k_predict.cu — N3: kernel-level and BB-level prediction.
//
// Kernel level, Fig 12 Step 4 / L279-281: "#insts = #insts^K' * #insts_sample / #insts^K'_sample ...
// The IPC of K is predicted to be the same as K'", so cycles(K) = cycles(K') * N_K / N_K' with N the analysed
// sample's instruction count (the A3 mass).  Exact u128 quotients rounded half up [N3-a]; one thread per kernel.
//
// BB level, Fig 7 Step 3, caption L201 / L208: the remaining warps' time is "accumulating the predicted time of their basic
// blocks"; a stable type's time is its mean at the latch, S_n / n (A5).  pred_dur_sum[w] = sum of S_n(k, b) over
// the warp's events of stable types, unpredicted[w] = its events of types never stable [N3-b].  A segmented sum
// over the trace: one thread per analysed warp (the kernel's row of the A5 tables stays in L1/L2; a warp's events
// are read in order, so each 32-byte sector is fetched once), grid-stride; warps longer than LONG_W events go to
// a work list that a second pass sums with one hardware warp each.  u64 overflow of a warp's sum is ERANGE.
#include "internal.h"

namespace photon {

namespace {

__global__ void k_kernel_predict(uint32_t K, const int64_t* __restrict__ match, const uint64_t* __restrict__ mass,
                                 const uint64_t* __restrict__ full_insts, const uint64_t* __restrict__ full_cycles,
                                 uint64_t* pred_insts, uint64_t* pred_cycles, DevErr* err) {
  for (uint32_t k = blockIdx.x * blockDim.x + threadIdx.x; k < K; k += gridDim.x * blockDim.x) {
    const int64_t r = match[k];
    if (r < 0) {
      pred_insts[k] = full_insts[k];
      pred_cycles[k] = full_cycles[k];
      continue;
    }
    if (r >= (int64_t)k || mass[r] == 0 || mass[k] >= kMassLimit || mass[r] >= kMassLimit) {
      latch(err, PHOTON_ERANGE, (int64_t)k);
      continue;
    }
    const u128 den = (u128)mass[r];
    const u128 qi = ((u128)full_insts[r] * mass[k] * 2 + den) / (2 * den);  // round half up
    const u128 qc = ((u128)full_cycles[r] * mass[k] * 2 + den) / (2 * den);
    if ((qi >> 64) != 0 || (qc >> 64) != 0) latch(err, PHOTON_ERANGE, (int64_t)k);
    pred_insts[k] = (uint64_t)qi;
    pred_cycles[k] = (uint64_t)qc;
  }
}

// One thread per analysed warp, 256 consecutive warps per CTA step (the block's first kernel by one binary search,
// each thread then steps forward); a thread walks its warp's events in aligned 16-byte words (eight events per
// load, independent table loads); the trace base is 16-byte aligned (photon_trace contract).
constexpr uint64_t LONG_W = 128;  // events above which a warp goes to the work list (pass 2; 128 measured best on C3)

__global__ void __launch_bounds__(256) k_bb_predict(const uint64_t* __restrict__ kwo, uint32_t K, uint32_t B,
                                                    const uint64_t* __restrict__ weo, uint64_t W, uint64_t E,
                                                    const uint16_t* __restrict__ bb,
                                                    const int64_t* __restrict__ first_stable,
                                                    const uint64_t* __restrict__ dur, uint64_t* pred,
                                                    uint32_t* unpred, uint64_t* long_list, uint32_t* n_long,
                                                    DevErr* err) {
  __shared__ uint32_t s_k0;
  for (uint64_t w0 = (uint64_t)blockIdx.x * 256; w0 < W; w0 += (uint64_t)gridDim.x * 256) {
    if (threadIdx.x == 0) {  // last kernel with kwo[k] <= w0
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
    const uint64_t s = umin64(weo[w], E), e = umin64(umax64(weo[w + 1], s), E);
    if (e - s > LONG_W) {  // a long warp: summed by a whole hardware warp in pass 2 (long warps are often
                           // contiguous, e.g. fully connected layers, so they are spread over the grid)
      long_list[atomicAdd(n_long, 1u)] = w | ((uint64_t)k << 40);
      continue;
    }
    const int64_t* fs = first_stable + (uint64_t)k * B;
    const uint64_t* ds = dur + (uint64_t)k * B;
    uint64_t lo = 0, hi = 0;  // u128 sum
    uint32_t miss = 0;
    bool bad = weo[w + 1] < weo[w];
    auto add1 = [&](uint32_t bv, uint64_t i) {
      if (bv >= B) {
        latch(err, PHOTON_ERANGE, (int64_t)i);
        return;
      }
      const int64_t f = fs[bv];
      const uint64_t x = f >= 0 ? ds[bv] : 0ull;
      miss += f < 0 ? 1u : 0u;
      lo += x;
      hi += lo < x;
    };
    // unaligned head, then whole 16-byte words (8 events per load, table loads independent), then the tail
    const uint64_t a8 = umin64((s + 7) & ~7ull, e), z8 = umax64(e & ~7ull, a8);
    for (uint64_t i = s; i < a8; ++i) add1(bb[i], i);
    for (uint64_t i0 = a8; i0 < z8; i0 += 8) {
      const uint4 q = *(const uint4*)(bb + i0);
      const uint32_t b8[8] = {q.x & 0xFFFFu, q.x >> 16, q.y & 0xFFFFu, q.y >> 16,
                              q.z & 0xFFFFu, q.z >> 16, q.w & 0xFFFFu, q.w >> 16};
      int64_t f[8];
      uint64_t v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        const uint32_t bu = b8[u] < B ? b8[u] : 0u;
        f[u] = fs[bu];
        v[u] = ds[bu];
      }
#pragma unroll
      for (int u = 0; u < 8; ++u) {
        if (b8[u] >= B) {
          latch(err, PHOTON_ERANGE, (int64_t)(i0 + u));
          continue;
        }
        const uint64_t x = f[u] >= 0 ? v[u] : 0ull;
        miss += f[u] < 0 ? 1u : 0u;
        lo += x;
        hi += lo < x;
      }
    }
    for (uint64_t i = z8; i < e; ++i) add1(bb[i], i);
    if (hi != 0 || bad) latch(err, PHOTON_ERANGE, (int64_t)w);
    pred[w] = lo;
    unpred[w] = miss;
  }
}

// pass 2: one hardware warp per listed long warp (grid-stride over the list), lanes stride its events coalesced,
// u128 shuffle reduction
__global__ void __launch_bounds__(256) k_bb_predict_long(uint32_t B, const uint64_t* __restrict__ weo, uint64_t E,
                                                         const uint16_t* __restrict__ bb,
                                                         const int64_t* __restrict__ first_stable,
                                                         const uint64_t* __restrict__ dur, uint64_t* pred,
                                                         uint32_t* unpred, const uint64_t* __restrict__ long_list,
                                                         const uint32_t* n_long, DevErr* err) {
  const int lane = threadIdx.x & 31;
  const uint32_t nl = *n_long;
  const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  for (uint64_t j = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5; j < nl; j += nw) {
    const uint64_t ent = long_list[j], w = ent & ((1ull << 40) - 1), k = ent >> 40;
    const uint64_t s = umin64(weo[w], E), e = umin64(umax64(weo[w + 1], s), E);
    const int64_t* fs = first_stable + k * B;
    const uint64_t* ds = dur + k * B;
    uint64_t lo = 0, hi = 0;
    uint32_t miss = 0;
    auto add = [&](uint32_t bv, uint64_t i) {
      if (bv >= B) {
        latch(err, PHOTON_ERANGE, (int64_t)i);
        return;
      }
      const int64_t f = fs[bv];
      const uint64_t x = f >= 0 ? ds[bv] : 0ull;
      miss += f < 0 ? 1u : 0u;
      lo += x;
      hi += lo < x;
    };
    // 16-byte vectors of 8 ids over the aligned middle (eight independent table lookups per lane and load), the
    // unaligned head and tail id by id
    const bool vec = ((uintptr_t)bb & 15) == 0;
    const uint64_t s8 = vec ? umin64((s + 7) & ~7ull, e) : e, e8 = vec ? umax64(e & ~7ull, s8) : e;
    for (uint64_t i = s + lane; i < s8; i += 32) add(bb[i], i);
#pragma unroll 2
    for (uint64_t i = s8 + 8 * (uint64_t)lane; i < e8; i += 256) {
      const uint4 v = __ldg(reinterpret_cast<const uint4*>(bb + i));
      const uint32_t w4[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
      for (int q = 0; q < 8; ++q) add((w4[q >> 1] >> ((q & 1) * 16)) & 0xFFFFu, i + q);
    }
    for (uint64_t i = e8 + lane; i < e; i += 32) add(bb[i], i);
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      const uint64_t ol = __shfl_xor_sync(0xffffffffu, lo, o), oh = __shfl_xor_sync(0xffffffffu, hi, o);
      lo += ol;
      hi += oh + (lo < ol);
      miss += __shfl_xor_sync(0xffffffffu, miss, o);
    }
    if (lane == 0) {
      if (hi != 0) latch(err, PHOTON_ERANGE, (int64_t)w);
      pred[w] = lo;
      unpred[w] = miss;
    }
  }
}

}  // namespace

cudaError_t launch_kernel_predict(uint32_t K, const int64_t* match, const uint64_t* mass, const uint64_t* full_insts,
                                  const uint64_t* full_cycles, uint64_t* pred_insts, uint64_t* pred_cycles,
                                  DevErr* err, cudaStream_t s) {
  if (K == 0) return cudaSuccess;
  note_launch(), k_kernel_predict<<<(unsigned)ceil_div(K, 256), 256, 0, s>>>(K, match, mass, full_insts, full_cycles,
                                                                             pred_insts, pred_cycles, err);
  return cudaGetLastError();
}

cudaError_t launch_bb_predict(const TraceDev& t, const int64_t* first_stable, const uint64_t* dur, uint64_t* pred,
                              uint32_t* unpred, uint64_t* long_list, uint32_t* n_long, DevErr* err, int num_sms,
                              cudaStream_t s) {
  if (t.W == 0) return cudaSuccess;
  cudaMemsetAsync(n_long, 0, 4, s);
  const unsigned grid = (unsigned)umin64(ceil_div(t.W, 256), (uint64_t)num_sms * 8);
  note_launch(), k_bb_predict<<<grid, 256, 0, s>>>(t.kwo, t.K, t.B, t.weo, t.W, t.E, t.bb, first_stable, dur, pred,
                                                   unpred, long_list, n_long, err);
  const unsigned g2 = (unsigned)umin64(ceil_div(umin64(t.W, t.E / (LONG_W + 1) + 1) * 32, 256),
                                       (uint64_t)num_sms * 16);
  note_launch(), k_bb_predict_long<<<g2 ? g2 : 1, 256, 0, s>>>(t.B, t.weo, t.E, t.bb, first_stable, dur, pred, unpred,
                                                                long_list, n_long, err);
  return cudaGetLastError();
}

}  // namespace photon
