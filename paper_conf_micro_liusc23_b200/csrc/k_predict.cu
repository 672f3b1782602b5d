// k_predict.cu — N3: kernel-level and BB-level prediction.
//
// Kernel level, Fig 12 Step 4 / L279-281: "#insts = #insts^K' * #insts_sample / #insts^K'_sample ...
// The IPC of K is predicted to be the same as K'", so cycles(K) = cycles(K') * N_K / N_K' with N the analysed
// sample's instruction count (the A3 mass).  Exact u128 quotients rounded half up [N3-a]; one thread per kernel.
//
// BB level, Fig 7 Step 3 / L204: the remaining warps' time is "accumulating the predicted time of their basic
// blocks"; a stable type's time is its mean at the latch, S_n / n (A5).  pred_dur_sum[w] = sum of S_n(k, b) over
// the warp's events of stable types, unpredicted[w] = its events of types never stable [N3-b].  A segmented sum
// over the trace: one hardware warp per analysed warp (coalesced u16 event loads, the kernel's row of the A5
// tables stays in L1/L2), grid-stride; u64 overflow of a warp's sum is latched as ERANGE.
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

__global__ void __launch_bounds__(256) k_bb_predict(const uint64_t* __restrict__ kwo, uint32_t K, uint32_t B,
                                                    const uint64_t* __restrict__ weo, uint64_t W, uint64_t E,
                                                    const uint16_t* __restrict__ bb,
                                                    const int64_t* __restrict__ first_stable,
                                                    const uint64_t* __restrict__ dur, uint64_t* pred,
                                                    uint32_t* unpred, DevErr* err) {
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t hw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t nhw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
  // a contiguous range of analysed warps per hardware warp: the kernel index only moves forward
  const uint64_t per = ceil_div(W, nhw), w0 = hw * per, w1 = umin64(w0 + per, W);
  uint32_t k = 0;
  if (w0 < w1) {  // last kernel with kwo[k] <= w0
    uint32_t lo = 0, hi2 = K - 1;
    while (lo < hi2) {
      const uint32_t mid = (lo + hi2 + 1) >> 1;
      if (kwo[mid] <= w0) lo = mid; else hi2 = mid - 1;
    }
    k = lo;
  }
  for (uint64_t w = w0; w < w1; ++w) {
    while (k + 1 < K && kwo[k + 1] <= w) ++k;
    const uint64_t s = umin64(weo[w], E), e = umin64(umax64(weo[w + 1], s), E);
    const int64_t* fs = first_stable + (uint64_t)k * B;
    const uint64_t* ds = dur + (uint64_t)k * B;
    uint64_t lo = 0, hi = 0;  // this lane's u128 sum
    uint32_t miss = 0;
    for (uint64_t i = s + lane; i < e; i += 32) {
      const uint32_t b = bb[i];
      if (b >= B) {
        latch(err, PHOTON_ERANGE, (int64_t)i);
        continue;
      }
      if (fs[b] >= 0) {
        const uint64_t v = ds[b];
        lo += v;
        hi += lo < v;
      } else {
        ++miss;
      }
    }
    for (int o = 16; o > 0; o >>= 1) {
      const uint64_t lo2 = __shfl_xor_sync(0xffffffffu, lo, o), hi2 = __shfl_xor_sync(0xffffffffu, hi, o);
      const uint64_t t = lo + lo2;
      hi = hi + hi2 + (t < lo);
      lo = t;
      miss += __shfl_xor_sync(0xffffffffu, miss, o);
    }
    if (lane == 0) {
      if (hi != 0 || weo[w + 1] < weo[w]) latch(err, PHOTON_ERANGE, (int64_t)w);
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
                              uint32_t* unpred, DevErr* err, int num_sms, cudaStream_t s) {
  if (t.W == 0) return cudaSuccess;
  const unsigned grid = (unsigned)umin64(ceil_div(t.W * 32, 256), (uint64_t)num_sms * 16);
  note_launch(), k_bb_predict<<<grid, 256, 0, s>>>(t.kwo, t.K, t.B, t.weo, t.W, t.E, t.bb, first_stable, dur, pred,
                                                   unpred, err);
  return cudaGetLastError();
}

}  // namespace photon
