// K1 core microbenchmark (profiles/round1/k1_core_microbench.txt): staging + table lookup + private-column accumulation per event, no warp boundaries.  MODE 0 = LDS+IADD+STS, 1 = atomicAdd, 4 = red.shared.add, 2 = lookups only, 3 = no table.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o mb profiles/k1_core_microbench.cu
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <vector>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
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
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

template <int NT, int Q, int MODE>
__global__ void __launch_bounds__(NT) kmb(const uint16_t* __restrict__ bb, uint64_t nchunks, const uint32_t* tblg,
                                          uint32_t* out) {
  constexpr int L = Q * 8;
  constexpr int CH = NT * L;  // events per chunk
  extern __shared__ __align__(128) uint8_t sm[];
  uint32_t* col = (uint32_t*)sm;                       // [16][NT]
  uint32_t* tbl = col + 16 * NT;                       // [4096]
  uint16_t* stage = (uint16_t*)(tbl + 4096);           // [2][CH]
  uint64_t* bar = (uint64_t*)(stage + 2 * CH);         // [2]
  const int t = threadIdx.x;
  for (int i = t; i < 4096; i += NT) tbl[i] = tblg[i];
  for (int i = t; i < 16 * NT; i += NT) col[i] = 0;
  if (t == 0) { mbar_init(&bar[0], 1); mbar_init(&bar[1], 1); }
  __syncthreads();
  uint64_t c = blockIdx.x;
  uint32_t ph[2] = {0, 0};
  if (t == 0 && c < nchunks) {
    mbar_arrive_expect_tx(&bar[0], CH * 2);
    bulk_g2s(stage, bb + c * CH, CH * 2, &bar[0]);
  }
  uint32_t acc = 0;
  uint32_t* mycol = col + t;
  int buf = 0;
  for (; c < nchunks; c += gridDim.x) {
    uint64_t cn = c + gridDim.x;
    if (t == 0 && cn < nchunks) {
      mbar_arrive_expect_tx(&bar[buf ^ 1], CH * 2);
      bulk_g2s(stage + (buf ^ 1) * CH, bb + cn * CH, CH * 2, &bar[buf ^ 1]);
    }
    while (!mbar_try_wait(&bar[buf], ph[buf])) {}
    ph[buf] ^= 1;
    const uint4* w = (const uint4*)(stage + buf * CH) + t * Q;
#pragma unroll 3
    for (int k = 0; k < Q; ++k) {
      uint4 v = w[k];
      uint32_t e[8] = {v.x & 0xffff, v.x >> 16, v.y & 0xffff, v.y >> 16, v.z & 0xffff, v.z >> 16, v.w & 0xffff, v.w >> 16};
#pragma unroll
      for (int i = 0; i < 8; ++i) {
        uint32_t te;
        if (MODE == 3) te = ((e[i] & 15u) * (NT * 4)) | (((e[i] >> 4) & 63u) << 16);
        else te = tbl[e[i]];
        uint32_t* p = (uint32_t*)((uint8_t*)mycol + (te & 0xFFFFu));
        uint32_t len = te >> 16;
        if (MODE == 0 || MODE == 3) { *p += len; }
        else if (MODE == 1) { atomicAdd(p, len); }
        else if (MODE == 4) { asm volatile("red.shared.add.u32 [%0], %1;" :: "r"(smem_u32(p)), "r"(len) : "memory"); }
        else { acc += te; }
      }
    }
    __syncthreads();  // buffer reuse
    buf ^= 1;
  }
  uint32_t s = acc;
  for (int j = 0; j < 16; ++j) s += col[j * NT + t];
  out[blockIdx.x * NT + t] = s;
}

template <int NT, int Q, int MODE>
float run(const uint16_t* d_bb, uint64_t E, const uint32_t* d_tbl, uint32_t* d_out, int ctas_per_sm) {
  constexpr int CH = NT * Q * 8;
  uint64_t nch = E / CH;
  size_t smem = 16 * NT * 4 + 4096 * 4 + 2 * CH * 2 + 16;
  cudaFuncSetAttribute(kmb<NT, Q, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int grid = 148 * ctas_per_sm;
  cudaEvent_t a, b;
  cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 3; ++i) kmb<NT, Q, MODE><<<grid, NT, smem>>>(d_bb, nch, d_tbl, d_out);
  cudaEventRecord(a);
  const int R = 10;
  for (int i = 0; i < R; ++i) kmb<NT, Q, MODE><<<grid, NT, smem>>>(d_bb, nch, d_tbl, d_out);
  cudaEventRecord(b);
  cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  ms /= R;
  cudaError_t err = cudaGetLastError();
  double ev = (double)nch * CH;
  printf("NT=%d Q=%d MODE=%d ctas/sm=%d smem=%zu: %.3f ms  %.3e ev/s  %.1f GB/s (%s)\n", NT, Q, MODE, ctas_per_sm,
         smem, ms, ev / ms * 1e3, ev * 2 / ms / 1e6, cudaGetErrorString(err));
  return ms;
}

int main() {
  const uint64_t E = 1ull << 30;  // 2 GB of events
  std::vector<uint16_t> h(E);
  uint64_t s = 12345;
  uint32_t prog = 0, left = 0;
  for (uint64_t i = 0; i < E; ++i) {
    if (left == 0) { s = s * 6364136223846793005ull + 1442695040888963407ull; prog = (s >> 33) & 255; left = 500 + ((s >> 20) & 1023); }
    --left;
    s = s * 6364136223846793005ull + 1442695040888963407ull;
    h[i] = (uint16_t)(prog * 16 + ((s >> 40) & 15));
  }
  std::vector<uint32_t> tb(4096);
  for (int b = 0; b < 4096; ++b) tb[b] = 0;  // filled per NT below (bin offset depends on NT)
  uint16_t* d_bb; uint32_t* d_tbl; uint32_t* d_out;
  cudaMalloc(&d_bb, E * 2);
  cudaMemcpy(d_bb, h.data(), E * 2, cudaMemcpyHostToDevice);
  cudaMalloc(&d_tbl, 4096 * 4);
  cudaMalloc(&d_out, 148 * 8 * 1024 * 4);
  auto mk = [&](int NT) {
    for (int b = 0; b < 4096; ++b) tb[b] = ((b & 15) * NT * 4) | ((1 + (b * 7919) % 64) << 16);
    cudaMemcpy(d_tbl, tb.data(), 4096 * 4, cudaMemcpyHostToDevice);
  };
  mk(256);
  run<256, 9, 2>(d_bb, E, d_tbl, d_out, 2);
  run<256, 9, 0>(d_bb, E, d_tbl, d_out, 2);
  run<256, 9, 1>(d_bb, E, d_tbl, d_out, 2);
  run<256, 9, 4>(d_bb, E, d_tbl, d_out, 2);
  run<256, 9, 3>(d_bb, E, d_tbl, d_out, 2);
  run<256, 17, 0>(d_bb, E, d_tbl, d_out, 2);
  run<256, 17, 4>(d_bb, E, d_tbl, d_out, 2);
  run<256, 9, 0>(d_bb, E, d_tbl, d_out, 3);
  run<256, 9, 4>(d_bb, E, d_tbl, d_out, 3);
  mk(512);
  run<512, 9, 0>(d_bb, E, d_tbl, d_out, 1);
  run<512, 9, 4>(d_bb, E, d_tbl, d_out, 1);
  run<512, 5, 0>(d_bb, E, d_tbl, d_out, 2);
  run<512, 5, 4>(d_bb, E, d_tbl, d_out, 2);
  mk(128);
  run<128, 9, 0>(d_bb, E, d_tbl, d_out, 6);
  run<128, 9, 4>(d_bb, E, d_tbl, d_out, 6);
  run<128, 9, 2>(d_bb, E, d_tbl, d_out, 6);
  return 0;
}
