// tracegen/gen.cpp — deterministic synthetic BB traces and timing streams shaped like the paper's workloads.
//
// This module is INPUT GENERATION ONLY.  It holds none of the method's arithmetic (no BBV, no grouping, no
// distance, no regression): it emits, per analysed warp, the sequence of executed basic-block ids, and per kernel
// the (bb, issue, retire) records of a simple wave model.  Both the CPU oracle and the CUDA path consume its
// output; it is the only code they share.  The recipe is documented in DESIGN.md §4 (input recipe).
//
// Determinism: every random draw is a counter-based splitmix64 of (seed, purpose, kernel, warp, i), so any warp
// range (a shard) or warp subset (the 1% sample) is generated independently and bit-identically, in any order and
// with any number of threads.
//
// Program templates follow the benchmark facts the paper gives:
//   ELEM 2 BBs (ReLU has two BBs, L364); VADD grid-stride; GEMM (16x16 work-group = 4 wavefronts of 64, L61;
//   body BBs end at s_barrier, L105-107); IM2COL; POOL; SOFTMAX; SPMV-like (Zipf nnz, final 1-instruction BB in
//   the last warp, L210/L231); C1 16-BB loop; C5 random loop nests.
#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <thread>
#include <vector>

namespace {

inline uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
  x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
  return x ^ (x >> 31);
}
inline uint64_t rng(uint64_t seed, uint64_t purpose, uint64_t a, uint64_t b = 0, uint64_t c = 0) {
  return splitmix64(seed ^ splitmix64(purpose ^ splitmix64(a ^ splitmix64(b ^ splitmix64(c)))));
}
inline double unif(uint64_t r) { return (double)(r >> 11) * (1.0 / 9007199254740992.0); }

enum Purpose : uint64_t {
  P_C1 = 1, P_VADD, P_SPMV, P_NEST, P_NEST_K, P_JIT, P_CLS, P_PROG, P_C5K, P_SEL
};

enum Tmpl : int { T_C1 = 0, T_ELEM, T_VADD, T_GEMM, T_IM2COL, T_POOL, T_SOFTMAX, T_SPMV, T_NEST };

struct Kern {
  int tmpl = 0;
  uint32_t bb_base = 0;  // global id of the template's local BB 0
  uint64_t n_warps = 0;
  int64_t p[10] = {0};
};

struct Gen {
  uint64_t seed = 0;
  std::vector<Kern> kerns;
  std::vector<uint32_t> bb_len;   // global BB table
  std::vector<uint64_t> kwoff;    // [K+1] prefix of n_warps
  std::vector<int> drift_class;   // per BB: 0 stable (ramp + jitter), 1 drift v/8, 2 drift v/2 (v = warp index)
};

// ---- program tables (local BB lengths) -------------------------------------------------------------------
const uint32_t LEN_C1[16] = {12, 4, 6, 3, 8, 5, 2, 7, 9, 3, 4, 6, 5, 2, 3, 10};
const uint32_t LEN_ELEM[2] = {10, 8};
const uint32_t LEN_VADD[4] = {8, 9, 3, 2};
const uint32_t LEN_GEMM[7] = {24, 14, 40, 3, 6, 8, 1};
const uint32_t LEN_IM2COL[5] = {16, 4, 6, 3, 5};
const uint32_t LEN_POOL[3] = {10, 7, 6};
const uint32_t LEN_SOFTMAX[4] = {12, 6, 9, 4};
const uint32_t LEN_SPMV[5] = {12, 4, 11, 6, 1};

// Appends the local BB sequence of warp `lw` (kernel-local index) of kernel `kk` (global index `k`) to out,
// or only counts it when out == nullptr.  Returns the event count.
template <class Emit>
uint64_t warp_seq(const Gen& g, uint32_t k, uint64_t lw, Emit&& emit) {
  const Kern& K = g.kerns[k];
  uint64_t n = 0;
  auto e = [&](uint32_t local) { emit(K.bb_base + local); ++n; };
  switch (K.tmpl) {
    case T_C1: {  // b0; loop b1..b14 x trip; b15.  trip 73 for ~97% of warps, else 72 or 74.
      uint64_t h = rng(g.seed, P_C1, k, lw) % 1000;
      int64_t trip = h < 970 ? K.p[0] : (h < 985 ? K.p[0] - 1 : K.p[0] + 1);
      e(0);
      for (int64_t t = 0; t < trip; ++t)
        for (uint32_t b = 1; b <= 14; ++b) e(b);
      e(15);
      break;
    }
    case T_ELEM: e(0); e(1); break;
    case T_VADD: {  // grid-stride loop: trips = base, +1 for the first p[1] warps (the tail)
      int64_t t = K.p[0] + ((int64_t)lw < K.p[1] ? 1 : 0);
      e(0);
      for (int64_t i = 0; i < t; ++i) { e(1); e(2); }
      e(3);
      break;
    }
    case T_GEMM: {  // p0 = kt, p1 = M, p2 = N; warp = wavefront q of work-group (i, j)
      int64_t kt = K.p[0], M = K.p[1], N = K.p[2];
      int64_t ncol = (N + 15) / 16;
      int64_t wg = (int64_t)(lw / 4), q = (int64_t)(lw % 4);
      int64_t i = wg / ncol, j = wg % ncol;
      bool valid = (i * 16 + 4 * q < M) && (j * 16 < N);
      e(0);
      for (int64_t t = 0; t < kt; ++t) { e(1); e(2); e(3); }
      e(4);
      if (valid) e(5);
      e(6);
      break;
    }
    case T_IM2COL: {  // p: Hout Wout Hin Win stride ksz pad Cin; warp = 64 consecutive output pixels of one row
      int64_t Ho = K.p[0], Wo = K.p[1], Hi = K.p[2], Wi = K.p[3], s = K.p[4], ks = K.p[5], pad = K.p[6];
      int64_t npix = Ho * Wo, wpr = (npix + 63) / 64;
      int64_t row = (int64_t)lw / wpr, chunk = (int64_t)lw % wpr;
      int64_t kk = row % (ks * ks), kh = kk / ks, kw = kk % ks;
      bool any_in = false, any_pad = false;
      for (int64_t l = 0; l < 64; ++l) {
        int64_t pix = chunk * 64 + l;
        if (pix >= npix) break;
        int64_t oh = pix / Wo, ow = pix % Wo;
        int64_t ih = oh * s + kh - pad, iw = ow * s + kw - pad;
        if (ih < 0 || ih >= Hi || iw < 0 || iw >= Wi) any_pad = true; else any_in = true;
      }
      e(0); e(1);
      if (any_in) e(2);
      if (any_pad) e(3);
      e(4);
      break;
    }
    case T_POOL: {
      e(0);
      for (int64_t i = 0; i < K.p[0]; ++i) e(1);
      e(2);
      break;
    }
    case T_SOFTMAX: {
      e(0);
      for (int64_t i = 0; i < K.p[0]; ++i) e(1);
      for (int64_t i = 0; i < K.p[0]; ++i) e(2);
      e(3);
      break;
    }
    case T_SPMV: {  // one row per warp; nnz ~ Zipf(1.5) capped at 256; last warp writes back (rare BB, L210)
      double u = unif(rng(g.seed, P_SPMV, k, lw));
      int64_t nnz = (int64_t)std::floor(std::pow(1.0 - u, -1.0 / 0.5));  // Pareto tail ~ Zipf(1.5)
      if (nnz < 1) nnz = 1;
      if (nnz > 256) nnz = 256;
      e(0); e(1);
      for (int64_t i = 0; i < nnz; ++i) e(2);
      e(3);
      if (lw + 1 == K.n_warps) e(4);
      break;
    }
    case T_NEST: {  // p0=a p1=c p2=t_out p3=t_in p4=irregular p5=tail permille
      int64_t a = K.p[0], c = K.p[1], tout = K.p[2], tin = K.p[3];
      if (K.p[4]) {  // irregular: geometric inner trips per warp with mean tin
        double u = unif(rng(g.seed, P_NEST, k, lw));
        double pr = 1.0 / (double)tin;
        tin = 1 + (int64_t)std::floor(std::log(1.0 - u) / std::log(1.0 - pr + 1e-12));
        if (tin > 4 * K.p[3] + 8) tin = 4 * K.p[3] + 8;
      } else if ((int64_t)(rng(g.seed, P_NEST, k, lw) % 1000) < K.p[5]) {
        tout += 1;  // the 2% tail
      }
      e(0);
      for (int64_t o = 0; o < tout; ++o) {
        for (int64_t b = 1; b < a; ++b) e((uint32_t)b);
        for (int64_t i = 0; i < tin; ++i)
          for (int64_t b = a; b < c; ++b) e((uint32_t)b);
        for (int64_t b = c; b < 15; ++b) e((uint32_t)b);
      }
      e(15);
      break;
    }
  }
  return n;
}

uint32_t add_prog(Gen& g, const uint32_t* lens, uint32_t n) {
  uint32_t base = (uint32_t)g.bb_len.size();
  for (uint32_t i = 0; i < n; ++i) g.bb_len.push_back(lens[i]);
  return base;
}

void finish(Gen& g) {
  g.kwoff.assign(g.kerns.size() + 1, 0);
  for (size_t k = 0; k < g.kerns.size(); ++k) g.kwoff[k + 1] = g.kwoff[k] + g.kerns[k].n_warps;
  g.drift_class.resize(g.bb_len.size());
  for (size_t b = 0; b < g.bb_len.size(); ++b) {
    double u = unif(rng(g.seed, P_CLS, b));
    g.drift_class[b] = u < 0.025 ? 1 : (u < 0.05 ? 2 : 0);
  }
}

Kern gemm(uint32_t base, int64_t M, int64_t N, int64_t Kd) {
  Kern k;
  k.tmpl = T_GEMM; k.bb_base = base;
  k.p[0] = (Kd + 15) / 16; k.p[1] = M; k.p[2] = N;
  k.n_warps = (uint64_t)(4 * ((M + 15) / 16) * ((N + 15) / 16));
  return k;
}
Kern elem(uint32_t base, int64_t n) {
  Kern k; k.tmpl = T_ELEM; k.bb_base = base; k.p[0] = n; k.n_warps = (uint64_t)((n + 63) / 64); return k;
}
Kern im2col(uint32_t base, int64_t Cin, int64_t Hi, int64_t Wi, int64_t ks, int64_t s, int64_t pad) {
  Kern k; k.tmpl = T_IM2COL; k.bb_base = base;
  int64_t Ho = (Hi + 2 * pad - ks) / s + 1, Wo = (Wi + 2 * pad - ks) / s + 1;
  k.p[0] = Ho; k.p[1] = Wo; k.p[2] = Hi; k.p[3] = Wi; k.p[4] = s; k.p[5] = ks; k.p[6] = pad; k.p[7] = Cin;
  k.n_warps = (uint64_t)(Cin * ks * ks * ((Ho * Wo + 63) / 64));
  return k;
}
Kern pool(uint32_t base, int64_t n_out, int64_t window) {
  Kern k; k.tmpl = T_POOL; k.bb_base = base; k.p[0] = window; k.n_warps = (uint64_t)((n_out + 63) / 64); return k;
}
Kern softmax(uint32_t base, int64_t n) {
  Kern k; k.tmpl = T_SOFTMAX; k.bb_base = base; k.n_warps = 4; k.p[0] = (n + 255) / 256; return k;
}

// C1: tiny — 1 kernel, 1024 warps, 16 BBs, ~1M events, ~97% dominant type.
void build_c1(Gen& g) {
  uint32_t base = add_prog(g, LEN_C1, 16);
  Kern k; k.tmpl = T_C1; k.bb_base = base; k.n_warps = 1024; k.p[0] = 73;
  g.kerns.push_back(k);
}

// C2: micro mix — 10 VADD + 10 GEMM kernels, 65536 warps each (4 BBs + 7 BBs = 11 BB ids).
void build_c2(Gen& g) {
  uint32_t vb = add_prog(g, LEN_VADD, 4), gb = add_prog(g, LEN_GEMM, 7);
  const int64_t vtrips[5] = {1, 2, 3, 4, 2};
  const int64_t vtail[5] = {0, 20000, 40000, 9000, 65000};  // warps with one extra trip
  const int64_t kts[5] = {8, 16, 32, 64, 128};
  for (int rep = 0; rep < 2; ++rep)
    for (int i = 0; i < 5; ++i) {
      Kern k; k.tmpl = T_VADD; k.bb_base = vb; k.n_warps = 65536; k.p[0] = vtrips[i]; k.p[1] = vtail[i];
      g.kerns.push_back(k);
    }
  for (int rep = 0; rep < 2; ++rep)
    for (int i = 0; i < 5; ++i) {
      // 65536 warps = 16384 work-groups.  kt in {16,64} use M mod 16 != 0 (edge wavefronts skip the store).
      int64_t M = (i == 1 || i == 3) ? 1016 : 1024, N = 4096;
      Kern k = gemm(gb, M, N, kts[i] * 16);
      k.n_warps = 65536;  // 4 * 64 * 256
      g.kerns.push_back(k);
    }
}

struct ConvSpec { int64_t Cin, Cout, H, ks, s, pad; };

// conv as {im2col (3x3/7x7 only), GEMM(M=Cout, N=Ho*Wo, K=Cin*ks*ks)}
void conv(Gen& g, uint32_t ib, uint32_t gb, const ConvSpec& c) {
  int64_t Ho = (c.H + 2 * c.pad - c.ks) / c.s + 1;
  if (c.ks > 1) g.kerns.push_back(im2col(ib, c.Cin, c.H, c.H, c.ks, c.s, c.pad));
  g.kerns.push_back(gemm(gb, c.Cout, Ho * Ho, c.Cin * c.ks * c.ks));
}

// C3: VGG-16 batch 1, 224x224 (~15.5 GFLOP, L37): 13 x {im2col, GEMM, bias+ReLU}, 5 max-pools,
// 3 FC {GEMM(N=1), bias(+ReLU)}, softmax.
void build_c3(Gen& g) {
  uint32_t ib = add_prog(g, LEN_IM2COL, 5), gb = add_prog(g, LEN_GEMM, 7), eb = add_prog(g, LEN_ELEM, 2);
  uint32_t pb = add_prog(g, LEN_POOL, 3), sb = add_prog(g, LEN_SOFTMAX, 4);
  const int64_t cfg[] = {64, 64, -1, 128, 128, -1, 256, 256, 256, -1, 512, 512, 512, -1, 512, 512, 512, -1};
  int64_t C = 3, H = 224;
  for (int64_t v : cfg) {
    if (v < 0) { H /= 2; g.kerns.push_back(pool(pb, C * H * H, 4)); continue; }
    conv(g, ib, gb, {C, v, H, 3, 1, 1});
    g.kerns.push_back(elem(eb, v * H * H));
    C = v;
  }
  const int64_t fc[3][2] = {{25088, 4096}, {4096, 4096}, {4096, 1000}};
  for (int i = 0; i < 3; ++i) {
    g.kerns.push_back(gemm(gb, fc[i][1], 1, fc[i][0]));
    g.kerns.push_back(elem(eb, fc[i][1]));
  }
  g.kerns.push_back(softmax(sb, 1000));
}

// C4: ResNet-152 batch 1: conv1 7x7/2 + BN-ReLU, max-pool, [3, 8, 36, 3] bottlenecks (v1.5: stride on the 3x3),
// projection on the first block of each stage, avg-pool, FC, softmax.
void build_c4(Gen& g) {
  uint32_t ib = add_prog(g, LEN_IM2COL, 5), gb = add_prog(g, LEN_GEMM, 7), eb = add_prog(g, LEN_ELEM, 2);
  uint32_t pb = add_prog(g, LEN_POOL, 3), sb = add_prog(g, LEN_SOFTMAX, 4);
  // BN-ReLU, BN, add+ReLU are distinct elementwise programs (different BB ids, same ELEM shape)
  uint32_t eb2 = add_prog(g, LEN_ELEM, 2), eb3 = add_prog(g, LEN_ELEM, 2);
  int64_t H = 224;
  conv(g, ib, gb, {3, 64, H, 7, 2, 3});
  H = 112;
  g.kerns.push_back(elem(eb, 64 * H * H));
  H = 56;
  g.kerns.push_back(pool(pb, 64 * H * H, 9));
  const int64_t blocks[4] = {3, 8, 36, 3}, width[4] = {64, 128, 256, 512};
  int64_t C = 64;
  for (int st = 0; st < 4; ++st) {
    for (int64_t bi = 0; bi < blocks[st]; ++bi) {
      int64_t w = width[st], s = (st > 0 && bi == 0) ? 2 : 1, Hout = H / s;
      conv(g, ib, gb, {C, w, H, 1, 1, 0});
      g.kerns.push_back(elem(eb, w * H * H));
      conv(g, ib, gb, {w, w, H, 3, s, 1});
      g.kerns.push_back(elem(eb, w * Hout * Hout));
      conv(g, ib, gb, {w, 4 * w, Hout, 1, 1, 0});
      g.kerns.push_back(elem(eb2, 4 * w * Hout * Hout));
      if (bi == 0) {  // projection shortcut (1x1, stride s)
        Kern pk = gemm(gb, 4 * w, Hout * Hout, C);
        g.kerns.push_back(pk);
        g.kerns.push_back(elem(eb2, 4 * w * Hout * Hout));
      }
      g.kerns.push_back(elem(eb3, 4 * w * Hout * Hout));
      C = 4 * w;
      H = Hout;
    }
  }
  g.kerns.push_back(pool(pb, C, 49));
  g.kerns.push_back(gemm(gb, 1000, 1, C));
  g.kerns.push_back(softmax(sb, 1000));
}

// C5: stress — 10^4 launches of 256 programs x 16 BBs (4096 BB ids), BB lengths U[1,64], half regular (one trip
// count + 2% tail), half irregular (geometric inner trips).  Program choice Zipf(1.1); warps log-uniform in
// [32, 8192]; trips scaled so E = 10^9 +- 1% (scaled by `scale`).
void build_c5(Gen& g, double scale, double corr) {
  const int NP = 256, NK = 10000;
  struct Prog { uint32_t base; int64_t a, c; bool irr; };
  std::vector<Prog> progs(NP);
  for (int p = 0; p < NP; ++p) {
    uint32_t lens[16];
    for (int i = 0; i < 16; ++i) lens[i] = 1 + (uint32_t)(rng(g.seed, P_PROG, p, i) % 64);
    progs[p].base = add_prog(g, lens, 16);
    progs[p].a = 2 + (int64_t)(rng(g.seed, P_PROG, p, 100) % 5);          // outer body  [1, a)
    progs[p].c = progs[p].a + 2 + (int64_t)(rng(g.seed, P_PROG, p, 101) % 6);  // inner body [a, c)
    progs[p].irr = (p % 2) == 1;
  }
  // Zipf(1.1) CDF over programs
  std::vector<double> cdf(NP);
  double z = 0;
  for (int p = 0; p < NP; ++p) { z += 1.0 / std::pow((double)(p + 1), 1.1); cdf[p] = z; }
  for (auto& v : cdf) v /= z;
  const int64_t tin_choices[4] = {2, 4, 8, 16};
  // per-launch draws, then a global trip scale so that total events ~ 1e9 * scale
  struct Draw { int prog; uint64_t warps; int64_t tin; double target; };
  std::vector<Draw> d(NK);
  for (int k = 0; k < NK; ++k) {
    double u = unif(rng(g.seed, P_C5K, k, 0));
    d[k].prog = (int)(std::lower_bound(cdf.begin(), cdf.end(), u) - cdf.begin());
    if (d[k].prog >= NP) d[k].prog = NP - 1;
    double lw = std::log(32.0) + unif(rng(g.seed, P_C5K, k, 1)) * (std::log(8192.0) - std::log(32.0));
    d[k].warps = (uint64_t)std::floor(std::exp(lw));
    d[k].tin = tin_choices[rng(g.seed, P_C5K, k, 2) % 4];
    d[k].target = std::exp(std::log(0.25) + unif(rng(g.seed, P_C5K, k, 3)) * (std::log(4.0) - std::log(0.25)));
  }
  double mult = 68.0;  // events per warp target multiplier, refined below
  for (int iter = 0; iter < 6; ++iter) {
    g.kerns.clear();
    double expect = 0;
    for (int k = 0; k < NK; ++k) {
      const Prog& P = progs[d[k].prog];
      Kern kk; kk.tmpl = T_NEST; kk.bb_base = P.base; kk.n_warps = d[k].warps;
      int64_t per_outer = (P.a - 1) + (P.c - P.a) * d[k].tin + (15 - P.c);
      double want = mult * d[k].target * scale;
      int64_t tout = (int64_t)std::floor((want - 2.0) / (double)per_outer + unif(rng(g.seed, P_C5K, k, 4)));
      if (tout < 1) tout = 1;
      kk.p[0] = P.a; kk.p[1] = P.c; kk.p[2] = tout; kk.p[3] = d[k].tin; kk.p[4] = P.irr ? 1 : 0; kk.p[5] = 20;
      expect += (double)kk.n_warps * (2.0 + (double)tout * (double)per_outer);
      g.kerns.push_back(kk);
    }
    double target_total = 1e9 * scale * corr;
    if (std::fabs(expect - target_total) < 0.002 * target_total) break;
    mult *= target_total / expect;
  }
}

// C6 (test mix, not a BASELINE config): every template at small size, incl. SpMV-like (many types, a rare BB)
// and C5-style nests, with repeats so kernel matching has work.  ~60K warps.
void build_c6(Gen& g) {
  uint32_t c1 = add_prog(g, LEN_C1, 16), vb = add_prog(g, LEN_VADD, 4), gb = add_prog(g, LEN_GEMM, 7);
  uint32_t ib = add_prog(g, LEN_IM2COL, 5), eb = add_prog(g, LEN_ELEM, 2), pb = add_prog(g, LEN_POOL, 3);
  uint32_t sb = add_prog(g, LEN_SOFTMAX, 4), spb = add_prog(g, LEN_SPMV, 5);
  uint32_t nb[4];
  for (int p = 0; p < 4; ++p) {
    uint32_t lens[16];
    for (int i = 0; i < 16; ++i) lens[i] = 1 + (uint32_t)(rng(g.seed, P_PROG, p, i) % 64);
    nb[p] = add_prog(g, lens, 16);
  }
  Kern k1; k1.tmpl = T_C1; k1.bb_base = c1; k1.n_warps = 777; k1.p[0] = 9; g.kerns.push_back(k1);
  for (int r = 0; r < 3; ++r) {
    Kern v; v.tmpl = T_VADD; v.bb_base = vb; v.n_warps = 3000 + 7 * r; v.p[0] = 2 + r % 2; v.p[1] = 1234;
    g.kerns.push_back(v);
  }
  g.kerns.push_back(gemm(gb, 100, 300, 64));
  g.kerns.push_back(gemm(gb, 100, 300, 80));
  g.kerns.push_back(gemm(gb, 100, 300, 64));
  g.kerns.push_back(gemm(gb, 8, 8, 64));     // 4 warps (< 64 cores: equal-warp rule)
  g.kerns.push_back(gemm(gb, 8, 8, 64));
  g.kerns.push_back(gemm(gb, 12, 8, 64));
  g.kerns.push_back(im2col(ib, 3, 30, 30, 3, 1, 1));
  g.kerns.push_back(im2col(ib, 4, 17, 17, 3, 2, 1));
  g.kerns.push_back(elem(eb, 100000));
  g.kerns.push_back(elem(eb, 1));
  g.kerns.push_back(pool(pb, 5000, 4));
  g.kerns.push_back(softmax(sb, 1000));
  for (int r = 0; r < 3; ++r) {
    Kern s; s.tmpl = T_SPMV; s.bb_base = spb; s.n_warps = 384 * (r + 1); g.kerns.push_back(s);
  }
  for (int r = 0; r < 8; ++r) {
    Kern n; n.tmpl = T_NEST; n.bb_base = nb[r % 4]; n.n_warps = 40 + 211 * r;
    n.p[0] = 3; n.p[1] = 7; n.p[2] = 2 + r / 4; n.p[3] = 4; n.p[4] = (r % 4) >= 2; n.p[5] = 20;
    g.kerns.push_back(n);
  }
}

struct Sel {  // a warp subset: global warps w0, w0+step, ... < w1
  uint64_t w0, w1, step;
  uint64_t count() const { return w1 > w0 ? (w1 - w0 + step - 1) / step : 0; }
  uint64_t at(uint64_t i) const { return w0 + i * step; }
};

uint32_t kernel_of(const Gen& g, uint64_t w) {
  return (uint32_t)(std::upper_bound(g.kwoff.begin(), g.kwoff.end(), w) - g.kwoff.begin() - 1);
}

template <class F>
void parallel_for(uint64_t n, int threads, F&& f) {
  if (threads <= 1 || n < 4096) { f(0, n); return; }
  std::vector<std::thread> ts;
  uint64_t chunk = (n + threads - 1) / threads;
  for (int t = 0; t < threads; ++t) {
    uint64_t a = t * chunk, b = std::min(n, a + chunk);
    if (a >= b) break;
    ts.emplace_back([&f, a, b] { f(a, b); });
  }
  for (auto& t : ts) t.join();
}

}  // namespace

extern "C" {

void tg_sel_counts(void* h, uint64_t w0, uint64_t w1, uint64_t step, uint64_t* out, int threads);

void* tg_create(int cfg, uint64_t seed, double scale) {
  Gen* g = new Gen();
  g->seed = seed;
  switch (cfg) {
    case 1: build_c1(*g); break;
    case 2: build_c2(*g); break;
    case 3: build_c3(*g); break;
    case 4: build_c4(*g); break;
    case 5: {
      // calibrate so the exact event total is 1e9*scale within 0.3% (the formula ignores tails/irregular trips)
      double sc = scale > 0 ? scale : 1.0, corr = 1.0;
      for (int it = 0; it < 4; ++it) {
        g->kerns.clear(); g->bb_len.clear();
        build_c5(*g, sc, corr);
        finish(*g);
        uint64_t W = g->kwoff.back();
        std::vector<uint64_t> cnt(W);
        tg_sel_counts(g, 0, W, 1, cnt.data(), 8);
        double E = 0;
        for (uint64_t c : cnt) E += (double)c;
        if (getenv("TG_DEBUG")) fprintf(stderr, "c5 iter %d corr %f E %.0f\n", it, corr, E);
        if (std::fabs(E - 1e9 * sc) < 0.003 * 1e9 * sc) break;
        corr *= 1e9 * sc / E;
      }
      break;
    }
    case 6: build_c6(*g); break;
    default: delete g; return nullptr;
  }
  finish(*g);
  return g;
}
void tg_free(void* h) { delete (Gen*)h; }
uint32_t tg_n_kernels(void* h) { return (uint32_t)((Gen*)h)->kerns.size(); }
uint32_t tg_n_bb(void* h) { return (uint32_t)((Gen*)h)->bb_len.size(); }
uint64_t tg_n_warps(void* h) { return ((Gen*)h)->kwoff.back(); }
void tg_bb_len(void* h, uint32_t* out) {
  Gen* g = (Gen*)h;
  std::memcpy(out, g->bb_len.data(), g->bb_len.size() * 4);
}
void tg_kernel_warps(void* h, uint64_t* out) {
  Gen* g = (Gen*)h;
  for (size_t k = 0; k < g->kerns.size(); ++k) out[k] = g->kerns[k].n_warps;
}
void tg_kernel_tmpl(void* h, int32_t* out) {
  Gen* g = (Gen*)h;
  for (size_t k = 0; k < g->kerns.size(); ++k) out[k] = g->kerns[k].tmpl;
}

// kernel id of each selected warp
void tg_sel_kernels(void* h, uint64_t w0, uint64_t w1, uint64_t step, uint32_t* out, int threads) {
  Gen* g = (Gen*)h;
  Sel s{w0, w1, step};
  parallel_for(s.count(), threads, [&](uint64_t a, uint64_t b) {
    for (uint64_t i = a; i < b; ++i) out[i] = kernel_of(*g, s.at(i));
  });
}

// event count of each selected warp
void tg_sel_counts(void* h, uint64_t w0, uint64_t w1, uint64_t step, uint64_t* out, int threads) {
  Gen* g = (Gen*)h;
  Sel s{w0, w1, step};
  parallel_for(s.count(), threads, [&](uint64_t a, uint64_t b) {
    uint32_t k = a < b ? kernel_of(*g, s.at(a)) : 0;
    for (uint64_t i = a; i < b; ++i) {
      uint64_t w = s.at(i);
      while (w >= g->kwoff[k + 1]) ++k;
      out[i] = warp_seq(*g, k, w - g->kwoff[k], [](uint32_t) {});
    }
  });
}

// events of the selected warps into bb[], at offsets off[i] (relative, off has count+1 entries)
void tg_sel_events(void* h, uint64_t w0, uint64_t w1, uint64_t step, const uint64_t* off, uint16_t* bb,
                   int threads) {
  Gen* g = (Gen*)h;
  Sel s{w0, w1, step};
  parallel_for(s.count(), threads, [&](uint64_t a, uint64_t b) {
    uint32_t k = a < b ? kernel_of(*g, s.at(a)) : 0;
    for (uint64_t i = a; i < b; ++i) {
      uint64_t w = s.at(i);
      while (w >= g->kwoff[k + 1]) ++k;
      uint16_t* p = bb + off[i];
      warp_seq(*g, k, w - g->kwoff[k], [&](uint32_t id) { *p++ = (uint16_t)id; });
    }
  });
}

// ---- timing streams (wave model) ------------------------------------------------------------
// Records of kernel k (all its warps): warp v issues its first BB at floor(v / 2560) * P; each later BB issues at
// the previous one's retire; retire = issue + d, d by the BB's class (stable ramp+jitter, or drifting).
// Records sorted by (retire, warp, seq).  Returns the record count; when out arrays are NULL only counts.
static void kernel_timing(const Gen* g, uint32_t k, uint16_t* bb, uint64_t* issue, uint64_t* retire) {
  const Kern& K = g->kerns[k];
  // wave period P: serial duration of warp 0 without ramp/jitter (4 ticks per instruction)
  uint64_t P = 0;
  warp_seq(*g, k, 0, [&](uint32_t id) { P += 4ull * g->bb_len[id]; });
  if (P == 0) P = 1;
  uint64_t waves = (K.n_warps + 2559) / 2560;
  double Tw = 0.25 * (double)(waves * P) + 1.0;
  struct Rec { uint64_t retire, issue, warp; uint32_t seq; uint16_t bb; };
  std::vector<Rec> recs;
  for (uint64_t v = 0; v < K.n_warps; ++v) {
    uint64_t t = (v / 2560) * P;
    uint32_t seq = 0;
    warp_seq(*g, k, v, [&](uint32_t id) {
      uint64_t len = g->bb_len[id];
      uint64_t d;
      int cls = g->drift_class[id];
      if (cls == 0) {
        double ramp = 4.0 * (double)len * std::max(0.0, 1.0 - (double)t / Tw);
        d = 4 * len + (uint64_t)ramp + (rng(g->seed, P_JIT, k, v, seq) & 7);
      } else {
        // drifting BB types: duration grows with the warp's launch order (bounded)
        d = 4 * len + (cls == 1 ? v / 8 : v / 2);
      }
      recs.push_back(Rec{t + d, t, v, seq, (uint16_t)id});
      t += d;
      ++seq;
    });
  }
  std::sort(recs.begin(), recs.end(), [](const Rec& a, const Rec& b) {
    if (a.retire != b.retire) return a.retire < b.retire;
    if (a.warp != b.warp) return a.warp < b.warp;
    return a.seq < b.seq;
  });
  for (size_t i = 0; i < recs.size(); ++i) {
    bb[i] = recs[i].bb;
    issue[i] = recs[i].issue;
    retire[i] = recs[i].retire;
  }
}

// Timing records of kernels [k0, k1) into arrays at rec_off[k - k0] (rec_off[i] = records before kernel k0+i,
// i.e. the kernel's event count prefix; the caller computes it from tg_sel_counts).  Parallel over kernels.
void tg_timing(void* h, uint32_t k0, uint32_t k1, const uint64_t* rec_off, uint16_t* bb, uint64_t* issue,
               uint64_t* retire, int threads) {
  const Gen* g = (const Gen*)h;
  std::vector<std::thread> ts;
  std::atomic<uint32_t> next{k0};
  int nt = threads < 1 ? 1 : threads;
  for (int t = 0; t < nt; ++t)
    ts.emplace_back([&] {
      for (;;) {
        uint32_t k = next.fetch_add(1);
        if (k >= k1) break;
        uint64_t o = rec_off[k - k0];
        kernel_timing(g, k, bb + o, issue + o, retire + o);
      }
    });
  for (auto& t : ts) t.join();
}

// Warp records of kernel k (N1): one record per warp, (issue, retire) of the whole warp.  Slot model: 2560 warp
// slots (64 CUs x 40, Table 1); warp v takes the slot freed by warp v - 2560 (its issue = that warp's retire), and
// runs its BBs back to back with the same per-BB durations as kernel_timing.  Records sorted by (retire, warp).
static void kernel_warp_timing(const Gen* g, uint32_t k, uint64_t* issue, uint64_t* retire) {
  const Kern& K = g->kerns[k];
  uint64_t P = 0;
  warp_seq(*g, k, 0, [&](uint32_t id) { P += 4ull * g->bb_len[id]; });
  if (P == 0) P = 1;
  uint64_t waves = (K.n_warps + 2559) / 2560;
  double Tw = 0.25 * (double)(waves * P) + 1.0;
  struct Rec { uint64_t retire, issue, warp; };
  std::vector<Rec> recs(K.n_warps);
  std::vector<uint64_t> slot(2560, 0);
  for (uint64_t v = 0; v < K.n_warps; ++v) {
    const uint64_t t0 = slot[v % 2560];
    uint64_t t = t0;
    uint32_t seq = 0;
    warp_seq(*g, k, v, [&](uint32_t id) {
      uint64_t len = g->bb_len[id];
      uint64_t d;
      int cls = g->drift_class[id];
      if (cls == 0) {
        double ramp = 4.0 * (double)len * std::max(0.0, 1.0 - (double)t / Tw);
        d = 4 * len + (uint64_t)ramp + (rng(g->seed, P_JIT, k, v, seq) & 7);
      } else {
        d = 4 * len + (cls == 1 ? v / 8 : v / 2);
      }
      t += d;
      ++seq;
    });
    if (t == t0) t = t0 + 1;  // an empty warp still occupies its slot for a tick
    slot[v % 2560] = t;
    recs[v] = Rec{t, t0, v};
  }
  std::sort(recs.begin(), recs.end(), [](const Rec& a, const Rec& b) {
    if (a.retire != b.retire) return a.retire < b.retire;
    return a.warp < b.warp;
  });
  for (size_t i = 0; i < recs.size(); ++i) {
    issue[i] = recs[i].issue;
    retire[i] = recs[i].retire;
  }
}

// Warp records of kernels [k0, k1) into arrays at rec_off[k - k0] (= warps before kernel k0+i).
void tg_warp_timing(void* h, uint32_t k0, uint32_t k1, const uint64_t* rec_off, uint64_t* issue, uint64_t* retire,
                    int threads) {
  const Gen* g = (const Gen*)h;
  std::vector<std::thread> ts;
  std::atomic<uint32_t> next{k0};
  int nt = threads < 1 ? 1 : threads;
  for (int t = 0; t < nt; ++t)
    ts.emplace_back([&] {
      for (;;) {
        uint32_t k = next.fetch_add(1);
        if (k >= k1) break;
        uint64_t o = rec_off[k - k0];
        kernel_warp_timing(g, k, issue + o, retire + o);
      }
    });
  for (auto& t : ts) t.join();
}

}  // extern "C"
