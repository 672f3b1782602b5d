// abi.cu — the C ABI of libphoton (include/photon.h): argument validation, workspace layout, launch sequencing.
// No computation happens here; every step of the path runs in the kernels of k_*.cu on the caller's stream.
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <utility>
#include <vector>

#include "internal.h"
#include <nvtx3/nvToolsExt.h>

using namespace photon;

struct photon_ctx {
  int device = 0;
  int num_sms = 148;
  std::string err;
  const void* last_ws = nullptr;
  // optional in-stream timing of each launch section (photon_profile)
  bool prof = false;
  std::vector<std::pair<cudaEvent_t, cudaEvent_t>> ev[PHOTON_PROF_N];
  size_t used[PHOTON_PROF_N] = {0};
  cudaEvent_t fork = nullptr;  // photon_warp_group2: the remap's dependency on the main stream
  // photon_analyse: two library streams and the events of its fork / join graph (created on first use)
  cudaStream_t sa = nullptr, sb = nullptr;
  cudaEvent_t aev[6] = {nullptr, nullptr, nullptr, nullptr, nullptr, nullptr};
};

namespace {

// one NVTX range per C-ABI call (header-only NVTX3: no cost unless a tool such as nsys / ncu is attached)
struct NvtxRange {
  explicit NvtxRange(const char* name) { nvtxRangePushA(name); }
  ~NvtxRange() { nvtxRangePop(); }
};

struct ProfScope {
  photon_ctx* c;
  int sec;
  cudaStream_t s;
  cudaEvent_t stop = nullptr;
  ProfScope(photon_ctx* c_, int sec_, cudaStream_t s_) : c(c_), sec(sec_), s(s_) {
    if (!c->prof) return;
    auto& v = c->ev[sec];
    if (c->used[sec] == v.size()) {
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      v.push_back({a, b});
    }
    auto& pr = v[c->used[sec]++];
    cudaEventRecord(pr.first, s);
    stop = pr.second;
  }
  ~ProfScope() {
    if (stop) cudaEventRecord(stop, s);
  }
};

int fail(photon_ctx* c, int code, const char* fmt, ...) {
  if (c) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    c->err = buf;
  }
  return code;
}

int cuda_fail(photon_ctx* c, cudaError_t e, const char* where) {
  return fail(c, PHOTON_ECUDA, "%s: %s", where, cudaGetErrorString(e));
}

#define CK(expr, where)                             \
  do {                                              \
    cudaError_t _e = (expr);                        \
    if (_e != cudaSuccess) return cuda_fail(ctx, _e, where); \
  } while (0)

bool aligned(const void* p, size_t a) { return ((uintptr_t)p % a) == 0; }

int check_trace(photon_ctx* ctx, const photon_trace* t) {
  if (!t) return fail(ctx, PHOTON_EINVAL, "trace is NULL");
  if (t->n_kernels == 0) return fail(ctx, PHOTON_EINVAL, "n_kernels must be >= 1");
  if (t->n_bb == 0 || t->n_bb > 65536) return fail(ctx, PHOTON_EINVAL, "n_bb must be in [1, 65536]");
  if (t->n_warps >= (1ull << 40) || t->n_events >= (1ull << 48)) return fail(ctx, PHOTON_EINVAL, "W or E too large");
  if (!t->kernel_warp_off || !t->warp_event_off || !t->bb_len) return fail(ctx, PHOTON_EINVAL, "NULL trace array");
  if (t->n_events && !t->bb) return fail(ctx, PHOTON_EINVAL, "bb is NULL");
  if (t->bb && !aligned(t->bb, 16)) return fail(ctx, PHOTON_EINVAL, "bb must be 16-byte aligned");
  return PHOTON_OK;
}

TraceDev to_dev(const photon_trace* t) {
  TraceDev d;
  d.kwo = t->kernel_warp_off; d.weo = t->warp_event_off; d.bb = t->bb; d.bb_len = t->bb_len; d.bb_bin = t->bb_bin;
  d.K = t->n_kernels; d.B = t->n_bb; d.W = t->n_warps; d.E = t->n_events;
  return d;
}

// ---- workspace layouts ----------------------------------------------------------------------------------
struct BbvWs {
  DevErr* err;
  BbvTables tb;         // per-BB tables (neutral / narrow / wide) and max_len
  uint64_t* kchunk;     // [K+1] kernel_bb_insts job prefix
  size_t bytes;
};
BbvWs bbv_layout(const photon_trace* t, void* base) {
  Carver c(base);
  BbvWs w;
  w.err = c.take<DevErr>(1);
  uint32_t P2 = next_pow2_u32(t->n_bb < 16 ? 16 : t->n_bb);
  w.tb.neutral = c.take<uint32_t>(P2);
  w.tb.narrow = c.take<uint32_t>(P2);
  w.tb.wide = c.take<uint32_t>(P2);
  w.tb.max_len = c.take<uint32_t>(4);
  w.kchunk = c.take<uint64_t>((size_t)t->n_kernels + 1);
  w.bytes = c.off + 256;
  return w;
}

// Entry pool: one entry per distinct (kernel, key) of each 32-warp block -- at most W -- bounded by 8x the
// type-table capacity (ECAPACITY beyond: the caller retries with a larger hint), plus room for every K1 worker's
// partly used last block of 64 entries (<= 160 SMs x 32 workers).
constexpr uint64_t kPoolSlack = 160ull * 32 * 64;
void carve_entries(Carver& c, uint64_t W, uint64_t cap, EntryPool& ep) {
  ep.cap = (W < 8 * cap ? W : 8 * cap) + kPoolSlack;
  ep.ent = c.take<TileEntry>(ep.cap);
  ep.slot = c.take<uint32_t>(ep.cap);
  ep.count = c.take<uint64_t>(1);
  ep.gid = c.take<uint32_t>(W + 1);
}

uint64_t ht_capacity(uint64_t hint, uint64_t W) {
  uint64_t h = hint ? hint : (W < (1ull << 18) ? W : (1ull << 18));
  uint64_t cap = 1024;
  while (cap < 2 * h) cap <<= 1;
  return cap;
}

struct HtWs {
  HashTable ht;
  CanonWs cw;
};
void carve_ht(Carver& c, uint64_t cap, uint32_t K, HtWs& w) {
  w.ht.hkey = c.take<uint64_t>(cap);
  w.ht.ready = c.take<uint32_t>(cap);
  w.ht.kern = c.take<uint32_t>(cap);
  w.ht.key = c.take<uint32_t>(cap * 16);
  w.ht.count = c.take<uint32_t>(cap);
  w.ht.first = c.take<uint64_t>(cap);
  w.ht.mask = cap - 1;
  w.cw.tcount = c.take<uint32_t>(K + 1);
  w.cw.cursor = c.take<uint32_t>(K + 1);
  w.cw.list = c.take<uint32_t>(cap);
  w.cw.canon = c.take<uint32_t>(cap);
  w.cw.scratch = c.take<uint32_t>(cap);
  w.cw.big = c.take<uint32_t>(K + 1);
  w.cw.nbig = c.take<uint32_t>(2);
}

struct GroupWs {
  BbvWs b;
  HtWs h;
  EntryPool ep;
  size_t bytes;
};
GroupWs group_layout(const photon_trace* t, uint64_t hint, void* base, size_t ws_bytes) {
  GroupWs g;
  g.b = bbv_layout(t, base);
  uint64_t cap = ht_capacity(hint, t->n_warps);
  if (base && ws_bytes) {
    // the capacity actually used is the largest power of two that fits (callers may pass a larger workspace)
    while (true) {
      Carver probe(nullptr);
      probe.off = g.b.bytes;
      HtWs tmp;
      EntryPool tp;
      carve_ht(probe, cap * 2, t->n_kernels, tmp);
      carve_entries(probe, t->n_warps, cap * 2, tp);
      if (probe.off + 256 > ws_bytes) break;
      cap *= 2;
    }
  }
  Carver c(base);
  c.off = g.b.bytes;
  carve_ht(c, cap, t->n_kernels, g.h);
  carve_entries(c, t->n_warps, cap, g.ep);
  g.bytes = c.off + 256;
  return g;
}

struct MatchLayout {
  DevErr* err;
  uint64_t* sig;
  uint64_t* mass;
  MatchWs mw;
  uint64_t* pairs;
  uint64_t* n_pairs;
  size_t bytes;
};
MatchLayout match_layout(uint32_t K, uint64_t T, uint64_t pair_cap, void* base) {
  Carver c(base);
  MatchLayout m;
  if (!pair_cap) pair_cap = 16ull * K + 65536;
  m.err = c.take<DevErr>(1);
  m.sig = c.take<uint64_t>(16 * (T ? T : 1));
  m.mass = c.take<uint64_t>(K + 1);
  m.mw.prof = c.take<float>(16ull * K + 16);
  m.mw.invn = c.take<double>(K + 1);
  m.mw.sigf = c.take<float>(16 * (T ? T : 1));
  m.mw.prof8 = c.take<uint32_t>(4ull * K + 4);
  m.mw.maybe = c.take<uint64_t>(pair_cap);
  m.mw.n_maybe = c.take<uint64_t>(1);
  m.mw.cand_cnt = c.take<uint32_t>(K + 1);
  m.mw.cand_off = c.take<uint64_t>(K + 1);
  m.mw.cand_cur = c.take<uint32_t>(K + 1);
  m.mw.cand = c.take<uint32_t>(pair_cap);
  m.mw.close_cnt = c.take<uint32_t>(K + 1);
  m.mw.state = c.take<uint8_t>(K + 1);
  m.mw.ulist = c.take<uint32_t>(2ull * K + 2);
  m.mw.flag = c.take<uint32_t>(4);
  m.mw.rcnt = c.take<uint32_t>(K + 2);
  {
    const uint64_t NB = ((uint64_t)K + 63) / 64;
    m.mw.border = c.take<uint32_t>(NB * 64 + 64);
    m.mw.bfs = c.take<int>((uint64_t)K + 1);
    m.mw.bandlo = c.take<uint32_t>(NB + 1);
    m.mw.bjobs = c.take<uint32_t>(NB + 1);
    m.mw.bjob_off = c.take<uint64_t>(NB + 1);
  }
  m.mw.pair_cap = pair_cap;
  m.pairs = c.take<uint64_t>(pair_cap);
  m.n_pairs = c.take<uint64_t>(1);
  m.bytes = c.off + 256;
  return m;
}

// match layout from ws_bytes: largest pair capacity that fits (T is fixed by the caller's bound)
MatchLayout match_layout_fit(uint32_t K, uint64_t T, void* base, size_t ws_bytes) {
  uint64_t cap = 16ull * K + 65536;
  MatchLayout m = match_layout(K, T, cap, nullptr);
  while (m.bytes > ws_bytes && cap > 1) { cap /= 2; m = match_layout(K, T, cap, nullptr); }
  for (;;) {
    MatchLayout bigger = match_layout(K, T, cap * 2, nullptr);
    if (bigger.bytes > ws_bytes) break;
    cap *= 2;
  }
  return match_layout(K, T, cap, base);
}

photon_match_params norm_params(photon_match_params p) {
  if (p.theta_den == 0) { p.theta_num = 1; p.theta_den = 20; }
  if (p.n_cores == 0) p.n_cores = 64;
  return p;
}

int check_match_params(photon_ctx* ctx, const photon_match_params& p) {
  if (p.theta_den == 0 || p.theta_den > (1u << 20) || p.theta_num > 2u * p.theta_den)
    return fail(ctx, PHOTON_EINVAL, "theta must be num/den with 1 <= den <= 2^20, num <= 2*den");
  return PHOTON_OK;
}

struct StableWs {
  DevErr* err;
  void* rest;
  size_t rest_bytes;
  size_t bytes;
};
StableWs stable_layout(const photon_timing* t, void* base) {
  Carver c(base);
  StableWs s;
  s.err = c.take<DevErr>(1);
  s.rest_bytes = stable_ws_bytes(*t);
  s.rest = c.take<uint8_t>(s.rest_bytes);
  s.bytes = c.off + 256;
  return s;
}

struct MergeWs {
  DevErr* err;
  HtWs h;
  size_t bytes;
};
MergeWs merge_layout(uint64_t n_rows, uint32_t K, void* base) {
  Carver c(base);
  MergeWs m;
  m.err = c.take<DevErr>(1);
  uint64_t cap = 1024;
  while (cap < 2 * n_rows) cap <<= 1;
  carve_ht(c, cap, K, m.h);
  m.bytes = c.off + 256;
  return m;
}

}  // namespace

extern "C" {

int photon_abi_version(void) { return PHOTON_ABI_VERSION; }

int photon_create(photon_ctx** out, int cuda_device) {
  NvtxRange nvtx_("photon_create");
  if (!out) return PHOTON_EINVAL;
  *out = nullptr;
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess || n == 0 || cuda_device < 0 || cuda_device >= n) {
    cudaGetLastError();
    return PHOTON_ECUDA;
  }
  photon_ctx* c = new (std::nothrow) photon_ctx();
  if (!c) return PHOTON_ECUDA;
  c->device = cuda_device;
  if (cudaDeviceGetAttribute(&c->num_sms, cudaDevAttrMultiProcessorCount, cuda_device) != cudaSuccess) {
    delete c;
    return PHOTON_ECUDA;
  }
  *out = c;
  return PHOTON_OK;
}

void photon_destroy(photon_ctx* ctx) {
  if (!ctx) return;
  for (auto& v : ctx->ev)
    for (auto& pr : v) { cudaEventDestroy(pr.first); cudaEventDestroy(pr.second); }
  if (ctx->fork) cudaEventDestroy(ctx->fork);
  for (auto& e : ctx->aev)
    if (e) cudaEventDestroy(e);
  if (ctx->sa) cudaStreamDestroy(ctx->sa);
  if (ctx->sb) cudaStreamDestroy(ctx->sb);
  delete ctx;
}

int photon_profile(photon_ctx* ctx, int enable) {
  NvtxRange nvtx_("photon_profile");
  if (!ctx) return PHOTON_EINVAL;
  ctx->prof = enable != 0;
  for (auto& u : ctx->used) u = 0;
  return PHOTON_OK;
}

int photon_profile_read(photon_ctx* ctx, void* stream, double* ms, uint64_t* launches) {
  NvtxRange nvtx_("photon_profile_read");
  if (!ctx || !ms || !launches) return PHOTON_EINVAL;
  CK(cudaStreamSynchronize((cudaStream_t)stream), "sync");
  for (int sec = 0; sec < PHOTON_PROF_N; ++sec) {
    double tot = 0;
    for (size_t i = 0; i < ctx->used[sec]; ++i) {
      float t = 0;
      CK(cudaEventElapsedTime(&t, ctx->ev[sec][i].first, ctx->ev[sec][i].second), "elapsed");
      tot += t;
    }
    ms[sec] = tot;
    launches[sec] = ctx->used[sec];
  }
  return PHOTON_OK;
}

uint64_t photon_launch_count(void) { return launch_counter().load(); }

const char* photon_last_error(const photon_ctx* ctx) { return ctx ? ctx->err.c_str() : "NULL ctx"; }

static int read_latch(photon_ctx* ctx, const void* ws, void* stream, int64_t* bad) {
  if (bad) *bad = -1;
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaStreamSynchronize(s), "cudaStreamSynchronize");
  CK(cudaGetLastError(), "pending CUDA error");
  if (!ws) return PHOTON_OK;
  DevErr e;
  CK(cudaMemcpy(&e, ws, sizeof e, cudaMemcpyDeviceToHost), "read error latch");
  if (bad) *bad = e.code ? e.index : -1;
  if (e.code) fail(ctx, e.code, "device-detected error %d at index %lld", e.code, (long long)e.index);
  return e.code;
}

int photon_check(photon_ctx* ctx, void* stream, int64_t* bad_index) {
  NvtxRange nvtx_("photon_check");
  if (!ctx) return PHOTON_EINVAL;
  return read_latch(ctx, ctx->last_ws, stream, bad_index);
}

int photon_ws_status(photon_ctx* ctx, const void* ws, void* stream, int64_t* bad_index) {
  NvtxRange nvtx_("photon_ws_status");
  if (!ctx) return PHOTON_EINVAL;
  return read_latch(ctx, ws, stream, bad_index);
}

// ---- A1 -----------------------------------------------------------------------------------------------------
size_t photon_bbv_workspace_bytes(const photon_trace* t) { return t ? bbv_layout(t, nullptr).bytes : 0; }

int photon_bbv_build(photon_ctx* ctx, const photon_trace* t, void* ws, size_t ws_bytes, uint32_t* warp_bbv16,
                     uint64_t* warp_insts, uint64_t* kernel_bb_insts, void* stream) {
  NvtxRange nvtx_("photon_bbv_build");
  if (!ctx) return PHOTON_EINVAL;
  int rc = check_trace(ctx, t);
  if (rc) return rc;
  if (!ws) return fail(ctx, PHOTON_EINVAL, "workspace is NULL");
  BbvWs w = bbv_layout(t, ws);
  if (ws_bytes < w.bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, w.bytes);
  if (warp_bbv16 && !aligned(warp_bbv16, 16)) return fail(ctx, PHOTON_EINVAL, "warp_bbv16 must be 16-byte aligned");
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  TraceDev d = to_dev(t);
  CK(cudaMemsetAsync(w.err, 0, sizeof(DevErr), s), "memset");
  CK(launch_validate_offsets(d, w.err, s), "validate");
  CK(launch_table_prep(d, w.tb, w.err, s), "table");
  if (warp_bbv16 || warp_insts) {
    ProfScope ps(ctx, PHOTON_PROF_BBV, s);
    CK(launch_bbv3(d, w.tb, warp_bbv16, warp_insts, nullptr, w.err, ctx->num_sms, s), "bbv");
  }
  if (kernel_bb_insts) {
    ProfScope ps(ctx, PHOTON_PROF_KBB, s);
    CK(launch_kernel_bb_insts(d, w.tb, kernel_bb_insts, w.kchunk, w.err, ctx->num_sms, s), "kbb");
  }
  return PHOTON_OK;
}

// ---- A2 -----------------------------------------------------------------------------------------------------
size_t photon_group_workspace_bytes(const photon_trace* t, uint64_t hint) {
  return t ? group_layout(t, hint, nullptr, 0).bytes : 0;
}

int photon_warp_group(photon_ctx* ctx, const photon_trace* t, const uint32_t* warp_bbv16, void* ws, size_t ws_bytes,
                      photon_types* out, void* stream) {
  NvtxRange nvtx_("photon_warp_group");
  return photon_warp_group2(ctx, t, warp_bbv16, ws, ws_bytes, out, stream, stream);
}

int photon_warp_group2(photon_ctx* ctx, const photon_trace* t, const uint32_t* warp_bbv16, void* ws, size_t ws_bytes,
                       photon_types* out, void* stream, void* remap_stream) {
  NvtxRange nvtx_("photon_warp_group2");
  if (!ctx) return PHOTON_EINVAL;
  int rc = check_trace(ctx, t);
  if (rc) return rc;
  if (!ws || !out) return fail(ctx, PHOTON_EINVAL, "workspace or output is NULL");
  if (!out->warp_type || !out->kernel_type_off || !out->type_key || !out->type_count || !out->type_first_warp ||
      !out->warp_sampling_ok)
    return fail(ctx, PHOTON_EINVAL, "NULL photon_types array");
  if (!aligned(out->type_key, 16)) return fail(ctx, PHOTON_EINVAL, "type_key must be 16-byte aligned");
  if (warp_bbv16 && !aligned(warp_bbv16, 16)) return fail(ctx, PHOTON_EINVAL, "warp_bbv16 must be 16-byte aligned");
  GroupWs g0 = group_layout(t, 0, nullptr, 0);
  if (ws_bytes < g0.b.bytes + 256) return fail(ctx, PHOTON_EWORKSPACE, "workspace too small");
  GroupWs g = group_layout(t, 1, ws, ws_bytes);  // largest table that fits
  if (g.bytes > ws_bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, g.bytes);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  TraceDev d = to_dev(t);
  DevErr* err = g.b.err;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  {
    ProfScope ps(ctx, PHOTON_PROF_PREP, s);
    CK(launch_ht_clear(g.h.ht, s), "ht_clear");
    CK(cudaMemsetAsync(g.ep.count, 0, 8, s), "memset");
    CK(launch_validate_offsets(d, err, s), "validate");
    if (!warp_bbv16) CK(launch_table_prep(d, g.b.tb, err, s), "table");
  }
  if (warp_bbv16) {
    ProfScope ps(ctx, PHOTON_PROF_GROUP_UNFUSED, s);
    CK(launch_group_from_bbv(d, warp_bbv16, g.ep, err, ctx->num_sms, s), "group_from_bbv");
  } else {
    ProfScope ps(ctx, PHOTON_PROF_BBV_FUSED, s);
    CK(launch_bbv3(d, g.b.tb, nullptr, nullptr, &g.ep, err, ctx->num_sms, s), "bbv_fused");
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_CANON, s);
    CK(launch_entries_insert(g.ep, g.h.ht, err, ctx->num_sms, s), "insert");
    CK(launch_canonicalise(g.h.ht, t->n_kernels, t->kernel_warp_off, nullptr, *out, g.h.cw, err, ctx->num_sms, s),
       "canon");
    cudaStream_t rs = (cudaStream_t)remap_stream;
    if (rs != s) {  // fork: the per-warp write on its own stream, after the canonical ids exist
      if (!ctx->fork) CK(cudaEventCreateWithFlags(&ctx->fork, cudaEventDisableTiming), "event");
      CK(cudaEventRecord(ctx->fork, s), "event");
      CK(cudaStreamWaitEvent(rs, ctx->fork, 0), "event");
    }
    CK(launch_remap_entries(g.ep, t->n_warps, g.h.cw.canon, out->warp_type, rs), "remap");
  }
  return PHOTON_OK;
}

int photon_types_total(photon_ctx* ctx, const photon_types* types, uint32_t K, uint64_t* total, void* stream) {
  NvtxRange nvtx_("photon_types_total");
  if (!ctx || !types || !total || !types->kernel_type_off) return PHOTON_EINVAL;
  CK(cudaStreamSynchronize((cudaStream_t)stream), "sync");
  CK(cudaMemcpy(total, types->kernel_type_off + K, 8, cudaMemcpyDeviceToHost), "read total");
  return PHOTON_OK;
}

// ---- A3 + A4 ------------------------------------------------------------------------------------------------
size_t photon_match_workspace_bytes(uint32_t K, uint64_t T, uint64_t pair_cap) {
  return match_layout(K, T, pair_cap, nullptr).bytes;
}

int photon_kernel_match(photon_ctx* ctx, uint32_t K, const photon_types* types, const uint64_t* warps_total,
                        photon_match_params params, void* ws, size_t ws_bytes, int64_t* match, double* match_dist,
                        void* stream) {
  NvtxRange nvtx_("photon_kernel_match");
  if (!ctx) return PHOTON_EINVAL;
  if (!types || !types->kernel_type_off || !types->type_key || !types->type_count || !warps_total || !match || !ws)
    return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (K == 0) return fail(ctx, PHOTON_EINVAL, "K must be >= 1");
  params = norm_params(params);
  int rc = check_match_params(ctx, params);
  if (rc) return rc;
  uint64_t T = types->capacity;
  MatchLayout m0 = match_layout(K, T, 1024, nullptr);
  if (ws_bytes < m0.bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, m0.bytes);
  MatchLayout m = match_layout_fit(K, T, ws, ws_bytes);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(m.err, 0, sizeof(DevErr), s), "memset");
  {
    ProfScope ps(ctx, PHOTON_PROF_SIG, s);
    CK(launch_sig_prof(K, types->kernel_type_off, types->type_key, types->type_count, m.sig, m.mass, m.mw, m.err,
                       s),
       "sig");
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_SCAN, s);
    CK(launch_match_scan(K, types->kernel_type_off, m.sig, m.mass, warps_total, params, 0, K, m.mw, m.pairs,
                         m.mw.pair_cap, m.n_pairs, m.err, ctx->num_sms, s, /*prof_ready=*/true, /*fused=*/true),
       "scan");
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_RESOLVE, s);
    CK(launch_match_resolve(K, types->kernel_type_off, m.sig, m.mass, warps_total, params, m.pairs, m.mw.pair_cap,
                            m.n_pairs, m.mw, match, match_dist, m.err, ctx->num_sms, s, /*fused=*/true),
       "resolve");
  }
  return PHOTON_OK;
}

// ---- the whole chain in one call, its independent parts overlapped -------------------------------------------
int photon_analyse(photon_ctx* ctx, const photon_trace* t, void* gws, size_t gws_bytes, photon_types* out,
                   const uint64_t* warps_total, photon_match_params params, void* mws, size_t mws_bytes,
                   int64_t* match, double* match_dist, void* stream) {
  NvtxRange nvtx_("photon_analyse");
  if (!ctx) return PHOTON_EINVAL;
  int rc = check_trace(ctx, t);
  if (rc) return rc;
  if (!gws || !mws || !out || !warps_total || !match) return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (!out->warp_type || !out->kernel_type_off || !out->type_key || !out->type_count || !out->type_first_warp ||
      !out->warp_sampling_ok)
    return fail(ctx, PHOTON_EINVAL, "NULL photon_types array");
  if (!aligned(out->type_key, 16)) return fail(ctx, PHOTON_EINVAL, "type_key must be 16-byte aligned");
  const uint32_t K = t->n_kernels;
  if (K == 0) return fail(ctx, PHOTON_EINVAL, "K must be >= 1");
  params = norm_params(params);
  rc = check_match_params(ctx, params);
  if (rc) return rc;
  GroupWs g0 = group_layout(t, 0, nullptr, 0);
  if (gws_bytes < g0.b.bytes + 256) return fail(ctx, PHOTON_EWORKSPACE, "group workspace too small");
  GroupWs g = group_layout(t, 1, gws, gws_bytes);
  if (g.bytes > gws_bytes) return fail(ctx, PHOTON_EWORKSPACE, "group workspace %zu < %zu bytes", gws_bytes, g.bytes);
  const uint64_t T = out->capacity;
  MatchLayout m0 = match_layout(K, T, 1024, nullptr);
  if (mws_bytes < m0.bytes) return fail(ctx, PHOTON_EWORKSPACE, "match workspace %zu < %zu bytes", mws_bytes, m0.bytes);
  MatchLayout m = match_layout_fit(K, T, mws, mws_bytes);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  if (!ctx->sa) {
    CK(cudaStreamCreateWithFlags(&ctx->sa, cudaStreamNonBlocking), "stream");
    CK(cudaStreamCreateWithFlags(&ctx->sb, cudaStreamNonBlocking), "stream");
    for (auto& e : ctx->aev) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming), "event");
  }
  cudaStream_t sa = ctx->sa, sb = ctx->sb;
  cudaEvent_t e_lists = ctx->aev[0], e_sorted = ctx->aev[1], e_prep = ctx->aev[2], e_filt = ctx->aev[3],
              e_remap = ctx->aev[4], e_clear = ctx->aev[5];
  ctx->last_ws = gws;
  TraceDev d = to_dev(t);
  DevErr* err = g.b.err;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  {
    ProfScope ps(ctx, PHOTON_PROF_PREP, s);
    // fork 0: the type table's clear and the offsets check run beside K1 (K1 needs neither: it reads offsets
    // defensively and the table is first written by the insertion, which joins them)
    CK(cudaEventRecord(e_prep, s), "event");
    CK(cudaStreamWaitEvent(sa, e_prep, 0), "event");
    CK(launch_ht_clear(g.h.ht, sa), "ht_clear");
    CK(launch_validate_offsets(d, err, sa), "validate");
    // the canonicalisation's and the resolution's per-call counters, zeroed here off the critical path
    CK(cudaMemsetAsync(g.h.cw.tcount, 0, sizeof(uint32_t) * K, sa), "memset");
    CK(cudaMemsetAsync(g.h.cw.nbig, 0, 8, sa), "memset");
    CK(cudaMemsetAsync(m.mw.state, 0, K, sa), "memset");
    CK(cudaMemsetAsync(m.err, 0, sizeof(DevErr), sa), "memset");  // the match part's error word (first latched after the join)
    CK(cudaEventRecord(e_clear, sa), "event");
    CK(launch_table_prep(d, g.b.tb, err, s, g.ep.count), "table");  // also zeroes the entry pool's count
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_BBV_FUSED, s);
    CK(launch_bbv3(d, g.b.tb, nullptr, nullptr, &g.ep, err, ctx->num_sms, s), "bbv_fused");
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_CANON, s);
    CK(cudaStreamWaitEvent(s, e_clear, 0), "event");  // join fork 0
    CK(launch_entries_insert(g.ep, g.h.ht, err, ctx->num_sms, s), "insert");
    CK(launch_canon_lists(g.h.ht, K, *out, g.h.cw, err, s, /*zeroed=*/true), "canon");
    // fork 1: the filter profiles, the pair filter and its candidate segments need only the unsorted table and its lists
    CK(cudaEventRecord(e_lists, s), "event");
    CK(cudaStreamWaitEvent(sb, e_lists, 0), "event");
    CK(launch_analyse_filter(K, out->kernel_type_off, g.h.cw.list, g.h.ht, m.mass, warps_total, params, m.mw,
                             m.n_pairs, m.err, sb),
       "filter");
    CK(cudaEventRecord(e_filt, sb), "event");
    // the canonical rows with A3 (g and g/N in row order, N summed by the sorting warp / CTA)
    CK(launch_canon_sort(g.h.ht, K, t->kernel_warp_off, nullptr, *out, g.h.cw, ctx->num_sms, s,
                         SigOut{m.sig, m.mw.sigf}, /*zeroed=*/true),
       "sort");
    // fork 2: the per-warp warp_type write
    CK(cudaEventRecord(e_sorted, s), "event");
    CK(cudaStreamWaitEvent(sa, e_sorted, 0), "event");
    CK(launch_remap_entries(g.ep, t->n_warps, g.h.cw.canon, out->warp_type, sa), "remap");
    CK(cudaEventRecord(e_remap, sa), "event");
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_SCAN, s);
    CK(cudaStreamWaitEvent(s, e_filt, 0), "event");  // the filter survivors, their segments, mass and 1/N
    CK(launch_analyse_exact(K, out->kernel_type_off, m.sig, m.mass, warps_total, params, m.mw, m.pairs,
                            m.mw.pair_cap, m.n_pairs, m.err, ctx->num_sms, s),
       "exact");
  }
  {
    ProfScope ps(ctx, PHOTON_PROF_RESOLVE, s);
    CK(launch_match_resolve(K, out->kernel_type_off, m.sig, m.mass, warps_total, params, m.pairs, m.mw.pair_cap,
                            m.n_pairs, m.mw, match, match_dist, m.err, ctx->num_sms, s, /*fused=*/true,
                            /*zeroed=*/true),
       "resolve");
  }
  CK(cudaStreamWaitEvent(s, e_remap, 0), "event");  // join: everything is ordered before later work on `stream`
  return PHOTON_OK;
}

// ---- N2: full-BBV exact grouping and tagged-stream ingest (k_full.cu) ------------------------------------------
namespace {
struct FullLayout {
  DevErr* err;
  FullWs f;
  HtWs h;
  size_t bytes;
};
// the hash table: a power of two >= 2 x hint (>= 1024), or >= 2W without a hint (every warp its own type)
uint64_t full_ht_cap(const photon_trace* t, uint64_t hint) {
  const uint64_t h = hint ? (hint < t->n_warps ? hint : t->n_warps) : t->n_warps;
  uint64_t cap = 1024;
  while (cap < 2 * h) cap <<= 1;
  return cap;
}
FullLayout full_layout(const photon_trace* t, void* base, uint64_t cap = 0) {
  Carver c(base);
  FullLayout L;
  const uint64_t W = t->n_warps + 1;
  L.err = c.take<DevErr>(1);
  L.f.h_lo = c.take<uint64_t>(W);
  L.f.h_hi = c.take<uint64_t>(W);
  L.f.list = c.take<uint64_t>(W);
  L.f.list2 = c.take<uint64_t>(W);
  L.f.kid = c.take<uint32_t>(W);
  L.f.wslot = c.take<uint32_t>(W);
  L.f.nlist = c.take<uint32_t>(4);
  L.f.htab = c.take<ulonglong2>((uint64_t)t->n_bb + 1);
  if (!cap) cap = full_ht_cap(t, 0);
  carve_ht(c, cap, t->n_kernels, L.h);
  L.bytes = c.off + 256;
  return L;
}
}  // namespace

size_t photon_group_full_workspace_bytes(const photon_trace* t, uint64_t type_capacity_hint) {
  if (!t) return 0;
  return full_layout(t, nullptr, full_ht_cap(t, type_capacity_hint)).bytes;
}

int photon_warp_group_full(photon_ctx* ctx, const photon_trace* t, const uint32_t* warp_bbv16, void* ws,
                           size_t ws_bytes, photon_types* out, void* stream) {
  NvtxRange nvtx_("photon_warp_group_full");
  if (!ctx) return PHOTON_EINVAL;
  int rc = check_trace(ctx, t);
  if (rc) return rc;
  if (!warp_bbv16 || !ws || !out || !out->kernel_type_off || !out->type_key || !out->type_count ||
      !out->type_first_warp || !out->warp_sampling_ok || !out->warp_type)
    return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (t->n_warps >= (1ull << 32)) return fail(ctx, PHOTON_EINVAL, "n_warps must be < 2^32");
  if (!aligned(warp_bbv16, 16)) return fail(ctx, PHOTON_EINVAL, "warp_bbv16 must be 16-byte aligned");
  if (!aligned(out->type_key, 16)) return fail(ctx, PHOTON_EINVAL, "type_key must be 16-byte aligned");
  // the largest table that fits the workspace (a hint-sized workspace gives a small table; ECAPACITY if it fills)
  const size_t need = photon_group_full_workspace_bytes(t, 1);
  if (ws_bytes < need) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, need);
  uint64_t cap = 1024;
  const uint64_t cap_max = full_ht_cap(t, 0);
  while (cap < cap_max && full_layout(t, nullptr, cap * 2).bytes <= ws_bytes) cap <<= 1;
  FullLayout L = full_layout(t, ws, cap);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(L.err, 0, sizeof(DevErr), s), "memset");
  TraceDev d = to_dev(t);
  CK(launch_validate_offsets(d, L.err, s), "validate");
  CK(launch_group_full(d, warp_bbv16, L.f, L.h.ht, L.h.cw, *out, L.err, ctx->num_sms, s), "group_full");
  return PHOTON_OK;
}

size_t photon_ingest_workspace_bytes(uint64_t n, uint64_t W) {
  (void)W;
  Carver c(nullptr);
  c.take<DevErr>(1);
  c.take<uint64_t>(n + 1);
  c.take<uint8_t>(radix_pairs_ws_bytes(n));
  return c.off + 256;
}

int photon_ingest_tagged(photon_ctx* ctx, uint64_t n, uint64_t W, const uint32_t* warp, const uint16_t* bb, void* ws,
                         size_t ws_bytes, uint16_t* bb_out, uint64_t* warp_event_off, void* stream) {
  NvtxRange nvtx_("photon_ingest_tagged");
  if (!ctx) return PHOTON_EINVAL;
  if ((n && (!warp || !bb || !bb_out)) || !warp_event_off || !ws) return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (W >= (1ull << 32) || n >= (1ull << 32)) return fail(ctx, PHOTON_EINVAL, "n and n_warps must be < 2^32");
  const size_t need = photon_ingest_workspace_bytes(n, W);
  if (ws_bytes < need) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, need);
  Carver c(ws);
  DevErr* err = c.take<DevErr>(1);
  uint64_t* key = c.take<uint64_t>(n + 1);
  void* sort_ws = c.take<uint8_t>(radix_pairs_ws_bytes(n));
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  CK(launch_ingest(n, W, warp, bb, key, sort_ws, bb_out, warp_event_off, err, s), "ingest");
  return PHOTON_OK;
}

// ---- N4: persisted signature pool (k_pool.cu) ----------------------------------------------------------------
size_t photon_pool_export_workspace_bytes(uint32_t K) {
  Carver c(nullptr);
  c.take<uint64_t>((size_t)K + 1);
  c.take<uint64_t>((size_t)K + 1);
  return c.off + 256;
}

int photon_pool_export(photon_ctx* ctx, uint32_t K, const photon_types* types, const uint64_t* warps_total,
                       const int64_t* match, void* ws, size_t ws_bytes, photon_types* pool, uint64_t* pool_wt,
                       uint32_t* pool_kid, uint32_t* n_pool, void* stream) {
  NvtxRange nvtx_("photon_pool_export");
  if (!ctx) return PHOTON_EINVAL;
  if (!types || !types->kernel_type_off || !types->type_key || !types->type_count || !warps_total || !match ||
      !pool || !pool->kernel_type_off || !pool->type_key || !pool->type_count || !pool_wt || !pool_kid || !n_pool ||
      !ws)
    return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (K == 0) return fail(ctx, PHOTON_EINVAL, "K must be >= 1");
  if (ws_bytes < photon_pool_export_workspace_bytes(K))
    return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, photon_pool_export_workspace_bytes(K));
  Carver c(ws);
  uint64_t* keep = c.take<uint64_t>((size_t)K + 1);
  uint64_t* ntypes = c.take<uint64_t>((size_t)K + 1);
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(launch_pool_export(K, *types, warps_total, match, keep, ntypes, *pool, pool_wt, pool_kid, n_pool,
                        (cudaStream_t)stream),
     "pool_export");
  return PHOTON_OK;
}

namespace {
struct PoolLayout {
  uint64_t* kto;
  uint32_t* key;
  uint64_t* cnt;
  uint64_t* wt;
  size_t off;  // start of the match workspace
};
PoolLayout pool_layout(uint32_t Kp, uint64_t Tp, uint32_t K, uint64_t T, void* base) {
  Carver c(base);
  PoolLayout p;
  p.kto = c.take<uint64_t>((size_t)Kp + K + 1);
  p.key = c.take<uint32_t>(16 * (Tp + T + 1));
  p.cnt = c.take<uint64_t>(Tp + T + 1);
  p.wt = c.take<uint64_t>((size_t)Kp + K + 1);
  p.off = (c.off + 255) & ~(size_t)255;
  return p;
}
}  // namespace

size_t photon_pool_match_workspace_bytes(uint32_t Kp, uint64_t Tp, uint32_t K, uint64_t T, uint64_t pair_cap) {
  return pool_layout(Kp, Tp, K, T, nullptr).off + match_layout(Kp + K, Tp + T, pair_cap, nullptr).bytes;
}

int photon_kernel_match_pooled(photon_ctx* ctx, uint32_t Kp, const photon_types* pool, const uint64_t* pool_wt,
                               uint64_t Tp, uint32_t K, const photon_types* types, const uint64_t* warps_total,
                               uint64_t T, photon_match_params params, void* ws, size_t ws_bytes, int64_t* match,
                               double* match_dist, void* stream) {
  NvtxRange nvtx_("photon_kernel_match_pooled");
  if (!ctx) return PHOTON_EINVAL;
  if (!pool || !pool->kernel_type_off || (Kp && (!pool->type_key || !pool->type_count || !pool_wt)) || !types ||
      !types->kernel_type_off || !types->type_key || !types->type_count || !warps_total || !match || !ws)
    return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (K == 0) return fail(ctx, PHOTON_EINVAL, "K must be >= 1");
  if ((uint64_t)Kp + K >= (1ull << 32)) return fail(ctx, PHOTON_EINVAL, "Kp + K too large");
  const PoolLayout p = pool_layout(Kp, Tp, K, T, ws);
  if (ws_bytes < photon_pool_match_workspace_bytes(Kp, Tp, K, T, 1024))
    return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes,
                photon_pool_match_workspace_bytes(Kp, Tp, K, T, 1024));
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(launch_pool_concat(Kp, *pool, pool_wt, K, *types, warps_total, p.kto, p.key, p.cnt, p.wt, Tp + T,
                        ctx->num_sms, (cudaStream_t)stream),
     "pool_concat");
  photon_types comb{};
  comb.capacity = Tp + T;
  comb.kernel_type_off = p.kto;
  comb.type_key = p.key;
  comb.type_count = p.cnt;
  return photon_kernel_match(ctx, Kp + K, &comb, p.wt, params, (uint8_t*)ws + p.off, ws_bytes - p.off, match,
                             match_dist, stream);
}

int photon_match_stats(photon_ctx* ctx, uint32_t K, uint64_t T, const void* ws, size_t ws_bytes, uint64_t* stats,
                       void* stream) {
  NvtxRange nvtx_("photon_match_stats");
  if (!ctx || !ws || !stats) return PHOTON_EINVAL;
  MatchLayout m = match_layout_fit(K, T, (void*)ws, ws_bytes);
  CK(cudaStreamSynchronize((cudaStream_t)stream), "sync");
  uint64_t nm = 0, np = 0;
  uint32_t rounds = 0;
  CK(cudaMemcpy(&nm, m.mw.n_maybe, 8, cudaMemcpyDeviceToHost), "stats");
  CK(cudaMemcpy(&np, m.n_pairs, 8, cudaMemcpyDeviceToHost), "stats");
  CK(cudaMemcpy(&rounds, m.mw.flag, 4, cudaMemcpyDeviceToHost), "stats");
  stats[0] = nm;
  stats[1] = np;
  stats[2] = rounds;
  stats[3] = m.mw.pair_cap;
  return PHOTON_OK;
}

int photon_sig_build(photon_ctx* ctx, uint32_t K, const uint64_t* kto, const uint32_t* type_key,
                     const uint64_t* type_count, uint32_t k_lo, uint32_t k_hi, uint64_t* sig, uint64_t* mass,
                     void* ws, size_t ws_bytes, void* stream) {
  NvtxRange nvtx_("photon_sig_build");
  if (!ctx) return PHOTON_EINVAL;
  if (!kto || !type_key || !type_count || !sig || !mass || k_hi > K || k_lo > k_hi || !ws)
    return fail(ctx, PHOTON_EINVAL, "bad sig_build arguments");
  if (ws_bytes < 256) return fail(ctx, PHOTON_EWORKSPACE, "sig_build workspace must be >= 256 bytes");
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  DevErr* err = (DevErr*)ws;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  CK(launch_sig_build(K, kto, type_key, type_count, k_lo, k_hi, sig, mass, err, s), "sig");
  return PHOTON_OK;
}

int photon_match_scan(photon_ctx* ctx, uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                      const uint64_t* warps_total, photon_match_params params, uint32_t k_lo, uint32_t k_hi, void* ws,
                      size_t ws_bytes, uint64_t* pairs, uint64_t pair_capacity, uint64_t* n_pairs, void* stream) {
  NvtxRange nvtx_("photon_match_scan");
  if (!ctx) return PHOTON_EINVAL;
  if (!kto || !sig || !mass || !warps_total || !ws || !pairs || !n_pairs || k_hi > K || k_lo > k_hi || K == 0)
    return fail(ctx, PHOTON_EINVAL, "bad match_scan arguments");
  params = norm_params(params);
  int rc = check_match_params(ctx, params);
  if (rc) return rc;
  MatchLayout m0 = match_layout(K, 1, 1024, nullptr);
  if (ws_bytes < m0.bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace too small");
  MatchLayout m = match_layout_fit(K, 1, ws, ws_bytes);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(m.err, 0, sizeof(DevErr), s), "memset");
  m.mw.sigf = nullptr;  // T is not known here: the exact screen converts the u64 signature on the fly
  CK(cudaMemsetAsync(pairs, 0xFF, sizeof(uint64_t) * pair_capacity, s), "memset");  // unused slots: PHOTON_PAIR_PAD
  CK(launch_match_scan(K, kto, sig, mass, warps_total, params, k_lo, k_hi, m.mw, pairs, pair_capacity, n_pairs, m.err,
                       ctx->num_sms, s),
     "scan");
  return PHOTON_OK;
}

int photon_match_resolve(photon_ctx* ctx, uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                         const uint64_t* warps_total, photon_match_params params, const uint64_t* pairs,
                         uint64_t n_pairs, void* ws, size_t ws_bytes, int64_t* match, double* match_dist,
                         void* stream) {
  NvtxRange nvtx_("photon_match_resolve");
  if (!ctx) return PHOTON_EINVAL;
  if (!kto || !sig || !mass || !warps_total || !ws || (n_pairs && !pairs) || !match || K == 0)
    return fail(ctx, PHOTON_EINVAL, "bad match_resolve arguments");
  params = norm_params(params);
  int rc = check_match_params(ctx, params);
  if (rc) return rc;
  // resolve needs cand arrays for n_pairs entries
  // (exactly the layout photon_match_workspace_bytes(K, 1, n_pairs) sized: a fitted layout could pick a larger
  // pair capacity than the buffer holds and carve the state arrays past its end)
  MatchLayout m = match_layout(K, 1, n_pairs ? n_pairs : 1, nullptr);
  if (ws_bytes < m.bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, m.bytes);
  m = match_layout(K, 1, n_pairs ? n_pairs : 1, ws);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(m.err, 0, sizeof(DevErr), s), "memset");
  CK(launch_match_resolve(K, kto, sig, mass, warps_total, params, pairs, n_pairs, nullptr, m.mw, match, match_dist,
                          m.err, ctx->num_sms, s),
     "resolve");
  return PHOTON_OK;
}

// ---- A5 -----------------------------------------------------------------------------------------------------
size_t photon_stable_workspace_bytes(const photon_timing* t) { return t ? stable_layout(t, nullptr).bytes : 0; }

int photon_bb_stable(photon_ctx* ctx, const photon_timing* t, const uint64_t* kbb, photon_stable_params p, void* ws,
                     size_t ws_bytes, int64_t* first_stable, uint64_t* dur, int64_t* switch_at, void* stream) {
  NvtxRange nvtx_("photon_bb_stable");
  if (!ctx) return PHOTON_EINVAL;
  if (!t || !t->kernel_rec_off || (t->n_records && (!t->bb || !t->issue || !t->retire)) || !kbb || !first_stable ||
      !switch_at || !ws)
    return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (t->n_kernels == 0 || t->n_bb == 0 || t->n_bb > 65536 || t->n_records >= (1ull << 32) ||
      (uint64_t)t->n_kernels * t->n_bb >= (1ull << 31))
    return fail(ctx, PHOTON_EINVAL, "bad timing sizes");
  if (p.window_n == 0) { p.window_n = 2048; }
  if (p.delta_den == 0) { p.delta_num = 3; p.delta_den = 100; }
  if (p.rate_den == 0) { p.rate_num = 95; p.rate_den = 100; }
  if (p.window_n < 2 || p.window_n > 8192 || p.delta_den > (1u << 16) || p.delta_num > p.delta_den ||
      p.rate_den > (1u << 16) || p.rate_num > p.rate_den)
    return fail(ctx, PHOTON_EINVAL, "bad stable params");
  StableWs w = stable_layout(t, ws);
  if (ws_bytes < w.bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, w.bytes);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(w.err, 0, sizeof(DevErr), s), "memset");
  ProfScope ps(ctx, PHOTON_PROF_STABLE, s);
  CK(launch_stable(*t, kbb, p, w.rest, w.rest_bytes, first_stable, dur, switch_at, w.err, ctx->num_sms, s), "stable");
  return PHOTON_OK;
}

// ---- N1 -----------------------------------------------------------------------------------------------------
size_t photon_warp_stable_workspace_bytes(const photon_timing* t) {
  return t ? 512 + warp_stable_ws_bytes(t->n_kernels, t->n_records) : 0;
}

int photon_warp_stable(photon_ctx* ctx, const photon_timing* t, const uint8_t* ok, photon_warp_stable_params p,
                       void* ws, size_t ws_bytes, int64_t* switch_at, uint64_t* dur, void* stream) {
  NvtxRange nvtx_("photon_warp_stable");
  if (!ctx) return PHOTON_EINVAL;
  if (!t || !t->kernel_rec_off || (t->n_records && (!t->issue || !t->retire)) || !switch_at || !ws)
    return fail(ctx, PHOTON_EINVAL, "NULL argument");
  if (t->n_kernels == 0 || t->n_records >= (1ull << 32)) return fail(ctx, PHOTON_EINVAL, "bad warp stream sizes");
  if (p.window_n == 0) p.window_n = 1024;
  if (p.delta_den == 0) { p.delta_num = 3; p.delta_den = 100; }
  if (p.window_n < 2 || p.window_n > 8192 || p.delta_den > (1u << 16) || p.delta_num > p.delta_den)
    return fail(ctx, PHOTON_EINVAL, "bad warp stable params");
  const size_t need = photon_warp_stable_workspace_bytes(t);
  if (ws_bytes < need) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, need);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  DevErr* err = (DevErr*)ws;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  ProfScope ps(ctx, PHOTON_PROF_STABLE, s);
  CK(launch_warp_stable(*t, ok, p.window_n, p.delta_num, p.delta_den, (uint8_t*)ws + 512, switch_at, dur, err,
                        ctx->num_sms, s),
     "warp_stable");
  return PHOTON_OK;
}

// ---- N3 -----------------------------------------------------------------------------------------------------
int photon_kernel_predict(photon_ctx* ctx, uint32_t K, const int64_t* match, const uint64_t* mass,
                          const uint64_t* full_insts, const uint64_t* full_cycles, void* ws, size_t ws_bytes,
                          uint64_t* pred_insts, uint64_t* pred_cycles, void* stream) {
  NvtxRange nvtx_("photon_kernel_predict");
  if (!ctx) return PHOTON_EINVAL;
  if (!match || !mass || !full_insts || !full_cycles || !pred_insts || !pred_cycles || !ws || K == 0)
    return fail(ctx, PHOTON_EINVAL, "bad kernel_predict arguments");
  if (ws_bytes < 256) return fail(ctx, PHOTON_EWORKSPACE, "kernel_predict workspace must be >= 256 bytes");
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  DevErr* err = (DevErr*)ws;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  CK(launch_kernel_predict(K, match, mass, full_insts, full_cycles, pred_insts, pred_cycles, err, s), "predict");
  return PHOTON_OK;
}

size_t photon_bb_predict_workspace_bytes(const photon_trace* t) {
  if (!t) return 0;
  Carver c(nullptr);
  c.take<DevErr>(1);
  c.take<uint32_t>(4);
  c.take<uint64_t>(t->n_warps + 1);
  return c.off + 256;
}

int photon_bb_predict(photon_ctx* ctx, const photon_trace* t, const int64_t* first_stable, const uint64_t* dur,
                      void* ws, size_t ws_bytes, uint64_t* pred, uint32_t* unpred, void* stream) {
  NvtxRange nvtx_("photon_bb_predict");
  if (!ctx) return PHOTON_EINVAL;
  int rc = check_trace(ctx, t);
  if (rc) return rc;
  if (!first_stable || !dur || !pred || !unpred || !ws) return fail(ctx, PHOTON_EINVAL, "NULL argument");
  // the long-warp work list packs (warp | kernel << 40): kernel ids must fit in 24 bits, warp ids in 40
  if (t->n_kernels >= (1u << 24) || t->n_warps >= (1ull << 40))
    return fail(ctx, PHOTON_EINVAL, "photon_bb_predict needs n_kernels < 2^24 and n_warps < 2^40");
  const size_t need = photon_bb_predict_workspace_bytes(t);
  if (ws_bytes < need) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, need);
  Carver c(ws);
  DevErr* err = c.take<DevErr>(1);
  uint32_t* n_long = c.take<uint32_t>(4);
  uint64_t* long_list = c.take<uint64_t>(t->n_warps + 1);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(err, 0, sizeof(DevErr), s), "memset");
  TraceDev d = to_dev(t);
  CK(launch_validate_offsets(d, err, s), "validate");
  CK(launch_bb_predict(d, first_stable, dur, pred, unpred, long_list, n_long, err, ctx->num_sms, s), "bb_predict");
  return PHOTON_OK;
}

// ---- multi-GPU helpers ------------------------------------------------------------------------------------
int photon_types_export(photon_ctx* ctx, uint32_t K_local, const photon_types* local, uint32_t kernel_base,
                        uint64_t warp_base, photon_type_row* rows, uint64_t row_capacity, uint64_t* n_rows,
                        void* stream) {
  NvtxRange nvtx_("photon_types_export");
  if (!ctx) return PHOTON_EINVAL;
  if (!local || !rows || K_local == 0 || row_capacity == 0) return fail(ctx, PHOTON_EINVAL, "bad export arguments");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(launch_types_export(K_local, *local, kernel_base, warp_base, rows, row_capacity, n_rows, (cudaStream_t)stream),
     "export");
  return PHOTON_OK;
}

size_t photon_merge_workspace_bytes(uint64_t n_rows, uint32_t K) { return merge_layout(n_rows, K, nullptr).bytes; }

int photon_types_merge(photon_ctx* ctx, const photon_type_row* rows, uint64_t n_rows, uint32_t K,
                       const uint64_t* kernel_warps, void* ws, size_t ws_bytes, photon_types* global, void* stream) {
  NvtxRange nvtx_("photon_types_merge");
  if (!ctx) return PHOTON_EINVAL;
  if ((n_rows && !rows) || K == 0 || !kernel_warps || !ws || !global || !global->kernel_type_off ||
      !global->type_key || !global->type_count || !global->type_first_warp || !global->warp_sampling_ok)
    return fail(ctx, PHOTON_EINVAL, "bad merge arguments");
  MergeWs m = merge_layout(n_rows, K, ws);
  if (ws_bytes < m.bytes) return fail(ctx, PHOTON_EWORKSPACE, "workspace %zu < %zu bytes", ws_bytes, m.bytes);
  cudaStream_t s = (cudaStream_t)stream;
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  ctx->last_ws = ws;
  CK(cudaMemsetAsync(m.err, 0, sizeof(DevErr), s), "memset");
  CK(launch_ht_clear(m.h.ht, s), "ht_clear");
  CK(launch_rows_insert(rows, n_rows, K, m.h.ht, m.err, s), "rows_insert");
  CK(launch_canonicalise(m.h.ht, K, nullptr, kernel_warps, *global, m.h.cw, m.err, ctx->num_sms, s), "canon");
  return PHOTON_OK;
}

int photon_types_remap(photon_ctx* ctx, uint32_t K_local, uint64_t W_local, const uint64_t* kernel_warp_off_local,
                       const photon_types* local, uint32_t kernel_base, uint64_t n_rows_merged, uint32_t K_global,
                       const void* merge_ws, size_t ws_bytes, uint32_t* warp_type_global, void* stream) {
  NvtxRange nvtx_("photon_types_remap");
  if (!ctx) return PHOTON_EINVAL;
  if (!local || !kernel_warp_off_local || !merge_ws || !warp_type_global || K_local == 0)
    return fail(ctx, PHOTON_EINVAL, "bad remap arguments");
  MergeWs m = merge_layout(n_rows_merged, K_global, (void*)merge_ws);
  if (ws_bytes < m.bytes) return fail(ctx, PHOTON_EWORKSPACE, "merge workspace mismatch");
  CK(cudaSetDevice(ctx->device), "cudaSetDevice");
  CK(launch_remap_direct(kernel_warp_off_local, K_local, W_local, *local, kernel_base, m.h.ht, m.h.cw.canon,
                         warp_type_global, m.err, (cudaStream_t)stream),
     "remap");
  return PHOTON_OK;
}

}  // extern "C"
