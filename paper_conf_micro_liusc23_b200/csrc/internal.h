// internal.h — host-side interface between the C ABI (abi.cu) and the kernel files.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "common.cuh"

namespace photon {

// ---- A1 / A2 (k_bbv3.cu) -------------------------------------------------------------------------------------
struct TraceDev {
  const uint64_t* kwo;
  const uint64_t* weo;
  const uint16_t* bb;
  const uint32_t* bb_len;
  const uint8_t* bb_bin;
  uint32_t K, B;
  uint64_t W, E;
};

// One distinct (kernel, key) of a 32-warp block, with its warp count and lowest warp (written by K1 / the unfused
// de-duplication, merged into the global type table by k_entries_insert).  count == 0 marks an unused entry.
struct alignas(16) TileEntry {
  uint32_t key[16];  // 16-byte aligned (vector stores)
  uint64_t first;
  uint32_t kernel;
  uint32_t count;
};
static_assert(sizeof(TileEntry) == 80, "TileEntry layout");
// The pool of entries: workers take blocks of entries with one atomic on `count`; every warp records its entry.
struct EntryPool {
  TileEntry* ent;     // [cap]
  uint64_t* count;    // [1] entries handed out (may exceed cap: ECAPACITY is latched)
  uint64_t cap;
  uint32_t* slot;     // [cap] hash-table slot of each entry (k_entries_insert)
  uint32_t* gid;      // [W] entry index of each warp
};

// Per-BB tables (k_table_prep): neutral (len << 4 | bin) for the BB distribution, and K1's packed entries in its
// narrow (u16 cells) and wide (u32 cells) formats; ids in [B, P2) are marked.  P2 = next pow2 >= max(B, 16).
struct BbvTables {
  uint32_t* neutral;  // [P2]
  uint32_t* narrow;   // [P2]
  uint32_t* wide;     // [P2]
  uint32_t* max_len;  // [1] max bb_len (device)
};
size_t bbv_table_bytes(uint32_t B);
cudaError_t launch_table_prep(const TraceDev& t, const BbvTables& tb, DevErr* err, cudaStream_t s,
                              uint64_t* zero = nullptr);  // zero: a u64 the kernel also zeroes (optional)
cudaError_t launch_validate_offsets(const TraceDev& t, DevErr* err, cudaStream_t s);
// K1 (k_bbv3.cu): streaming BBV pass; fused with A2's per-worker de-duplication when ep != nullptr
cudaError_t launch_bbv3(const TraceDev& t, const BbvTables& tb, uint32_t* warp_bbv16, uint64_t* warp_insts,
                        const EntryPool* ep, DevErr* err, int num_sms, cudaStream_t s);
// A2 de-duplication from materialised BBVs (unfused path)
cudaError_t launch_group_from_bbv(const TraceDev& t, const uint32_t* warp_bbv16, const EntryPool& ep, DevErr* err,
                                  int num_sms, cudaStream_t s);
cudaError_t launch_kernel_bb_insts(const TraceDev& t, const BbvTables& tb, uint64_t* kbb, uint64_t* kchunk_off,
                                   DevErr* err, int num_sms, cudaStream_t s);

// ---- A2 insertion + canonicalisation (k_types.cu) ------------------------------------------------------------
cudaError_t launch_ht_clear(const HashTable& ht, cudaStream_t s);
cudaError_t launch_entries_insert(const EntryPool& ep, const HashTable& ht, DevErr* err, int num_sms,
                                  cudaStream_t s);
cudaError_t launch_remap_entries(const EntryPool& ep, uint64_t W, const uint32_t* canon, uint32_t* warp_type,
                                 cudaStream_t s);
struct CanonWs {
  uint32_t* tcount;   // [K] types per kernel
  uint32_t* cursor;   // [K]
  uint32_t* list;     // [cap] slot ids grouped by kernel
  uint32_t* canon;    // [cap] slot -> kernel-local canonical id
  uint32_t* scratch;  // [cap] sort scratch (large kernels)
  uint32_t* big;      // [K] kernels with > 32 types: mid-size from the front, large ones from the back
  uint32_t* nbig;     // [2] counters (mid, large)
};
// From the hash table to canonical photon_types (kernel_type_off, rows, warp_sampling_ok) and the slot->id map.
cudaError_t launch_canonicalise(const HashTable& ht, uint32_t K, const uint64_t* kwo_or_null,
                                const uint64_t* kernel_warps_or_null, const photon_types& out, const CanonWs& cw,
                                DevErr* err, int num_sms, cudaStream_t s);
// multi-GPU helpers
cudaError_t launch_types_export(uint32_t K, const photon_types& local, uint32_t kernel_base, uint64_t warp_base,
                                photon_type_row* rows, uint64_t row_cap, uint64_t* n_rows, cudaStream_t s);
cudaError_t launch_rows_insert(const photon_type_row* rows, uint64_t n, uint32_t K, const HashTable& ht,
                               DevErr* err, cudaStream_t s);
// warp_type_global[v] = canonical id (in the merged table) of local warp v's type (direct hash lookup)
cudaError_t launch_remap_direct(const uint64_t* kwo_local, uint32_t K_local, uint64_t W_local,
                                const photon_types& local, uint32_t kernel_base, const HashTable& ht,
                                const uint32_t* canon, uint32_t* warp_type_global, DevErr* err, cudaStream_t s);

// ---- A3/A4 (k_match.cu) -----------------------------------------------------------------------------------
struct MatchWs {
  float* prof;         // [K][16] normalised per-bin profile (filter)
  double* invn;        // [K] 1 / N_k (fp64 screen of the exact check)
  float* sigf;         // [16 T] g / N in fp32 (screen of the exact check; nullptr: converted on the fly)
  uint32_t* prof8;     // [K][4] the profile quantised to u8 (round(255 P)), packed 4 bins per word (coarse filter)
  uint64_t* maybe;     // [pair_cap] profile-filter survivors
  uint64_t* n_maybe;   // [1]
  uint32_t* cand_cnt;  // [K]
  uint64_t* cand_off;  // [K+1]
  uint32_t* cand_cur;  // [K]
  uint32_t* cand;      // [pair_cap] r per (k, r), grouped by k
  uint32_t* close_cnt; // [K] fused path: close candidates in k's segment of cand (starting at cand_off[k])
  uint8_t* state;      // [K] 0 undecided, 1 representative, 2 matched
  uint32_t* ulist;     // [2K] undecided-kernel lists (resolution rounds)
  uint32_t* flag;      // [4]
  uint32_t* rcnt;      // [K+2] undecided count of each resolution round
  uint32_t* border;    // [NB * 64] band order: sorted position -> kernel (k_match.cu)
  int* bfs;            // [K] the sorted projections
  uint32_t* bandlo;    // [NB] first r-block of each k-block's band
  uint32_t* bjobs;     // [NB] filter jobs of each k-block
  uint64_t* bjob_off;  // [NB + 1]
  uint64_t pair_cap;
};
cudaError_t launch_sig_build(uint32_t K, const uint64_t* kto, const uint32_t* type_key, const uint64_t* type_count,
                             uint32_t k_lo, uint32_t k_hi, uint64_t* sig, uint64_t* mass, DevErr* err, cudaStream_t s);
cudaError_t launch_match_scan(uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                              const uint64_t* wt, photon_match_params p, uint32_t k_lo, uint32_t k_hi,
                              const MatchWs& mw, uint64_t* pairs, uint64_t pair_cap, uint64_t* n_pairs, DevErr* err,
                              int num_sms, cudaStream_t s, bool prof_ready = false, bool fused = false);
// photon_analyse: the match split around the canonical sort (k_match.cu)
cudaError_t launch_analyse_filter(uint32_t K, const uint64_t* kto, const uint32_t* list, const HashTable& ht,
                                  uint64_t* mass, const uint64_t* wt, photon_match_params p, const MatchWs& mw,
                                  uint64_t* n_pairs, DevErr* err, cudaStream_t sb);
cudaError_t launch_analyse_exact(uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                                 const uint64_t* wt, photon_match_params p, const MatchWs& mw, uint64_t* pairs,
                                 uint64_t pair_cap, uint64_t* n_pairs, DevErr* err, int num_sms, cudaStream_t s);
// the canonicalisation in two parts (photon_analyse overlaps work with the second)
// zeroed: the caller zeroed the per-call counters (cw.tcount / cw.nbig / mw.state) earlier, off the critical path
cudaError_t launch_canon_lists(const HashTable& ht, uint32_t K, const photon_types& out, const CanonWs& cw,
                               DevErr* err, cudaStream_t s, bool zeroed = false);
// A3 emitted with the rows (photon_analyse): sig = count * key (u64) and sigf = RN32(sig * RN64(1 / N_k)) in row
// order, N_k summed by the sorting warp / CTA (nullptr: rows only)
struct SigOut {
  uint64_t* sig;
  float* sigf;
};
cudaError_t launch_canon_sort(const HashTable& ht, uint32_t K, const uint64_t* kwo, const uint64_t* kernel_warps,
                              const photon_types& out, const CanonWs& cw, int num_sms, cudaStream_t s,
                              SigOut so = SigOut{nullptr, nullptr}, bool zeroed = false);
// the single-GPU fused A3: signatures + the filter profiles in one pass (launch_match_scan(prof_ready = true))
cudaError_t launch_sig_prof(uint32_t K, const uint64_t* kto, const uint32_t* type_key, const uint64_t* type_count,
                            uint64_t* sig, uint64_t* mass, const MatchWs& mw, DevErr* err, cudaStream_t s);
cudaError_t launch_match_resolve(uint32_t K, const uint64_t* kto, const uint64_t* sig, const uint64_t* mass,
                                 const uint64_t* wt, photon_match_params p, const uint64_t* pairs, uint64_t n_pairs,
                                 const uint64_t* n_pairs_dev, const MatchWs& mw, int64_t* match, double* match_dist,
                                 DevErr* err, int num_sms, cudaStream_t s, bool fused = false, bool zeroed = false);

// ---- A5 (k_stable.cu) -------------------------------------------------------------------------------------
size_t stable_ws_bytes(const photon_timing& t);
// N1: warp-level stability over per-kernel warp streams (groups = kernels)
size_t warp_stable_ws_bytes(uint32_t K, uint64_t R);
cudaError_t launch_warp_stable(const photon_timing& t, const uint8_t* ok, uint32_t n, uint32_t dnum, uint32_t dden,
                               void* ws, int64_t* switch_at, uint64_t* dur, DevErr* err, int num_sms,
                               cudaStream_t s);
// ---- N2 (k_full.cu): full-BBV exact grouping and tagged-stream ingest ----------------------------------------
struct FullWs {
  uint64_t *h_lo, *h_hi;  // [W] order-independent 128-bit hash of each warp's event multiset
  uint32_t *kid, *wslot;  // [W] kernel of each warp; its hash-table slot
  uint64_t* list;         // [W] work list of long warps (> 16 events)
  uint64_t* list2;        // [W] long warps whose sequence differs from their type's first (count verification)
  uint32_t* nlist;        // [2] the two lengths
  ulonglong2* htab;       // [B] the two 64-bit mixes of every BB id
};
size_t radix_pairs_ws_bytes(uint64_t n);
cudaError_t launch_radix_pairs(uint64_t* key, uint64_t n, uint32_t bits, void* ws, uint64_t** key_out,
                               uint32_t** perm_out, cudaStream_t s);
cudaError_t launch_group_full(const TraceDev& t, const uint32_t* bbv16, const FullWs& f, const HashTable& ht,
                              const CanonWs& cw, const photon_types& out, DevErr* err, int num_sms, cudaStream_t s);
cudaError_t launch_ingest(uint64_t n, uint64_t W, const uint32_t* warp, const uint16_t* bb, uint64_t* key,
                          void* sort_ws, uint16_t* bb_out, uint64_t* off, DevErr* err, cudaStream_t s);
// ---- N4 (k_pool.cu): persisted signature pool --------------------------------------------------------------
cudaError_t launch_pool_export(uint32_t K, const photon_types& ty, const uint64_t* wt, const int64_t* match,
                               uint64_t* keep, uint64_t* ntypes, const photon_types& pool, uint64_t* pwt,
                               uint32_t* pkid, uint32_t* n_pool, cudaStream_t s);
cudaError_t launch_pool_concat(uint32_t Kp, const photon_types& pool, const uint64_t* pwt, uint32_t K,
                               const photon_types& ty, const uint64_t* wt, uint64_t* okto, uint32_t* okey,
                               uint64_t* ocnt, uint64_t* owt, uint64_t T_bound, int num_sms, cudaStream_t s);
// ---- N3 (k_predict.cu) --------------------------------------------------------------------------------------
cudaError_t launch_kernel_predict(uint32_t K, const int64_t* match, const uint64_t* mass, const uint64_t* full_insts,
                                  const uint64_t* full_cycles, uint64_t* pred_insts, uint64_t* pred_cycles,
                                  DevErr* err, cudaStream_t s);
cudaError_t launch_bb_predict(const TraceDev& t, const int64_t* first_stable, const uint64_t* dur, uint64_t* pred,
                              uint32_t* unpred, uint64_t* long_list, uint32_t* n_long, DevErr* err, int num_sms,
                              cudaStream_t s);
cudaError_t launch_stable(const photon_timing& t, const uint64_t* kbb, photon_stable_params p, void* ws,
                          size_t ws_bytes, int64_t* first_stable, uint64_t* dur, int64_t* switch_at, DevErr* err,
                          int num_sms, cudaStream_t s);

}  // namespace photon
