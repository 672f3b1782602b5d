"""Multi-GPU driver: warps sharded across ranks (one process per GPU), merged with torch.distributed collectives.

DESIGN.md §6.  The trace is cut into contiguous warp ranges (one per rank, ~equal events; a kernel may straddle two
shards).  Per rank:

  1. fused BBV + warp-type pass on the local shard (libphoton);                              no communication
  2. local type rows (global kernel id, 16-bin key, count, lowest global warp) -> variable-length ALL-GATHER
  3. merge all rows into the canonical global type tables (identical on every rank); remap local warps to global
     canonical ids;                                                                            no communication
  4. GPU-BBV signatures of the kernels this rank owns (first warp in its range) -> ALL-REDUCE (SUM) of the
     zero-padded signature / mass buffers (north_star: "kernel signatures are merged with an all-reduce")
  5. close-pair scan of a k-range of equal triangle area -> variable-length ALL-GATHER of the pairs
  6. launch-order resolution of the union (replicated; its result does not depend on pair order).

The collectives go through `Comm` (torch.distributed with NCCL on GPUs; gloo in the CPU tests) and the compute
through a backend object; `GpuBackend` calls libphoton's C ABI.  The CPU tests substitute a brute-force backend to
check this host logic (sharding, padding, ownership, ranges) against the single-process oracle.
"""
from __future__ import annotations

import math
from typing import Optional, Sequence

import numpy as np

ROW_BYTES = 88  # photon_type_row: kernel u32, pad u32, key 16 x u32, count u64, first_warp u64


def shard_ranges(warp_counts: np.ndarray, n: int) -> np.ndarray:
    """[n+1] warp cut points with ~equal events per shard (binary search on the event prefix)."""
    pref = np.zeros(len(warp_counts) + 1, np.uint64)
    np.cumsum(warp_counts, out=pref[1:])
    E = int(pref[-1])
    cuts = [0] + [int(np.searchsorted(pref, (E * s) // n, side="left")) for s in range(1, n)] + [len(warp_counts)]
    return np.maximum.accumulate(np.array(cuts, np.int64))


def owned_kernels(kernel_warp_off: np.ndarray, w0: int, w1: int, is_last: bool):
    """Kernels whose first warp lies in [w0, w1) (empty kernels at the very end belong to the last rank)."""
    kwo = np.asarray(kernel_warp_off, np.int64)
    K = len(kwo) - 1
    starts = kwo[:K]
    lo = int(np.searchsorted(starts, w0, side="left"))
    hi = K if is_last else int(np.searchsorted(starts, w1, side="left"))
    return lo, hi


def triangle_range(K: int, rank: int, world: int):
    """k in [lo, hi): ranks get ~equal shares of the lower-triangle pair work (k-rows have k pairs each)."""
    lo = int(math.floor(K * math.sqrt(rank / world)))
    hi = K if rank == world - 1 else int(math.floor(K * math.sqrt((rank + 1) / world)))
    return lo, hi


class Comm:
    """The collectives the driver needs, over a torch.distributed process group."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)

    def allgather_varlen(self, x):
        """Concatenate a variable-length tensor (first dim) across ranks, in rank order."""
        import torch
        n = torch.tensor([x.shape[0]], dtype=torch.int64, device=x.device)
        ns = [torch.zeros_like(n) for _ in range(self.world)]
        self.dist.all_gather(ns, n, group=self.group)
        counts = [int(v.item()) for v in ns]
        m = max(counts) if counts else 0
        if m == 0:
            return x[:0], counts
        pad = torch.zeros((m,) + tuple(x.shape[1:]), dtype=x.dtype, device=x.device)
        pad[: x.shape[0]] = x
        outs = [torch.empty_like(pad) for _ in range(self.world)]
        self.dist.all_gather(outs, pad, group=self.group)
        return torch.cat([o[:c] for o, c in zip(outs, counts)]), counts

    def allreduce_sum(self, x):
        self.dist.all_reduce(x, op=self.dist.ReduceOp.SUM, group=self.group)
        return x


class GpuBackend:
    """libphoton calls used by the sharded chain (all on the rank's device and current stream)."""

    def __init__(self, ph):
        self.ph = ph
        self.torch = ph.torch

    def local_rows(self, d, kernel_base: int, warp_base: int, check: bool):
        ty = self.ph.photon_warp_group(d, check=check)
        T = self.ph.photon_types_total(ty, d.n_kernels)
        rows = self.torch.empty((max(T, 1), ROW_BYTES), dtype=self.torch.uint8, device=self.ph.device)
        if T:
            self.ph.photon_types_export(d.n_kernels, ty, kernel_base, warp_base, rows)
        return ty, rows[:T]

    def merge(self, rows, K: int, kernel_warps):
        n = int(rows.shape[0])
        cap = max(n, 1)
        g = self.ph.alloc_types(K, 0, cap)
        g["warp_type"] = None
        ws = self.ph.photon_types_merge(rows, n, K, kernel_warps, g)
        g["_merge"] = (ws, n)
        return g

    def remap(self, d, ty_local, g, kernel_base: int, K: int):
        out = self.ph.empty(d.n_warps, "int32")
        ws, n = g["_merge"]
        self.ph.photon_types_remap(d.n_kernels, d.n_warps, d.kernel_warp_off, ty_local, kernel_base, n, K, ws, out)
        return out

    def types_total(self, g, K: int) -> int:
        return self.ph.photon_types_total(g, K)

    def sig_build(self, g, K: int, T: int, k_lo: int, k_hi: int):
        sig = self.torch.zeros(16 * max(T, 1), dtype=self.torch.int64, device=self.ph.device)
        mass = self.torch.zeros(K, dtype=self.torch.int64, device=self.ph.device)
        if k_hi > k_lo:
            self.ph.photon_sig_build(K, g["kernel_type_off"], g["type_key"], g["type_count"], k_lo, k_hi, sig, mass)
        return sig, mass

    def match_scan(self, g, K, sig, mass, warps_total, params, k_lo, k_hi, cap):
        pairs = self.torch.empty(max(cap, 1), dtype=self.torch.int64, device=self.ph.device)
        n = self.torch.zeros(1, dtype=self.torch.int64, device=self.ph.device)
        self.ph.photon_match_scan(K, g["kernel_type_off"], sig, mass, warps_total, params, k_lo, k_hi, pairs, n)
        cnt = int(n.item())
        if cnt > cap:
            return None
        return pairs[:cnt]

    def match_resolve(self, g, K, sig, mass, warps_total, params, pairs):
        match = self.ph.empty(K, "int64")
        dist = self.ph.empty(K, "float64")
        self.ph.photon_match_resolve(K, g["kernel_type_off"], sig, mass, warps_total, params, pairs,
                                     int(pairs.shape[0]), match, dist)
        return match, dist


class ShardedAnalysis:
    """One rank's part of the sharded A1 -> A4 chain.  Every rank returns the same global type tables and match;
    warp_type covers the rank's own warps (global canonical ids)."""

    def __init__(self, ph_or_backend, n_kernels: int, kernel_warps: np.ndarray, trace, d, theta=(1, 20),
                 n_cores: int = 64, pool_all_prior: int = 0, comm: Optional[Comm] = None,
                 kernel_warp_off_global: Optional[np.ndarray] = None):
        self.be = ph_or_backend if hasattr(ph_or_backend, "local_rows") else GpuBackend(ph_or_backend)
        self.comm = comm if comm is not None else Comm()
        self.K = int(n_kernels)
        self.kernel_warps = np.asarray(kernel_warps, np.uint64)
        self.tr = trace
        self.d = d
        self.theta = theta
        self.n_cores = n_cores
        self.pool_all_prior = pool_all_prior
        kwo = kernel_warp_off_global
        if kwo is None:
            kwo = np.zeros(self.K + 1, np.uint64)
            np.cumsum(self.kernel_warps, out=kwo[1:])
        self.kwo_global = kwo
        w0 = int(trace.warp_base)
        w1 = w0 + int(trace.n_warps)
        self.own = owned_kernels(kwo, w0, w1, self.comm.rank == self.comm.world - 1)
        self.tri = triangle_range(self.K, self.comm.rank, self.comm.world)
        self.pair_cap = 16 * self.K + 65536
        self._dev_tensors = None

    def _tensors(self, like):
        import torch
        if self._dev_tensors is None:
            dev = like.device
            analysed = np.diff(np.asarray(self.kwo_global, np.uint64)).astype(np.uint64)  # dominance denominator W_k
            self._dev_tensors = dict(
                kernel_warps=torch.from_numpy(analysed.view(np.int64)).to(dev),
                warps_total=torch.from_numpy(self.kernel_warps.view(np.int64)).to(dev))  # launched (warp rule)
        return self._dev_tensors

    def run(self, check: bool = False) -> dict:
        be, comm = self.be, self.comm
        # 1-2: local types -> rows -> all-gather
        ty_local, rows = be.local_rows(self.d, int(self.tr.kernel_base), int(self.tr.warp_base), check)
        rows_all, _ = comm.allgather_varlen(rows)
        t = self._tensors(rows_all)
        # 3: merged canonical tables (same on every rank) + local warps -> global ids
        g = be.merge(rows_all, self.K, t["kernel_warps"])
        warp_type = be.remap(self.d, ty_local, g, int(self.tr.kernel_base), self.K)
        T = be.types_total(g, self.K)
        # 4: signatures of owned kernels -> all-reduce
        sig, mass = be.sig_build(g, self.K, T, self.own[0], self.own[1])
        comm.allreduce_sum(sig)
        comm.allreduce_sum(mass)
        # 5: pair scan of this rank's k-range -> all-gather
        from ._lib import MatchParams
        params = MatchParams(int(self.theta[0]), int(self.theta[1]), int(self.n_cores), int(self.pool_all_prior))
        while True:
            pairs = be.match_scan(g, self.K, sig, mass, t["warps_total"], params, self.tri[0], self.tri[1],
                                  self.pair_cap)
            ok = 1 if pairs is not None else 0
            import torch
            flag = torch.tensor([1 - ok], dtype=torch.int64, device=sig.device)
            comm.allreduce_sum(flag)  # every rank retries together if any ran out of pair capacity
            if int(flag.item()) == 0:
                break
            self.pair_cap *= 4
        pairs_all, _ = comm.allgather_varlen(pairs)
        # 6: launch-order resolution (replicated)
        match, dist = be.match_resolve(g, self.K, sig, mass, t["warps_total"], params, pairs_all)
        g.update(warp_type=warp_type, match=match, match_dist=dist, sig=sig, mass=mass, total_types=T)
        return g
