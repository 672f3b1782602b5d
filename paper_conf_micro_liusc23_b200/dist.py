"""Multi-GPU driver: one process per GPU, torch.distributed (NCCL on GPUs, gloo in the CPU tests) for the plumbing.

DESIGN.md §6.  Two independent sharded paths, both following SURVEY.md §8(e):

ShardedAnalysis (A1 -> A4).  The trace is cut into contiguous warp ranges (one per rank, ~equal events; a kernel
may straddle two shards).  Per rank:

  1. fused BBV + warp-type pass on the local shard (libphoton);                              no communication
  2. local type rows (global kernel id, 16-bin key, count, lowest global warp) -> ALL-GATHER of fixed-capacity
     row buffers (padding rows, PHOTON_ROW_PAD, are skipped by the merge)
  3. merge all rows into the canonical global type tables (identical on every rank); remap local warps to global
     canonical ids;                                                                            no communication
  4. GPU-BBV signatures of the kernels this rank owns (first warp in its range), zeros elsewhere -> ALL-REDUCE
     (SUM) of the signature / mass buffers (north_star: "kernel signatures are merged with an all-reduce")
  5. close-pair scan of a k-range of equal triangle area -> ALL-GATHER of fixed-capacity pair buffers (unused
     slots hold PHOTON_PAIR_PAD, skipped by the resolution)
  6. launch-order resolution of the union (replicated; its result does not depend on pair order).

ShardedStable (A5).  Kernels are independent in the stability test (L229: "the last n basic blocks from the same
type" of one kernel's stream), so each rank tests a contiguous kernel range of the timing stream with no
communication, then the per-kernel outputs (first_stable, stable_dur_sum, switch_at) are ALL-GATHERed.

Both are graph-ready: `plan()` sizes every buffer once (the only host synchronisations: local type count, pair
count), `step()` then issues kernels and collectives only -- no host read, no allocation -- so it can be captured
in one CUDA graph per rank (`capture()`), and `check()` (outside the timed region) raises if a device error was
latched or a fixed capacity overflowed.  The compute goes through a backend object: `GpuBackend` calls
libphoton's C ABI; the CPU tests substitute a brute-force backend to check this host logic against the oracle.
"""
from __future__ import annotations

import math
from typing import Optional

import numpy as np

from ._lib import PAIR_PAD, ROW_PAD

ROW_BYTES = 88  # photon_type_row: kernel u32, pad u32, key 16 x u32, count u64, first_warp u64


class CapacityOverflow(RuntimeError):
    """A fixed-capacity exchange buffer was too small for this step: re-plan (sizes grow) and run again."""


def shard_ranges(warp_counts: np.ndarray, n: int) -> np.ndarray:
    """[n+1] warp cut points with ~equal events per shard (binary search on the event prefix)."""
    pref = np.zeros(len(warp_counts) + 1, np.uint64)
    np.cumsum(warp_counts, out=pref[1:])
    E = int(pref[-1])
    cuts = [0] + [int(np.searchsorted(pref, (E * s) // n, side="left")) for s in range(1, n)] + [len(warp_counts)]
    return np.maximum.accumulate(np.array(cuts, np.int64))


def kernel_ranges(kernel_rec_counts: np.ndarray, n: int) -> np.ndarray:
    """[n+1] kernel cut points with ~equal timing records per rank (A5 shards: whole kernels)."""
    return shard_ranges(np.asarray(kernel_rec_counts, np.uint64), n)


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
    """The collectives the drivers need, over a torch.distributed process group (fixed sizes only)."""

    def __init__(self, group=None):
        import torch.distributed as dist
        self.dist = dist
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)

    def allgather(self, out, x):
        """out [world * n] <- every rank's x [n] (flattened, rank order)."""
        self.dist.all_gather_into_tensor(out.view(-1), x.reshape(-1), group=self.group)
        return out

    def allreduce_sum(self, x):
        self.dist.all_reduce(x, op=self.dist.ReduceOp.SUM, group=self.group)
        return x

    def allreduce_max_host(self, v: int, like) -> int:
        """Plan-time only (synchronises): the maximum of a host integer over ranks."""
        import torch
        t = torch.tensor([int(v)], dtype=torch.int64, device=like.device)
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX, group=self.group)
        return int(t.item())


class GpuBackend:
    """libphoton calls used by the sharded drivers (all on the rank's device and current stream; no host reads
    except local_total / pair_count, which only plan() and check() call)."""

    def __init__(self, ph):
        self.ph = ph
        self.torch = ph.torch

    def zeros(self, n, dtype):
        return self.torch.zeros(max(int(n), 1), dtype=getattr(self.torch, dtype), device=self.ph.device)

    def local_types(self, d, check: bool, out=None):
        return self.ph.photon_warp_group(d, check=check, out=out)

    def local_total(self, ty, K_local: int) -> int:
        return self.ph.photon_types_total(ty, K_local)

    def export(self, ty, d, kernel_base: int, warp_base: int, rows, n_dev):
        self.ph.photon_types_export(d.n_kernels, ty, kernel_base, warp_base, rows, n_dev)

    def alloc_global(self, K: int, cap: int):
        g = self.ph.alloc_types(K, 0, cap)
        g["warp_type"] = None
        return g

    def merge(self, rows, n_rows: int, K: int, kernel_warps, g):
        g["_merge"] = (self.ph.photon_types_merge(rows, n_rows, K, kernel_warps, g), n_rows)
        return g

    def remap(self, d, ty_local, g, kernel_base: int, K: int, out):
        ws, n = g["_merge"]
        self.ph.photon_types_remap(d.n_kernels, d.n_warps, d.kernel_warp_off, ty_local, kernel_base, n, K, ws, out)
        return out

    def types_total(self, g, K: int) -> int:
        return self.ph.photon_types_total(g, K)

    def sig_build(self, g, K: int, k_lo: int, k_hi: int, sig, mass):
        g["_sig_ws"] = self.ph.photon_sig_build(K, g["kernel_type_off"], g["type_key"], g["type_count"], k_lo, k_hi,
                                                sig, mass)

    def match_scan(self, g, K, sig, mass, warps_total, params, k_lo, k_hi, pairs, n_dev, ws_pairs=0):
        g["_scan_ws"] = self.ph.photon_match_scan(K, g["kernel_type_off"], sig, mass, warps_total, params, k_lo, k_hi,
                                                  pairs, n_dev, ws_pairs=ws_pairs)

    def scan_overflow(self, g) -> bool:
        """Plan-time (synchronises): did the filter's candidate list overflow the scan workspace?"""
        from ._lib import ECAPACITY
        rc, _ = self.ph.ws_status(g["_scan_ws"])
        return rc == ECAPACITY

    def pair_count(self, n_dev) -> int:
        return int(n_dev.item())

    def match_resolve(self, g, K, sig, mass, warps_total, params, pairs_all, match, dist):
        g["_resolve_ws"] = self.ph.photon_match_resolve(K, g["kernel_type_off"], sig, mass, warps_total, params,
                                                        pairs_all, int(pairs_all.shape[0]), match, dist)

    def check(self, g, ty_local):
        from ._lib import ECAPACITY
        for ws in (ty_local.get("_ws"), g.get("_merge", (None,))[0], g.get("_sig_ws"), g.get("_scan_ws"),
                   g.get("_resolve_ws")):
            if ws is not None:
                rc, bad = self.ph.ws_status(ws)
                if rc == ECAPACITY:
                    raise CapacityOverflow(f"a device table or candidate list overflowed (index {bad})")
                self.ph.check(ws)

    # A5
    def stable(self, tm, kbb, n, delta, rate, out):
        return self.ph.photon_bb_stable(tm, kbb, n, delta, rate, check=False, out=out)

    def check_stable(self, out):
        self.ph.check(out["_ws"])


class ShardedAnalysis:
    """One rank's part of the sharded A1 -> A4 chain.  Every rank returns the same global type tables and match;
    warp_type covers the rank's own warps (global canonical ids)."""

    def __init__(self, ph_or_backend, n_kernels: int, kernel_warps: np.ndarray, trace, d, theta=(1, 20),
                 n_cores: int = 64, pool_all_prior: int = 0, comm: Optional[Comm] = None,
                 kernel_warp_off_global: Optional[np.ndarray] = None, want_dist: bool = False,
                 pair_slack: float = 1.25):
        self.be = ph_or_backend if hasattr(ph_or_backend, "local_types") else GpuBackend(ph_or_backend)
        self.comm = comm if comm is not None else Comm()
        self.K = int(n_kernels)
        self.kernel_warps = np.asarray(kernel_warps, np.uint64)
        self.tr = trace
        self.d = d
        self.theta = theta
        self.n_cores = n_cores
        self.pool_all_prior = pool_all_prior
        self.want_dist = want_dist
        self.pair_slack = pair_slack
        kwo = kernel_warp_off_global
        if kwo is None:
            kwo = np.zeros(self.K + 1, np.uint64)
            np.cumsum(self.kernel_warps, out=kwo[1:])
        self.kwo_global = kwo
        w0 = int(trace.warp_base)
        w1 = w0 + int(trace.n_warps)
        self.own = owned_kernels(kwo, w0, w1, self.comm.rank == self.comm.world - 1)
        self.tri = triangle_range(self.K, self.comm.rank, self.comm.world)
        self.buf = None  # fixed-capacity buffers, set by plan()

    def _params(self):
        from ._lib import MatchParams
        return MatchParams(int(self.theta[0]), int(self.theta[1]), int(self.n_cores), int(self.pool_all_prior))

    def plan(self, row_cap: int = 0, pair_cap: int = 0):
        """Size every exchange buffer (synchronises: the local type count and the pair count are read once).
        Capacities passed explicitly are used as they are."""
        be, comm, W = self.be, self.comm, self.comm.world
        ty = be.local_types(self.d, check=True)
        T_local = be.local_total(ty, self.d.n_kernels)
        b = dict(ty=ty, n_rows_dev=be.zeros(1, "int64"), n_pairs_dev=be.zeros(1, "int64"))
        like = b["n_rows_dev"]
        if not row_cap:  # explicit capacities are taken as given (check() reports an overflow)
            row_cap = comm.allreduce_max_host(max(T_local, 1), like)
        b["row_cap"] = row_cap
        b["rows"] = be.zeros(row_cap * ROW_BYTES, "uint8").view(row_cap, ROW_BYTES)
        b["rows_all"] = be.zeros(W * row_cap * ROW_BYTES, "uint8").view(W * row_cap, ROW_BYTES)
        n_rows = W * row_cap  # merged types <= rows: sizes the global tables and the signature buffer
        b["g"] = be.alloc_global(self.K, n_rows)
        b["warp_type"] = be.zeros(self.d.n_warps, "int32")
        b["sig"] = be.zeros(16 * n_rows, "int64")
        b["mass"] = be.zeros(self.K, "int64")
        b["match"] = be.zeros(self.K, "int64")
        b["dist"] = be.zeros(self.K, "float64") if self.want_dist else None
        # t: analysed warps per kernel (dominance denominator W_k) and launched warps (warp rule)
        import torch
        analysed = np.diff(np.asarray(self.kwo_global, np.uint64)).astype(np.uint64)
        dev = like.device
        b["kernel_warps"] = torch.from_numpy(analysed.view(np.int64).copy()).to(dev)
        b["warps_total"] = torch.from_numpy(self.kernel_warps.view(np.int64).copy()).to(dev)
        self.buf = b
        # a sizing pass for the pair capacity and the scan workspace (the filter's candidate list): the scan
        # alone, its counts read on the host
        ws_cap = 16 * self.K + 65536
        if not pair_cap:
            self._front()
            b["pairs"] = be.zeros(ws_cap, "int64")
            for _ in range(12):
                be.match_scan(b["g"], self.K, b["sig"], b["mass"], b["warps_total"], self._params(), self.tri[0],
                              self.tri[1], b["pairs"], b["n_pairs_dev"], ws_pairs=ws_cap)
                n = be.pair_count(b["n_pairs_dev"])
                if n > int(b["pairs"].shape[0]):  # close pairs dropped (this also latches ECAPACITY)
                    b["pairs"] = be.zeros(n, "int64")
                    ws_cap = max(ws_cap, n)
                elif be.scan_overflow(b["g"]):  # the filter's candidate list overflowed
                    ws_cap = min(4 * ws_cap, self.K * (self.K - 1) // 2 + 1024)
                else:
                    break
            pair_cap = int(comm.allreduce_max_host(n, like) * self.pair_slack) + 1024
            ws_cap = comm.allreduce_max_host(ws_cap, like)
        b["pair_cap"], b["ws_cap"] = pair_cap, max(ws_cap, pair_cap)
        b["pairs"] = be.zeros(pair_cap, "int64")
        b["pairs_all"] = be.zeros(W * pair_cap, "int64")
        return self

    def _front(self):
        """Steps 1-4 (types, rows exchange, merge + remap, signatures)."""
        be, comm, b = self.be, self.comm, self.buf
        ty = be.local_types(self.d, check=False, out=b["ty"])
        b["ty"] = ty
        be.export(ty, self.d, int(self.tr.kernel_base), int(self.tr.warp_base), b["rows"], b["n_rows_dev"])
        comm.allgather(b["rows_all"], b["rows"])
        g = be.merge(b["rows_all"], int(b["rows_all"].shape[0]), self.K, b["kernel_warps"], b["g"])
        be.remap(self.d, ty, g, int(self.tr.kernel_base), self.K, b["warp_type"])
        be.sig_build(g, self.K, self.own[0], self.own[1], b["sig"], b["mass"])
        comm.allreduce_sum(b["sig"])
        comm.allreduce_sum(b["mass"])
        return g

    def step(self) -> dict:
        """One sync-free pass (kernels and collectives only): returns the result tables (device tensors)."""
        if self.buf is None:
            self.plan()
        be, comm, b = self.be, self.comm, self.buf
        g = self._front()
        be.match_scan(g, self.K, b["sig"], b["mass"], b["warps_total"], self._params(), self.tri[0], self.tri[1],
                      b["pairs"], b["n_pairs_dev"], ws_pairs=b["ws_cap"])
        comm.allgather(b["pairs_all"], b["pairs"])
        be.match_resolve(g, self.K, b["sig"], b["mass"], b["warps_total"], self._params(), b["pairs_all"],
                         b["match"], b["dist"])
        g.update(warp_type=b["warp_type"], match=b["match"], match_dist=b["dist"], sig=b["sig"], mass=b["mass"])
        return g

    def check(self):
        """After step()s (synchronises): device errors, and every rank's fixed capacities (CapacityOverflow)."""
        be, b = self.be, self.buf
        err, flags = None, 0
        try:
            be.check(b["g"], b["ty"])
        except CapacityOverflow:
            flags |= 4
        except Exception as e:  # a latched device error: every rank must leave check() the same way
            err, flags = e, flags | 8
        flags |= int(be.pair_count(b["n_rows_dev"]) > b["row_cap"]) | 2 * int(be.pair_count(b["n_pairs_dev"]) >
                                                                             b["pair_cap"])
        flags = self.comm.allreduce_max_host(flags, b["n_rows_dev"])  # collective: the ranks agree
        if err is not None:
            raise err
        if flags & 8:
            raise RuntimeError("a device error was latched on another rank")
        if flags:
            raise CapacityOverflow(f"exchange capacity exceeded (rows {b['row_cap']}, pairs {b['pair_cap']})")

    def run(self, check: bool = True) -> dict:
        """plan (first call) + step (+ check, re-planning with larger buffers after an overflow)."""
        if self.buf is None:
            self.plan()
        for _ in range(4):
            res = self.step()
            if not check:
                return res
            try:
                self.check()
                res["total_types"] = self.be.types_total(res, self.K)
                return res
            except CapacityOverflow:
                self.plan()  # measured sizes
        raise CapacityOverflow("exchange capacity kept overflowing")

    def capture(self):
        """One CUDA graph of step() on this rank (plan() first; NCCL collectives are captured with the kernels)."""
        import torch
        if self.buf is None:
            self.plan()
        s = torch.cuda.Stream(device=self.buf["sig"].device)
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):  # warm the captured sequence once outside the graph
            self.step()
        torch.cuda.current_stream().wait_stream(s)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            self.result = self.step()
        return graph


def complete_kbb(kbb_local, n_kernels_local: int, n_bb: int, kernel_base: int, own, comm: Comm):
    """kernel_bb_insts rows [own[1] - own[0], B] of this rank's OWNED kernels, complete.  A kernel straddling
    shards has partial rows on the ranks after its owner, as their first local kernel: every rank contributes that
    one row (all-gather of its kernel id + [B] counts), and each owner adds the rows of its kernels.  Setup-time
    helper (torch ops; not part of a timed step)."""
    import torch
    B, k0 = int(n_bb), int(kernel_base)
    kb = kbb_local.reshape(n_kernels_local, B)
    row = torch.zeros(B + 1, dtype=torch.int64, device=kb.device)
    row[0] = -1
    if n_kernels_local and k0 < own[0]:  # the first local kernel started on an earlier rank
        row[0] = k0
        row[1:] = kb[0]
    allr = torch.empty(comm.world * (B + 1), dtype=torch.int64, device=kb.device)
    comm.allgather(allr, row)
    allr = allr.view(comm.world, B + 1).cpu()
    lo, hi = own
    out = kb[lo - k0:hi - k0].clone()
    for r in range(comm.world):
        k = int(allr[r, 0])
        if r != comm.rank and lo <= k < hi:
            out[k - lo] += allr[r, 1:].to(out.device)
    return out.reshape(-1)


class ShardedStable:
    """One rank's part of the kernel-sharded A5: the rank's kernels [k_lo, k_hi) (of `cuts`) tested locally, the
    outputs all-gathered into [world, kmax, B] buffers (kmax = the largest kernel range)."""

    def __init__(self, ph_or_backend, tm_local, kbb_local, cuts, n_bb: int, n: int = 2048, delta=(3, 100),
                 rate=(95, 100), comm: Optional[Comm] = None):
        self.be = ph_or_backend if hasattr(ph_or_backend, "stable") else GpuBackend(ph_or_backend)
        self.comm = comm if comm is not None else Comm()
        self.cuts = np.asarray(cuts, np.int64)
        self.k_lo, self.k_hi = int(self.cuts[self.comm.rank]), int(self.cuts[self.comm.rank + 1])
        self.kmax = max(int(np.diff(self.cuts).max()), 1)
        self.B = int(n_bb)
        self.tm, self.kbb = tm_local, kbb_local
        self.prm = (n, delta, rate)
        self.buf = None

    def plan(self):
        be, W, KB = self.be, self.comm.world, self.kmax * self.B
        self.buf = b = dict(first_stable=be.zeros(KB, "int64"), stable_dur_sum=be.zeros(KB, "int64"),
                            switch_at=be.zeros(self.kmax, "int64"))
        b["fs_all"] = be.zeros(W * KB, "int64")
        b["ds_all"] = be.zeros(W * KB, "int64")
        b["sw_all"] = be.zeros(W * self.kmax, "int64")
        return self

    def step(self):
        if self.buf is None:
            self.plan()
        b, comm = self.buf, self.comm
        n, delta, rate = self.prm
        if self.k_hi > self.k_lo:  # a rank without kernels still joins the all-gathers
            self.be.stable(self.tm, self.kbb, n, delta, rate, b)
        comm.allgather(b["fs_all"], b["first_stable"])
        comm.allgather(b["ds_all"], b["stable_dur_sum"])
        comm.allgather(b["sw_all"], b["switch_at"])
        return b

    def check(self):
        if self.k_hi > self.k_lo:
            self.be.check_stable(self.buf)

    def tables(self):
        """The global [K, B] / [K] outputs assembled from the gathered buffers (outside any timed region)."""
        import torch
        b, W, KB = self.buf, self.comm.world, self.kmax * self.B
        cnt = np.diff(self.cuts)
        fs = torch.cat([b["fs_all"][r * KB:r * KB + int(cnt[r]) * self.B] for r in range(W)])
        ds = torch.cat([b["ds_all"][r * KB:r * KB + int(cnt[r]) * self.B] for r in range(W)])
        sw = torch.cat([b["sw_all"][r * self.kmax:r * self.kmax + int(cnt[r])] for r in range(W)])
        return fs, ds, sw

    def capture(self):
        import torch
        if self.buf is None:
            self.plan()
        s = torch.cuda.Stream(device=self.buf["fs_all"].device)
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            self.step()
        torch.cuda.current_stream().wait_stream(s)
        graph = torch.cuda.CUDAGraph()
        with torch.cuda.graph(graph):
            self.step()
        return graph
