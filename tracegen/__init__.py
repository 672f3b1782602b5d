"""Seeded synthetic inputs for the Photon hot path (shared by the CPU oracle, the CUDA path, tests and bench).

This module is input generation only: it holds none of the method's arithmetic.  The C++ core (gen.cpp) draws
every random number from a counter-based splitmix64 keyed by (seed, purpose, kernel, warp, i), so a shard
(contiguous warp range) or a sample (every `step`-th warp, the paper's 1% sample, L208/L258) is generated
independently and bit-identically.  Recipes: DESIGN.md §4.

Configs (BASELINE.json "configs"):
  1 tiny (1 kernel, 1024 warps, 16 BBs, ~1M events)      2 micro mix (10 VADD + 10 GEMM, 64K warps each)
  3 VGG-16 batch 1                                         4 ResNet-152 batch 1
  5 stress (10^4 kernels, 10^9 events, 4096 BB ids)        6 test mix (every template, small; not a BASELINE config)
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field
from typing import Optional, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libtracegen.so")
_SRC = os.path.join(_HERE, "gen.cpp")

CONFIG_NAMES = {1: "C1-tiny", 2: "C2-micro-mix", 3: "C3-vgg16", 4: "C4-resnet152", 5: "C5-stress", 6: "C6-test-mix"}


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", _SO, _SRC, "-lpthread"])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u64, u32, vp, i32 = ctypes.c_uint64, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_int
        L.tg_create.restype = vp
        L.tg_create.argtypes = [i32, u64, ctypes.c_double]
        L.tg_free.argtypes = [vp]
        L.tg_n_kernels.restype = u32
        L.tg_n_kernels.argtypes = [vp]
        L.tg_n_bb.restype = u32
        L.tg_n_bb.argtypes = [vp]
        L.tg_n_warps.restype = u64
        L.tg_n_warps.argtypes = [vp]
        L.tg_bb_len.argtypes = [vp, vp]
        L.tg_kernel_warps.argtypes = [vp, vp]
        L.tg_kernel_tmpl.argtypes = [vp, vp]
        L.tg_sel_kernels.argtypes = [vp, u64, u64, u64, vp, i32]
        L.tg_sel_counts.argtypes = [vp, u64, u64, u64, vp, i32]
        L.tg_sel_events.argtypes = [vp, u64, u64, u64, vp, vp, i32]
        L.tg_timing.argtypes = [vp, u32, u32, vp, vp, vp, vp, i32]
        L.tg_warp_timing.argtypes = [vp, u32, u32, vp, vp, vp, i32]
        _lib = L
    return _lib


def _threads(threads: Optional[int]) -> int:
    if threads:
        return threads
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:  # pragma: no cover
        return os.cpu_count() or 1


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data


@dataclass
class Trace:
    """Functional BB trace, CSR by kernel then warp (the layout of photon_trace, include/photon.h)."""
    kernel_warp_off: np.ndarray        # u64 [K+1]
    warp_event_off: np.ndarray         # u64 [W+1]
    bb: np.ndarray                     # u16 [E]
    bb_len: np.ndarray                 # u32 [B]
    bb_bin: Optional[np.ndarray]       # u8  [B] or None (bin = b & 15)
    warps_total: np.ndarray            # u64 [K] launched warps per kernel (kernel-match warp rule)
    name: str = ""
    kernel_base: int = 0               # global id of local kernel 0 (shards)
    warp_base: int = 0                 # global index of local warp 0 (shards)

    @property
    def n_kernels(self) -> int:
        return len(self.kernel_warp_off) - 1

    @property
    def n_warps(self) -> int:
        return len(self.warp_event_off) - 1

    @property
    def n_events(self) -> int:
        return len(self.bb)

    @property
    def n_bb(self) -> int:
        return len(self.bb_len)


@dataclass
class Timing:
    """Per-kernel timing streams (photon_timing): records sorted by retire within each kernel."""
    kernel_rec_off: np.ndarray  # u64 [K+1]
    bb: np.ndarray              # u16 [R]
    issue: np.ndarray           # u64 [R]
    retire: np.ndarray          # u64 [R]
    n_bb: int = 0

    @property
    def n_kernels(self) -> int:
        return len(self.kernel_rec_off) - 1

    @property
    def n_records(self) -> int:
        return len(self.bb)


class Generator:
    """Handle on one config's kernel list (cheap to create; events are produced on demand)."""

    def __init__(self, cfg: int, seed: Optional[int] = None, scale: float = 1.0):
        self.cfg = int(cfg)
        self.seed = int(self.cfg if seed is None else seed)
        L = _L()
        self._h = L.tg_create(self.cfg, self.seed, float(scale))
        if not self._h:
            raise ValueError(f"unknown config {cfg}")
        self.n_kernels = L.tg_n_kernels(self._h)
        self.n_bb = L.tg_n_bb(self._h)
        self.n_warps = L.tg_n_warps(self._h)
        self.bb_len = np.empty(self.n_bb, np.uint32)
        L.tg_bb_len(self._h, _ptr(self.bb_len))
        self.kernel_warps = np.empty(self.n_kernels, np.uint64)
        L.tg_kernel_warps(self._h, _ptr(self.kernel_warps))
        self.kernel_tmpl = np.empty(self.n_kernels, np.int32)
        L.tg_kernel_tmpl(self._h, _ptr(self.kernel_tmpl))
        self.kwoff = np.zeros(self.n_kernels + 1, np.uint64)
        np.cumsum(self.kernel_warps, out=self.kwoff[1:])

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and _lib is not None:
            _lib.tg_free(h)
            self._h = None

    # -- warp selections ---------------------------------------------------------------------------------------
    def warp_counts(self, w0: int = 0, w1: Optional[int] = None, step: int = 1, threads=None) -> np.ndarray:
        w1 = self.n_warps if w1 is None else w1
        n = max(0, (w1 - w0 + step - 1) // step)
        out = np.empty(n, np.uint64)
        _L().tg_sel_counts(self._h, w0, w1, step, _ptr(out), _threads(threads))
        return out

    def trace(self, w0: int = 0, w1: Optional[int] = None, step: int = 1, threads=None,
              bb_bin: Optional[np.ndarray] = None) -> Trace:
        """Trace of global warps w0, w0+step, ... < w1.  Local kernels = the kernels spanned by [w0, w1)
        (kernels with no selected warp keep an empty row so kernel ids stay contiguous)."""
        L = _L()
        w1 = self.n_warps if w1 is None else int(w1)
        w0 = int(w0)
        if not (0 <= w0 <= w1 <= self.n_warps) or step < 1:
            raise ValueError("bad warp selection")
        T = _threads(threads)
        n = max(0, (w1 - w0 + step - 1) // step)
        kid = np.empty(n, np.uint32)
        L.tg_sel_kernels(self._h, w0, w1, step, _ptr(kid), T)
        counts = np.empty(n, np.uint64)
        L.tg_sel_counts(self._h, w0, w1, step, _ptr(counts), T)
        off = np.zeros(n + 1, np.uint64)
        np.cumsum(counts, out=off[1:])
        E = int(off[-1])
        bb = np.empty(max(E, 1), np.uint16)[:E]
        L.tg_sel_events(self._h, w0, w1, step, _ptr(off), _ptr(bb), T)
        if w1 > w0:
            k_first = int(np.searchsorted(self.kwoff, w0, side="right") - 1)
            k_last = int(np.searchsorted(self.kwoff, w1 - 1, side="right") - 1)
        else:
            k_first = k_last = 0
        K = k_last - k_first + 1
        per_k = np.bincount(kid.astype(np.int64) - k_first, minlength=K).astype(np.uint64) if n else np.zeros(K, np.uint64)
        kwo = np.zeros(K + 1, np.uint64)
        np.cumsum(per_k, out=kwo[1:])
        return Trace(kernel_warp_off=kwo, warp_event_off=off, bb=bb, bb_len=self.bb_len.copy(),
                     bb_bin=None if bb_bin is None else np.asarray(bb_bin, np.uint8),
                     warps_total=self.kernel_warps[k_first:k_last + 1].copy(),
                     name=f"{CONFIG_NAMES.get(self.cfg, self.cfg)}", kernel_base=k_first, warp_base=w0)

    def kernels_trace(self, k0: int, k1: int, **kw) -> Trace:
        """Trace of all warps of kernels [k0, k1)."""
        return self.trace(int(self.kwoff[k0]), int(self.kwoff[k1]), **kw)

    def timing(self, k0: int = 0, k1: Optional[int] = None, threads=None) -> Timing:
        """Timing streams of kernels [k0, k1) (one record per BB execution of every warp, wave model)."""
        L = _L()
        k1 = self.n_kernels if k1 is None else int(k1)
        T = _threads(threads)
        w0, w1 = int(self.kwoff[k0]), int(self.kwoff[k1])
        counts = self.warp_counts(w0, w1, 1, threads)
        per_k = np.add.reduceat(counts, (self.kwoff[k0:k1] - w0).astype(np.int64)) if k1 > k0 else np.zeros(0, np.uint64)
        # reduceat misbehaves for empty kernels; recompute those as 0
        empty = self.kernel_warps[k0:k1] == 0
        per_k = np.where(empty, 0, per_k).astype(np.uint64)
        off = np.zeros(k1 - k0 + 1, np.uint64)
        np.cumsum(per_k, out=off[1:])
        R = int(off[-1])
        bb = np.empty(R, np.uint16)
        iss = np.empty(R, np.uint64)
        ret = np.empty(R, np.uint64)
        L.tg_timing(self._h, k0, k1, _ptr(off), _ptr(bb), _ptr(iss), _ptr(ret), T)
        return Timing(kernel_rec_off=off, bb=bb, issue=iss, retire=ret, n_bb=self.n_bb)


    def warp_timing(self, k0: int = 0, k1: Optional[int] = None, threads=None) -> Timing:
        """N1 warp streams of kernels [k0, k1): one (issue, retire) record per warp, slot model, sorted by retire
        within each kernel (bb is all zero, n_bb = 1)."""
        L = _L()
        k1 = self.n_kernels if k1 is None else int(k1)
        per_k = np.asarray(self.kernel_warps[k0:k1], np.uint64)
        off = np.zeros(k1 - k0 + 1, np.uint64)
        np.cumsum(per_k, out=off[1:])
        R = int(off[-1])
        iss = np.empty(R, np.uint64)
        ret = np.empty(R, np.uint64)
        L.tg_warp_timing(self._h, k0, k1, _ptr(off), _ptr(iss), _ptr(ret), _threads(threads))
        return Timing(kernel_rec_off=off, bb=np.zeros(R, np.uint16), issue=iss, retire=ret, n_bb=1)


def make_trace(cfg: int, seed: Optional[int] = None, scale: float = 1.0, **kw) -> Trace:
    return Generator(cfg, seed, scale).trace(**kw)


def shard_bounds(warp_counts: np.ndarray, n_shards: int) -> np.ndarray:
    """Cut W warps into n_shards contiguous ranges of ~E/n_shards events each (warp boundaries).
    Returns int64 [n_shards+1] warp indices.  (Input partitioning only; the method does not depend on it.)"""
    W = len(warp_counts)
    pref = np.zeros(W + 1, np.uint64)
    np.cumsum(warp_counts, out=pref[1:])
    E = int(pref[-1])
    cuts = [0]
    for s in range(1, n_shards):
        target = (E * s) // n_shards
        cuts.append(int(np.searchsorted(pref, target, side="left")))
    cuts.append(W)
    cuts = np.maximum.accumulate(np.array(cuts, np.int64))
    return cuts


# ---------------------------------------------------------------------------------------------------------------
# Hand-made traces for tests
def trace_from_warps(kernels, bb_len, bb_bin=None, warps_total=None) -> Trace:
    """kernels: list (per kernel) of lists (per warp) of BB-id sequences."""
    offs, bbs, kwo = [0], [], [0]
    for warps in kernels:
        for seq in warps:
            bbs.extend(seq)
            offs.append(offs[-1] + len(seq))
        kwo.append(kwo[-1] + len(warps))
    K = len(kernels)
    wt = np.array([len(w) for w in kernels] if warps_total is None else warps_total, np.uint64)
    return Trace(kernel_warp_off=np.array(kwo, np.uint64), warp_event_off=np.array(offs, np.uint64),
                 bb=np.array(bbs, np.uint16), bb_len=np.array(bb_len, np.uint32),
                 bb_bin=None if bb_bin is None else np.array(bb_bin, np.uint8), warps_total=wt, name="hand")


def random_trace(seed: int, n_kernels: int, max_warps: int, max_events: int, n_bb: int,
                 custom_bins: bool = False, max_len: int = 64, dup_p: float = 0.6) -> Trace:
    """Small random trace with deliberate duplicates (so grouping has non-trivial types), empty warps and
    ragged lengths.  Uses numpy's PCG64 seeded generator (input generation only)."""
    rs = np.random.default_rng(seed)
    bb_len = rs.integers(1, max_len + 1, n_bb, dtype=np.uint32)
    bb_bin = rs.integers(0, 16, n_bb, dtype=np.uint8) if custom_bins else None
    kernels = []
    for _ in range(n_kernels):
        nw = int(rs.integers(0, max_warps + 1))
        protos = [rs.integers(0, n_bb, int(rs.integers(0, max_events + 1))).tolist() for _ in range(3)]
        warps = []
        for _ in range(nw):
            if rs.random() < dup_p:
                warps.append(list(protos[int(rs.integers(0, 3))]))
            else:
                warps.append(rs.integers(0, n_bb, int(rs.integers(0, max_events + 1))).tolist())
        kernels.append(warps)
    if all(len(w) == 0 for w in kernels):
        kernels[0].append([0])
    return trace_from_warps(kernels, bb_len, bb_bin)
