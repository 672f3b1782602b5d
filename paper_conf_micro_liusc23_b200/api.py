"""Thin Python binding of libphoton (same names as the C ABI, argument marshalling only).

PyTorch supplies device memory and streams; every step of the path runs in libphoton's sm_100a kernels.  There
is no CPU fallback: constructing `Photon` without a CUDA device or without the built library raises.

Unsigned device arrays are carried in signed torch tensors of the same width (u64 -> int64, u32 -> int32,
u16 -> int16); the bits are what the C ABI sees.
"""
from __future__ import annotations

import ctypes
from dataclasses import dataclass
from typing import Dict, Optional, Tuple

import numpy as np

from . import _lib
from ._lib import PhotonError, PhotonUnavailable

_NP2T = {np.dtype(np.uint64): "int64", np.dtype(np.int64): "int64", np.dtype(np.uint32): "int32",
         np.dtype(np.int32): "int32", np.dtype(np.uint16): "int16", np.dtype(np.uint8): "uint8",
         np.dtype(np.float64): "float64"}


def _torch():
    import torch
    return torch


def to_device(a: np.ndarray, device, pin: bool = False, non_blocking: bool = False):
    """numpy -> torch tensor with the same bits (unsigned carried in signed tensors of equal width)."""
    torch = _torch()
    a = np.ascontiguousarray(a)
    view = {8: np.int64, 4: np.int32, 2: np.int16, 1: np.uint8}[a.dtype.itemsize] if a.dtype.kind in "ui" else a.dtype
    t = torch.from_numpy(a.view(view))
    if pin:
        t = t.pin_memory()
    return t.to(device, non_blocking=non_blocking) if device is not None else t


def to_numpy(t, dtype) -> np.ndarray:
    return t.detach().cpu().numpy().view(dtype)


@dataclass
class DeviceTrace:
    """photon_trace in device memory."""
    kernel_warp_off: "object"  # int64 [K+1]
    warp_event_off: "object"   # int64 [W+1]
    bb: "object"               # int16 [E]
    bb_len: "object"           # int32 [B]
    bb_bin: Optional["object"]  # uint8 [B] or None
    warps_total: "object"      # int64 [K]
    n_kernels: int
    n_bb: int
    n_warps: int
    n_events: int

    @staticmethod
    def from_host(trace, device, non_blocking: bool = False) -> "DeviceTrace":
        """`trace` has numpy fields kernel_warp_off, warp_event_off, bb, bb_len, bb_bin, warps_total."""
        f = lambda a: to_device(a, device, non_blocking=non_blocking)
        return DeviceTrace(f(trace.kernel_warp_off), f(trace.warp_event_off), f(trace.bb), f(trace.bb_len),
                           None if trace.bb_bin is None else f(trace.bb_bin), f(trace.warps_total),
                           len(trace.kernel_warp_off) - 1, len(trace.bb_len), len(trace.warp_event_off) - 1,
                           len(trace.bb))

    def c(self) -> _lib.Trace:
        p = lambda t: t.data_ptr() if (t is not None and t.numel() > 0) else None
        return _lib.Trace(self.n_kernels, self.n_bb, self.n_warps, self.n_events, p(self.kernel_warp_off),
                          p(self.warp_event_off), p(self.bb), p(self.bb_len), p(self.bb_bin))


@dataclass
class DeviceTiming:
    kernel_rec_off: "object"  # int64 [K+1]
    bb: "object"              # int16 [R]
    issue: "object"           # int64 [R]
    retire: "object"          # int64 [R]
    n_kernels: int
    n_bb: int
    n_records: int

    @staticmethod
    def from_host(tm, device, n_bb: Optional[int] = None) -> "DeviceTiming":
        f = lambda a: to_device(a, device)
        return DeviceTiming(f(tm.kernel_rec_off), f(tm.bb), f(tm.issue), f(tm.retire), len(tm.kernel_rec_off) - 1,
                            int(n_bb if n_bb is not None else tm.n_bb), len(tm.bb))

    def c(self) -> _lib.Timing:
        p = lambda t: t.data_ptr() if t.numel() > 0 else None
        return _lib.Timing(self.n_kernels, self.n_bb, self.n_records, p(self.kernel_rec_off), p(self.bb),
                           p(self.issue), p(self.retire))


def ht_capacity(hint: int, n_warps: int) -> int:
    """Mirror of abi.cu's hash-table sizing (power of two >= 2 x expected types, >= 1024)."""
    h = hint if hint else min(n_warps, 1 << 18)
    cap = 1024
    while cap < 2 * h:
        cap <<= 1
    return cap


class Photon:
    """One libphoton context on one CUDA device."""

    def __init__(self, device=None):
        torch = _torch()
        if not torch.cuda.is_available():
            raise PhotonUnavailable("libphoton needs a CUDA device (sm_100a); none is visible")
        self.torch = torch
        self.device = torch.device("cuda", torch.cuda.current_device() if device is None else int(device))
        self.L = _lib.load()
        ctx = ctypes.c_void_p()
        rc = self.L.photon_create(ctypes.byref(ctx), self.device.index)
        if rc != 0:
            raise PhotonUnavailable(f"photon_create failed ({rc})")
        self.ctx = ctx
        self._ws: Dict[str, object] = {}
        self._hint: Dict[tuple, int] = {}   # table sizes that worked, reused by later unchecked calls
        self._pcap: Dict[int, int] = {}

    def __del__(self):
        if getattr(self, "ctx", None) is not None and getattr(self, "L", None) is not None:
            self.L.photon_destroy(self.ctx)
            self.ctx = None

    # -- plumbing ---------------------------------------------------------------------------------------------
    def stream_ptr(self, stream=None) -> int:
        s = stream if stream is not None else self.torch.cuda.current_stream(self.device)
        return s.cuda_stream

    def workspace(self, tag: str, nbytes: int):
        """Cached device workspace (grows, never shrinks); returns a view of exactly nbytes."""
        ws = self._ws.get(tag)
        if ws is None or ws.numel() < nbytes:
            ws = self.torch.empty(max(nbytes, 256), dtype=self.torch.uint8, device=self.device)
            self._ws[tag] = ws
        return ws[:max(nbytes, 256)]

    def _rc(self, rc: int):
        if rc != 0:
            raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode())

    def ws_status(self, ws, stream=None) -> Tuple[int, int]:
        bad = ctypes.c_int64(-1)
        rc = self.L.photon_ws_status(self.ctx, ws.data_ptr(), self.stream_ptr(stream), ctypes.byref(bad))
        return rc, bad.value

    def check(self, ws, stream=None):
        rc, bad = self.ws_status(ws, stream)
        if rc != 0:
            raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)

    def empty(self, n, dtype):
        return self.torch.empty(max(int(n), 0), dtype=getattr(self.torch, dtype), device=self.device)

    # -- A1 ----------------------------------------------------------------------------------------------------
    def photon_bbv_build(self, t: DeviceTrace, bbv16: bool = True, insts: bool = True, kbb: bool = False,
                         stream=None, check: bool = True, out: Optional[dict] = None) -> dict:
        ct = t.c()
        nb = self.L.photon_bbv_workspace_bytes(ctypes.byref(ct))
        ws = self.workspace("bbv", nb)
        o = out if out is not None else {}
        if bbv16 and "warp_bbv16" not in o:
            o["warp_bbv16"] = self.empty(16 * t.n_warps, "int32")
        if insts and "warp_insts" not in o:
            o["warp_insts"] = self.empty(t.n_warps, "int64")
        if kbb and "kernel_bb_insts" not in o:
            o["kernel_bb_insts"] = self.empty(t.n_kernels * t.n_bb, "int64")
        p = lambda k: o[k].data_ptr() if (k in o and o[k].numel()) else None
        self._rc(self.L.photon_bbv_build(self.ctx, ctypes.byref(ct), ws.data_ptr(), ws.numel(),
                                         p("warp_bbv16") if bbv16 else None, p("warp_insts") if insts else None,
                                         p("kernel_bb_insts") if kbb else None, self.stream_ptr(stream)))
        if check:
            self.check(ws, stream)
        return o

    # -- A2 ----------------------------------------------------------------------------------------------------
    def alloc_types(self, n_kernels: int, n_warps: int, capacity: int) -> dict:
        cap = max(1, capacity)
        return dict(capacity=cap, warp_type=self.empty(n_warps, "int32"),
                    kernel_type_off=self.empty(n_kernels + 1, "int64"), type_key=self.empty(16 * cap, "int32"),
                    type_count=self.empty(cap, "int64"), type_first_warp=self.empty(cap, "int64"),
                    warp_sampling_ok=self.empty(n_kernels, "uint8"))

    @staticmethod
    def _types_fit(ty: Optional[dict], n_kernels: int, n_warps: int, capacity: int) -> bool:
        """A previous result's tables may be reused only when every array has exactly this trace's sizes (the
        kernels write W / K / K+1 entries and up to `capacity` rows)."""
        if ty is None or ty.get("capacity", 0) < capacity:
            return False
        need = dict(warp_type=n_warps, kernel_type_off=n_kernels + 1, warp_sampling_ok=n_kernels,
                    type_key=16 * ty["capacity"], type_count=ty["capacity"], type_first_warp=ty["capacity"])
        return all(ty.get(k) is not None and ty[k].numel() == n for k, n in need.items())

    @staticmethod
    def types_c(ty: dict) -> _lib.Types:
        p = lambda k: ty[k].data_ptr() if (ty.get(k) is not None and ty[k].numel()) else None
        return _lib.Types(ty["capacity"], p("warp_type"), p("kernel_type_off"), p("type_key"), p("type_count"),
                          p("type_first_warp"), p("warp_sampling_ok"))

    def photon_warp_group(self, t: DeviceTrace, warp_bbv16=None, capacity_hint: int = 0, stream=None,
                          check: bool = True, out: Optional[dict] = None, remap_stream=None) -> dict:
        """remap_stream (optional): warp_type is written there (photon_warp_group2) -- join it before reading."""
        key = (t.n_kernels, t.n_warps)
        hint = max(capacity_hint, self._hint.get(key, 0))
        for _ in range(8):
            ct = t.c()
            nb = self.L.photon_group_workspace_bytes(ctypes.byref(ct), hint)
            ws = self.workspace("group", nb)
            cap = min(max(t.n_warps, 1), ht_capacity(hint, t.n_warps))
            ty = out if self._types_fit(out, t.n_kernels, t.n_warps, cap) else self.alloc_types(t.n_kernels, t.n_warps, cap)
            tc = self.types_c(ty)
            self._rc(self.L.photon_warp_group2(self.ctx, ctypes.byref(ct),
                                               None if warp_bbv16 is None else warp_bbv16.data_ptr(), ws.data_ptr(),
                                               ws.numel(), ctypes.byref(tc), self.stream_ptr(stream),
                                               self.stream_ptr(remap_stream if remap_stream is not None else stream)))
            ty["_ws"] = ws
            if not check:
                return ty
            rc, bad = self.ws_status(ws, stream)
            if rc == _lib.ECAPACITY:
                hint = max(2 * ht_capacity(hint, t.n_warps), 1 << 12)
                out = None
                continue
            if rc != 0:
                raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)
            self._hint[key] = hint
            return ty
        raise PhotonError(_lib.ECAPACITY, "type table kept overflowing")

    def photon_types_total(self, ty: dict, n_kernels: int, stream=None) -> int:
        v = ctypes.c_uint64(0)
        tc = self.types_c(ty)
        self._rc(self.L.photon_types_total(self.ctx, ctypes.byref(tc), n_kernels, ctypes.byref(v),
                                           self.stream_ptr(stream)))
        return int(v.value)

    # -- A3 + A4 -----------------------------------------------------------------------------------------------
    @staticmethod
    def match_params(theta=(1, 20), n_cores=64, pool_all_prior=0) -> _lib.MatchParams:
        return _lib.MatchParams(int(theta[0]), int(theta[1]), int(n_cores), int(pool_all_prior))

    def photon_kernel_match(self, n_kernels: int, ty: dict, warps_total, theta=(1, 20), n_cores=64,
                            pool_all_prior=0, want_dist: bool = True, pair_capacity: int = 0, stream=None,
                            check: bool = True, out: Optional[dict] = None) -> dict:
        K = n_kernels
        cap = max(pair_capacity or (16 * K + 65536), self._pcap.get(K, 0))
        for _ in range(8):
            nb = self.L.photon_match_workspace_bytes(K, ty["capacity"], cap)
            ws = self.workspace("match", nb)
            o = out if out is not None else {}
            o.setdefault("match", self.empty(K, "int64"))
            if want_dist:
                o.setdefault("match_dist", self.empty(K, "float64"))
            tc = self.types_c(ty)
            self._rc(self.L.photon_kernel_match(self.ctx, K, ctypes.byref(tc), warps_total.data_ptr(),
                                                self.match_params(theta, n_cores, pool_all_prior), ws.data_ptr(),
                                                ws.numel(), o["match"].data_ptr(),
                                                o["match_dist"].data_ptr() if want_dist else None,
                                                self.stream_ptr(stream)))
            o["_ws"] = ws
            if not check:
                return o
            rc, bad = self.ws_status(ws, stream)
            if rc == _lib.ECAPACITY:
                cap *= 4
                continue
            if rc != 0:
                raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)
            self._pcap[K] = cap
            return o
        raise PhotonError(_lib.ECAPACITY, "pair table kept overflowing")

    def match_stats(self, n_kernels: int, ty: dict, m: dict, stream=None) -> dict:
        st = (ctypes.c_uint64 * 4)()
        ws = m["_ws"]
        self._rc(self.L.photon_match_stats(self.ctx, n_kernels, ty["capacity"], ws.data_ptr(), ws.numel(), st,
                                           self.stream_ptr(stream)))
        return dict(filter_pairs=int(st[0]), close_pairs=int(st[1]), rounds=int(st[2]), pair_capacity=int(st[3]))

    # -- N2: full-BBV exact grouping and tagged-stream ingest (L154, L161) -------------------------------------
    def photon_warp_group_full(self, t: DeviceTrace, warp_bbv16=None, stream=None, check: bool = True,
                               out: Optional[dict] = None) -> dict:
        """Warp types keyed on the full BBV (N2); warp_bbv16 from photon_bbv_build (computed when None).  `out` (a
        previous result for the same trace) is reused instead of allocating new tables."""
        if warp_bbv16 is None:
            warp_bbv16 = self.photon_bbv_build(t, bbv16=True, insts=False, stream=stream, check=check)["warp_bbv16"]
        ct = t.c()
        cap = max(t.n_warps, 1)
        ty = out if self._types_fit(out, t.n_kernels, t.n_warps, cap) else self.alloc_types(t.n_kernels, t.n_warps, cap)
        # the hash table is sized from the types a checked call found before (a table for every warp otherwise)
        key = ("full", t.n_kernels, t.n_warps)
        hint = self._hint.get(key, 0)
        for _ in range(8):
            ws = self.workspace("group_full", self.L.photon_group_full_workspace_bytes(ctypes.byref(ct), hint))
            self._rc(self.L.photon_warp_group_full(self.ctx, ctypes.byref(ct), warp_bbv16.data_ptr(), ws.data_ptr(),
                                                   ws.numel(), ctypes.byref(self.types_c(ty)),
                                                   self.stream_ptr(stream)))
            ty["_ws"] = ws
            if not check:
                return ty
            rc, bad = self.ws_status(ws, stream)
            if rc == _lib.ECAPACITY and hint:
                hint = 0  # the full-size table cannot overflow
                continue
            if rc != 0:
                raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)
            if key not in self._hint:
                self._hint[key] = max(2 * self.photon_types_total(ty, t.n_kernels, stream), 512)
            return ty
        raise PhotonError(_lib.ECAPACITY, "full-BBV type table kept overflowing")

    def photon_ingest_tagged(self, warp, bb, n_warps: int, stream=None, check: bool = True) -> dict:
        """Interleaved (warp, bb) tagged events -> CSR by warp (stable): dict(bb, warp_event_off)."""
        n = int(warp.numel())
        ws = self.workspace("ingest", self.L.photon_ingest_workspace_bytes(n, n_warps))
        out = dict(bb=self.empty(n, "int16"), warp_event_off=self.empty(n_warps + 1, "int64"))
        self._rc(self.L.photon_ingest_tagged(self.ctx, n, n_warps, warp.data_ptr() if n else None,
                                             bb.data_ptr() if n else None, ws.data_ptr(), ws.numel(),
                                             out["bb"].data_ptr() if n else None, out["warp_event_off"].data_ptr(),
                                             self.stream_ptr(stream)))
        if check:
            self.check(ws, stream)
        return out

    # -- N4: persisted signature pool (L402) -------------------------------------------------------------------
    def photon_pool_export(self, n_kernels: int, ty: dict, warps_total, match, stream=None) -> dict:
        """The representatives of a run (match < 0) as a pool: dict(n_pool, capacity, kernel_type_off, type_key,
        type_count, warps_total, kernel_id) of device tensors.  Syncs once to read the pool's size."""
        K = n_kernels
        ws = self.workspace("pool", self.L.photon_pool_export_workspace_bytes(K))
        pool = dict(capacity=ty["capacity"], kernel_type_off=self.empty(K + 1, "int64"),
                    type_key=self.empty(16 * ty["capacity"], "int32"), type_count=self.empty(ty["capacity"], "int64"))
        pwt, pkid, npool = self.empty(K, "int64"), self.empty(K, "int32"), self.empty(1, "int32")
        pc = self.types_c(pool)
        self._rc(self.L.photon_pool_export(self.ctx, K, ctypes.byref(self.types_c(ty)), warps_total.data_ptr(),
                                           match.data_ptr(), ws.data_ptr(), ws.numel(), ctypes.byref(pc),
                                           pwt.data_ptr(), pkid.data_ptr(), npool.data_ptr(),
                                           self.stream_ptr(stream)))
        self.torch.cuda.synchronize(self.device)
        Kp = int(npool.item())
        T = int(pool["kernel_type_off"][Kp].item())
        return dict(n_pool=Kp, capacity=max(T, 1), kernel_type_off=pool["kernel_type_off"][:Kp + 1],
                    type_key=pool["type_key"][:16 * max(T, 1)], type_count=pool["type_count"][:max(T, 1)],
                    warps_total=pwt[:Kp], kernel_id=pkid[:Kp])

    def photon_kernel_match_pooled(self, pool: dict, n_kernels: int, ty: dict, warps_total, theta=(1, 20),
                                   n_cores=64, pool_all_prior=0, want_dist: bool = True, stream=None) -> dict:
        """A4 against a pool (N4): match / match_dist over [0, Kp + K); index < Kp = a pooled kernel."""
        Kp, K = pool["n_pool"], n_kernels
        Tp, T = pool["capacity"], ty["capacity"]
        cap = 1024
        for _ in range(8):
            nb = self.L.photon_pool_match_workspace_bytes(Kp, Tp, K, T, max(cap, 16 * (Kp + K) + 65536))
            ws = self.workspace("pool_match", nb)
            off = (self.L.photon_pool_match_workspace_bytes(Kp, Tp, K, T, 1024)
                   - self.L.photon_match_workspace_bytes(Kp + K, Tp + T, 1024))
            o = dict(match=self.empty(Kp + K, "int64"))
            if want_dist:
                o["match_dist"] = self.empty(Kp + K, "float64")
            self._rc(self.L.photon_kernel_match_pooled(
                self.ctx, Kp, ctypes.byref(self.types_c(pool)), pool["warps_total"].data_ptr() if Kp else None, Tp,
                K, ctypes.byref(self.types_c(ty)), warps_total.data_ptr(), T,
                self.match_params(theta, n_cores, pool_all_prior), ws.data_ptr(), ws.numel(), o["match"].data_ptr(),
                o["match_dist"].data_ptr() if want_dist else None, self.stream_ptr(stream)))
            rc, bad = self.ws_status(ws[off:], stream)
            if rc == _lib.ECAPACITY:
                cap *= 4
                continue
            if rc != 0:
                raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)
            return o
        raise PhotonError(_lib.ECAPACITY, "pair table kept overflowing")

    @staticmethod
    def save_pool(pool: dict, path: str):
        """Persist a pool (host .npz; the analysis data is micro-architecture agnostic, L402)."""
        import numpy as np
        np.savez(path, **{k: (v.cpu().numpy() if hasattr(v, "cpu") else np.asarray(v)) for k, v in pool.items()})

    def load_pool(self, path: str) -> dict:
        import numpy as np
        z = np.load(path)
        out = {}
        for k in z.files:
            v = z[k]
            out[k] = int(v) if v.ndim == 0 else self.torch.from_numpy(v).to(self.device)
        return out

    def photon_gpu_bbv(self, n_kernels: int, ty: dict, stream=None, check: bool = True) -> dict:
        """A3 (L178, Fig 5): every kernel's GPU-BBV signature g_k (sig [16T] u64 in the rows' order, so
        sig_off = 16 * kernel_type_off) and its mass N_k = sum(g_k) (mass [K] u64), via photon_sig_build."""
        K = n_kernels
        o = dict(sig=self.empty(16 * ty["capacity"], "int64"), mass=self.empty(max(K, 1), "int64"))
        ws = self.photon_sig_build(K, ty["kernel_type_off"], ty["type_key"], ty["type_count"], 0, K, o["sig"],
                                   o["mass"], stream=stream)
        if check:
            self.check(ws, stream)
        o["mass"] = o["mass"][:K]
        return o

    # split form (multi-GPU driver)
    def photon_sig_build(self, K, kto, type_key, type_count, k_lo, k_hi, sig, mass, stream=None):
        ws = self.workspace("sig", 256)
        self._rc(self.L.photon_sig_build(self.ctx, K, kto.data_ptr(), type_key.data_ptr(), type_count.data_ptr(),
                                         k_lo, k_hi, sig.data_ptr() if sig.numel() else None, mass.data_ptr(),
                                         ws.data_ptr(), ws.numel(), self.stream_ptr(stream)))
        return ws

    def photon_match_scan(self, K, kto, sig, mass, warps_total, params, k_lo, k_hi, pairs, n_pairs, stream=None,
                          ws_pairs: int = 0):
        """ws_pairs: room for the filter's candidate list in the workspace (default: the pair buffer's size; a
        candidate list that does not fit latches ECAPACITY in the workspace)."""
        nb = self.L.photon_match_workspace_bytes(K, 1, max(int(ws_pairs), pairs.numel()))
        ws = self.workspace("scan", nb)
        self._rc(self.L.photon_match_scan(self.ctx, K, kto.data_ptr(), sig.data_ptr() if sig.numel() else None,
                                          mass.data_ptr(), warps_total.data_ptr(), params, k_lo, k_hi, ws.data_ptr(),
                                          ws.numel(), pairs.data_ptr(), pairs.numel(), n_pairs.data_ptr(),
                                          self.stream_ptr(stream)))
        return ws

    def photon_match_resolve(self, K, kto, sig, mass, warps_total, params, pairs, n_pairs: int, match, match_dist,
                             stream=None):
        nb = self.L.photon_match_workspace_bytes(K, 1, max(n_pairs, 1))
        ws = self.workspace("resolve", nb)
        self._rc(self.L.photon_match_resolve(self.ctx, K, kto.data_ptr(), sig.data_ptr() if sig.numel() else None,
                                             mass.data_ptr(), warps_total.data_ptr(), params,
                                             pairs.data_ptr() if n_pairs else None, n_pairs, ws.data_ptr(),
                                             ws.numel(), match.data_ptr(),
                                             None if match_dist is None else match_dist.data_ptr(),
                                             self.stream_ptr(stream)))
        return ws

    # -- A5 ----------------------------------------------------------------------------------------------------
    def photon_bb_stable(self, tm: DeviceTiming, kernel_bb_insts, n: int = 2048, delta=(3, 100), rate=(95, 100),
                         want_dur: bool = True, stream=None, check: bool = True, out: Optional[dict] = None) -> dict:
        ct = tm.c()
        nb = self.L.photon_stable_workspace_bytes(ctypes.byref(ct))
        ws = self.workspace("stable", nb)
        o = out if out is not None else {}
        o.setdefault("first_stable", self.empty(tm.n_kernels * tm.n_bb, "int64"))
        if want_dur:
            o.setdefault("stable_dur_sum", self.empty(tm.n_kernels * tm.n_bb, "int64"))
        o.setdefault("switch_at", self.empty(tm.n_kernels, "int64"))
        prm = _lib.StableParams(int(n), int(delta[0]), int(delta[1]), int(rate[0]), int(rate[1]))
        self._rc(self.L.photon_bb_stable(self.ctx, ctypes.byref(ct), kernel_bb_insts.data_ptr(), prm, ws.data_ptr(),
                                         ws.numel(), o["first_stable"].data_ptr(),
                                         o["stable_dur_sum"].data_ptr() if want_dur else None,
                                         o["switch_at"].data_ptr(), self.stream_ptr(stream)))
        o["_ws"] = ws
        if check:
            self.check(ws, stream)
        return o

    # -- N1: warp-level stability (L249, L262, Fig 10) --------------------------------------------------------
    def photon_warp_stable(self, tm: DeviceTiming, warp_sampling_ok=None, n: int = 1024, delta=(3, 100),
                           want_dur: bool = True, stream=None, check: bool = True, out: Optional[dict] = None) -> dict:
        """switch_at [K] (first stable warp retirement per kernel, -1 = none) and dur_sum [K] (S_n there)."""
        ct = tm.c()
        ws = self.workspace("warp_stable", self.L.photon_warp_stable_workspace_bytes(ctypes.byref(ct)))
        o = out if out is not None else {}
        o.setdefault("switch_at", self.empty(tm.n_kernels, "int64"))
        if want_dur:
            o.setdefault("dur_sum", self.empty(tm.n_kernels, "int64"))
        prm = _lib.WarpStableParams(int(n), int(delta[0]), int(delta[1]))
        ok = None if warp_sampling_ok is None else warp_sampling_ok.data_ptr()
        self._rc(self.L.photon_warp_stable(self.ctx, ctypes.byref(ct), ok, prm, ws.data_ptr(), ws.numel(),
                                           o["switch_at"].data_ptr(), o["dur_sum"].data_ptr() if want_dur else None,
                                           self.stream_ptr(stream)))
        o["_ws"] = ws
        if check:
            self.check(ws, stream)
        return o

    # -- N3: kernel- and BB-level prediction (Fig 12 Step 4 / L279-281; Fig 7 Step 3) -------------------------
    def photon_kernel_predict(self, match, mass, full_insts, full_cycles, stream=None, check: bool = True) -> dict:
        """pred_insts / pred_cycles [K] of every kernel from its representative (round half up)."""
        K = int(match.numel())
        ws = self.workspace("kpredict", 256)
        o = {"pred_insts": self.empty(K, "int64"), "pred_cycles": self.empty(K, "int64")}
        self._rc(self.L.photon_kernel_predict(self.ctx, K, match.data_ptr(), mass.data_ptr(), full_insts.data_ptr(),
                                              full_cycles.data_ptr(), ws.data_ptr(), ws.numel(),
                                              o["pred_insts"].data_ptr(), o["pred_cycles"].data_ptr(),
                                              self.stream_ptr(stream)))
        o["_ws"] = ws
        if check:
            self.check(ws, stream)
        return o

    def photon_bb_predict(self, t: DeviceTrace, first_stable, stable_dur_sum, stream=None, check: bool = True,
                          out: Optional[dict] = None) -> dict:
        """pred_dur_sum [W] (sum of the stable types' S_n over each warp's events) and unpredicted [W]; `out` (a
        previous result for the same trace) is reused."""
        ct = t.c()
        ws = self.workspace("bpredict", self.L.photon_bb_predict_workspace_bytes(ctypes.byref(ct)))
        o = out if out is not None else {}
        o.setdefault("pred_dur_sum", self.empty(t.n_warps, "int64"))
        o.setdefault("unpredicted", self.empty(t.n_warps, "int32"))
        self._rc(self.L.photon_bb_predict(self.ctx, ctypes.byref(ct), first_stable.data_ptr(),
                                          stable_dur_sum.data_ptr(), ws.data_ptr(), ws.numel(),
                                          o["pred_dur_sum"].data_ptr(), o["unpredicted"].data_ptr(),
                                          self.stream_ptr(stream)))
        o["_ws"] = ws
        if check:
            self.check(ws, stream)
        return o

    # -- multi-GPU helpers -------------------------------------------------------------------------------------
    def photon_types_export(self, K_local, ty, kernel_base, warp_base, rows, n_rows=None, stream=None):
        """rows: [row_capacity, 88] uint8 (padded with PHOTON_ROW_PAD rows); n_rows: device int64 [1] or None."""
        tc = self.types_c(ty)
        self._rc(self.L.photon_types_export(self.ctx, K_local, ctypes.byref(tc), kernel_base, warp_base,
                                            rows.data_ptr(), int(rows.shape[0]),
                                            None if n_rows is None else n_rows.data_ptr(), self.stream_ptr(stream)))

    def photon_types_merge(self, rows, n_rows, K, kernel_warps, out: dict, stream=None):
        nb = self.L.photon_merge_workspace_bytes(n_rows, K)
        ws = self.workspace("merge", nb)
        tc = self.types_c(out)
        self._rc(self.L.photon_types_merge(self.ctx, rows.data_ptr() if n_rows else None, n_rows, K,
                                           kernel_warps.data_ptr(), ws.data_ptr(), ws.numel(), ctypes.byref(tc),
                                           self.stream_ptr(stream)))
        return ws

    def photon_types_remap(self, K_local, W_local, kwo_local, ty_local, kernel_base, n_rows, K, merge_ws,
                           warp_type_global, stream=None):
        tc = self.types_c(ty_local)
        self._rc(self.L.photon_types_remap(self.ctx, K_local, W_local, kwo_local.data_ptr(), ctypes.byref(tc),
                                           kernel_base, n_rows, K, merge_ws.data_ptr(), merge_ws.numel(),
                                           warp_type_global.data_ptr() if W_local else None,
                                           self.stream_ptr(stream)))

    # -- CUDA graphs ------------------------------------------------------------------------------------------
    def capture(self, fn):
        """Capture fn() -- a sync-free sequence of libphoton calls on the current stream (check=False, buffers
        reused through `out=`) -- in one CUDA graph.  fn runs once eagerly on the capture stream first (so every
        cached workspace already has its final size and nothing is allocated inside the graph).  Returns
        (graph, the captured call's result); graph.replay() re-runs the whole sequence with one launch."""
        torch = self.torch
        s = torch.cuda.Stream(device=self.device)
        s.wait_stream(torch.cuda.current_stream(self.device))
        with torch.cuda.stream(s):
            fn()
        torch.cuda.current_stream(self.device).wait_stream(s)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            res = fn()
        return g, res

    # -- the benchmarked chain ---------------------------------------------------------------------------------
    def analyse(self, t: DeviceTrace, theta=(1, 20), n_cores=64, pool_all_prior=0, want_dist=False, stream=None,
                check: bool = True, capacity_hint: int = 0, pair_capacity: int = 0, out: Optional[dict] = None) -> dict:
        """A1 -> A2 -> A3 -> A4 on one device in one call (photon_analyse: fused BBV + grouping pass, canonical
        tables, signatures, match; the library overlaps the independent parts on its own streams).  With
        check=False nothing synchronises (errors stay latched in the returned workspaces).  `out` (a previous result
        for the same trace) is reused instead of allocating new output tables."""
        K, W = t.n_kernels, t.n_warps
        key = (K, W)
        hint = max(capacity_hint, self._hint.get(key, 0))
        pcap = max(pair_capacity or (16 * K + 65536), self._pcap.get(K, 0))
        prm = self.match_params(theta, n_cores, pool_all_prior)
        ok = lambda k: out is not None and out.get(k) is not None and out[k].numel() == K
        for _ in range(12):
            ct = t.c()
            gws = self.workspace("group", self.L.photon_group_workspace_bytes(ctypes.byref(ct), hint))
            cap = min(max(W, 1), ht_capacity(hint, W))
            ty = out if self._types_fit(out, K, W, cap) else self.alloc_types(K, W, cap)
            mws = self.workspace("match", self.L.photon_match_workspace_bytes(K, ty["capacity"], pcap))
            match = out["match"] if ok("match") else self.empty(K, "int64")
            dist = None
            if want_dist:
                dist = out["match_dist"] if ok("match_dist") else self.empty(K, "float64")
            tc = self.types_c(ty)
            self._rc(self.L.photon_analyse(self.ctx, ctypes.byref(ct), gws.data_ptr(), gws.numel(), ctypes.byref(tc),
                                           t.warps_total.data_ptr(), prm, mws.data_ptr(), mws.numel(),
                                           match.data_ptr(), None if dist is None else dist.data_ptr(),
                                           self.stream_ptr(stream)))
            ty.update(match=match, match_dist=dist, _ws=gws, _mws=mws)
            if not check:
                return ty
            rc, bad = self.ws_status(gws, stream)
            if rc == _lib.ECAPACITY:  # the type table filled: a larger one
                hint = max(2 * ht_capacity(hint, W), 1 << 12)
                out = None
                continue
            if rc != 0:
                raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)
            rc, bad = self.ws_status(mws, stream)
            if rc == _lib.ECAPACITY:  # the pair list filled: a larger one
                pcap *= 4
                continue
            if rc != 0:
                raise PhotonError(rc, self.L.photon_last_error(self.ctx).decode(), bad)
            self._hint[key] = hint
            self._pcap[K] = pcap
            return ty
        raise PhotonError(_lib.ECAPACITY, "type table or pair list kept overflowing")
