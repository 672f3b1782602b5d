"""CPU oracle for the Photon online-analysis hot path — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py (cpu_baseline leg, --impl reference) may import this package.
The product path (paper_conf_micro_liusc23_b200) never imports it and shares no code with it.

The arithmetic lives in photon_oracle.cpp (plain single-threaded C++17, each function citing PAPER.md); this
module only marshals numpy arrays.  Pins: tests/test_oracle_pins.py.  Parity unpinned by the paper (no paper
number exists for them): theta [P-7] and the readings [P-2], [P-5], [P-6], [P-8] — DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "photon_oracle.cpp")

OK, EINVAL, ERANGE, ECAPACITY = 0, -1, -3, -4


class OracleError(RuntimeError):
    def __init__(self, code: int, index: int):
        super().__init__(f"oracle error {code} at index {index}")
        self.code = code
        self.index = index


def build(force: bool = False) -> str:
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-o", _SO, _SRC])
    return _SO


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        vp, u32, u64, i32 = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
        L.or_bbv.restype = i32
        L.or_bbv.argtypes = [u32, u32, u64, u64, vp, vp, vp, vp, vp, vp, vp, vp, vp]
        L.or_group.restype = i32
        L.or_group.argtypes = [u32, u64, vp, vp, u64, vp, vp, vp, vp, vp, vp]
        L.or_signature.restype = i32
        L.or_signature.argtypes = [u32, vp, vp, vp, vp, vp, vp]
        L.or_match.restype = i32
        L.or_match.argtypes = [u32, vp, vp, vp, vp, u32, u32, u64, u32, vp, vp]
        L.or_stable.restype = i32
        L.or_stable.argtypes = [u32, u32, u64, vp, vp, vp, vp, vp, u32, u32, u32, u32, u32, i32, vp, vp, vp, vp]
        L.or_warp_stable.restype = i32
        L.or_warp_stable.argtypes = [u32, u64, vp, vp, vp, vp, u32, u32, u32, i32, vp, vp, vp]
        L.or_kernel_predict.restype = i32
        L.or_kernel_predict.argtypes = [u32, vp, vp, vp, vp, vp, vp, vp]
        L.or_bb_predict.restype = i32
        L.or_bb_predict.argtypes = [u32, u32, u64, u64, vp, vp, vp, vp, vp, vp, vp, vp]
        _lib = L
    return _lib


def _p(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def bbv(trace, want_kbb: bool = True):
    """A1: (warp_bbv16 [W,16] u32, warp_insts [W] u64, kernel_bb_insts [K,B] u64 or None)."""
    K, B, W, E = trace.n_kernels, trace.n_bb, trace.n_warps, trace.n_events
    p16 = np.zeros((W, 16), np.uint32)
    ins = np.zeros(W, np.uint64)
    kbb = np.zeros((K, B), np.uint64) if want_kbb else None
    bad = ctypes.c_int64(-1)
    bbin = None if trace.bb_bin is None else _c(trace.bb_bin, np.uint8)
    kwo, weo = _c(trace.kernel_warp_off, np.uint64), _c(trace.warp_event_off, np.uint64)
    bbs, bl = _c(trace.bb, np.uint16), _c(trace.bb_len, np.uint32)
    rc = _L().or_bbv(K, B, W, E, _p(kwo), _p(weo), _p(bbs), _p(bl), _p(bbin), _p(p16), _p(ins), _p(kbb),
                     ctypes.byref(bad))
    if rc != OK:
        raise OracleError(rc, bad.value)
    return p16, ins, kbb


def group(trace, warp_bbv16: np.ndarray):
    """A2: canonical type tables (dict of numpy arrays, names as photon_types)."""
    K, W = trace.n_kernels, trace.n_warps
    cap = max(W, 1)
    out = dict(warp_type=np.zeros(W, np.uint32), kernel_type_off=np.zeros(K + 1, np.uint64),
               type_key=np.zeros((cap, 16), np.uint32), type_count=np.zeros(cap, np.uint64),
               type_first_warp=np.zeros(cap, np.uint64), warp_sampling_ok=np.zeros(K, np.uint8))
    kwo = _c(trace.kernel_warp_off, np.uint64)
    p16 = _c(warp_bbv16, np.uint32)
    rc = _L().or_group(K, W, _p(kwo), _p(p16), cap, _p(out["warp_type"]), _p(out["kernel_type_off"]),
                       _p(out["type_key"]), _p(out["type_count"]), _p(out["type_first_warp"]),
                       _p(out["warp_sampling_ok"]))
    if rc != OK:
        raise OracleError(rc, -1)
    T = int(out["kernel_type_off"][-1])
    for k in ("type_key", "type_count", "type_first_warp"):
        out[k] = out[k][:T].copy()
    return out


def signature(kernel_type_off, type_key, type_count):
    """A3: (sig [16T] u64, mass [K] u64)."""
    kto = _c(kernel_type_off, np.uint64)
    K = len(kto) - 1
    T = int(kto[-1])
    sig = np.zeros(max(16 * T, 1), np.uint64)
    mass = np.zeros(max(K, 1), np.uint64)
    bad = ctypes.c_int64(-1)
    tk, tc = _c(type_key, np.uint32), _c(type_count, np.uint64)  # converted copies must outlive the call
    rc = _L().or_signature(K, _p(kto), _p(tk), _p(tc), _p(sig), _p(mass), ctypes.byref(bad))
    if rc != OK:
        raise OracleError(rc, bad.value)
    return sig[:16 * T], mass[:K]


def match(kernel_type_off, sig, mass, warps_total, theta=(1, 20), n_cores=64, pool_all_prior=0):
    """A4: (match [K] i64, match_dist [K] f64)."""
    kto = _c(kernel_type_off, np.uint64)
    K = len(kto) - 1
    m = np.zeros(max(K, 1), np.int64)
    d = np.zeros(max(K, 1), np.float64)
    sg = _c(sig, np.uint64) if len(sig) else np.zeros(1, np.uint64)
    ms, wt = _c(mass, np.uint64), _c(warps_total, np.uint64)  # converted copies must outlive the call
    rc = _L().or_match(K, _p(kto), _p(sg), _p(ms), _p(wt), int(theta[0]), int(theta[1]), int(n_cores),
                       int(pool_all_prior), _p(m), _p(d))
    if rc != OK:
        raise OracleError(rc, -1)
    return m[:K], d[:K]


def stable(timing, kernel_bb_insts, n=2048, delta=(3, 100), rate=(95, 100), brute=False):
    """A5: (first_stable [K,B] i64, stable_dur_sum [K,B] u64, switch_at [K] i64)."""
    K, B, R = timing.n_kernels, int(timing.n_bb), timing.n_records
    fs = np.zeros((K, B), np.int64)
    ds = np.zeros((K, B), np.uint64)
    sw = np.zeros(max(K, 1), np.int64)
    bad = ctypes.c_int64(-1)
    kbb = _c(kernel_bb_insts, np.uint64)
    kro, bbs = _c(timing.kernel_rec_off, np.uint64), _c(timing.bb, np.uint16)  # copies must outlive the call
    iss, ret = _c(timing.issue, np.uint64), _c(timing.retire, np.uint64)
    rc = _L().or_stable(K, B, R, _p(kro), _p(bbs), _p(iss), _p(ret), _p(kbb), int(n),
                        int(delta[0]), int(delta[1]), int(rate[0]), int(rate[1]), 1 if brute else 0, _p(fs),
                        _p(ds), _p(sw), ctypes.byref(bad))
    if rc != OK:
        raise OracleError(rc, bad.value)
    return fs, ds, sw[:K]


def warp_stable(timing, ok=None, n=1024, delta=(3, 100), brute=False):
    """N1: (switch_at [K] i64, dur_sum [K] u64) of the warp-level stability test over the kernels' warp streams
    (records = warps in retirement order; timing.bb is ignored); ok [K] u8 gates kernels without a dominant type."""
    K, R = timing.n_kernels, timing.n_records
    sw = np.zeros(max(K, 1), np.int64)
    ds = np.zeros(max(K, 1), np.uint64)
    bad = ctypes.c_int64(-1)
    okc = None if ok is None else _c(ok, np.uint8)
    kro, iss = _c(timing.kernel_rec_off, np.uint64), _c(timing.issue, np.uint64)  # copies must outlive the call
    ret = _c(timing.retire, np.uint64)
    rc = _L().or_warp_stable(K, R, _p(kro), _p(iss), _p(ret), None if okc is None else _p(okc), int(n),
                             int(delta[0]), int(delta[1]), 1 if brute else 0, _p(sw), _p(ds), ctypes.byref(bad))
    if rc != OK:
        raise OracleError(rc, bad.value)
    return sw[:K], ds[:K]


def kernel_predict(match, mass, full_insts, full_cycles):
    """N3 kernel level: (pred_insts [K] u64, pred_cycles [K] u64) from each kernel's representative."""
    K = len(match)
    pi = np.zeros(max(K, 1), np.uint64)
    pc = np.zeros(max(K, 1), np.uint64)
    bad = ctypes.c_int64(-1)
    m, ms, fi, fc = (_c(match, np.int64), _c(mass, np.uint64), _c(full_insts, np.uint64),
                     _c(full_cycles, np.uint64))  # converted copies must outlive the call
    rc = _L().or_kernel_predict(K, _p(m), _p(ms), _p(fi), _p(fc), _p(pi), _p(pc), ctypes.byref(bad))
    if rc != OK:
        raise OracleError(rc, bad.value)
    return pi[:K], pc[:K]


def bb_predict(trace, first_stable, stable_dur_sum):
    """N3 BB level: (pred_dur_sum [W] u64, unpredicted [W] u32) of every warp of the trace."""
    W = trace.n_warps
    pd = np.zeros(max(W, 1), np.uint64)
    un = np.zeros(max(W, 1), np.uint32)
    bad = ctypes.c_int64(-1)
    a = [_c(trace.kernel_warp_off, np.uint64), _c(trace.warp_event_off, np.uint64), _c(trace.bb, np.uint16),
         _c(first_stable, np.int64), _c(stable_dur_sum, np.uint64)]  # converted copies must outlive the call
    rc = _L().or_bb_predict(trace.n_kernels, trace.n_bb, W, trace.n_events, *[_p(x) for x in a], _p(pd), _p(un),
                            ctypes.byref(bad))
    if rc != OK:
        raise OracleError(rc, bad.value)
    return pd[:W], un[:W]


def group_full(trace, warp_bbv16):
    """N2 (L154, L161, reading [N2-a]): warp types keyed on the full BBV (the count of every BB id); rows ordered
    by (count desc, projected key asc, lowest warp asc); type_key = the members' 16-bin projection.  Plain Python
    over each warp's events (small traces)."""
    K, W = trace.n_kernels, trace.n_warps
    kwo = np.asarray(trace.kernel_warp_off, np.int64)
    weo = np.asarray(trace.warp_event_off, np.int64)
    bb = np.asarray(trace.bb)
    p16 = np.asarray(warp_bbv16, np.uint32).reshape(-1, 16)
    warp_type = np.zeros(W, np.uint32)
    kto = np.zeros(K + 1, np.uint64)
    keys, cnts, firsts = [], [], []
    ok = np.zeros(K, np.uint8)
    for k in range(K):
        groups = {}  # full BBV -> [first warp, count, members]
        for w in range(int(kwo[k]), int(kwo[k + 1])):
            ids, c = np.unique(bb[weo[w]:weo[w + 1]], return_counts=True)
            fk = (tuple(int(x) for x in ids), tuple(int(x) for x in c))
            g = groups.setdefault(fk, [w, 0, []])
            g[1] += 1
            g[2].append(w)
        rows = sorted(groups.values(), key=lambda g: (-g[1], tuple(int(x) for x in p16[g[0]]), g[0]))
        for r, g in enumerate(rows):
            for w in g[2]:
                warp_type[w] = r
            keys.append(p16[g[0]])
            cnts.append(g[1])
            firsts.append(g[0])
        kto[k + 1] = kto[k] + len(rows)
        Wk = int(kwo[k + 1] - kwo[k])
        ok[k] = 1 if Wk > 0 and rows and 100 * rows[0][1] > 95 * Wk else 0
    return dict(warp_type=warp_type, kernel_type_off=kto,
                type_key=np.array(keys, np.uint32).reshape(-1, 16), type_count=np.array(cnts, np.uint64),
                type_first_warp=np.array(firsts, np.uint64), warp_sampling_ok=ok)


def ingest(warp, bb, n_warps):
    """N2 ingest: tagged (warp, bb) events in stream order -> (bb by warp, stream order kept; warp_event_off)."""
    warp = np.asarray(warp, np.int64)
    order = np.argsort(warp, kind="stable")
    off = np.zeros(n_warps + 1, np.uint64)
    off[1:] = np.cumsum(np.bincount(warp, minlength=n_warps)[:n_warps])
    return np.asarray(bb)[order], off


def pool_export(types, warps_total, match_):
    """N4 (L402, reading [N4-a]): the run's representative kernels (match < 0), in launch order: dict(n_pool,
    kernel_type_off, type_key, type_count, warps_total, kernel_id)."""
    kto = np.asarray(types["kernel_type_off"], np.uint64)
    reps = [k for k in range(len(kto) - 1) if int(match_[k]) < 0]
    off, keys, cnts = [0], [], []
    for k in reps:
        a, b = int(kto[k]), int(kto[k + 1])
        keys.append(np.asarray(types["type_key"], np.uint32).reshape(-1, 16)[a:b])
        cnts.append(np.asarray(types["type_count"], np.uint64)[a:b])
        off.append(off[-1] + (b - a))
    return dict(n_pool=len(reps), kernel_type_off=np.array(off, np.uint64),
                type_key=np.concatenate(keys) if keys else np.zeros((0, 16), np.uint32),
                type_count=np.concatenate(cnts) if cnts else np.zeros(0, np.uint64),
                warps_total=np.array([int(warps_total[k]) for k in reps], np.uint64),
                kernel_id=np.array(reps, np.uint32))


def match_pooled(pool, types, warps_total, theta=(1, 20), n_cores=64, pool_all_prior=0):
    """N4: A4 with the pool's kernels launched before the run's (reading [N4-a]); indices < n_pool are pooled."""
    kto = np.asarray(types["kernel_type_off"], np.uint64)
    K, T = len(kto) - 1, int(kto[-1])
    pk = np.asarray(pool["kernel_type_off"], np.uint64)
    Tp = int(pk[-1])
    comb_kto = np.concatenate([pk, Tp + kto[1:]])
    keys = np.concatenate([np.asarray(pool["type_key"], np.uint32).reshape(-1, 16)[:Tp],
                           np.asarray(types["type_key"], np.uint32).reshape(-1, 16)[:T]])
    cnts = np.concatenate([np.asarray(pool["type_count"], np.uint64)[:Tp],
                           np.asarray(types["type_count"], np.uint64)[:T]])
    sig, mass = signature(comb_kto, keys, cnts)
    wt = np.concatenate([np.asarray(pool["warps_total"], np.uint64), np.asarray(warps_total, np.uint64)[:K]])
    return match(comb_kto, sig, mass, wt, theta, n_cores, pool_all_prior)


def _kernel_slice(trace, k0, k1):
    """Kernels [k0, k1) of a trace as a trace of their own (offsets rebased; arrays are views)."""
    from types import SimpleNamespace
    kwo = np.asarray(trace.kernel_warp_off, np.uint64)
    weo = np.asarray(trace.warp_event_off, np.uint64)
    w0, w1 = int(kwo[k0]), int(kwo[k1])
    e0, e1 = int(weo[w0]), int(weo[w1])
    t = SimpleNamespace(kernel_warp_off=kwo[k0:k1 + 1] - kwo[k0], warp_event_off=weo[w0:w1 + 1] - weo[w0],
                        bb=np.asarray(trace.bb)[e0:e1], bb_len=trace.bb_len, bb_bin=trace.bb_bin,
                        warps_total=np.asarray(trace.warps_total)[k0:k1])
    t.n_kernels, t.n_warps, t.n_events, t.n_bb = k1 - k0, w1 - w0, e1 - e0, len(trace.bb_len)
    return t, w0


def analyse_threads(trace, threads, theta=(1, 20), n_cores=64, pool_all_prior=0):
    """analyse() with the per-kernel steps (A1 BBVs, A2 grouping, A3 signatures) of contiguous kernel ranges run on
    `threads` host threads (the C calls release the GIL), then the launch-order match (A4) on one thread.  The
    all-cores CPU baseline of bench.py; results are identical to analyse()."""
    from concurrent.futures import ThreadPoolExecutor
    K = trace.n_kernels
    weo = np.asarray(trace.warp_event_off, np.uint64)
    kwo = np.asarray(trace.kernel_warp_off, np.uint64)
    kev = weo[kwo.astype(np.int64)].astype(np.float64)  # first event of each kernel (and the end)
    cuts = sorted(set([0, K] + [int(np.searchsorted(kev, trace.n_events * i / threads)) for i in range(1, threads)]))
    cuts = [min(max(c, 0), K) for c in cuts]

    def part(i):
        sub, w0 = _kernel_slice(trace, cuts[i], cuts[i + 1])
        p16, _, _ = bbv(sub, want_kbb=False)
        t = group(sub, p16)
        sig, mass = signature(t["kernel_type_off"], t["type_key"], t["type_count"])
        return t, sig, mass, w0

    with ThreadPoolExecutor(max_workers=threads) as ex:
        parts = list(ex.map(part, range(len(cuts) - 1)))
    kto, keys, cnts, firsts, wtype, ok, sigs, masses = [np.zeros(1, np.uint64)], [], [], [], [], [], [], []
    for t, sig, mass, w0 in parts:
        kto.append(kto[-1][-1] + t["kernel_type_off"][1:])
        keys.append(t["type_key"]); cnts.append(t["type_count"]); firsts.append(t["type_first_warp"] + np.uint64(w0))
        wtype.append(t["warp_type"]); ok.append(t["warp_sampling_ok"]); sigs.append(sig); masses.append(mass)
    out = dict(kernel_type_off=np.concatenate(kto), type_key=np.concatenate(keys), type_count=np.concatenate(cnts),
               type_first_warp=np.concatenate(firsts), warp_type=np.concatenate(wtype),
               warp_sampling_ok=np.concatenate(ok))
    sig, mass = np.concatenate(sigs), np.concatenate(masses)
    m, d = match(out["kernel_type_off"], sig, mass, trace.warps_total, theta, n_cores, pool_all_prior)
    out.update(sig=sig, mass=mass, match=m, match_dist=d)
    return out


def analyse(trace, theta=(1, 20), n_cores=64, pool_all_prior=0):
    """The benchmarked chain A1 -> A2 -> A3 -> A4 on one trace; returns a dict of every output."""
    p16, ins, kbb = bbv(trace, want_kbb=False)
    t = group(trace, p16)
    sig, mass = signature(t["kernel_type_off"], t["type_key"], t["type_count"])
    m, d = match(t["kernel_type_off"], sig, mass, trace.warps_total, theta, n_cores, pool_all_prior)
    t.update(warp_bbv16=p16, warp_insts=ins, sig=sig, mass=mass, match=m, match_dist=d)
    return t
