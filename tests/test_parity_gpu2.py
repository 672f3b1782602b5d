"""GPU parity, round 2: the cases VERDICT r1 listed as untested, element by element against the CPU oracle.

- A5 (photon_bb_stable, PAPER.md L229 / Eq. 1 L222-225 / L208) on C2, on all of C5 in kernel batches (the B > 256
  radix path at full scale), and on constructed streams for the method's degenerate cases: S_2n = 0 [P-17],
  den = 0 [P-16], a switch weight of exactly 95% and just above [P-14][P-15], a kernel of zero total weight.
- K1 (photon_bbv_build / photon_warp_group, L154 / L161 / L178) on warps far longer than one staging chunk, mixed
  with tiny and empty warps, fused and unfused, for B <= 4096 and B > 4096, with BB lengths up to the 2^17 bound.
- A3 (photon_sig_build = photon_gpu_bbv, L178, Fig 5): sig and mass against oracle.signature, and N3's kernel
  prediction (L279-281) fed by the GPU's own mass.
- Reuse of a previous result's tables (out=) equals a fresh call, and a mismatched result is not reused.
"""
import numpy as np
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ph():
    from paper_conf_micro_liusc23_b200 import Photon
    return Photon(0)


def _dev(ph, tr):
    from paper_conf_micro_liusc23_b200 import DeviceTrace
    return DeviceTrace.from_host(tr, ph.device)


def _np(t, dt):
    from paper_conf_micro_liusc23_b200 import to_numpy
    return to_numpy(t, dt)


def _check_types(ty, ref):
    T = int(ref["kernel_type_off"][-1])
    assert np.array_equal(_np(ty["kernel_type_off"], np.uint64), ref["kernel_type_off"])
    assert np.array_equal(_np(ty["warp_type"], np.uint32), ref["warp_type"])
    assert np.array_equal(_np(ty["type_key"], np.uint32).reshape(-1, 16)[:T], ref["type_key"])
    assert np.array_equal(_np(ty["type_count"], np.uint64)[:T], ref["type_count"])
    assert np.array_equal(_np(ty["type_first_warp"], np.uint64)[:T], ref["type_first_warp"])
    assert np.array_equal(_np(ty["warp_sampling_ok"], np.uint8), ref["warp_sampling_ok"])


# ---- A5 ----------------------------------------------------------------------------------------------------------
def _check_stable(ph, tm, kbb, n=2048, delta=(3, 100), rate=(95, 100)):
    from paper_conf_micro_liusc23_b200 import DeviceTiming, to_device
    o = ph.photon_bb_stable(DeviceTiming.from_host(tm, ph.device),
                            to_device(np.ascontiguousarray(kbb, np.uint64), ph.device), n, delta, rate)
    fs, ds, sw = oracle.stable(tm, kbb, n, delta, rate)
    K, B = tm.n_kernels, int(tm.n_bb)
    gfs = _np(o["first_stable"], np.int64).reshape(K, B)
    assert np.array_equal(gfs, fs)
    assert np.array_equal(_np(o["stable_dur_sum"], np.uint64).reshape(K, B), ds)
    assert np.array_equal(_np(o["switch_at"], np.int64), sw)
    return fs, ds, sw


def test_stable_c2(ph):
    g = tg.Generator(2)
    _, _, kbb = oracle.bbv(g.trace())
    fs, _, sw = _check_stable(ph, g.timing(), kbb)
    assert (fs >= 0).sum() > 20 and (sw >= 0).sum() > 10


@pytest.mark.slow
def test_stable_c5_all_kernels_in_batches(ph):
    # every C5 kernel (10^9 records in all), 1000 kernels (~10^8 records) per call; B = 4096 > 256 takes the
    # composite-key radix path
    g = tg.Generator(5)
    n_stable = n_switch = 0
    for k0 in range(0, g.n_kernels, 1000):
        k1 = min(k0 + 1000, g.n_kernels)
        _, _, kbb = oracle.bbv(g.kernels_trace(k0, k1))
        fs, _, sw = _check_stable(ph, g.timing(k0, k1), kbb)
        n_stable += int((fs >= 0).sum())
        n_switch += int((sw >= 0).sum())
    assert n_stable > 10000 and n_switch > 100


def _one_kernel_streams(streams, n_bb):
    """streams: per kernel, a list of (bb, issue, retire) records already in retirement order."""
    offs = np.cumsum([0] + [len(s) for s in streams]).astype(np.uint64)
    cat = lambda i, dt: np.array([r[i] for s in streams for r in s], dt)
    return tg.Timing(kernel_rec_off=offs, bb=cat(0, np.uint16), issue=cat(1, np.uint64), retire=cat(2, np.uint64),
                     n_bb=n_bb)


def test_stable_degenerate_cases(ph):
    # the oracle pins of test_oracle_pins.test_detector_constructed_streams, run on the GPU together, n = 2048
    n = 2048
    xs = [100 * i for i in range(3 * n)]
    line = [(0, x, x + 423) for x in xs]                       # L227 MM line scaled: stable at its 2n-th execution
    mix = line + [(1, xs[-1] + 50, xs[-1] + 473)]              # + a rare BB executed once (L210)
    zero = [(0, i, i) for i in range(2 * n + 5)]               # S_2n = 0 [P-17]
    flat = sorted([(0, 1000, 1000 + 5 + (i % 3)) for i in range(2 * n)], key=lambda r: r[2])  # den = 0 [P-16]
    tm = _one_kernel_streams([line, mix, mix, mix, zero, flat, mix], 2)
    kbb = np.array([[7, 0], [994, 6], [950, 50], [951, 49], [1, 0], [1, 0], [0, 0]], np.uint64)
    fs, ds, sw = _check_stable(ph, tm, kbb, n)
    p = 2 * n - 1
    assert fs[:, 0].tolist() == [p, p, p, p, -1, -1, p] and (fs[:, 1] == -1).all()
    assert int(ds[0, 0]) == 423 * n
    # switch: 99.4% -> yes; exactly 95% -> no (strict, L208 "larger than"); 95.1% -> yes; zero total weight -> no
    assert sw.tolist() == [p, p, -1, p, -1, -1, -1]
    # the rate parameter path (rate_num/rate_den other than 95/100)
    _check_stable(ph, tm, kbb, n, rate=(950, 1000))
    _check_stable(ph, tm, kbb, n, rate=(951, 1000))


@pytest.mark.parametrize("n", [16, 2048])
def test_stable_wide_time_ranges(ph, n):
    # k_window's fast path stages run spans as 32-bit times shifted by the run's first retire time and needs every
    # shifted time within 2^((61 - ceil(log2 n)) / 2); these streams force the general path (huge issue gaps, huge
    # durations: issue far before the first retire) and switch between the two paths inside one group
    rng = np.random.default_rng(n)
    streams = []
    for kind in range(4):
        m = 3 * n + 9000 if kind != 3 else 6 * n + 20000
        if kind == 0:    # gaps up to 2^25: every run spans more than the range
            gaps = rng.integers(1, 1 << 25, m)
            dur = np.full(m, 1000) + (rng.random(m) < 0.2) * rng.integers(0, 50, m)
        elif kind == 1:  # durations ~2^33: shifted issue times far below the range
            gaps = rng.integers(1, 64, m)
            dur = (1 << 33) + rng.integers(0, 1000, m)
        elif kind == 2:  # noisy, never stable, wide
            gaps = rng.integers(1, 1 << 24, m)
            dur = rng.integers(1, 1 << 30, m)
        else:            # narrow for a while, then wide gaps, then narrow again (both paths in one group)
            gaps = np.where((np.arange(m) > 2 * n + 3000) & (np.arange(m) < 3 * n + 9000),
                            rng.integers(1, 1 << 26, m), rng.integers(1, 40, m))
            i = np.arange(m)
            dur = np.where(i < 3 * n + 9000, 50 + 3 * i, 500)  # drifting mean: stable only after the wide part
        x = np.cumsum(gaps).astype(np.uint64) + np.uint64(5)
        y = x + dur.astype(np.uint64)
        assert int(y.max()) < (1 << 40)
        bb = (rng.random(m) < 0.1).astype(np.uint16)  # two BBs per kernel
        o = np.argsort(y, kind="stable")
        streams.append(list(zip(bb[o].tolist(), x[o].tolist(), y[o].tolist())))
    tm = _one_kernel_streams(streams, 2)
    kbb = np.array([[9, 1], [5, 5], [1, 1], [3, 1]], np.uint64)
    fs, _, _ = _check_stable(ph, tm, kbb, n)
    assert (fs >= 0).sum() >= 2


# ---- K1 on long warps ---------------------------------------------------------------------------------------------
def _trace_from_lengths(seed, kernels, n_bb, max_len, dup_every=3):
    """kernels: per kernel a list of warp lengths.  Every `dup_every`-th warp repeats the previous warp of the same
    length (so long warps also form multi-member types); events drawn from a per-kernel 16-BB program."""
    rs = np.random.default_rng(seed)
    bb_len = rs.integers(1, max_len + 1, n_bb, dtype=np.uint64).astype(np.uint32)
    seqs, kwo = [], [0]
    for k, lens in enumerate(kernels):
        prog = rs.choice(n_bb, size=min(16, n_bb), replace=False).astype(np.uint16)
        last = {}
        for i, L in enumerate(lens):
            if i % dup_every == dup_every - 1 and L in last:
                s = last[L]
            else:
                s = prog[rs.integers(0, len(prog), L)] if L else np.zeros(0, np.uint16)
                if L and rs.random() < 0.3:  # a stray id from anywhere in [0, B)
                    s = s.copy()
                    s[rs.integers(0, L)] = rs.integers(0, n_bb)
            last[L] = s
            seqs.append(s)
        kwo.append(kwo[-1] + len(lens))
    offs = np.zeros(len(seqs) + 1, np.uint64)
    offs[1:] = np.cumsum([len(s) for s in seqs])
    return tg.Trace(kernel_warp_off=np.array(kwo, np.uint64), warp_event_off=offs,
                    bb=np.concatenate(seqs).astype(np.uint16) if seqs else np.zeros(0, np.uint16), bb_len=bb_len,
                    bb_bin=None, warps_total=np.array([len(x) for x in kernels], np.uint64), name="long")


def _long_kernels(rs):
    big = [45000, 100000, 18431, 18432, 18433, 36864, 20000, 40000, 40000, 40000, 73000]
    k0 = []
    for L in big:  # each long warp between tiny and empty ones
        k0 += [0, 1, 3, L, 0, 2]
    k1 = [5] * 300 + [70000, 70000, 70000] + list(rs.integers(0, 40, 500))
    k2 = list(rs.integers(0, 9, 700)) + [55555] + [0] * 50
    k3 = [40000, 40000, 41000]
    return [k0, k1, k2, [], k3]


@pytest.mark.parametrize("n_bb,max_len", [(300, 64), (4096, 64), (4096, (1 << 17) - 1), (5000, 64), (70, 40000)])
def test_k1_long_warps(ph, n_bb, max_len):
    rs = np.random.default_rng(n_bb + max_len)
    kernels = _long_kernels(rs)
    if max_len >= 1 << 16:  # keep every warp's instruction total below 2^32 (the documented bound)
        kernels = [[min(L, 30000) for L in ks] for ks in kernels]
    tr = _trace_from_lengths(n_bb, kernels, n_bb, max_len)
    d = _dev(ph, tr)
    o = ph.photon_bbv_build(d, bbv16=True, insts=True, kbb=True)
    p16, ins, kb = oracle.bbv(tr, want_kbb=True)
    assert np.array_equal(_np(o["warp_bbv16"], np.uint32).reshape(-1, 16), p16)
    assert np.array_equal(_np(o["warp_insts"], np.uint64), ins)
    assert np.array_equal(_np(o["kernel_bb_insts"], np.uint64).reshape(tr.n_kernels, tr.n_bb), kb)
    ref = oracle.group(tr, p16)
    assert (ref["type_count"] > 1).any()
    _check_types(ph.photon_warp_group(d), ref)                               # fused
    _check_types(ph.photon_warp_group(d, warp_bbv16=o["warp_bbv16"]), ref)   # unfused


@pytest.mark.parametrize("n_bb", [300, 5000])
def test_k1_long_warps_unfused_grouping(ph, n_bb):
    # the same kind of traces through the unfused grouping (materialised BBVs -> k_group3_from_bbv); B = 5000 >
    # 4096 reads the BB table through L1 instead of shared memory
    rs = np.random.default_rng(n_bb)
    tr = _trace_from_lengths(n_bb + 1, _long_kernels(rs), n_bb, 64)
    d = _dev(ph, tr)
    p16, ins, _ = oracle.bbv(tr, want_kbb=False)
    o = ph.photon_bbv_build(d, bbv16=True, insts=True)
    assert np.array_equal(_np(o["warp_bbv16"], np.uint32).reshape(-1, 16), p16)
    assert np.array_equal(_np(o["warp_insts"], np.uint64), ins)
    _check_types(ph.photon_warp_group(d, o["warp_bbv16"]), oracle.group(tr, p16))


# ---- A3 ------------------------------------------------------------------------------------------------------------
def _check_sig(ph, tr):
    d = _dev(ph, tr)
    ty = ph.photon_warp_group(d)
    ref = oracle.analyse(tr)
    _check_types(ty, ref)
    g = ph.photon_gpu_bbv(tr.n_kernels, ty)
    sig, mass = oracle.signature(ref["kernel_type_off"], ref["type_key"], ref["type_count"])
    T = int(ref["kernel_type_off"][-1])
    assert np.array_equal(_np(g["sig"], np.uint64)[:16 * T], sig)
    assert np.array_equal(_np(g["mass"], np.uint64), mass)
    return d, ty, g, ref


def test_sig_c4_and_prediction_from_gpu_mass(ph):
    from paper_conf_micro_liusc23_b200 import to_device
    tr = tg.make_trace(4)
    d, ty, g, ref = _check_sig(ph, tr)
    m = ph.photon_kernel_match(tr.n_kernels, ty, d.warps_total)
    assert np.array_equal(_np(m["match"], np.int64), ref["match"])
    rs = np.random.default_rng(44)
    K = tr.n_kernels
    fi = rs.integers(1, 1 << 40, K).astype(np.uint64)
    fc = rs.integers(1, 1 << 40, K).astype(np.uint64)
    o = ph.photon_kernel_predict(m["match"], g["mass"], to_device(fi, ph.device), to_device(fc, ph.device))
    pi, pc = oracle.kernel_predict(ref["match"], ref["mass"], fi, fc)
    assert np.array_equal(_np(o["pred_insts"], np.uint64), pi)
    assert np.array_equal(_np(o["pred_cycles"], np.uint64), pc)


def test_sig_c6_and_random(ph):
    _check_sig(ph, tg.make_trace(6))
    _check_sig(ph, tg.random_trace(5, n_kernels=6, max_warps=500, max_events=80, n_bb=40))


@pytest.mark.slow
def test_sig_c5(ph):
    _check_sig(ph, tg.make_trace(5))


# ---- out= reuse ------------------------------------------------------------------------------------------------
def _same(a, b, keys):
    import torch
    for k in keys:
        assert torch.equal(a[k], b[k]), k


def test_out_reuse_analyse_and_full(ph):
    keys = ("warp_type", "kernel_type_off", "warp_sampling_ok", "match")
    tr6, tr1 = tg.make_trace(6), tg.make_trace(1)
    d6, d1 = _dev(ph, tr6), _dev(ph, tr1)
    fresh6 = ph.analyse(d6)
    again6 = ph.analyse(d6, out=fresh6)
    for k in keys:
        assert again6[k] is fresh6[k]  # reused in place
    ref6 = oracle.analyse(tr6)
    _check_types(again6, ref6)
    assert np.array_equal(_np(again6["match"], np.int64), ref6["match"])
    # a result of another trace (different W and K) must not be written into
    r1 = ph.analyse(d1, out=fresh6)
    assert r1["warp_type"] is not fresh6["warp_type"] and r1["match"] is not fresh6["match"]
    _check_types(r1, oracle.analyse(tr1))
    # N2 binding
    f6 = ph.photon_warp_group_full(d6)
    g6 = ph.photon_warp_group_full(d6, out=f6)
    assert g6["warp_type"] is f6["warp_type"]
    p16, _, _ = oracle.bbv(tr6, want_kbb=False)
    rf = oracle.group_full(tr6, p16)
    assert np.array_equal(_np(g6["warp_type"], np.uint32), rf["warp_type"])
    h1 = ph.photon_warp_group_full(d1, out=f6)
    assert h1["warp_type"] is not f6["warp_type"]
    p16, _, _ = oracle.bbv(tr1, want_kbb=False)
    assert np.array_equal(_np(h1["warp_type"], np.uint32), oracle.group_full(tr1, p16)["warp_type"])


@pytest.mark.parametrize("cfg", [6, 1])
def test_chain_cuda_graph_replay_matches_oracle(ph, cfg):
    # bench.py times the chain as one CUDA graph replay per step: the replayed result must equal the oracle
    import torch
    from paper_conf_micro_liusc23_b200 import DeviceTrace
    g = tg.Generator(cfg)
    tr = g.trace()
    d = DeviceTrace.from_host(tr, ph.device)
    r0 = ph.analyse(d, check=True)
    graph, r = ph.capture(lambda: ph.analyse(d, check=False, out=r0))
    for k in ("warp_type", "match"):
        r[k].fill_(-7)  # the replay must rewrite every output
    graph.replay()
    graph.replay()
    torch.cuda.synchronize()
    ph.check(r["_ws"])
    ph.check(r["_mws"])
    ref = oracle.analyse(tr)
    T = int(ref["kernel_type_off"][-1])
    assert np.array_equal(_np(r["kernel_type_off"], np.uint64), ref["kernel_type_off"])
    assert np.array_equal(_np(r["type_key"], np.uint32).reshape(-1, 16)[:T], ref["type_key"])
    assert np.array_equal(_np(r["type_count"], np.uint64)[:T], ref["type_count"])
    assert np.array_equal(_np(r["warp_type"], np.uint32), ref["warp_type"])
    assert np.array_equal(_np(r["warp_sampling_ok"], np.uint8), ref["warp_sampling_ok"])
    assert np.array_equal(_np(r["match"], np.int64), ref["match"])


def test_group_full_table_hint_overflow_retry(ph):
    # N2 sizes its hash table from the types a checked call found before on a trace of the same shape; a later
    # trace of that shape with many more types overflows the small table (ECAPACITY) and the checked call retries
    # with the full-size table -- both results equal the oracle
    rs = np.random.default_rng(3)
    few = [[[1, 2, 3] * 6 for _ in range(600)], [[4, 5] * 9 for _ in range(600)]]
    many = [[list(rs.integers(0, 40, 18)) for _ in range(600)], [list(rs.integers(0, 40, 18)) for _ in range(600)]]
    for kernels in (few, many):
        tr = tg.trace_from_warps(kernels, bb_len=rs.integers(1, 9, 40).tolist())
        d = _dev(ph, tr)
        p16, _, _ = oracle.bbv(tr, want_kbb=False)
        ref = oracle.group_full(tr, p16)
        ty = ph.photon_warp_group_full(d)
        T = int(ref["kernel_type_off"][-1])
        assert np.array_equal(_np(ty["kernel_type_off"], np.uint64), ref["kernel_type_off"])
        assert np.array_equal(_np(ty["warp_type"], np.uint32), ref["warp_type"])
        assert np.array_equal(_np(ty["type_count"], np.uint64)[:T], ref["type_count"])
