"""GPU parity: libphoton (through its C ABI) vs the CPU oracle, element by element on the same seeded inputs.

Bar (BASELINE.json north_star): bit-exact BBVs, warp types, type tables, dominance, matches and stability /
switch decisions; reported fp64 distances within 1e-6 relative.
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


def check_bbv(ph, tr, kbb=True):
    d = _dev(ph, tr)
    o = ph.photon_bbv_build(d, bbv16=True, insts=True, kbb=kbb)
    p16, ins, kb = oracle.bbv(tr, want_kbb=kbb)
    assert np.array_equal(_np(o["warp_bbv16"], np.uint32).reshape(-1, 16), p16)
    assert np.array_equal(_np(o["warp_insts"], np.uint64), ins)
    if kbb:
        assert np.array_equal(_np(o["kernel_bb_insts"], np.uint64).reshape(tr.n_kernels, tr.n_bb), kb)
    return d, o, p16


def check_types(ph, tr, ty, ref):
    T = int(ref["kernel_type_off"][-1])
    assert np.array_equal(_np(ty["kernel_type_off"], np.uint64), ref["kernel_type_off"])
    assert np.array_equal(_np(ty["warp_type"], np.uint32), ref["warp_type"])
    assert np.array_equal(_np(ty["type_key"], np.uint32).reshape(-1, 16)[:T], ref["type_key"])
    assert np.array_equal(_np(ty["type_count"], np.uint64)[:T], ref["type_count"])
    assert np.array_equal(_np(ty["type_first_warp"], np.uint64)[:T], ref["type_first_warp"])
    assert np.array_equal(_np(ty["warp_sampling_ok"], np.uint8), ref["warp_sampling_ok"])


def check_match(ph, tr, ty, ref, theta=(1, 20), n_cores=64, pool=0):
    d = _dev(ph, tr)
    m = ph.photon_kernel_match(tr.n_kernels, ty, d.warps_total, theta, n_cores, pool, want_dist=True)
    sig, mass = oracle.signature(ref["kernel_type_off"], ref["type_key"], ref["type_count"])
    om, od = oracle.match(ref["kernel_type_off"], sig, mass, tr.warps_total, theta, n_cores, pool)
    gm = _np(m["match"], np.int64)
    gd = _np(m["match_dist"], np.float64)
    assert np.array_equal(gm, om)
    fin = np.isfinite(od)
    assert np.array_equal(np.isfinite(gd), fin)
    np.testing.assert_allclose(gd[fin], od[fin], rtol=1e-6, atol=0)


def full_chain(ph, tr, thetas=((1, 20),), pools=(0,), n_cores=64):
    d, o, p16 = check_bbv(ph, tr)
    ref = oracle.group(tr, p16)
    ty = ph.photon_warp_group(d)  # fused single pass
    check_types(ph, tr, ty, ref)
    ty2 = ph.photon_warp_group(d, warp_bbv16=o["warp_bbv16"])  # unfused
    check_types(ph, tr, ty2, ref)
    for th in thetas:
        for pool in pools:
            check_match(ph, tr, ty, ref, th, n_cores, pool)
    return ty, ref


def test_worked_example(ph):
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_example.json")))
    tr = tg.trace_from_warps(g["kernels"], g["bb_len"])
    full_chain(ph, tr, thetas=((1, 20), (1, 2), (4, 11), (2, 5)), n_cores=2)


@pytest.mark.parametrize("seed", range(10))
def test_random_small(ph, seed):
    custom = seed % 2 == 1
    n_bb = [7, 16, 40, 300, 5000, 9000, 65536, 33, 17, 4096][seed]
    tr = tg.random_trace(seed, n_kernels=1 + seed % 7, max_warps=600, max_events=90, n_bb=n_bb, custom_bins=custom)
    full_chain(ph, tr, thetas=((1, 20), (1, 5), (1, 2)), pools=(0, 1))


@pytest.mark.parametrize("cfg", [1, 6])
def test_k1_fused_and_unfused_grouping_match(ph, cfg):
    # the fused K1 (BBV + de-dup in one pass) and the unfused path (materialised BBVs -> k_group3_from_bbv) must
    # both give the oracle's types (C1: blocks of several chunks; C6: every template, tiny warps)
    tr = tg.make_trace(cfg)
    d, o, p16 = check_bbv(ph, tr)
    ref = oracle.group(tr, p16)
    check_types(ph, tr, ph.photon_warp_group(d), ref)
    check_types(ph, tr, ph.photon_warp_group(d, o["warp_bbv16"]), ref)


def test_empty_warps_kernels_and_ragged(ph):
    kernels = [[[], [], [0, 1]], [], [[2] * 1000 + [1] * 3], [[]], [[0, 1, 2, 3, 4, 5, 6]] * 300 + [[1]]]
    tr = tg.trace_from_warps(kernels, bb_len=[3, 1, 7, 2, 9, 4, 5], warps_total=[3, 64, 1, 1, 301])
    full_chain(ph, tr, thetas=((1, 20), (2, 1)), pools=(0, 1))


@pytest.mark.parametrize("cfg", [1, 6])
def test_config_small(ph, cfg):
    tr = tg.make_trace(cfg)
    full_chain(ph, tr, thetas=((1, 100), (1, 20), (1, 10), (1, 5)), pools=(0, 1))


def test_config_c6_sample_1pct(ph):
    # the paper's 1% sample (L208/L258): every 100th warp, warps_total = launched warps
    g = tg.Generator(6)
    tr = g.trace(0, g.n_warps, step=100)
    full_chain(ph, tr, thetas=((1, 20),), pools=(0, 1))


@pytest.mark.parametrize("cfg", [2, 3, 4])
def test_config_full(ph, cfg):
    tr = tg.make_trace(cfg)
    full_chain(ph, tr, thetas=((1, 100), (1, 20), (1, 10), (1, 5)), pools=(0, 1))


@pytest.mark.slow
def test_config_c5_full(ph):
    """C5 at full size (10^9 events): the oracle runs the whole chain too (~30 s)."""
    tr = tg.make_trace(5)
    d = _dev(ph, tr)
    ty = ph.photon_warp_group(d)
    ref = oracle.analyse(tr)
    check_types(ph, tr, ty, ref)
    m = ph.photon_kernel_match(tr.n_kernels, ty, d.warps_total, (1, 20), 64, 0)
    assert np.array_equal(_np(m["match"], np.int64), ref["match"])


# ---- error paths ------------------------------------------------------------------------------------------------
def test_errors(ph):
    from paper_conf_micro_liusc23_b200 import PhotonError
    tr = tg.trace_from_warps([[[0, 1, 2, 1], [1, 5, 0]]], bb_len=[1, 2, 3])  # bb 5 >= B at event 5
    with pytest.raises(PhotonError) as ei:
        ph.photon_bbv_build(_dev(ph, tr))
    assert ei.value.code == -3 and ei.value.index == 5
    with pytest.raises(PhotonError) as ei:
        ph.photon_warp_group(_dev(ph, tr))
    assert ei.value.code == -3
    tr = tg.trace_from_warps([[[0] * 3]], bb_len=[(1 << 16) + 5])
    tr.bb = np.array([0] * 70000, np.uint16)  # 70000 * (2^16+5) >= 2^32: per-warp instructions overflow
    tr.warp_event_off = np.array([0, 70000], np.uint64)
    with pytest.raises(PhotonError) as ei:
        ph.photon_bbv_build(_dev(ph, tr))
    assert ei.value.code == -3 and ei.value.index == 0
    tr = tg.trace_from_warps([[[0], [1]]], bb_len=[1, 2])
    tr.warp_event_off = np.array([0, 2, 2], np.uint64)  # [W] != E... E = 2 here; make it non-monotone instead
    tr.warp_event_off = np.array([0, 3, 2], np.uint64)
    with pytest.raises(PhotonError) as ei:
        ph.photon_bbv_build(_dev(ph, tr))
    assert ei.value.code == -3
    tr = tg.trace_from_warps([[[0]]], bb_len=[0])  # length 0 is invalid
    with pytest.raises(PhotonError) as ei:
        ph.photon_bbv_build(_dev(ph, tr))
    assert ei.value.code == -1


def test_capacity_retry(ph):
    # every warp its own type: a hint of 1 forces ECAPACITY, the binding retries with a larger table
    rs = np.random.default_rng(3)
    kernels = [[list(rs.integers(0, 16, 20)) for _ in range(5000)]]
    tr = tg.trace_from_warps(kernels, bb_len=list(range(1, 17)))
    d = _dev(ph, tr)
    ty = ph.photon_warp_group(d, capacity_hint=1)
    p16, _, _ = oracle.bbv(tr, want_kbb=False)
    check_types(ph, tr, ty, oracle.group(tr, p16))


# ---- A5 ------------------------------------------------------------------------------------------------------
def check_stable(ph, tm, kbb, n, delta=(3, 100), rate=(95, 100)):
    from paper_conf_micro_liusc23_b200 import DeviceTiming, to_device
    dt = DeviceTiming.from_host(tm, ph.device)
    kb = to_device(np.ascontiguousarray(kbb, np.uint64), ph.device)
    o = ph.photon_bb_stable(dt, kb, n, delta, rate)
    fs, ds, sw = oracle.stable(tm, kbb, n, delta, rate)
    K, B = tm.n_kernels, int(tm.n_bb)
    assert np.array_equal(_np(o["first_stable"], np.int64).reshape(K, B), fs)
    assert np.array_equal(_np(o["stable_dur_sum"], np.uint64).reshape(K, B), ds)
    assert np.array_equal(_np(o["switch_at"], np.int64), sw)
    return fs


@pytest.mark.parametrize("n", [8, 32, 64])
def test_stable_c6(ph, n):
    g = tg.Generator(6)
    tm = g.timing()
    _, _, kbb = oracle.bbv(g.trace())
    fs = check_stable(ph, tm, kbb, n)
    assert (fs >= 0).any()


def test_stable_c1(ph):
    g = tg.Generator(1)
    tm = g.timing()
    _, _, kbb = oracle.bbv(g.trace())
    check_stable(ph, tm, kbb, 2048)
    check_stable(ph, tm, kbb, 512, delta=(1, 100))


@pytest.mark.parametrize("cfg", [3, 4])
def test_stable_configs(ph, cfg):
    g = tg.Generator(cfg)
    tm = g.timing()
    _, _, kbb = oracle.bbv(g.trace())
    check_stable(ph, tm, kbb, 2048)


def test_stable_paper_lines(ph):
    # L227 lines (stable) and L145 (not), one kernel per line, n = 64
    from fractions import Fraction
    n = 64
    recs = []
    for a in ["1.00", "0.99", "32.87", "0.97", "0.9701", "1.03", "1.0299"]:
        xs = [10_000 * (i + 1) for i in range(3 * n)]
        ys = [int(Fraction(a) * x + 10 ** 9) for x in xs]
        recs.append((xs, ys))
    off = np.cumsum([0] + [len(x) for x, _ in recs]).astype(np.uint64)
    tm = tg.Timing(kernel_rec_off=off, bb=np.zeros(int(off[-1]), np.uint16),
                   issue=np.concatenate([np.array(x, np.uint64) for x, _ in recs]),
                   retire=np.concatenate([np.array(y, np.uint64) for _, y in recs]), n_bb=1)
    fs = check_stable(ph, tm, np.ones((len(recs), 1), np.uint64), n)
    assert fs[:, 0].tolist() == [2 * n - 1, 2 * n - 1, -1, -1, 2 * n - 1, -1, 2 * n - 1]


def test_stable_errors(ph):
    from paper_conf_micro_liusc23_b200 import PhotonError
    tm = tg.Timing(kernel_rec_off=np.array([0, 3], np.uint64), bb=np.zeros(3, np.uint16),
                   issue=np.array([1, 2, 3], np.uint64), retire=np.array([5, 4, 9], np.uint64), n_bb=1)
    with pytest.raises(PhotonError) as ei:
        check_stable(ph, tm, np.ones((1, 1), np.uint64), 2)
    assert ei.value.code == -3 and ei.value.index == 1


def test_stable_late_multirun(ph):
    # groups that stabilise only after many 8192-position runs, never stabilise, or stabilise at once, interleaved
    # in one kernel (and repeated over 40 kernels so the ticket batches hold > 32 groups)
    rng = np.random.default_rng(11)
    offs, bbs, iss, ret = [0], [], [], []
    for k in range(40):
        L = 3000 + 700 * k
        late = L // 2 + 5 * k
        n_rec = 3 * L
        x = np.cumsum(rng.integers(1, 50, n_rec)).astype(np.uint64) + np.uint64(10 ** 6 * k)
        bb = np.tile(np.arange(3, dtype=np.uint16), L)
        dur = np.empty(n_rec, np.uint64)
        j = np.repeat(np.arange(L), 3)
        dur[0::3] = np.where(j[0::3] < late, rng.integers(1, 5000, L), 100)          # late stabiliser
        dur[1::3] = rng.integers(1, 5000, L)                                          # never
        dur[2::3] = 200                                                                # immediate
        y = x + dur
        order = np.argsort(y, kind="stable")
        bbs.append(bb[order]); iss.append(x[order]); ret.append(y[order])
        offs.append(offs[-1] + n_rec)
    tm = tg.Timing(kernel_rec_off=np.array(offs, np.uint64), bb=np.concatenate(bbs), issue=np.concatenate(iss),
                   retire=np.concatenate(ret), n_bb=3)
    kbb = np.ones((40, 3), np.uint64)
    fs = check_stable(ph, tm, kbb, 256)
    assert (fs[:, 0] > 0).all() and (fs[:, 2] >= 0).all()


@pytest.mark.parametrize("B", [256, 257, 1000, 5000, 9000])
def test_stable_many_bb(ph, B):
    # B <= 256: job multisplit on BB ids; 256 < B <= 8192: on per-kernel compacted ids (kernels with > 256 local ids
    # keep their counters in global memory); B > 8192: composite-key radix sort -- all must agree with the oracle
    rng = np.random.default_rng(B)
    offs, bbs, iss, ret = [0], [], [], []
    for k in range(6):
        n_rec = 30000 + 9000 * k
        x = np.cumsum(rng.integers(1, 20, n_rec)).astype(np.uint64)
        bb = (rng.zipf(1.3, n_rec) % B).astype(np.uint16)
        dur = np.where(rng.random(n_rec) < 0.9, 40 + (bb.astype(np.uint64) % 7), rng.integers(1, 400, n_rec))
        y = x + dur.astype(np.uint64)
        o = np.argsort(y, kind="stable")
        bbs.append(bb[o]); iss.append(x[o]); ret.append(y[o])
        offs.append(offs[-1] + n_rec)
    offs.insert(3, offs[2])  # an empty kernel in the middle
    tm = tg.Timing(kernel_rec_off=np.array(offs, np.uint64), bb=np.concatenate(bbs), issue=np.concatenate(iss),
                   retire=np.concatenate(ret), n_bb=B)
    kbb = rng.integers(0, 1000, (7, B)).astype(np.uint64)
    fs = check_stable(ph, tm, kbb, 16)
    assert (fs >= 0).sum() > 10


@pytest.mark.parametrize("K", [3000, 6000])
def test_match_many_kernels_synthetic(ph, K):
    # K > 2048 takes the cooperative (grid-barrier) resolution; type tables are synthetic clusters of near-copies
    # (many close pairs, long launch-order chains), checked against the oracle's signature + match
    from paper_conf_micro_liusc23_b200 import to_device
    rng = np.random.default_rng(K)
    n_tmpl = 40
    tmpl = rng.integers(1, 400, (n_tmpl, 4, 16)).astype(np.uint32)
    T = rng.integers(1, 5, K)
    kto = np.zeros(K + 1, np.uint64)
    kto[1:] = np.cumsum(T)
    keys, counts = [], []
    for k in range(K):
        t = rng.integers(0, n_tmpl)
        for r in range(T[k]):
            key = tmpl[t, r].astype(np.int64) + rng.integers(-2, 3, 16) * (rng.random(16) < 0.3)
            keys.append(np.clip(key, 0, None).astype(np.uint32))
            counts.append(int(rng.integers(50, 60) if r == 0 else rng.integers(1, 8)))
    keys = np.array(keys, np.uint32)
    counts = np.array(counts, np.uint64)
    wt = np.where(rng.random(K) < 0.5, 64 + rng.integers(0, 200, K), rng.integers(1, 4, K) * 16).astype(np.uint64)
    ty = ph.alloc_types(K, 1, len(counts))
    ty["kernel_type_off"].copy_(to_device(kto, ph.device))
    ty["type_key"].copy_(to_device(keys.reshape(-1), ph.device))
    ty["type_count"].copy_(to_device(counts, ph.device))
    m = ph.photon_kernel_match(K, ty, to_device(wt, ph.device), (1, 20), 64, 0, want_dist=True)
    sig, mass = oracle.signature(kto, keys, counts)
    om, od = oracle.match(kto, sig, mass, wt, (1, 20), 64, 0)
    gm = _np(m["match"], np.int64)
    assert (om >= 0).sum() > K // 4  # the clusters really produce matches
    assert np.array_equal(gm, om)
    # without match_dist (the timed chain's setting) the same decisions
    m2 = ph.photon_kernel_match(K, ty, to_device(wt, ph.device), (1, 20), 64, 0, want_dist=False)
    assert np.array_equal(_np(m2["match"], np.int64), om)
    gd = _np(m["match_dist"], np.float64)
    fin = np.isfinite(od)
    assert np.array_equal(np.isfinite(gd), fin)
    np.testing.assert_allclose(gd[fin], od[fin], rtol=1e-6, atol=0)


# ---- N1: warp-level stability (L249, L262, Fig 10) ---------------------------------------------------------------
def check_warp_stable(ph, tm, ok, n, delta=(3, 100)):
    from paper_conf_micro_liusc23_b200 import DeviceTiming, to_device
    dt = DeviceTiming.from_host(tm, ph.device)
    okd = None if ok is None else to_device(np.ascontiguousarray(ok, np.uint8), ph.device)
    o = ph.photon_warp_stable(dt, okd, n, delta)
    sw, ds = oracle.warp_stable(tm, ok, n, delta)
    assert np.array_equal(_np(o["switch_at"], np.int64), sw)
    assert np.array_equal(_np(o["dur_sum"], np.uint64), ds)
    return sw


@pytest.mark.parametrize("cfg", [3, 4, 2])
def test_warp_stable_configs_gated_by_dominance(ph, cfg):
    # the slot-model warp streams of every kernel, gated by A2's warp_sampling_ok of the same trace (the fused GPU
    # path computes it; the oracle's dominance decision must agree first)
    g = tg.Generator(cfg)
    tr = g.trace()
    ty = ph.photon_warp_group(_dev(ph, tr))
    p16, _, _ = oracle.bbv(tr, want_kbb=False)
    ok = oracle.group(tr, p16)["warp_sampling_ok"]
    assert np.array_equal(_np(ty["warp_sampling_ok"], np.uint8), ok)
    tm = g.warp_timing()
    sw = check_warp_stable(ph, tm, ok, 1024)
    sw_all = check_warp_stable(ph, tm, None, 1024)
    assert (sw_all >= 0).any()
    assert np.all(sw[ok == 0] == -1)


@pytest.mark.parametrize("n", [2, 64, 1024])
def test_warp_stable_c4_prefix_windows(ph, n):
    check_warp_stable(ph, tg.Generator(4).warp_timing(0, 60), None, n)
    check_warp_stable(ph, tg.Generator(4).warp_timing(0, 60), None, n, delta=(1, 100))


def test_warp_stable_paper_lines_and_errors(ph):
    from fractions import Fraction
    from paper_conf_micro_liusc23_b200 import PhotonError
    n = 64
    recs = []
    for a in ["1.00", "0.99", "32.87", "0.97", "0.9701", "1.03", "1.0299"]:
        xs = [10_000 * (i + 1) for i in range(3 * n)]
        ys = [int(Fraction(a) * x + 10 ** 9) for x in xs]
        recs.append((xs, ys))
    recs.append(([5] * 10, [6] * 10))  # too short to evaluate
    off = np.cumsum([0] + [len(x) for x, _ in recs]).astype(np.uint64)
    tm = tg.Timing(kernel_rec_off=off, bb=np.zeros(int(off[-1]), np.uint16),
                   issue=np.concatenate([np.array(x, np.uint64) for x, _ in recs]),
                   retire=np.concatenate([np.array(y, np.uint64) for _, y in recs]), n_bb=1)
    sw = check_warp_stable(ph, tm, None, n)
    assert sw.tolist() == [2 * n - 1, 2 * n - 1, -1, -1, 2 * n - 1, -1, 2 * n - 1, -1]
    ok = np.array([1, 0, 1, 1, 1, 1, 0, 1], np.uint8)
    sw = check_warp_stable(ph, tm, ok, n)
    assert sw.tolist() == [2 * n - 1, -1, -1, -1, 2 * n - 1, -1, -1, -1]
    bad = tg.Timing(kernel_rec_off=np.array([0, 3], np.uint64), bb=np.zeros(3, np.uint16),
                    issue=np.array([1, 2, 3], np.uint64), retire=np.array([5, 4, 9], np.uint64), n_bb=1)
    with pytest.raises(PhotonError) as ei:
        check_warp_stable(ph, bad, None, 2)
    assert ei.value.code == -3 and ei.value.index == 1


# ---- N3: kernel- and BB-level prediction (Fig 12 Step 4 / L279-281; Fig 7 Step 3) -------------------------------
def test_kernel_predict_chain_c4(ph):
    # ResNet-152: the GPU chain's matches and masses feed the prediction; synthetic "detailed simulation" counts for
    # the representatives; compared element by element with the oracle on the same inputs
    from paper_conf_micro_liusc23_b200 import to_device
    tr = tg.Generator(4).trace()
    d = _dev(ph, tr)
    r = ph.analyse(d)
    match = _np(r["match"], np.int64)
    ref = oracle.analyse(tr)
    assert np.array_equal(match, ref["match"])
    mass = ref["mass"]
    rs = np.random.default_rng(4)
    fi = rs.integers(1, 1 << 40, len(match)).astype(np.uint64)
    fc = rs.integers(1, 1 << 40, len(match)).astype(np.uint64)
    dv = lambda a, dt: to_device(np.ascontiguousarray(a, dt), ph.device)
    o = ph.photon_kernel_predict(dv(match, np.int64), dv(mass, np.uint64), dv(fi, np.uint64), dv(fc, np.uint64))
    pi, pc = oracle.kernel_predict(match, mass, fi, fc)
    assert np.array_equal(_np(o["pred_insts"], np.uint64), pi)
    assert np.array_equal(_np(o["pred_cycles"], np.uint64), pc)
    assert (match >= 0).sum() > 100  # the repeated conv4_x blocks are predicted, not simulated


def test_kernel_predict_errors(ph):
    from paper_conf_micro_liusc23_b200 import PhotonError, to_device
    dv = lambda a, dt: to_device(np.ascontiguousarray(a, dt), ph.device)
    with pytest.raises(PhotonError) as ei:  # representative index must precede the kernel
        ph.photon_kernel_predict(dv([-1, 1], np.int64), dv([3, 2], np.uint64), dv([5, 5], np.uint64),
                                 dv([5, 5], np.uint64))
    assert ei.value.code == -3 and ei.value.index == 1


@pytest.mark.parametrize("cfg", [3, 6])
def test_bb_predict_from_gpu_stability(ph, cfg):
    # A5 on the GPU gives first_stable / S_n; the per-warp BB-level prediction over the same config's trace
    from paper_conf_micro_liusc23_b200 import DeviceTiming, to_device
    g = tg.Generator(cfg)
    tr = g.trace()
    d = _dev(ph, tr)
    kbb = ph.photon_bbv_build(d, bbv16=False, insts=False, kbb=True)["kernel_bb_insts"]
    n = 2048 if cfg == 3 else 32
    st = ph.photon_bb_stable(DeviceTiming.from_host(g.timing(), ph.device), kbb, n)
    o = ph.photon_bb_predict(d, st["first_stable"], st["stable_dur_sum"])
    fs = _np(st["first_stable"], np.int64).reshape(tr.n_kernels, tr.n_bb)
    ds = _np(st["stable_dur_sum"], np.uint64).reshape(tr.n_kernels, tr.n_bb)
    pd, un = oracle.bb_predict(tr, fs, ds)
    assert np.array_equal(_np(o["pred_dur_sum"], np.uint64), pd)
    assert np.array_equal(_np(o["unpredicted"], np.uint32), un)
    assert (pd > 0).any() and (un > 0).any()


def test_bb_predict_random_tables(ph):
    from paper_conf_micro_liusc23_b200 import to_device
    for seed in range(4):
        tr = tg.random_trace(seed, n_kernels=1 + seed, max_warps=700, max_events=300, n_bb=[7, 300, 5000, 16][seed])
        rs = np.random.default_rng(seed)
        fs = np.where(rs.random((tr.n_kernels, tr.n_bb)) < 0.6, 1, -1).astype(np.int64)
        ds = rs.integers(1, 1 << 50, (tr.n_kernels, tr.n_bb)).astype(np.uint64)
        o = ph.photon_bb_predict(_dev(ph, tr), to_device(fs, ph.device), to_device(ds, ph.device))
        pd, un = oracle.bb_predict(tr, fs, ds)
        assert np.array_equal(_np(o["pred_dur_sum"], np.uint64), pd)
        assert np.array_equal(_np(o["unpredicted"], np.uint32), un)


def test_bb_predict_long_warp_list(ph):
    # warps above 128 events go to the device work list (pass 2): contiguous runs of long warps (as C3's fully
    # connected layers) next to tiny ones, a long warp of 9000 events, a bad id inside a long warp
    from paper_conf_micro_liusc23_b200 import PhotonError, to_device
    rs = np.random.default_rng(7)
    kernels = [[list(rs.integers(0, 9, 4)) for _ in range(300)],
               [list(rs.integers(0, 9, int(rs.integers(129, 700)))) for _ in range(200)],
               [list(rs.integers(0, 9, int(n))) for n in rs.integers(0, 200, 500)] + [list(rs.integers(0, 9, 9000))]]
    tr = tg.trace_from_warps(kernels, bb_len=list(range(1, 10)))
    fs = np.where(rs.random((tr.n_kernels, tr.n_bb)) < 0.7, 1, -1).astype(np.int64)
    ds = rs.integers(1, 1 << 50, (tr.n_kernels, tr.n_bb)).astype(np.uint64)
    o = ph.photon_bb_predict(_dev(ph, tr), to_device(fs, ph.device), to_device(ds, ph.device))
    pd, un = oracle.bb_predict(tr, fs, ds)
    assert np.array_equal(_np(o["pred_dur_sum"], np.uint64), pd)
    assert np.array_equal(_np(o["unpredicted"], np.uint32), un)
    bad = int(tr.warp_event_off[300]) + 77  # inside the first long warp
    tr.bb = tr.bb.copy()
    tr.bb[bad] = 9
    with pytest.raises(PhotonError) as ei:
        ph.photon_bb_predict(_dev(ph, tr), to_device(fs, ph.device), to_device(ds, ph.device))
    assert ei.value.code == -3 and ei.value.index == bad


# ---- N4: persisted signature pool (L402) -------------------------------------------------------------------
@pytest.mark.parametrize("cfg", [6, 4])
def test_pool_reuse(ph, cfg, tmp_path):
    # run A -> pool of its representatives (device export, persisted to disk and reloaded); run B matched against
    # it: pool, match and distances equal the oracle's on the same split
    g = tg.Generator(cfg)
    h = g.n_kernels // 2
    a, b = g.kernels_trace(0, h), g.kernels_trace(h, g.n_kernels)
    da, db = _dev(ph, a), _dev(ph, b)
    ty_a = ph.photon_warp_group(da)
    m_a = ph.photon_kernel_match(a.n_kernels, ty_a, da.warps_total)
    pool = ph.photon_pool_export(a.n_kernels, ty_a, da.warps_total, m_a["match"])
    ra = oracle.group(a, oracle.bbv(a, want_kbb=False)[0])
    sa, ma_ = oracle.signature(ra["kernel_type_off"], ra["type_key"], ra["type_count"])
    ref_m_a, _ = oracle.match(ra["kernel_type_off"], sa, ma_, a.warps_total)
    assert np.array_equal(_np(m_a["match"], np.int64), ref_m_a)
    rp = oracle.pool_export(ra, a.warps_total, ref_m_a)
    Kp = rp["n_pool"]
    assert pool["n_pool"] == Kp
    assert np.array_equal(_np(pool["kernel_type_off"], np.uint64), rp["kernel_type_off"])
    Tp = int(rp["kernel_type_off"][-1])
    assert np.array_equal(_np(pool["type_key"], np.uint32).reshape(-1, 16)[:Tp], rp["type_key"])
    assert np.array_equal(_np(pool["type_count"], np.uint64)[:Tp], rp["type_count"])
    assert np.array_equal(_np(pool["warps_total"], np.uint64), rp["warps_total"])
    assert np.array_equal(_np(pool["kernel_id"], np.uint32), rp["kernel_id"])
    path = str(tmp_path / "pool.npz")
    ph.save_pool(pool, path)
    pool2 = ph.load_pool(path)
    ty_b = ph.photon_warp_group(db)
    rb = oracle.group(b, oracle.bbv(b, want_kbb=False)[0])
    for th in ((1, 20), (1, 5)):
        o = ph.photon_kernel_match_pooled(pool2, b.n_kernels, ty_b, db.warps_total, theta=th)
        rm, rd = oracle.match_pooled(rp, rb, b.warps_total, theta=th)
        assert np.array_equal(_np(o["match"], np.int64), rm)
        got = _np(o["match_dist"], np.float64)
        fin = np.isfinite(rd)
        assert np.array_equal(np.isfinite(got), fin)
        assert np.allclose(got[fin], rd[fin], rtol=1e-6, atol=0)
        if th == (1, 20):
            assert (rm[Kp:] >= 0).sum() > 0  # some of run B reuses run A


# ---- N2: full-BBV exact grouping and tagged-stream ingest (L154, L161) ------------------------------------------
@pytest.mark.parametrize("which", ["c6", "c1", "rand5000", "ragged", "perm", pytest.param("c3", marks=pytest.mark.slow)])
def test_group_full(ph, which):
    if which == "c6":
        tr = tg.make_trace(6)
    elif which == "c3":  # the bench's N2 workload at full size (1.75M warps, 9% long)
        tr = tg.make_trace(3)
    elif which == "perm":  # long warps that are permutations of each other (the histogram verification, ids in
        rs = np.random.default_rng(5)  # three 4096-id chunks), near-misses differing in one event, short ones
        kernels = []
        for k in range(6):
            base = rs.integers(0, 9000, 40 + 30 * k).tolist()
            ws = [base]
            for j in range(12):
                p = list(rs.permutation(base))
                if j % 5 == 4:
                    p[0] = (p[0] + 4096) % 9000  # same length, another id in another chunk
                ws.append([int(v) for v in p])
            sh = rs.integers(0, 9000, 9).tolist()
            ws += [sh, [int(v) for v in rs.permutation(sh)], sh[::-1]]
            kernels.append(ws)
        tr = tg.trace_from_warps(kernels, bb_len=rs.integers(1, 9, 9000).tolist())
    elif which == "c1":
        tr = tg.make_trace(1)
    elif which == "rand5000":
        tr = tg.random_trace(11, n_kernels=5, max_warps=400, max_events=60, n_bb=5000, dup_p=0.7)
    else:
        kernels = [[[], [], [0, 1]], [], [[2] * 1000 + [1] * 3], [[]], [[0, 1, 2, 3, 4, 5, 6]] * 300 + [[1]],
                   [[1, 0], [0, 1], [1, 1, 0], [0, 1, 1], [2]]]
        tr = tg.trace_from_warps(kernels, bb_len=[3, 1, 7, 2, 9, 4, 5])
    d = _dev(ph, tr)
    p16, _, _ = oracle.bbv(tr, want_kbb=False)
    ref = oracle.group_full(tr, p16)
    ty = ph.photon_warp_group_full(d)
    T = int(ref["kernel_type_off"][-1])
    assert np.array_equal(_np(ty["kernel_type_off"], np.uint64), ref["kernel_type_off"])
    assert np.array_equal(_np(ty["warp_type"], np.uint32), ref["warp_type"])
    assert np.array_equal(_np(ty["type_key"], np.uint32).reshape(-1, 16)[:T], ref["type_key"].reshape(-1, 16))
    assert np.array_equal(_np(ty["type_count"], np.uint64)[:T], ref["type_count"])
    assert np.array_equal(_np(ty["type_first_warp"], np.uint64)[:T], ref["type_first_warp"])
    assert np.array_equal(_np(ty["warp_sampling_ok"], np.uint8), ref["warp_sampling_ok"])


def test_ingest_tagged(ph):
    import torch
    tr = tg.make_trace(6)
    W, weo = tr.n_warps, tr.warp_event_off.astype(np.int64)
    owner = np.repeat(np.arange(W), np.diff(weo)).astype(np.uint32)
    # interleave warps in slices of the generator's 2560-slot wave order: event i of warp w at key (w % 2560, i, w)
    pos = np.arange(len(owner)) - weo[owner]
    order = np.lexsort((owner, pos, owner % 2560))
    warp, bb = owner[order], tr.bb[order]
    out = ph.photon_ingest_tagged(torch.from_numpy(warp.astype(np.int32)).to(ph.device),
                                  torch.from_numpy(bb.astype(np.int16)).to(ph.device), W)
    rb, roff = oracle.ingest(warp, bb, W)
    assert np.array_equal(_np(out["warp_event_off"], np.uint64), roff)
    assert np.array_equal(_np(out["bb"], np.uint16), rb)
    assert np.array_equal(rb, tr.bb)  # and it is the CSR trace back
    from paper_conf_micro_liusc23_b200 import PhotonError
    bad = warp.copy()
    bad[7] = W
    with pytest.raises(PhotonError) as ei:
        ph.photon_ingest_tagged(torch.from_numpy(bad.astype(np.int32)).to(ph.device),
                                torch.from_numpy(bb.astype(np.int16)).to(ph.device), W)
    assert ei.value.code == -3 and ei.value.index == 7
