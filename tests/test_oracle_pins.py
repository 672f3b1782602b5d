"""Pins of the CPU oracle against things other than itself (CPU only, -m "not gpu").

Each pin names the PAPER.md passage (L<n>) or the mathematical fact it rests on.  None of them re-calls the
oracle's own formula: the references are the paper's printed numbers, a hand-worked example, exact Fraction
arithmetic written independently here, numpy's least squares / bincount, brute force on tiny inputs, and
invariants (so a dropped term, a wrong sign or index, or a transposed operand fails one of them).
"""
import itertools
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import tracegen as tg

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------------------------------------------------------
# Worked GPU-BBV example (tests/golden/worked_example.json, derived by hand from L178 + readings)
def test_worked_example_full_chain():
    g = _gold("worked_example.json")
    e = g["expect"]
    tr = tg.trace_from_warps(g["kernels"], g["bb_len"])
    p16, ins, kbb = oracle.bbv(tr)
    assert p16[:, :3].tolist() == e["warp_bbv16_nonzero"] and not p16[:, 3:].any()
    assert ins.tolist() == e["warp_insts"]
    assert kbb.tolist() == e["kernel_bb_insts"]
    t = oracle.group(tr, p16)
    assert t["warp_type"].tolist() == e["warp_type"]
    assert t["kernel_type_off"].tolist() == e["kernel_type_off"]
    assert t["type_key"][:, :3].tolist() == e["type_key_nonzero"]
    assert t["type_count"].tolist() == e["type_count"]
    assert t["type_first_warp"].tolist() == e["type_first_warp"]
    assert t["warp_sampling_ok"].tolist() == e["warp_sampling_ok"]
    sig, mass = oracle.signature(t["kernel_type_off"], t["type_key"], t["type_count"])
    assert mass.tolist() == e["mass"]
    a = {str(i): int(v) for i, v in enumerate(sig[:32]) if v}
    b = {str(i): int(v) for i, v in enumerate(sig[32:48]) if v}
    assert a == e["sig_nonzero_A"] and b == e["sig_nonzero_B"]
    for key, theta, cores in [("match_theta_1_20_cores_64", (1, 20), 64), ("match_theta_1_2_cores_64", (1, 2), 64),
                              ("match_theta_1_2_cores_2", (1, 2), 2), ("match_theta_4_11_cores_2", (4, 11), 2),
                              ("match_theta_2_5_cores_2", (2, 5), 2)]:
        m, d = oracle.match(t["kernel_type_off"], sig, mass, tr.warps_total, theta, cores)
        assert m.tolist() == e[key], key
        # matched or not, kernel B reports D(A, B) = 216/594: its representative, else the nearest representative
        assert d[1] == pytest.approx(e["D_AB_num"] / e["D_AB_den"], rel=1e-12)
        assert np.isinf(d[0])


# ---------------------------------------------------------------------------------------------------------------
# A1: BBV.  Pins: invariant sum_j p_w[j] = I_w = sum_e len(bb_e); identity fold for B <= 16 equals the full BBV
# computed with numpy.bincount; brute-force recount; single-BB warp p = count x len.
def _brute_bbv(tr):
    bins = (np.arange(tr.n_bb) & 15) if tr.bb_bin is None else tr.bb_bin
    out = np.zeros((tr.n_warps, 16), np.int64)
    for w in range(tr.n_warps):
        for e in range(int(tr.warp_event_off[w]), int(tr.warp_event_off[w + 1])):
            b = int(tr.bb[e])
            out[w, int(bins[b])] += int(tr.bb_len[b])
    return out


@pytest.mark.parametrize("seed,custom", [(1, False), (2, True), (3, True), (4, False)])
def test_bbv_bruteforce_and_invariants(seed, custom):
    tr = tg.random_trace(seed, n_kernels=4, max_warps=12, max_events=40, n_bb=40, custom_bins=custom)
    p16, ins, kbb = oracle.bbv(tr)
    assert np.array_equal(p16.astype(np.int64), _brute_bbv(tr))
    for w in range(tr.n_warps):
        ev = tr.bb[int(tr.warp_event_off[w]):int(tr.warp_event_off[w + 1])]
        assert int(ins[w]) == int(tr.bb_len[ev.astype(np.int64)].astype(np.int64).sum())
        assert int(p16[w].astype(np.int64).sum()) == int(ins[w])
    # BB distribution: rows sum to the kernel's instructions
    for k in range(tr.n_kernels):
        w0, w1 = int(tr.kernel_warp_off[k]), int(tr.kernel_warp_off[k + 1])
        assert int(kbb[k].sum()) == int(ins[w0:w1].sum())


def test_bbv_identity_fold_equals_full_bbv():
    # B <= 16 with the default fold: the projection is the identity, so p_w = full BBV = bincount x len
    tr = tg.random_trace(7, n_kernels=3, max_warps=10, max_events=60, n_bb=16)
    p16, _, _ = oracle.bbv(tr)
    for w in range(tr.n_warps):
        ev = tr.bb[int(tr.warp_event_off[w]):int(tr.warp_event_off[w + 1])].astype(np.int64)
        full = np.bincount(ev, minlength=16) * tr.bb_len.astype(np.int64)
        assert np.array_equal(p16[w].astype(np.int64), full)


def test_bbv_single_bb_warp_and_empty_warp():
    # single-BB warp: p = count x len; empty warp (L231 empty-task warps execute almost nothing): key all zeros
    tr = tg.trace_from_warps([[[5] * 7, [], [5]]], bb_len=[1] * 5 + [13])
    p16, ins, _ = oracle.bbv(tr)
    assert p16[0, 5] == 7 * 13 and p16[0].sum() == 7 * 13
    assert not p16[1].any() and ins[1] == 0
    assert p16[2, 5] == 13


def test_bbv_range_errors():
    tr = tg.trace_from_warps([[[0, 1, 9]]], bb_len=[1, 2, 3])  # bb 9 >= B
    with pytest.raises(oracle.OracleError) as ei:
        oracle.bbv(tr)
    assert ei.value.code == oracle.ERANGE and ei.value.index == 2
    tr = tg.trace_from_warps([[[0], [1]]], bb_len=[1, 2])
    tr.warp_event_off = np.array([0, 1, 0], np.uint64)  # non-monotone (and [W] != E)
    with pytest.raises(oracle.OracleError):
        oracle.bbv(tr)
    tr = tg.trace_from_warps([[[0] * 3]], bb_len=[(1 << 31) + 5])  # I_w >= 2^32
    with pytest.raises(oracle.OracleError) as ei:
        oracle.bbv(tr)
    assert ei.value.code == oracle.ERANGE and ei.value.index == 0


# ---------------------------------------------------------------------------------------------------------------
# A2: grouping.  Pins: partition (each warp exactly one type, counts sum to W_k); brute-force O(W^2): same type
# <=> equal key; canonical ids invariant under warp permutation; order = count desc then key asc (checked against
# Python's sorted on tuples); dominance boundary exactly 95% -> 0, above -> 1 (L249 strict).
@pytest.mark.parametrize("seed", [11, 12, 13])
def test_group_partition_bruteforce(seed):
    tr = tg.random_trace(seed, n_kernels=5, max_warps=30, max_events=20, n_bb=20, custom_bins=True)
    p16, _, _ = oracle.bbv(tr)
    t = oracle.group(tr, p16)
    kto = t["kernel_type_off"]
    for k in range(tr.n_kernels):
        w0, w1 = int(tr.kernel_warp_off[k]), int(tr.kernel_warp_off[k + 1])
        rows = range(int(kto[k]), int(kto[k + 1]))
        assert sum(int(t["type_count"][r]) for r in rows) == w1 - w0
        for a, b in itertools.product(range(w0, w1), repeat=2):
            assert (t["warp_type"][a] == t["warp_type"][b]) == bool(np.array_equal(p16[a], p16[b]))
        for w in range(w0, w1):
            assert np.array_equal(t["type_key"][int(kto[k]) + int(t["warp_type"][w])], p16[w])
        # canonical order by Python's own tuple sort
        keyed = sorted(((-int(t["type_count"][r]), tuple(int(x) for x in t["type_key"][r])) for r in rows))
        assert [(-c, key) for c, key in keyed] == [(int(t["type_count"][r]), tuple(int(x) for x in t["type_key"][r]))
                                                   for r in rows]
        for r in rows:
            members = [w for w in range(w0, w1) if np.array_equal(p16[w], t["type_key"][r])]
            assert t["type_first_warp"][r] == min(members)
        Wk = w1 - w0
        dom = int(t["type_count"][int(kto[k])]) if Wk else 0
        assert t["warp_sampling_ok"][k] == (1 if Wk and Fraction(dom, Wk) > Fraction(95, 100) else 0)


def test_group_permutation_invariance():
    tr = tg.random_trace(21, n_kernels=1, max_warps=40, max_events=15, n_bb=10)
    p16, _, _ = oracle.bbv(tr)
    t = oracle.group(tr, p16)
    perm = np.random.default_rng(5).permutation(tr.n_warps)
    tr2 = tg.trace_from_warps([[tr.bb[int(tr.warp_event_off[w]):int(tr.warp_event_off[w + 1])].tolist()
                                for w in perm]], tr.bb_len)
    p2, _, _ = oracle.bbv(tr2)
    t2 = oracle.group(tr2, p2)
    assert np.array_equal(t["type_key"], t2["type_key"]) and np.array_equal(t["type_count"], t2["type_count"])
    assert np.array_equal(t2["warp_type"], t["warp_type"][perm])


@pytest.mark.parametrize("n_dom,n_all,ok", [(19, 20, 0), (95, 100, 0), (96, 100, 1), (20, 20, 1), (1, 1, 1),
                                            (190, 201, 0), (191, 201, 1)])
def test_dominance_boundary(n_dom, n_all, ok):
    # L249 "accounts for more than 95%": strict; 19/20 = 95% exactly -> no warp sampling
    warps = [[0, 1]] * n_dom + [[0]] * (n_all - n_dom)
    tr = tg.trace_from_warps([warps], bb_len=[3, 4])
    p16, _, _ = oracle.bbv(tr)
    assert oracle.group(tr, p16)["warp_sampling_ok"][0] == ok


# ---------------------------------------------------------------------------------------------------------------
# A3 / A4: signature, distance, matching.  Pins: sum g = N; Fraction distance of the normalised weighted BBVs
# built here from the type table (independent code); metric properties; strict threshold boundary; brute-force
# launch-order resolution on random tiny lists; scenario pins.
def _frac_gpu_bbv(t, k):
    """GPU BBV of kernel k as Fractions, built the L178 way: weights c_t/W, weighted BBVs listed, then [P-5]
    scaled to unit mass.  Written independently of the oracle (which works on integers g, N)."""
    kto = t["kernel_type_off"]
    rows = range(int(kto[k]), int(kto[k + 1]))
    W = sum(int(t["type_count"][r]) for r in rows)
    vec = []
    for r in rows:
        wgt = Fraction(int(t["type_count"][r]), W)
        vec.extend(wgt * int(x) for x in t["type_key"][r])
    s = sum(vec)
    return [v / s for v in vec] if s else vec


def _frac_dist(a, b):
    L = max(len(a), len(b))
    a = a + [Fraction(0)] * (L - len(a))
    b = b + [Fraction(0)] * (L - len(b))
    return sum(abs(x - y) for x, y in zip(a, b))


def _pipeline(tr):
    p16, _, _ = oracle.bbv(tr)
    t = oracle.group(tr, p16)
    sig, mass = oracle.signature(t["kernel_type_off"], t["type_key"], t["type_count"])
    return t, sig, mass


def test_signature_mass_and_distance_metric_properties():
    tr = tg.random_trace(31, n_kernels=6, max_warps=12, max_events=12, n_bb=12, dup_p=0.8)
    t, sig, mass = _pipeline(tr)
    kto = t["kernel_type_off"]
    for k in range(tr.n_kernels):
        assert int(sig[16 * int(kto[k]):16 * int(kto[k + 1])].astype(object).sum()) == int(mass[k])
    vecs = [_frac_gpu_bbv(t, k) for k in range(tr.n_kernels)]
    nz = [k for k in range(tr.n_kernels) if mass[k] > 0]
    for a in nz:
        assert _frac_dist(vecs[a], vecs[a]) == 0
        for b in nz:
            dab = _frac_dist(vecs[a], vecs[b])
            assert dab == _frac_dist(vecs[b], vecs[a]) and 0 <= dab <= 2
            for c in nz:
                assert _frac_dist(vecs[a], vecs[c]) <= dab + _frac_dist(vecs[b], vecs[c])
    # oracle's reported distance for a forced match (theta = 2 + pool_all_prior) equals the Fraction value
    for a, b in itertools.combinations(nz, 2):
        sub = tg.trace_from_warps([_warps_of(tr, a), _warps_of(tr, b)], tr.bb_len)
        t2, s2, m2 = _pipeline(sub)
        d_exact = _frac_dist(_frac_gpu_bbv(t2, 0), _frac_gpu_bbv(t2, 1))
        if d_exact < 2:
            mm, dd = oracle.match(t2["kernel_type_off"], s2, m2, [1000, 1000], theta=(2, 1), n_cores=64)
            assert mm[1] == 0 and dd[1] == pytest.approx(float(d_exact), rel=1e-12, abs=0)


def _warps_of(tr, k):
    return [tr.bb[int(tr.warp_event_off[w]):int(tr.warp_event_off[w + 1])].tolist()
            for w in range(int(tr.kernel_warp_off[k]), int(tr.kernel_warp_off[k + 1]))]


def _brute_resolve(vecs, masses, wt, theta, cores, pool_all):
    """Launch-order leader clustering (L271 Fig 12 Steps 2-3, [P-8][P-9][P-10]) on Fraction distances."""
    K = len(vecs)
    rep, match = [False] * K, [-1] * K
    for k in range(K):
        best = None
        for r in range(k):
            if not (pool_all or rep[r]) or masses[k] == 0 or masses[r] == 0:
                continue
            if not (wt[k] == wt[r] or min(wt[k], wt[r]) >= cores):
                continue
            if _frac_dist(vecs[k], vecs[r]) < theta:
                cand = (abs(wt[k] - wt[r]), r)
                best = cand if best is None or cand < best else best
        if best is None:
            rep[k] = True
        else:
            match[k] = best[1]
    return match


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("theta", [(1, 100), (1, 20), (1, 10), (1, 5), (1, 2)])
def test_match_bruteforce_random(seed, theta):
    rs = np.random.default_rng(100 + seed)
    # few prototypes with small perturbations so many pairs are near the threshold
    protos = [[int(x) for x in rs.integers(0, 6, int(rs.integers(1, 8)))] for _ in range(3)]
    kernels = []
    for _ in range(9):
        p = protos[int(rs.integers(0, 3))]
        warps = [list(p) for _ in range(int(rs.integers(1, 8)))]
        if rs.random() < 0.5:
            warps.append(p + [int(rs.integers(0, 6))])
        kernels.append(warps)
    wt = [int(x) for x in rs.choice([16, 32, 64, 100, 128, 128], size=len(kernels))]
    tr = tg.trace_from_warps(kernels, bb_len=[1, 2, 3, 5, 8, 13], warps_total=wt)
    t, sig, mass = _pipeline(tr)
    vecs = [_frac_gpu_bbv(t, k) for k in range(len(kernels))]
    for pool_all in (0, 1):
        m, d = oracle.match(t["kernel_type_off"], sig, mass, wt, theta, 64, pool_all)
        assert m.tolist() == _brute_resolve(vecs, [int(x) for x in mass], wt, Fraction(*theta), 64, pool_all)
        for k in range(len(kernels)):
            if m[k] >= 0:
                assert d[k] == pytest.approx(float(_frac_dist(vecs[k], vecs[int(m[k])])), rel=1e-12)
            else:  # a representative: the minimum D to any earlier member of the pool [P-8] (warp rule ignored)
                pool = [r for r in range(k) if (pool_all or m[r] < 0) and int(mass[r]) > 0]
                if int(mass[k]) == 0 or not pool:
                    assert np.isinf(d[k])
                else:
                    want = min(_frac_dist(vecs[k], vecs[r]) for r in pool)
                    assert d[k] == pytest.approx(float(want), rel=1e-12)


def test_match_scenarios():
    a, b = [0, 1, 1, 2], [0, 2, 2, 2, 1]
    # identical repeat matches its first occurrence; chain: k2 matches k0 (representative), not k1 (matched)
    tr = tg.trace_from_warps([[a] * 4, [a] * 4, [a] * 4, [b] * 4], [2, 3, 1], warps_total=[100, 100, 100, 100])
    t, sig, mass = _pipeline(tr)
    m, d = oracle.match(t["kernel_type_off"], sig, mass, tr.warps_total)
    assert m.tolist() == [-1, 0, 0, -1] and d[1] == 0.0 and np.isinf(d[0])
    # the representative k3 reports its distance to the only earlier representative, k0
    v = [_frac_gpu_bbv(t, k) for k in range(4)]
    assert d[3] == pytest.approx(float(_frac_dist(v[3], v[0])), rel=1e-12) and 0 < d[3] < 2
    # fewer warps than GPU cores (64): unequal counts never match; equal counts do (L271 Fig 12 note, L277)
    m, _ = oracle.match(t["kernel_type_off"], sig, mass, np.array([32, 33, 32, 32], np.uint64))
    assert m.tolist() == [-1, -1, 0, -1]
    # closest warp count wins; a tie goes to the earliest representative (pool = all prior so 0 and 1 compete)
    m, _ = oracle.match(t["kernel_type_off"], sig, mass, np.array([100, 140, 120, 100], np.uint64),
                        pool_all_prior=1)
    assert m[2] == 0  # |120-100| = |120-140| = 20: tie -> earliest
    m, _ = oracle.match(t["kernel_type_off"], sig, mass, np.array([100, 130, 120, 100], np.uint64),
                        pool_all_prior=1)
    assert m[2] == 1
    # empty signature never matches [P-19]
    tr = tg.trace_from_warps([[[]], [[]]], [1])
    t, sig, mass = _pipeline(tr)
    m, d = oracle.match(t["kernel_type_off"], sig, mass, [64, 64], theta=(2, 1))
    assert m.tolist() == [-1, -1] and np.isinf(d).all()


def test_match_theta_exact_boundary():
    # D = 4/11 exactly (worked example): theta = 4/11 -> not close (strict); 4/11 + tiny -> close
    g = _gold("worked_example.json")
    tr = tg.trace_from_warps(g["kernels"], g["bb_len"], warps_total=[100, 100])
    t, sig, mass = _pipeline(tr)
    assert oracle.match(t["kernel_type_off"], sig, mass, tr.warps_total, (4, 11))[0].tolist() == [-1, -1]
    assert oracle.match(t["kernel_type_off"], sig, mass, tr.warps_total, (400001, 1100000))[0].tolist() == [-1, 0]
    assert oracle.match(t["kernel_type_off"], sig, mass, tr.warps_total, (399999, 1100000))[0].tolist() == [-1, -1]


# ---------------------------------------------------------------------------------------------------------------
# A5: Eq. 1 slope and the stability detector.
def _exact_slope(xs, ys):
    """Eq. 1 (L222-225) in exact rationals, written from the textbook normal equations."""
    n = len(xs)
    xm = Fraction(sum(xs), n)
    ym = Fraction(sum(ys), n)
    sxy = sum((x - xm) * (y - ym) for x, y in zip(xs, ys))
    sxx = sum((x - xm) ** 2 for x in xs)
    return sxy / sxx


def _timing_one_kernel(xs, ys, bbs=None):
    R = len(xs)
    return tg.Timing(kernel_rec_off=np.array([0, R], np.uint64),
                     bb=np.array(bbs if bbs is not None else [0] * R, np.uint16),
                     issue=np.array(xs, np.uint64), retire=np.array(ys, np.uint64), n_bb=1 if bbs is None else max(bbs) + 1)


def _line_stream(a: Fraction, b: Fraction, n: int, count: int, x0=10_000, dx=10_000, offset=10 ** 9):
    xs = [x0 + dx * i for i in range(count)]
    ys = [int(a * x + b + offset) for x in xs]  # a*x integral for the chosen a and dx
    return xs, ys


@pytest.mark.parametrize("entry", _gold("paper_lines.json")["lines"] + _gold("paper_lines.json")["boundary"])
def test_eq1_paper_lines_and_boundary(entry):
    a = Fraction(entry["a"])
    b = Fraction(entry.get("b", "0")) * 100  # microseconds -> ticks, keeps the line (slope is unit-free)
    n = 8
    xs, ys = _line_stream(a, b, n, 2 * n)
    # the closed form agrees with numpy's least squares and with the exact rational slope
    assert _exact_slope(xs, ys) == a
    assert np.polyfit(np.array(xs, float), np.array(ys, float), 1)[0] == pytest.approx(float(a), rel=1e-9)
    fs, ds, sw = oracle.stable(_timing_one_kernel(xs, ys), np.array([[1]], np.uint64), n=n)
    assert (fs[0, 0] == 2 * n - 1) == entry["stable"], entry
    if entry["stable"]:
        assert int(ds[0, 0]) == sum(y - x for x, y in zip(xs[n:], ys[n:]))  # S_n of the last n
        assert sw[0] == 2 * n - 1


def test_eq1_float_hazard_at_boundary():
    # a = 0.97 exactly (|1-a| = delta): numpy.polyfit's float slope lands on the wrong side of |1-a| < 0.03 and a
    # float detector would call it stable; the exact integer test (the oracle's) does not [P-15][P-16]
    xs, ys = _line_stream(Fraction(97, 100), Fraction(0), 8, 16, x0=0, dx=1000, offset=10 ** 6)
    fa = np.polyfit(np.array(xs, float), np.array(ys, float), 1)[0]
    assert _exact_slope(xs, ys) == Fraction(97, 100)
    assert abs(1 - fa) < 0.03  # the float hazard is real on this stream
    fs, _, _ = oracle.stable(_timing_one_kernel(xs, ys), np.array([[1]], np.uint64), n=8)
    assert fs[0, 0] == -1


@pytest.mark.parametrize("seed", range(8))
def test_stability_bruteforce_fraction(seed):
    """Random small streams of 3 BB types: first-stable positions equal a from-scratch Fraction recomputation
    of cond1 (Eq. 1, |1-a| < delta) and cond2 (mean check) at every execution, in both oracle modes."""
    rs = np.random.default_rng(seed)
    n = int(rs.choice([2, 3, 5, 8]))
    R = 120
    types = rs.integers(0, 3, R)
    t = 0
    xs, ys = [], []
    for i in range(R):
        t += int(rs.integers(0, 4))
        d = int(rs.choice([5, 5, 5, 6])) if rs.random() < 0.8 else int(rs.integers(0, 12))
        xs.append(t)
        ys.append(t + d)
    order = sorted(range(R), key=lambda i: (ys[i], i))
    xs = [xs[i] for i in order]
    ys = [ys[i] for i in order]
    bbs = [int(types[i]) for i in range(R)]
    tm = _timing_one_kernel(xs, ys, bbs)
    tm.n_bb = 3
    kbb = np.array([[50, 30, 20]], np.uint64)
    delta = Fraction(3, 100) if seed % 2 else Fraction(1, 5)
    expect = [-1, -1, -1]
    for b in range(3):
        idx = [i for i in range(R) if bbs[i] == b]
        for j in range(2 * n, len(idx) + 1):
            win = idx[j - n:j]
            win2 = idx[j - 2 * n:j]
            wx = [xs[i] for i in win]
            wy = [ys[i] for i in win]
            if len(set(wx)) < 2:
                c1 = False
            else:
                c1 = abs(1 - _exact_slope(wx, wy)) < delta
            sn = sum(ys[i] - xs[i] for i in win)
            s2n = sum(ys[i] - xs[i] for i in win2)
            c2 = s2n > 0 and abs(Fraction(sn, n) - Fraction(s2n, 2 * n)) < delta * Fraction(s2n, 2 * n)
            if c1 and c2:
                expect[b] = idx[j - 1]
                break
    for brute in (True, False):
        fs, ds, sw = oracle.stable(tm, kbb, n=n, delta=(delta.numerator, delta.denominator), brute=brute)
        assert fs[0].tolist() == expect
    # switch [P-14]: order stable BBs by position, first point where the weight share exceeds 95%
    st = sorted((p, b) for b, p in enumerate(expect) if p >= 0)
    acc, want = 0, -1
    for p, b in st:
        acc += int(kbb[0, b])
        if Fraction(acc, 100) > Fraction(95, 100):
            want = p
            break
    assert sw[0] == want


def test_detector_constructed_streams():
    n = 2048
    # L227 MM line scaled x100: y = x + 423, single type -> stable at exactly its 2n-th execution (position 4095)
    xs = [100 * i for i in range(3 * n)]
    ys = [x + 423 for x in xs]
    fs, ds, sw = oracle.stable(_timing_one_kernel(xs, ys), np.array([[7]], np.uint64), n=n)
    assert fs[0, 0] == 2 * n - 1 and int(ds[0, 0]) == 423 * n and sw[0] == 2 * n - 1
    # SpMV-like mix (L210): a stable 99.4%-weight BB + a 0.6% BB executed once (rare, never stable) -> switches
    xs2 = xs + [xs[-1] + 50]
    ys2 = ys + [ys[-1] + 60]
    tm = _timing_one_kernel(xs2, ys2, [0] * len(xs) + [1])
    fs, _, sw = oracle.stable(tm, np.array([[994, 6]], np.uint64), n=n)
    assert fs[0].tolist() == [2 * n - 1, -1] and sw[0] == 2 * n - 1
    # exactly 95% weight stable -> no switch (strict, L208 "larger than"); 95.1% -> switch
    fs, _, sw = oracle.stable(tm, np.array([[950, 50]], np.uint64), n=n)
    assert sw[0] == -1
    fs, _, sw = oracle.stable(tm, np.array([[951, 49]], np.uint64), n=n)
    assert sw[0] == 2 * n - 1
    # all issue times equal: den = 0 -> not stable [P-16]
    xs3 = [1000] * (2 * n)
    ys3 = [1000 + 5 + (i % 3) for i in range(2 * n)]
    ys3.sort()
    fs, _, _ = oracle.stable(_timing_one_kernel(xs3, ys3), np.array([[1]], np.uint64), n=n)
    assert fs[0, 0] == -1
    # zero durations: S_2n = 0 -> not stable [P-17]
    xs4 = list(range(2 * n))
    fs, _, _ = oracle.stable(_timing_one_kernel(xs4, xs4), np.array([[1]], np.uint64), n=n)
    assert fs[0, 0] == -1


def test_detector_ramp_then_flat_bruteforce():
    # durations ramp down then flatten (the warm-up of L227): compare both oracle modes with a direct recomputation
    n = 16
    xs, ys = [], []
    t = 0
    for i in range(12 * n):
        d = 200 - 4 * i if i < 40 else 40
        xs.append(t)
        ys.append(t + d)
        t += 7
    order = sorted(range(len(xs)), key=lambda i: (ys[i], i))
    xs = [xs[i] for i in order]
    ys = [ys[i] for i in order]
    want = -1
    for j in range(2 * n, len(xs) + 1):
        wx, wy = xs[j - n:j], ys[j - n:j]
        c1 = abs(1 - _exact_slope(wx, wy)) < Fraction(3, 100)
        sn = sum(y - x for x, y in zip(wx, wy))
        s2n = sum(y - x for x, y in zip(xs[j - 2 * n:j], ys[j - 2 * n:j]))
        c2 = s2n > 0 and abs(2 * sn - s2n) * 100 < 3 * s2n
        if c1 and c2:
            want = j - 1
            break
    assert want > 2 * n  # the ramp delays stability past the first evaluable window
    for brute in (True, False):
        fs, _, _ = oracle.stable(_timing_one_kernel(xs, ys), np.array([[1]], np.uint64), n=n, brute=brute)
        assert fs[0, 0] == want


def test_stable_range_errors():
    tm = _timing_one_kernel([5, 6], [4, 9])  # retire < issue
    with pytest.raises(oracle.OracleError) as ei:
        oracle.stable(tm, np.array([[1]], np.uint64), n=2)
    assert ei.value.index == 0
    tm = _timing_one_kernel([1, 2], [9, 8])  # not retire-sorted
    with pytest.raises(oracle.OracleError) as ei:
        oracle.stable(tm, np.array([[1]], np.uint64), n=2)
    assert ei.value.index == 1
    tm = _timing_one_kernel([1, 1 << 40], [9, (1 << 40) + 1])  # time >= 2^40
    with pytest.raises(oracle.OracleError):
        oracle.stable(tm, np.array([[1]], np.uint64), n=2)


def test_oracle_modes_agree_on_generated_timing():
    g = tg.Generator(6)
    tm = g.timing(0, 6)
    tr = g.kernels_trace(0, 6)
    _, _, kbb = oracle.bbv(tr)
    a = oracle.stable(tm, kbb, n=32, brute=True)
    b = oracle.stable(tm, kbb, n=32, brute=False)
    for x, y in zip(a, b):
        assert np.array_equal(x, y)
    assert (a[0] >= 0).any()  # something stabilises


# ---- N1: warp-level stability (L249, L262, Fig 10) ---------------------------------------------------------------
def _warp_stream(kernels):
    """kernels: list of (xs, ys) warp records, each kernel retire-sorted; returns a photon_timing-like Timing."""
    off = np.zeros(len(kernels) + 1, np.uint64)
    off[1:] = np.cumsum([len(x) for x, _ in kernels])
    xs = np.array([v for x, _ in kernels for v in x], np.uint64)
    ys = np.array([v for _, y in kernels for v in y], np.uint64)
    return tg.Timing(kernel_rec_off=off, bb=np.zeros(len(xs), np.uint16), issue=xs, retire=ys, n_bb=1)


def test_warp_stable_constructed_and_gating():
    n = 1024  # L262 "we set n=1024"
    xs = [100 * i for i in range(3 * n)]
    ys = [x + 423 for x in xs]  # the L227 MM line, as warps
    # a kernel whose warp durations drift (a = 1.2): never within 3% of 1
    dx = [100 * i for i in range(3 * n)]
    dy = [int(Fraction(6, 5) * x) + 500 for x in dx]
    tm = _warp_stream([(xs, ys), (dx, dy), (xs, ys)])
    sw, ds = oracle.warp_stable(tm, np.array([1, 1, 0], np.uint8), n=n)
    # first evaluable retirement (the 2n-th warp) is stable; S_n = 423 n; the prediction is S_n / n = 423 ticks
    assert sw.tolist() == [2 * n - 1, -1, -1] and int(ds[0]) == 423 * n
    sw, _ = oracle.warp_stable(tm, None, n=n)  # no gate: the third kernel switches too
    assert sw.tolist() == [2 * n - 1, -1, 2 * n - 1]
    # fewer than 2n warps: never evaluable [P-11]
    sw, _ = oracle.warp_stable(_warp_stream([(xs[:2 * n - 1], ys[:2 * n - 1])]), None, n=n)
    assert sw[0] == -1


@pytest.mark.parametrize("entry", _gold("paper_lines.json")["lines"] + _gold("paper_lines.json")["boundary"])
def test_warp_stable_paper_lines(entry):
    # L262: "the a of the least square method on the last n warps ... is close to 1 (|a-1| < delta)"; the same Eq. 1
    # lines (L145, L227) and the strict 0.97 / 1.03 boundaries decide the warp-sampling switch
    a = Fraction(entry["a"])
    b = Fraction(entry.get("b", "0")) * 100
    n = 8
    xs, ys = _line_stream(a, b, n, 2 * n)
    sw, ds = oracle.warp_stable(_warp_stream([(xs, ys)]), None, n=n)
    assert (sw[0] == 2 * n - 1) == entry["stable"], entry


@pytest.mark.parametrize("seed", range(6))
def test_warp_stable_bruteforce_fraction(seed):
    """Random warp streams: the switch position equals a from-scratch Fraction recomputation of cond1 (Eq. 1 over
    the last n warps) and cond2 (mean of the last n vs the last 2n) at every retirement, in both oracle modes."""
    rs = np.random.default_rng(100 + seed)
    n = int(rs.choice([2, 3, 4, 8]))
    kernels, expect, ok = [], [], []
    for k in range(3):
        R = int(rs.integers(0, 80))
        t, xs, ys = 0, [], []
        for i in range(R):
            t += int(rs.integers(0, 5))
            d = 20 + int(rs.integers(0, 3)) if rs.random() < 0.85 else int(rs.integers(5, 40))
            xs.append(t)
            ys.append(t + d)
        order = sorted(range(R), key=lambda i: (ys[i], i))
        xs, ys = [xs[i] for i in order], [ys[i] for i in order]
        kernels.append((xs, ys))
        g = int(rs.integers(0, 4) > 0)
        ok.append(g)
        want = -1
        for j in range(2 * n, R + 1):
            wx, wy = xs[j - n:j], ys[j - n:j]
            c1 = len(set(wx)) >= 2 and abs(1 - _exact_slope(wx, wy)) < Fraction(3, 100)
            sn = sum(y - x for x, y in zip(wx, wy))
            s2n = sum(y - x for x, y in zip(xs[j - 2 * n:j], ys[j - 2 * n:j]))
            c2 = s2n > 0 and abs(Fraction(sn, n) - Fraction(s2n, 2 * n)) < Fraction(3, 100) * Fraction(s2n, 2 * n)
            if c1 and c2:
                want = j - 1
                break
        expect.append(want if g else -1)
    tm = _warp_stream(kernels)
    for brute in (True, False):
        sw, _ = oracle.warp_stable(tm, np.array(ok, np.uint8), n=n, brute=brute)
        assert sw.tolist() == expect


def test_warp_stable_generated_modes_agree_and_range_errors():
    tm = tg.Generator(4).warp_timing(0, 30)  # ResNet-152 stem and first blocks, slot-model warp streams
    a = oracle.warp_stable(tm, None, n=64, brute=True)
    b = oracle.warp_stable(tm, None, n=64, brute=False)
    assert np.array_equal(a[0], b[0]) and np.array_equal(a[1], b[1])
    assert 0 < (a[0] >= 0).sum() < len(a[0])  # some kernels switch, some do not
    with pytest.raises(oracle.OracleError) as ei:
        oracle.warp_stable(_warp_stream([([1, 2], [9, 8])]), None, n=2)  # not retire-sorted
    assert ei.value.index == 1


# ---- N3: kernel- and BB-level prediction (Fig 12 Step 4 / L279-281, Fig 7 Step 3) ------------------------------
def _half_up(num: Fraction) -> int:
    return int((num + Fraction(1, 2)) // 1)


def test_kernel_predict_formula_and_rounding():
    # #insts = #insts^K' * #insts_sample / #insts^K'_sample (L279-281); IPC(K) = IPC(K') => the same ratio scales
    # the cycles; a representative keeps its simulated counts
    match = np.array([-1, 0, 0, -1, 3], np.int64)
    mass = np.array([3, 2, 1, 4, 2], np.uint64)          # N_k: instructions of the analysed sample (A3 masses)
    full_i = np.array([1000, 0, 0, 7, 0], np.uint64)
    full_c = np.array([3, 0, 0, 5, 0], np.uint64)
    pi, pc = oracle.kernel_predict(match, mass, full_i, full_c)
    assert pi.tolist() == [1000, 667, 333, 7, 4]          # 2000/3 -> 667, 1000/3 -> 333, 7*2/4 = 3.5 -> 4 (half up)
    assert pc.tolist() == [3, 2, 1, 5, 3]                 # 5*2/4 = 2.5 -> 3
    rs = np.random.default_rng(5)
    for _ in range(200):
        K = int(rs.integers(1, 6))
        match = np.array([-1] + [int(rs.integers(-1, k)) for k in range(1, K)], np.int64)
        mass = rs.integers(1, 1 << 40, K).astype(np.uint64)
        fi = rs.integers(0, 1 << 62, K).astype(np.uint64)
        fc = rs.integers(0, 1 << 62, K).astype(np.uint64)
        exact = [max(_half_up(Fraction(int(fi[r]) * int(mass[k]), int(mass[r]))),
                     _half_up(Fraction(int(fc[r]) * int(mass[k]), int(mass[r])))) if r >= 0 else 0
                 for k, r in enumerate(int(x) for x in match)]
        if max(exact) >= 1 << 64:  # a prediction that does not fit u64 is a range error, not a wrapped value
            with pytest.raises(oracle.OracleError):
                oracle.kernel_predict(match, mass, fi, fc)
            continue
        pi, pc = oracle.kernel_predict(match, mass, fi, fc)
        for k in range(K):
            r = int(match[k])
            if r < 0:
                assert (int(pi[k]), int(pc[k])) == (int(fi[k]), int(fc[k]))
            else:
                assert int(pi[k]) == _half_up(Fraction(int(fi[r]) * int(mass[k]), int(mass[r])))
                assert int(pc[k]) == _half_up(Fraction(int(fc[r]) * int(mass[k]), int(mass[r])))


def test_bb_predict_worked_example_and_invariants():
    # the worked example's kernel A (L178 pipeline): warps [0,1,1,2] x3 and [0,1,2]; types 0 and 1 stable with
    # S_n = 40 and 90 (n = 10: mean durations 4 and 9 ticks), type 2 never stable (a rare BB: interval model, out)
    g = _gold("worked_example.json")
    tr = tg.trace_from_warps(g["kernels"], g["bb_len"])
    K, B = tr.n_kernels, tr.n_bb
    fs = np.full((K, B), -1, np.int64)
    ds = np.zeros((K, B), np.uint64)
    fs[0, 0], ds[0, 0] = 5, 40
    fs[0, 1], ds[0, 1] = 9, 90
    pd, un = oracle.bb_predict(tr, fs, ds)
    W0 = int(tr.kernel_warp_off[1])
    assert pd[:W0].tolist() == [40 + 2 * 90, 40 + 2 * 90, 40 + 90, 40 + 2 * 90]
    assert un[:W0].tolist() == [1, 1, 1, 1]
    assert pd[W0:].tolist() == [0] * (tr.n_warps - W0) and un[W0:].tolist() == [4] * (tr.n_warps - W0)
    # invariant on a generated trace: per kernel, sum_w pred = sum_b (executions of b) * S_n(b) over stable b, with
    # the executions taken independently from the A1 BB distribution (kernel_bb_insts / len)
    g6 = tg.Generator(6)
    tr6 = g6.kernels_trace(0, 10)
    _, _, kbb = oracle.bbv(tr6)
    rs = np.random.default_rng(9)
    fs = np.where(rs.random((tr6.n_kernels, tr6.n_bb)) < 0.7, 1, -1).astype(np.int64)
    ds = rs.integers(1, 1 << 30, (tr6.n_kernels, tr6.n_bb)).astype(np.uint64)
    pd, un = oracle.bb_predict(tr6, fs, ds)
    kwo = np.asarray(tr6.kernel_warp_off, np.int64)
    blen = np.asarray(tr6.bb_len, np.uint64)
    for k in range(tr6.n_kernels):
        execs = kbb[k] // blen
        want = sum(int(execs[b]) * int(ds[k, b]) for b in range(tr6.n_bb) if fs[k, b] >= 0)
        miss = sum(int(execs[b]) for b in range(tr6.n_bb) if fs[k, b] < 0)
        assert sum(int(x) for x in pd[kwo[k]:kwo[k + 1]]) == want
        assert int(un[kwo[k]:kwo[k + 1]].sum()) == miss


# N4: persisted signature pool (L402, reading [N4-a]).  Pins: a run matched against its own pool has no
# representative left and each of its representatives reuses its own pooled copy at distance 0; the pooled
# decisions for run B equal an independent Fraction brute force over A's representatives followed by B.
def _split_runs(seed):
    tr = tg.random_trace(seed, n_kernels=10, max_warps=10, max_events=12, n_bb=10, dup_p=0.8)
    h = tr.n_kernels // 2
    return tr, tg.trace_from_warps([_warps_of(tr, k) for k in range(h)], tr.bb_len,
                                   warps_total=tr.warps_total[:h]), \
        tg.trace_from_warps([_warps_of(tr, k) for k in range(h, tr.n_kernels)], tr.bb_len,
                            warps_total=tr.warps_total[h:])


@pytest.mark.parametrize("seed", range(4))
def test_pool_self_reuse(seed):
    _, a, _ = _split_runs(40 + seed)
    t, sig, mass = _pipeline(a)
    m, _ = oracle.match(t["kernel_type_off"], sig, mass, a.warps_total)
    pool = oracle.pool_export(t, a.warps_total, m)
    assert pool["n_pool"] == int((m < 0).sum()) and list(pool["kernel_id"]) == [k for k in range(a.n_kernels) if m[k] < 0]
    mp, dp = oracle.match_pooled(pool, t, a.warps_total)
    Kp = pool["n_pool"]
    cur = mp[Kp:]
    assert (mp[:Kp] < 0).all()  # pooled representatives stay representatives
    for k in range(a.n_kernels):
        if mass[k] == 0:
            assert cur[k] < 0  # N = 0 never matches [P-19]
            continue
        assert 0 <= cur[k] < Kp  # every kernel reuses a pooled representative
        if m[k] < 0:  # a representative finds its own copy (distance 0, equal warps, earliest such)
            assert cur[k] == list(pool["kernel_id"]).index(k) and dp[Kp + k] == 0.0


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("theta", [(1, 20), (1, 5)])
def test_pool_matches_bruteforce(seed, theta):
    _, a, b = _split_runs(60 + seed)
    ta, sa, ma_ = _pipeline(a)
    m_a, _ = oracle.match(ta["kernel_type_off"], sa, ma_, a.warps_total, theta=theta)
    pool = oracle.pool_export(ta, a.warps_total, m_a)
    tb, _, mb_ = _pipeline(b)
    mp, _ = oracle.match_pooled(pool, tb, b.warps_total, theta=theta)
    reps = [k for k in range(a.n_kernels) if m_a[k] < 0]
    vecs = [_frac_gpu_bbv(ta, k) for k in reps] + [_frac_gpu_bbv(tb, k) for k in range(b.n_kernels)]
    masses = [int(ma_[k]) for k in reps] + [int(x) for x in mb_]
    wt = [int(a.warps_total[k]) for k in reps] + [int(x) for x in b.warps_total]
    ref = _brute_resolve(vecs, masses, wt, Fraction(*theta), 64, 0)
    assert list(mp) == ref


# N2: full-BBV grouping (reading [N2-a]) and tagged ingest.  Pins: with B <= 16 and the identity fold the full BBV
# IS the projected one, so the types equal A2's; brute force on tiny traces (same type <=> equal event multisets,
# counts = class sizes, the row order rule recomputed); refinement of the projected grouping; ingest of a random
# order-preserving interleaving gives back the CSR.
def test_group_full_equals_projected_when_fold_is_identity():
    for tr in (tg.make_trace(1), tg.random_trace(5, n_kernels=4, max_warps=60, max_events=30, n_bb=16, dup_p=0.7)):
        p16, _, _ = oracle.bbv(tr, want_kbb=False)
        a, b = oracle.group(tr, p16), oracle.group_full(tr, p16)
        T = int(a["kernel_type_off"][-1])
        for f in ("warp_type", "kernel_type_off", "warp_sampling_ok"):
            assert np.array_equal(a[f], b[f]), f
        assert np.array_equal(a["type_key"][:T], b["type_key"])
        assert np.array_equal(a["type_count"][:T], b["type_count"])
        assert np.array_equal(a["type_first_warp"][:T], b["type_first_warp"])


@pytest.mark.parametrize("seed", range(4))
def test_group_full_bruteforce_and_refinement(seed):
    import collections
    tr = tg.random_trace(70 + seed, n_kernels=3, max_warps=40, max_events=10, n_bb=40, dup_p=0.7)
    p16, _, _ = oracle.bbv(tr, want_kbb=False)
    t = oracle.group_full(tr, p16)
    proj = oracle.group(tr, p16)
    kwo, weo = tr.kernel_warp_off, tr.warp_event_off
    for k in range(tr.n_kernels):
        ws = list(range(int(kwo[k]), int(kwo[k + 1])))
        ms = {w: collections.Counter(tr.bb[int(weo[w]):int(weo[w + 1])].tolist()) for w in ws}
        for a in ws:
            for b in ws:
                assert (t["warp_type"][a] == t["warp_type"][b]) == (ms[a] == ms[b])
                if ms[a] == ms[b]:
                    assert proj["warp_type"][a] == proj["warp_type"][b]  # refinement
        o = int(t["kernel_type_off"][k])
        n = int(t["kernel_type_off"][k + 1]) - o
        rows = []
        for r in range(n):
            mem = [w for w in ws if t["warp_type"][w] == r]
            assert int(t["type_count"][o + r]) == len(mem) and int(t["type_first_warp"][o + r]) == min(mem)
            assert np.array_equal(t["type_key"][o + r], p16[min(mem)])
            rows.append((-len(mem), tuple(int(x) for x in p16[min(mem)]), min(mem)))
        assert rows == sorted(rows)


def test_ingest_interleaved_stream():
    tr = tg.random_trace(9, n_kernels=3, max_warps=50, max_events=20, n_bb=30)
    rs = np.random.default_rng(9)
    W, weo = tr.n_warps, tr.warp_event_off.astype(np.int64)
    owner = np.repeat(np.arange(W), np.diff(weo))
    order = np.argsort(rs.random(len(owner)), kind="stable")  # a random interleaving ...
    order = np.concatenate([np.sort(order[owner[order] == w]) for w in range(W)])[np.argsort(
        np.concatenate([np.flatnonzero(owner[order] == w) for w in range(W)]), kind="stable")]  # ... keeping each warp's order
    warp, bb = owner[order], tr.bb[order]
    for w in range(W):  # the stream keeps each warp's event order
        assert np.array_equal(bb[warp == w], tr.bb[weo[w]:weo[w + 1]])
    out_bb, off = oracle.ingest(warp, bb, W)
    assert np.array_equal(off, tr.warp_event_off.astype(np.uint64)) and np.array_equal(out_bb, tr.bb)


# ---------------------------------------------------------------------------------------------------------------
# The all-cores CPU baseline (bench.py cpu_baseline): the same oracle functions over kernel ranges on host threads
# must give exactly analyse()'s tables and decisions.
@pytest.mark.parametrize("which", ["c6", "c4", "random"])
def test_analyse_threads_equals_analyse(which):
    if which == "random":
        tr = tg.random_trace(3, n_kernels=7, max_warps=300, max_events=60, n_bb=40)
    else:
        tr = tg.make_trace(6 if which == "c6" else 4)
    a = oracle.analyse(tr)
    for threads in (1, 3, 8):
        b = oracle.analyse_threads(tr, threads)
        for k in ("kernel_type_off", "type_key", "type_count", "type_first_warp", "warp_type", "warp_sampling_ok",
                  "sig", "mass", "match"):
            assert np.array_equal(np.asarray(a[k]), np.asarray(b[k])), (k, threads)
        assert np.array_equal(np.isinf(a["match_dist"]), np.isinf(b["match_dist"]))
        fin = np.isfinite(a["match_dist"])
        assert np.array_equal(a["match_dist"][fin], b["match_dist"][fin])
