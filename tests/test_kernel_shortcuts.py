"""CPU checks (no GPU) of the arithmetic shortcuts the CUDA path takes where it does not follow the oracle's steps
literally -- each restated here in numpy and compared with the plain definition on random inputs:

* the pair filter's band order (k_match.cu): with f(q) = sum of bins 0-7 minus bins 8-15 of the u8 profile,
  |f(k) - f(r)| <= sum_j |q_k[j] - q_r[j]|, so no pair the coarse test keeps is ever outside the band, and the
  tile skipping rule (smallest f of a k-block minus largest f of an r-block >= the threshold) drops only such pairs;
* the switch point (k_stable.cu k_switch): the least t_b with rate_den * acc(t_b) > rate_num * total over the
  stable BBs equals the binary search over t of the plain definition;
* A5's latched-record lookup (k_stable.cu locate_record): the r-th record of id b in a 64-record slice found from
  two records per lane and a scan of the per-lane match counts equals the plain walk.
These pin the kernels' reasoning, not the kernels (their outputs are compared with the oracle by the -m gpu
tests)."""
import numpy as np
import pytest


def band_f(q):
    return q[..., :8].sum(-1).astype(np.int64) - q[..., 8:].sum(-1).astype(np.int64)


@pytest.mark.parametrize("seed", range(4))
def test_band_projection_bounds_the_coarse_distance(seed):
    rng = np.random.default_rng(seed)
    K = 300
    # profiles clustered like C5's programs: a few centres plus noise, quantised to u8 with unit mass
    centres = rng.dirichlet(np.ones(16), size=8)
    P = centres[rng.integers(0, 8, K)] + rng.normal(0, 0.01, (K, 16)).clip(-0.005, None)
    P = np.abs(P)
    P /= P.sum(1, keepdims=True)
    q = np.rint(P * 255).astype(np.int64)
    f = band_f(q)
    sad = np.abs(q[:, None, :] - q[None, :, :]).sum(-1)
    assert np.all(np.abs(f[:, None] - f[None, :]) <= sad)
    for theta in (1 / 100, 1 / 20, 1 / 10, 1 / 5):
        thr8 = int(np.ceil(255 * theta + 17))
        order = np.argsort(f, kind="stable")
        fs = f[order]
        FT = 16  # small tiles so the test has many
        nb = (K + FT - 1) // FT
        kept_by_tiles = np.zeros((K, K), bool)
        for kb in range(nb):
            fmin = fs[kb * FT]
            for rb in range(kb + 1):
                last = min(rb * FT + FT - 1, K - 1)
                if not fs[last] > fmin - thr8:  # skipped tile
                    continue
                for i in range(kb * FT, min(kb * FT + FT, K)):
                    for j in range(rb * FT, min(rb * FT + FT, K)):
                        if j < i:
                            kept_by_tiles[order[i], order[j]] = kept_by_tiles[order[j], order[i]] = True
        coarse = sad < thr8
        np.fill_diagonal(coarse, False)
        assert not np.any(coarse & ~kept_by_tiles)  # every coarse survivor lies in an enumerated tile


def switch_plain(fs, w, rnum, rden):
    """PAPER.md L208-210 [P-14] by the definition: least t with rden * acc(t) > rnum * total (binary search)."""
    total = int(w.sum())
    st = fs >= 0
    if total == 0 or not rden * int(w[st].sum()) > rnum * total:
        return -1
    lo, hi = 0, int(fs.max())
    while lo < hi:
        mid = (lo + hi) // 2
        acc = int(w[st & (fs <= mid)].sum())
        if rden * acc > rnum * total:
            hi = mid
        else:
            lo = mid + 1
    return lo


def switch_compacted(fs, w, rnum, rden):
    total = int(w.sum())
    st = np.flatnonzero(fs >= 0)
    if total == 0 or not rden * int(w[st].sum()) > rnum * total:
        return -1
    best = None
    for i in st:
        acc = int(w[st][fs[st] <= fs[i]].sum())
        if rden * acc > rnum * total and (best is None or fs[i] < best):
            best = int(fs[i])
    return best


@pytest.mark.parametrize("seed", range(6))
def test_switch_by_compacted_list_equals_the_binary_search(seed):
    rng = np.random.default_rng(100 + seed)
    for _ in range(200):
        B = int(rng.integers(1, 40))
        n_st = int(rng.integers(0, B + 1))
        fs = np.full(B, -1, np.int64)
        pos = rng.choice(10_000, size=n_st, replace=False)  # one record each: distinct positions
        fs[rng.choice(B, size=n_st, replace=False)] = pos
        w = rng.integers(0, 1000, B).astype(np.int64)
        if rng.random() < 0.2:
            w[:] = 0
        assert switch_compacted(fs, w, 95, 100) == switch_plain(fs, w, 95, 100)


@pytest.mark.parametrize("seed", range(4))
def test_slice_rank_lookup_equals_the_walk(seed):
    rng = np.random.default_rng(200 + seed)
    for _ in range(300):
        ids = rng.integers(0, 5, 64)
        b = int(rng.integers(0, 5))
        matches = np.flatnonzero(ids == b)
        if len(matches) == 0:
            continue
        r = int(rng.integers(0, len(matches)))
        walk = int(matches[r])
        # two records per lane, an exclusive scan of the lanes' match counts, the lane holding the r-th match
        m = (ids == b).reshape(32, 2).astype(np.int64)
        c2 = m.sum(1)
        ex2 = np.cumsum(c2) - c2
        lane = int(np.flatnonzero((r >= ex2) & (r < ex2 + c2))[0])
        got = 2 * lane + (0 if (r == ex2[lane] and m[lane, 0]) else 1)
        assert got == walk
