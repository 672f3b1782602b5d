"""The seeded input generator: determinism, shard/sample independence, workload shapes (CPU only)."""
import numpy as np
import pytest

import tracegen as tg


def test_deterministic_and_seeded():
    a = tg.make_trace(6)
    b = tg.make_trace(6)
    c = tg.make_trace(6, seed=99)
    assert np.array_equal(a.bb, b.bb) and np.array_equal(a.warp_event_off, b.warp_event_off)
    assert not (len(a.bb) == len(c.bb) and np.array_equal(a.bb, c.bb))


@pytest.mark.parametrize("cfg", [1, 2, 6])
def test_shards_are_slices_of_the_whole(cfg):
    g = tg.Generator(cfg)
    full = g.trace(0, min(g.n_warps, 200000))
    cuts = tg.shard_bounds(g.warp_counts(0, full.n_warps), 3)
    for s in range(3):
        sh = g.trace(int(cuts[s]), int(cuts[s + 1]))
        e0, e1 = int(full.warp_event_off[cuts[s]]), int(full.warp_event_off[cuts[s + 1]])
        assert np.array_equal(sh.bb, full.bb[e0:e1])
        assert np.array_equal(sh.warp_event_off, full.warp_event_off[cuts[s]:cuts[s + 1] + 1] - e0)
        assert sh.warp_base == cuts[s]


def test_sample_every_100th_warp():
    g = tg.Generator(6)
    full = g.trace()
    smp = g.trace(0, g.n_warps, step=100)
    assert smp.n_warps == (g.n_warps + 99) // 100
    for i in range(smp.n_warps):
        w = 100 * i
        assert np.array_equal(smp.bb[int(smp.warp_event_off[i]):int(smp.warp_event_off[i + 1])],
                              full.bb[int(full.warp_event_off[w]):int(full.warp_event_off[w + 1])])
    assert smp.n_kernels == full.n_kernels and int(smp.kernel_warp_off[-1]) == smp.n_warps
    assert np.array_equal(smp.warps_total, full.warps_total)


def test_config_shapes():
    c1 = tg.make_trace(1)
    assert c1.n_kernels == 1 and c1.n_warps == 1024 and c1.n_bb == 16 and abs(c1.n_events - 1.05e6) < 0.05e6
    g2 = tg.Generator(2)
    assert g2.n_kernels == 20 and g2.n_warps == 20 * 65536 and g2.n_bb == 11
    g3 = tg.Generator(3)
    assert g3.n_kernels == 51 and 1.5e6 < g3.n_warps < 2e6
    g4 = tg.Generator(4)
    assert 400 < g4.n_kernels < 430
    g5 = tg.Generator(5)
    assert g5.n_kernels == 10000 and g5.n_bb == 4096
    wk = g5.kernel_warps
    assert wk.min() >= 32 and wk.max() <= 8192 and 0.08 < (wk < 64).mean() < 0.18


def test_timing_sorted_and_shaped():
    g = tg.Generator(6)
    tm = g.timing(0, 5)
    tr = g.kernels_trace(0, 5)
    assert tm.n_records == tr.n_events
    for k in range(tm.n_kernels):
        a, b = int(tm.kernel_rec_off[k]), int(tm.kernel_rec_off[k + 1])
        assert (np.diff(tm.retire[a:b].astype(np.int64)) >= 0).all()
        assert (tm.retire[a:b] >= tm.issue[a:b]).all()
        # same multiset of BB ids as the functional trace of the kernel
        w0, w1 = int(tr.kernel_warp_off[k]), int(tr.kernel_warp_off[k + 1])
        ev = tr.bb[int(tr.warp_event_off[w0]):int(tr.warp_event_off[w1])]
        assert np.array_equal(np.sort(ev), np.sort(tm.bb[a:b]))
