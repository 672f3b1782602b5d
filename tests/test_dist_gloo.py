"""Multi-process (world_size 2, 3 and 4, gloo on CPU) tests of the sharded drivers' host logic (dist.py).

The compute is the numpy stand-in (tests/dist_numpy_backend.py); what is under test is the driver: shard cuts at
warp boundaries (a kernel may straddle shards), kernel ownership for the signature all-reduce, triangle ranges
for the pair scan, the fixed-capacity padded all-gathers (row and pair padding skipped by the merge and the
resolution; capacity overflow detected and re-planned), and the kernel-sharded A5 with its output all-gather and
the straddling-kernel completion of kernel_bb_insts.  Every rank's result must equal the single-process oracle
on the whole trace.
"""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _prefix(g, max_warps=3000):
    W = min(g.n_warps, max_warps)
    kmax = int(np.searchsorted(g.kwoff, W, side="right")) - 1  # whole kernels only
    return kmax, int(g.kwoff[kmax])


def _worker(rank, world, port, cfg, theta, out_dir, tight):
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import tracegen as tg
    from dist_numpy_backend import NumpyBackend
    from paper_conf_micro_liusc23_b200.dist import (CapacityOverflow, Comm, ShardedAnalysis, ShardedStable,
                                                    complete_kbb, kernel_ranges, shard_ranges)
    import oracle
    g = tg.Generator(cfg)
    kmax, W = _prefix(g)
    counts = g.warp_counts(0, W)
    cuts = shard_ranges(counts, world)
    tr = g.trace(int(cuts[rank]), int(cuts[rank + 1]))
    comm = Comm()
    sa = ShardedAnalysis(NumpyBackend(), kmax, g.kernel_warps[:kmax], tr, tr, theta=theta, comm=comm,
                         kernel_warp_off_global=g.kwoff[:kmax + 1], want_dist=True)
    overflowed = 0
    if tight:  # capacities too small on purpose: check() must detect it on every rank, run() must re-plan
        sa.plan(row_cap=1, pair_cap=1)
        sa.step()
        try:
            sa.check()
        except CapacityOverflow:
            overflowed = 1
        sa.buf = None
    res = sa.run(check=True)
    # A5 (kernel shards by records) on the same kernels
    tm_all = g.timing(0, kmax)
    rec = np.diff(tm_all.kernel_rec_off.astype(np.int64))
    kc = kernel_ranges(rec, world)
    k0, k1 = int(kc[rank]), int(kc[rank + 1])
    _, _, kbb_all = oracle.bbv(g.kernels_trace(0, kmax))
    kbb = torch.from_numpy(kbb_all[k0:k1].reshape(-1).view(np.int64).copy())
    st = ShardedStable(NumpyBackend(), g.timing(k0, k1), kbb, kc, g.n_bb, n=64, comm=comm)
    st.step()
    fs, ds, sw = st.tables()
    # kernel_bb_insts of owned kernels from the warp shard's partial rows (straddling kernels completed)
    _, _, kbb_loc = oracle.bbv(tr)
    kl = complete_kbb(torch.from_numpy(kbb_loc.reshape(-1).view(np.int64).copy()), tr.n_kernels, g.n_bb,
                      int(tr.kernel_base), sa.own, comm)
    np.savez(os.path.join(out_dir, f"r{rank}.npz"), kto=res["kernel_type_off"], key=res["type_key"],
             count=res["type_count"], first=res["type_first_warp"], ok=res["warp_sampling_ok"],
             match=res["match"].numpy(), dist=res["match_dist"].numpy(), wt=res["warp_type"].numpy(),
             w0=cuts[rank], w1=cuts[rank + 1], over=overflowed, fs=fs.numpy(), ds=ds.numpy(), sw=sw.numpy(),
             own=np.array(sa.own), kbb_own=kl.numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg,theta,tight", [(2, 6, (1, 20), False), (3, 6, (1, 5), True),
                                                   (4, 6, (1, 20), False), (2, 1, (1, 20), True),
                                                   (4, 1, (1, 5), False)])
def test_sharded_chain_matches_oracle(tmp_path, world, cfg, theta, tight):
    import oracle
    import tracegen as tg
    mp.spawn(_worker, args=(world, _free_port(), cfg, theta, str(tmp_path), tight), nprocs=world, join=True)
    g = tg.Generator(cfg)
    kmax, W = _prefix(g)
    tr = g.kernels_trace(0, kmax)
    ref = oracle.analyse(tr, theta=theta)
    T = int(ref["kernel_type_off"][-1])
    p16, _, kbb = oracle.bbv(tr)
    fs, ds, sw = oracle.stable(g.timing(0, kmax), kbb, 64)
    wt = np.zeros(tr.n_warps, np.uint32)
    for r in range(world):
        z = np.load(tmp_path / f"r{r}.npz")
        assert np.array_equal(z["kto"], ref["kernel_type_off"])
        assert np.array_equal(z["key"][:T], ref["type_key"])
        assert np.array_equal(z["count"][:T], ref["type_count"])
        assert np.array_equal(z["first"][:T], ref["type_first_warp"])
        assert np.array_equal(z["ok"], ref["warp_sampling_ok"])
        assert np.array_equal(z["match"], ref["match"])
        assert np.array_equal(z["dist"], ref["match_dist"])
        assert int(z["over"]) == int(tight)
        wt[int(z["w0"]):int(z["w1"])] = z["wt"][:int(z["w1"]) - int(z["w0"])]
        assert np.array_equal(z["fs"], fs.reshape(-1)) and np.array_equal(z["ds"].view(np.uint64), ds.reshape(-1))
        assert np.array_equal(z["sw"], sw)
        lo, hi = z["own"]
        assert np.array_equal(z["kbb_own"].view(np.uint64), kbb[lo:hi].reshape(-1))
    assert np.array_equal(wt, ref["warp_type"])


def test_partition_helpers():
    from paper_conf_micro_liusc23_b200.dist import kernel_ranges, owned_kernels, shard_ranges, triangle_range
    counts = np.array([5, 0, 7, 1, 1, 30, 2, 2], np.uint64)
    cuts = shard_ranges(counts, 3)
    assert cuts[0] == 0 and cuts[-1] == len(counts) and (np.diff(cuts) >= 0).all()
    kwo = np.array([0, 2, 2, 5, 8], np.uint64)  # kernel 1 empty
    owners = [owned_kernels(kwo, int(cuts[r]), int(cuts[r + 1]), r == 2) for r in range(3)]
    covered = sorted(k for lo, hi in owners for k in range(lo, hi))
    assert covered == list(range(4))  # every kernel owned exactly once
    K = 1000
    rng = [triangle_range(K, r, 8) for r in range(8)]
    assert rng[0][0] == 0 and rng[-1][1] == K and all(rng[i][1] == rng[i + 1][0] for i in range(7))
    work = [sum(range(lo, hi)) for lo, hi in rng]
    assert max(work) < 1.2 * (sum(work) / 8)
    kc = kernel_ranges(np.array([10, 0, 10, 10, 50, 5, 5], np.uint64), 4)
    assert kc[0] == 0 and kc[-1] == 7 and (np.diff(kc) >= 0).all()
