"""Multi-process (world_size 2 and 3, gloo on CPU) tests of the sharded chain's host logic (dist.py).

The compute is the numpy stand-in (tests/dist_numpy_backend.py); what is under test is the driver: shard cuts at
warp boundaries (a kernel may straddle shards), kernel ownership for the signature all-reduce, triangle ranges
for the pair scan, and the variable-length all-gathers.  Every rank's merged result must equal the
single-process oracle on the whole trace, and the union of the ranks' warp types must equal the oracle's.
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


def _worker(rank, world, port, cfg, theta, out_dir):
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import tracegen as tg
    from dist_numpy_backend import NumpyBackend
    from paper_conf_micro_liusc23_b200.dist import Comm, ShardedAnalysis, shard_ranges
    g = tg.Generator(cfg)
    W = min(g.n_warps, 3000)
    kmax = int(np.searchsorted(g.kwoff, W, side="right")) - 1  # whole kernels only
    W = int(g.kwoff[kmax])
    counts = g.warp_counts(0, W)
    cuts = shard_ranges(counts, world)
    tr = g.trace(int(cuts[rank]), int(cuts[rank + 1]))
    res = ShardedAnalysis(NumpyBackend(), kmax, g.kernel_warps[:kmax], tr, tr, theta=theta, comm=Comm(),
                          kernel_warp_off_global=g.kwoff[:kmax + 1]).run()
    np.savez(os.path.join(out_dir, f"r{rank}.npz"), kto=res["kernel_type_off"], key=res["type_key"],
             count=res["type_count"], first=res["type_first_warp"], ok=res["warp_sampling_ok"],
             match=res["match"].numpy(), wt=res["warp_type"], w0=cuts[rank], w1=cuts[rank + 1])
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg,theta", [(2, 6, (1, 20)), (3, 6, (1, 5)), (2, 1, (1, 20))])
def test_sharded_chain_matches_oracle(tmp_path, world, cfg, theta):
    import oracle
    import tracegen as tg
    mp.spawn(_worker, args=(world, _free_port(), cfg, theta, str(tmp_path)), nprocs=world, join=True)
    g = tg.Generator(cfg)
    W = min(g.n_warps, 3000)
    kmax = int(np.searchsorted(g.kwoff, W, side="right")) - 1
    tr = g.kernels_trace(0, kmax)
    ref = oracle.analyse(tr, theta=theta)
    T = int(ref["kernel_type_off"][-1])
    wt = np.zeros(tr.n_warps, np.uint32)
    for r in range(world):
        z = np.load(tmp_path / f"r{r}.npz")
        assert np.array_equal(z["kto"], ref["kernel_type_off"])
        assert np.array_equal(z["key"][:T], ref["type_key"])
        assert np.array_equal(z["count"][:T], ref["type_count"])
        assert np.array_equal(z["first"][:T], ref["type_first_warp"])
        assert np.array_equal(z["ok"], ref["warp_sampling_ok"])
        assert np.array_equal(z["match"], ref["match"])
        wt[int(z["w0"]):int(z["w1"])] = z["wt"]
    assert np.array_equal(wt, ref["warp_type"])


def test_partition_helpers():
    from paper_conf_micro_liusc23_b200.dist import owned_kernels, shard_ranges, triangle_range
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
