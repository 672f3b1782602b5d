"""Sharded chain with the real libphoton backend on ONE GPU: G shards run in G threads (one libphoton context
each) and a thread-barrier "fake collective" stands in for NCCL (NCCL cannot put two ranks on one device).  The
merged results must be identical to the single-process oracle for every G."""
import threading

import numpy as np
import pytest

import oracle
import tracegen as tg

pytestmark = pytest.mark.gpu


class FakeComm:
    """all_gather / all_reduce across threads of one process (rank order preserved)."""

    def __init__(self, world, shared, rank):
        self.world, self.rank, self.s = world, rank, shared

    def _exchange(self, x):
        import torch
        torch.cuda.synchronize()  # the other threads read x on their own streams: it must be complete
        s = self.s
        s["slots"][self.rank] = x
        s["bar"].wait()
        vals = list(s["slots"])
        s["bar"].wait()
        return vals

    def _done(self):
        import torch
        torch.cuda.synchronize()

    def allgather_varlen(self, x):
        import torch
        vals = self._exchange(x)
        out = torch.cat(vals)
        self._done()
        self.s["bar"].wait()
        return out, [v.shape[0] for v in vals]

    def allreduce_sum(self, x):
        vals = self._exchange(x.clone())
        tot = vals[0].clone()
        for v in vals[1:]:
            tot += v
        x.copy_(tot)
        self._done()  # keep the slot tensors alive and read until every thread has summed them
        self.s["bar"].wait()
        return x


@pytest.mark.parametrize("cfg,world", [(6, 2), (6, 3), (1, 2), (3, 4)])
def test_sharded_gpu_matches_oracle(cfg, world):
    import torch
    from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon, to_numpy
    from paper_conf_micro_liusc23_b200.dist import ShardedAnalysis, shard_ranges
    g = tg.Generator(cfg)
    cuts = shard_ranges(g.warp_counts(), world)
    shared = {"slots": [None] * world, "bar": threading.Barrier(world)}
    results, errors = [None] * world, []

    def run(rank):
        try:
            torch.cuda.set_device(0)
            ph = Photon(0)
            tr = g.trace(int(cuts[rank]), int(cuts[rank + 1]))
            d = DeviceTrace.from_host(tr, ph.device)
            res = ShardedAnalysis(ph, g.n_kernels, g.kernel_warps, tr, d, comm=FakeComm(world, shared, rank)).run(
                check=True)
            torch.cuda.synchronize()
            results[rank] = {k: (to_numpy(v, np.uint64 if k in ("kernel_type_off", "type_count", "type_first_warp")
                                         else np.uint32 if k in ("type_key", "warp_type") else
                                         np.uint8 if k == "warp_sampling_ok" else np.int64))
                                 for k, v in res.items() if k in ("kernel_type_off", "type_key", "type_count",
                                                                  "type_first_warp", "warp_sampling_ok",
                                                                  "warp_type", "match")}
        except BaseException as e:  # pragma: no cover - surfaced below
            errors.append(e)
            shared["bar"].abort()

    ths = [threading.Thread(target=run, args=(r,)) for r in range(world)]
    for t in ths:
        t.start()
    for t in ths:
        t.join()
    if errors:
        raise errors[0]
    ref = oracle.analyse(g.trace())
    T = int(ref["kernel_type_off"][-1])
    wt = np.concatenate([results[r]["warp_type"] for r in range(world)])
    assert np.array_equal(wt, ref["warp_type"])
    for r in range(world):
        x = results[r]
        assert np.array_equal(x["kernel_type_off"], ref["kernel_type_off"])
        assert np.array_equal(x["type_key"].reshape(-1, 16)[:T], ref["type_key"])
        assert np.array_equal(x["type_count"][:T], ref["type_count"])
        assert np.array_equal(x["type_first_warp"][:T], ref["type_first_warp"])
        assert np.array_equal(x["warp_sampling_ok"], ref["warp_sampling_ok"])
        assert np.array_equal(x["match"], ref["match"])
