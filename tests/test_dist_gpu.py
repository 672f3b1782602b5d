"""Sharded drivers with the real libphoton backend on ONE GPU.

1. G shards run in G threads (one libphoton context each) and a thread-barrier "fake collective" stands in for
   NCCL (NCCL cannot put two ranks on one device): the merged results of the chain (A1 -> A4) and of the
   kernel-sharded A5 must be identical to the single-process oracle for every G.
2. A real NCCL process group of world size 1: the whole per-rank step (kernels + NCCL collectives) captured in one
   CUDA graph per driver and replayed, with the same oracle comparison -- the graph-ready path bench.py times.
"""
import os
import socket
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
        self.s["bar"].wait()  # keep the slot tensors alive and read until every thread is done with them

    def allgather(self, out, x):
        import torch
        vals = self._exchange(x.reshape(-1))
        out.view(-1).copy_(torch.cat(vals))
        self._done()
        return out

    def allreduce_sum(self, x):
        vals = self._exchange(x.clone())
        tot = vals[0].clone()
        for v in vals[1:]:
            tot += v
        x.copy_(tot)
        self._done()
        return x

    def allreduce_max_host(self, v, like):
        import torch
        t = torch.tensor([int(v)], dtype=torch.int64, device=like.device)
        vals = self._exchange(t)
        m = max(int(u.item()) for u in vals)
        self._done()
        return m


_KEYS = {"kernel_type_off": np.uint64, "type_count": np.uint64, "type_first_warp": np.uint64,
         "type_key": np.uint32, "warp_type": np.uint32, "warp_sampling_ok": np.uint8, "match": np.int64}


def _host(res):
    from paper_conf_micro_liusc23_b200 import to_numpy
    return {k: to_numpy(res[k], dt) for k, dt in _KEYS.items()}


def _compare(ref, x, T):
    assert np.array_equal(x["kernel_type_off"], ref["kernel_type_off"])
    assert np.array_equal(x["type_key"].reshape(-1, 16)[:T], ref["type_key"])
    assert np.array_equal(x["type_count"][:T], ref["type_count"])
    assert np.array_equal(x["type_first_warp"][:T], ref["type_first_warp"])
    assert np.array_equal(x["warp_sampling_ok"], ref["warp_sampling_ok"])
    assert np.array_equal(x["match"], ref["match"])


@pytest.mark.parametrize("cfg,world", [(6, 2), (6, 3), (1, 2), (3, 4)])
def test_sharded_gpu_matches_oracle(cfg, world):
    import torch
    from paper_conf_micro_liusc23_b200 import DeviceTiming, DeviceTrace, Photon, to_device
    from paper_conf_micro_liusc23_b200.dist import ShardedAnalysis, ShardedStable, kernel_ranges, shard_ranges
    g = tg.Generator(cfg)
    cuts = shard_ranges(g.warp_counts(), world)
    tm_all = g.timing()
    kc = kernel_ranges(np.diff(tm_all.kernel_rec_off.astype(np.int64)), world)
    _, _, kbb_all = oracle.bbv(g.trace())
    shared = {"slots": [None] * world, "bar": threading.Barrier(world)}
    results, stab, errors = [None] * world, [None] * world, []

    def run(rank):
        try:
            torch.cuda.set_device(0)
            ph = Photon(0)
            tr = g.trace(int(cuts[rank]), int(cuts[rank + 1]))
            d = DeviceTrace.from_host(tr, ph.device)
            comm = FakeComm(world, shared, rank)
            res = ShardedAnalysis(ph, g.n_kernels, g.kernel_warps, tr, d, comm=comm).run(check=True)
            torch.cuda.synchronize()
            results[rank] = _host(res)
            k0, k1 = int(kc[rank]), int(kc[rank + 1])
            st = ShardedStable(ph, DeviceTiming.from_host(g.timing(k0, k1), ph.device, n_bb=g.n_bb),
                               to_device(np.ascontiguousarray(kbb_all[k0:k1].reshape(-1)), ph.device), kc, g.n_bb,
                               comm=comm)
            st.step()
            st.check()
            stab[rank] = [t.cpu().numpy() for t in st.tables()]
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
    wt = np.concatenate([results[r]["warp_type"][:int(cuts[r + 1] - cuts[r])] for r in range(world)])
    assert np.array_equal(wt, ref["warp_type"])
    fs, ds, sw = oracle.stable(tm_all, kbb_all, 2048)
    for r in range(world):
        _compare(ref, results[r], T)
        assert np.array_equal(stab[r][0], fs.reshape(-1))
        assert np.array_equal(stab[r][1].view(np.uint64), ds.reshape(-1))
        assert np.array_equal(stab[r][2], sw)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.fixture(scope="module")
def nccl1():
    import torch
    import torch.distributed as dist
    torch.cuda.set_device(0)
    if not dist.is_initialized():
        dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{_free_port()}", rank=0, world_size=1,
                                device_id=torch.device("cuda", 0))
    yield
    dist.destroy_process_group()


@pytest.mark.parametrize("cfg", [6, 3])
def test_sharded_step_cuda_graph_nccl(nccl1, cfg):
    """plan() once, then the step captured in one CUDA graph (kernels + NCCL collectives) and replayed 3 times:
    identical to the oracle, no capacity overflow, no latched device error."""
    import torch
    from paper_conf_micro_liusc23_b200 import DeviceTiming, DeviceTrace, Photon, to_device
    from paper_conf_micro_liusc23_b200.dist import ShardedAnalysis, ShardedStable
    g = tg.Generator(cfg)
    ph = Photon(0)
    tr = g.trace()
    d = DeviceTrace.from_host(tr, ph.device)
    sa = ShardedAnalysis(ph, g.n_kernels, g.kernel_warps, tr, d).plan()
    graph = sa.capture()
    for _ in range(3):
        graph.replay()
    torch.cuda.synchronize()
    sa.check()
    ref = oracle.analyse(tr)
    x = _host(sa.result)
    _compare(ref, x, int(ref["kernel_type_off"][-1]))
    assert np.array_equal(x["warp_type"][:tr.n_warps], ref["warp_type"])
    tm = g.timing()
    _, _, kbb = oracle.bbv(tr)
    st = ShardedStable(ph, DeviceTiming.from_host(tm, ph.device), to_device(np.ascontiguousarray(kbb.reshape(-1)),
                                                                            ph.device),
                       np.array([0, g.n_kernels]), g.n_bb).plan()
    gs = st.capture()
    gs.replay()
    torch.cuda.synchronize()
    st.check()
    fs, ds, sw = oracle.stable(tm, kbb, 2048)
    a, b, c = (t.cpu().numpy() for t in st.tables())
    assert np.array_equal(a, fs.reshape(-1)) and np.array_equal(b.view(np.uint64), ds.reshape(-1))
    assert np.array_equal(c, sw)
