"""CPU stand-in for libphoton in the multi-process tests of paper_conf_micro_liusc23_b200.dist (test code only).

It implements the backend calls ShardedAnalysis makes with plain numpy / the CPU oracle, so the driver's host
logic (shard cuts, kernel ownership, triangle ranges, fixed-capacity padded all-gathers, the all-reduce merge,
kernel-sharded A5) runs for real over gloo on CPU and is checked against the single-process oracle.  Exported rows use the 88-byte
photon_type_row layout of include/photon.h.
"""
from fractions import Fraction

import numpy as np
import torch

import oracle

ROW = np.dtype([("kernel", "<u4"), ("pad", "<u4"), ("key", "<u4", (16,)), ("count", "<u8"), ("first", "<u8")])
assert ROW.itemsize == 88


PAD64 = -1  # PHOTON_PAIR_PAD as int64


class NumpyBackend:
    """The fixed-capacity backend interface of dist.GpuBackend on CPU tensors ("device" = CPU)."""

    def zeros(self, n, dtype):
        return torch.zeros(max(int(n), 1), dtype=getattr(torch, dtype))

    def local_types(self, tr, check, out=None):
        p16, _, _ = oracle.bbv(tr, want_kbb=False)
        ty = oracle.group(tr, p16)
        ty["_p16"] = p16
        return ty

    def local_total(self, ty, K_local):
        return int(ty["kernel_type_off"][-1])

    def export(self, ty, tr, kernel_base, warp_base, rows, n_dev):
        T = int(ty["kernel_type_off"][-1])
        cap = int(rows.shape[0])
        rec = np.zeros(cap, ROW)
        rec["kernel"] = 0xFFFFFFFF  # PHOTON_ROW_PAD
        for k in range(tr.n_kernels):
            for r in range(int(ty["kernel_type_off"][k]), int(ty["kernel_type_off"][k + 1])):
                if r < cap:
                    rec[r] = (kernel_base + k, 0, ty["type_key"][r], ty["type_count"][r],
                              ty["type_first_warp"][r] + warp_base)
        rows.copy_(torch.from_numpy(rec.view(np.uint8).reshape(cap, 88).copy()))
        n_dev[0] = T

    def alloc_global(self, K, cap):
        return {}

    def merge(self, rows, n_rows, K, kernel_warps, g):
        rec = rows.numpy().reshape(-1).view(ROW)[:n_rows]
        acc = {}
        for x in rec:
            if int(x["kernel"]) == 0xFFFFFFFF:
                continue
            key = (int(x["kernel"]), tuple(int(v) for v in x["key"]))
            c, f = acc.get(key, (0, 1 << 62))
            acc[key] = (c + int(x["count"]), min(f, int(x["first"])))
        per = [[] for _ in range(K)]
        for (k, key), (c, f) in acc.items():
            per[k].append((-c, key, f))
        kto = [0]
        keys, counts, firsts, ok = [], [], [], []
        wk = kernel_warps.numpy().view(np.uint64)
        for k in range(K):
            per[k].sort()
            for negc, key, f in per[k]:
                keys.append(key)
                counts.append(-negc)
                firsts.append(f)
            kto.append(len(keys))
            c0 = -per[k][0][0] if per[k] else 0
            ok.append(1 if wk[k] > 0 and 100 * c0 > 95 * int(wk[k]) else 0)
        g.update(kernel_type_off=np.array(kto, np.uint64), type_key=np.array(keys, np.uint32).reshape(-1, 16),
                 type_count=np.array(counts, np.uint64), type_first_warp=np.array(firsts, np.uint64),
                 warp_sampling_ok=np.array(ok, np.uint8))
        return g

    def remap(self, tr, ty_local, g, kernel_base, K, out):
        index = {}
        for k in range(K):
            for r in range(int(g["kernel_type_off"][k]), int(g["kernel_type_off"][k + 1])):
                index[(k, tuple(int(v) for v in g["type_key"][r]))] = r - int(g["kernel_type_off"][k])
        p16 = ty_local["_p16"]
        for kl in range(tr.n_kernels):
            for w in range(int(tr.kernel_warp_off[kl]), int(tr.kernel_warp_off[kl + 1])):
                out[w] = index.get((kernel_base + kl, tuple(int(v) for v in p16[w])), -1)  # -1: rows dropped
        return out

    def pair_count(self, n_dev):
        return int(n_dev[0])

    def check(self, g, ty_local):
        pass

    def types_total(self, g, K):
        return int(g["kernel_type_off"][-1])

    def sig_build(self, g, K, k_lo, k_hi, sig, mass):
        kto = g["kernel_type_off"]
        sig.zero_()
        mass.zero_()  # other ranks' kernels: zero (the all-reduce sums the ranks' buffers)
        for k in range(k_lo, k_hi):
            for r in range(int(kto[k]), int(kto[k + 1])):
                v = g["type_key"][r].astype(np.int64) * int(g["type_count"][r])
                sig[16 * r:16 * r + 16] = torch.from_numpy(v)
                mass[k] += int(v.sum())

    @staticmethod
    def _dnum(g, sig, mass, k, r):
        kto = g["kernel_type_off"]
        a = sig[16 * int(kto[k]):16 * int(kto[k + 1])].tolist()
        b = sig[16 * int(kto[r]):16 * int(kto[r + 1])].tolist()
        L = max(len(a), len(b))
        a += [0] * (L - len(a))
        b += [0] * (L - len(b))
        Nk, Nr = int(mass[k]), int(mass[r])
        return sum(abs(x * Nr - y * Nk) for x, y in zip(a, b))

    def scan_overflow(self, g):
        return False

    def match_scan(self, g, K, sig, mass, warps_total, params, k_lo, k_hi, pairs, n_dev, ws_pairs=0):
        s, m = sig.numpy(), mass.numpy()
        wt = warps_total.numpy().view(np.uint64)
        out = []
        for k in range(k_lo, k_hi):
            for r in range(k):
                Nk, Nr = int(m[k]), int(m[r])
                if Nk == 0 or Nr == 0:
                    continue
                Wk, Wr = int(wt[k]), int(wt[r])
                if not (Wk == Wr or min(Wk, Wr) >= params.n_cores):
                    continue
                if params.theta_den * self._dnum(g, s, m, k, r) < params.theta_num * Nk * Nr:
                    out.append((k << 32) | r)
        pairs.fill_(PAD64)
        cap = int(pairs.shape[0])
        for i, p in enumerate(out[:cap]):
            pairs[i] = p
        n_dev[0] = len(out)

    def match_resolve(self, g, K, sig, mass, warps_total, params, pairs, match_out, dist_out):
        s, m = sig.numpy(), mass.numpy()
        wt = warps_total.numpy().view(np.uint64)
        cand = [[] for _ in range(K)]
        for p in pairs.tolist():
            if p == PAD64:
                continue
            cand[p >> 32].append(p & 0xFFFFFFFF)
        rep = [False] * K
        match = np.full(K, -1, np.int64)
        dist = np.full(K, np.inf)
        for k in range(K):
            best = None
            for r in sorted(cand[k]):
                if params.pool_all_prior or rep[r]:
                    c = (abs(int(wt[k]) - int(wt[r])), r)
                    best = c if best is None or c < best else best
            if best is None:
                rep[k] = True
                pool = [r for r in range(k) if (params.pool_all_prior or rep[r]) and int(m[r]) > 0]
                if int(m[k]) > 0 and pool:  # a representative: its minimum distance to the earlier pool
                    dist[k] = float(min(Fraction(self._dnum(g, s, m, k, r), int(m[k]) * int(m[r])) for r in pool))
            else:
                match[k] = best[1]
                dist[k] = float(Fraction(self._dnum(g, s, m, k, best[1]), int(m[k]) * int(m[best[1]])))
        match_out.copy_(torch.from_numpy(match))
        if dist_out is not None:
            dist_out.copy_(torch.from_numpy(dist))

    # A5 (kernel shards): the oracle on the rank's timing slice
    def stable(self, tm, kbb, n, delta, rate, out):
        K = tm.n_kernels
        fs, ds, sw = oracle.stable(tm, kbb.numpy().view(np.uint64).reshape(K, -1), n, delta, rate)
        out["first_stable"][:fs.size] = torch.from_numpy(fs.reshape(-1).copy())
        out["stable_dur_sum"][:ds.size] = torch.from_numpy(ds.reshape(-1).view(np.int64).copy())
        out["switch_at"][:K] = torch.from_numpy(sw.copy())
        return out

    def check_stable(self, out):
        pass
