"""CPU stand-in for libphoton in the multi-process tests of paper_conf_micro_liusc23_b200.dist (test code only).

It implements the backend calls ShardedAnalysis makes with plain numpy / the CPU oracle, so the driver's host
logic (shard cuts, kernel ownership, triangle ranges, variable-length all-gathers, all-reduce merge) runs for
real over gloo on CPU and is checked against the single-process oracle.  Exported rows use the 88-byte
photon_type_row layout of include/photon.h.
"""
from fractions import Fraction

import numpy as np
import torch

import oracle

ROW = np.dtype([("kernel", "<u4"), ("pad", "<u4"), ("key", "<u4", (16,)), ("count", "<u8"), ("first", "<u8")])
assert ROW.itemsize == 88


class NumpyBackend:
    def local_rows(self, tr, kernel_base, warp_base, check):
        p16, _, _ = oracle.bbv(tr, want_kbb=False)
        ty = oracle.group(tr, p16)
        T = int(ty["kernel_type_off"][-1])
        rows = np.zeros(T, ROW)
        for k in range(tr.n_kernels):
            for r in range(int(ty["kernel_type_off"][k]), int(ty["kernel_type_off"][k + 1])):
                rows[r] = (kernel_base + k, 0, ty["type_key"][r], ty["type_count"][r],
                           ty["type_first_warp"][r] + warp_base)
        ty["_p16"] = p16
        return ty, torch.from_numpy(rows.view(np.uint8).reshape(T, 88).copy())

    def merge(self, rows, K, kernel_warps):
        rec = rows.numpy().reshape(-1).view(ROW) if rows.shape[0] else np.zeros(0, ROW)
        acc = {}
        for x in rec:
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
        return dict(kernel_type_off=np.array(kto, np.uint64), type_key=np.array(keys, np.uint32).reshape(-1, 16),
                    type_count=np.array(counts, np.uint64), type_first_warp=np.array(firsts, np.uint64),
                    warp_sampling_ok=np.array(ok, np.uint8))

    def remap(self, tr, ty_local, g, kernel_base, K):
        index = {}
        for k in range(K):
            for r in range(int(g["kernel_type_off"][k]), int(g["kernel_type_off"][k + 1])):
                index[(k, tuple(int(v) for v in g["type_key"][r]))] = r - int(g["kernel_type_off"][k])
        out = np.zeros(tr.n_warps, np.uint32)
        p16 = ty_local["_p16"]
        for kl in range(tr.n_kernels):
            for w in range(int(tr.kernel_warp_off[kl]), int(tr.kernel_warp_off[kl + 1])):
                out[w] = index[(kernel_base + kl, tuple(int(v) for v in p16[w]))]
        return out

    def types_total(self, g, K):
        return int(g["kernel_type_off"][-1])

    def sig_build(self, g, K, T, k_lo, k_hi):
        kto = g["kernel_type_off"]
        sig = np.zeros(16 * max(T, 1), np.int64)
        mass = np.zeros(K, np.int64)
        for k in range(k_lo, k_hi):
            for r in range(int(kto[k]), int(kto[k + 1])):
                v = g["type_key"][r].astype(np.int64) * int(g["type_count"][r])
                sig[16 * r:16 * r + 16] = v
                mass[k] += int(v.sum())
        return torch.from_numpy(sig), torch.from_numpy(mass)

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

    def match_scan(self, g, K, sig, mass, warps_total, params, k_lo, k_hi, cap):
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
        if len(out) > cap:
            return None
        return torch.tensor(out, dtype=torch.int64)

    def match_resolve(self, g, K, sig, mass, warps_total, params, pairs):
        s, m = sig.numpy(), mass.numpy()
        wt = warps_total.numpy().view(np.uint64)
        cand = [[] for _ in range(K)]
        for p in pairs.tolist():
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
        return torch.from_numpy(match), torch.from_numpy(dist)
