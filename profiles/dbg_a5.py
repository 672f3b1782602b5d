import sys; sys.path.insert(0, '/root/repo'); sys.path.insert(0, '.')
import numpy as np, tracegen as tg, oracle
from paper_conf_micro_liusc23_b200 import Photon, DeviceTiming, to_device, to_numpy
ph = Photon(0)
g = tg.Generator(2)
for k0, k1 in [(19, 20), (18, 20), (10, 20), (0, 20)]:
    tm = g.timing(k0, k1); _, _, kbb = oracle.bbv(g.kernels_trace(k0, k1))
    o = ph.photon_bb_stable(DeviceTiming.from_host(tm, ph.device), to_device(kbb, ph.device), 2048)
    fs, ds, sw = oracle.stable(tm, kbb, 2048)
    gfs = to_numpy(o["first_stable"], np.int64).reshape(fs.shape)
    bad = np.argwhere(gfs != fs)
    print(k0, k1, "records", tm.n_records, "mismatch", len(bad), bad[:5].tolist(), flush=True)
