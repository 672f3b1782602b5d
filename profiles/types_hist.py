import os, sys; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, tracegen as tg
from paper_conf_micro_liusc23_b200 import DeviceTrace, Photon
ph=Photon(0); d=DeviceTrace.from_host(tg.Generator(5).trace(), ph.device)
r=ph.analyse(d)
kto=r["kernel_type_off"].cpu().numpy().view(np.uint64).astype(np.int64)
t=np.diff(kto)
print("K",len(t),"T",kto[-1],"hist", np.histogram(t,[0,1,2,4,8,16,32,64,128,256,4096,10**9]))
