import sys, time
sys.path.insert(0, '/root/repo')
import torch
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
for hg in (0.03, 0.0):
    for ncyc in (200, 1313, 100000):
        with Hydro(HydroConfig(n=(128,)*3, t_stop=0.3, hg_coef=hg)) as h:
            h.step(1); torch.cuda.synchronize()
            t0 = time.perf_counter(); info = h.step(ncyc); el = time.perf_counter() - t0
        print(hg, ncyc, info["cycle"], info["status"], round(el, 3), flush=True)
