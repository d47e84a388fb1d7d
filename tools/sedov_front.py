import sys; sys.path.insert(0, ".")
import numpy as np, time
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
t0=time.time()
with Hydro(HydroConfig(n=(448,448,448))) as h:
    c=0
    while c < 12000:
        h.step(500); c+=500
        b=h.box((0,0,0),(128,1,1), names=("u",))
        u=np.abs(b["u"][0,0,:]); front=int(np.nonzero(u)[0].max()) if u.any() else -1
        print(c, h.info()["t"], front, round(time.time()-t0,1), flush=True)
        if front > 75: break
