from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
for path in ("two",):
    h = Hydro(HydroConfig(n=(16,16,16), path=path, graph=False))
    print(path, h.step(2))
