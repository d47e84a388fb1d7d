"""Two ranks on one GPU through the product path (probe whether NCCL accepts it)."""
import os
import sys
import numpy as np
import torch
import torch.distributed as dist
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "."))
from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig

rank = int(os.environ["RANK"]); ws = int(os.environ["WORLD_SIZE"])
torch.cuda.set_device(0)
dist.init_process_group("gloo")
n = (24, 20, 16)
cfg = HydroConfig(n=n, ndom=(2, 1, 1), nranks=ws, rank=rank, device=0)
try:
    h = Hydro(cfg)
    info = h.step(10)
    f = h.fields(["x", "e", "rho"])
    print(rank, "ok", info, float(f["e"].sum()), flush=True)
except Exception as ex:
    print(rank, "FAILED", ex, flush=True)
dist.destroy_process_group()
