"""Paper shape sweeps on one B200 (Figs. 12-18).

The paper times the 3-D Sedov problem on meshes whose y and z sizes are fixed per figure while
one dimension is swept (Fig. 12: x = z = 320, y swept; Figs. 13-18: (y, z) in {240, 360, 480} x
{320, 160}, x swept), for its "Default" mode (one domain per GPU) and its MPS mode (four ranks,
i.e. four y-slab domains, per GPU).  Here each point runs the same mesh twice on one GPU: one
domain, and four y-slab domains (the intra-GPU halo copy standing in for MPS's four ranks;
DESIGN.md §12).  Zones are cubic (h = 1.2/128); timing as in bench.py (CUDA events around
`steps` graph-replayed cycles after `warmup` cycles).  One JSON line per run.

The paper's node has 4 GPUs.  Under torchrun (one process per GPU) the same mesh is split by the
hierarchical rule into one block per GPU ("Default") or four y-slabs per GPU
(MPS analogue), the halo crosses GPUs through the peer transport, the time is the max over
ranks and rank 0 prints:

    python tools/shape_sweep.py [--figs 12,13,...] [--steps 20] [--max-zones 4.1e7]
    torchrun --nproc-per-node 4 --master-addr 127.0.0.1 tools/shape_sweep.py --figs 12
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

# figure -> (swept axis, fixed sizes of the other two axes, swept values)
FIGS = {
    12: ("y", {"x": 320, "z": 320}, [32, 64, 128, 192, 256, 320, 400]),
    13: ("x", {"y": 240, "z": 320}, [32, 64, 128, 256, 384, 512]),
    14: ("x", {"y": 240, "z": 160}, [32, 64, 128, 256, 512, 768, 1024]),
    15: ("x", {"y": 360, "z": 320}, [32, 64, 128, 256, 352]),
    16: ("x", {"y": 360, "z": 160}, [32, 64, 128, 256, 512, 704]),
    17: ("x", {"y": 480, "z": 320}, [32, 64, 128, 256]),
    18: ("x", {"y": 480, "z": 160}, [32, 64, 128, 256, 512]),
}


def run_point(n, dpg, steps, warmup, ngpu=1, rank=0, local=0, dist=None):
    import torch
    from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig, decompose_hierarchical
    h = 1.2 / 128
    ndom, cuts, d2r = decompose_hierarchical(n, ngpu, dpg)
    cfg = HydroConfig(n=n, extent=tuple(h * v for v in n), ndom=ndom, cuts=cuts,
                      dom_to_rank=d2r, rank=rank, nranks=ngpu, device=local, transport="peer")
    with Hydro(cfg) as hyd:
        stream = torch.cuda.current_stream()
        hyd.step(warmup, stream=stream.cuda_stream)
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        info = hyd.step(steps, stream=stream.cuda_stream)
        b.record(stream)
        torch.cuda.synchronize()
        ms = a.elapsed_time(b)
        if dist:
            t = torch.tensor([ms], device="cpu" if dist.get_backend() == "gloo" else "cuda")
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
        kt = hyd.time_kernels(min(steps, 10))
    zones = n[0] * n[1] * n[2]
    return {"zones": zones, "ms_per_cycle": ms / steps, "zone_cycles_per_s": zones * steps / (ms * 1e-3),
            "status": info["status"], "kernel_ms": kt}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--figs", default=",".join(str(k) for k in FIGS))
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--max-zones", type=float, default=4.1e7)
    args = ap.parse_args()
    import torch
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    share = os.environ.get("HYDRO_SHARE_GPU") == "1"  # testing: every rank on device 0 (gloo)
    if share:
        local = 0
    torch.cuda.set_device(local)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo" if share else "nccl")
    for fig in (int(f) for f in args.figs.split(",")):
        axis, fixed, values = FIGS[fig]
        for v in values:
            size = dict(fixed)
            size[axis] = v
            n = (size["x"], size["y"], size["z"])
            if n[0] * n[1] * n[2] > args.max_zones:
                continue
            for dpg in (1, 4):
                if n[1] < 4 * dpg * (2 if ws > 1 else 1):
                    continue
                r = run_point(n, dpg, args.steps, args.warmup, ws, rank, local, dist)
                r.update({"figure": fig, "swept": axis, "mesh": list(n), "gpus": ws,
                          "domains_per_gpu": dpg,
                          "mode": "1 domain/GPU (Default)" if dpg == 1
                          else "4 y-slab domains/GPU (MPS analogue)"})
                if rank == 0:
                    print(json.dumps(r), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
