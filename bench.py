"""Benchmark: zone-cycles/s of the fp64 Lagrangian hydro cycle (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config sedov512] [--impl ours|reference]

A "step" is one full cycle of the hot path (S1-S9: zone stage, node/energy stage, halo exchange,
dt reduction) over the whole mesh.  Default workload at every N: BASELINE.json configs[2],
"Sedov blast 3D 512^3 zones strong-scaled, 8 domains over 1/2/4/8 B200" (the configuration the
metric "zone-cycles/sec fp64 at 1/2/4/8 B200" is quoted on; 8 domains of 256^3 by the
hierarchical rule: 8 per GPU at N=1, 4 at N=2, ...).  The same JSON line
carries configs[3] (weak scaling, 384^3 per GPU as 4 y-slabs) as a second object, "weak384",
timed the same way in the same run.  Other BASELINE configs are selectable with --config.

value: zone-cycles/s over all ranks, device-timed with CUDA events on the launching stream,
max over ranks.  e2e: the same metric through the public API with host buffers (N=1:
hydro_run_batch, pinned host state in and out every step, copies overlapped with the cycles;
N>1: hydro_domain_unpack / hydro_domain_pack of each rank's own domains from / into pinned host
memory around the cycles).  roofline: the dominant kernel's algorithmic bytes / its mean
duration (hydro_time_kernels, CUDA events) against the measured HBM copy bandwidth.
selfcheck: a fresh context of the benchmarked configuration, 40 cycles, whose corner window
[0,48)^3 is compared with the oracle on a 48^3 box of the same zone size.
cpu_baseline / --impl reference: the oracle (test infrastructure) on the host cores, on a
bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

CONFIGS = {
    "sedov32": "Sedov blast 3D 32^3 zones, single domain, 100 cycles fp64",
    "sedov128": "Sedov blast 3D 128^3 zones, single domain on 1xB200",
    "sedov512": "Sedov blast 3D 512^3 zones strong-scaled, 8 domains over 1/2/4/8 B200 with "
                "NCCL halo exchange",
    "weak384": "weak scaling 384^3 zones per GPU, 1/2/4/8 B200 (multi-domain per GPU)",
    "uneven448": "unevenly sized domains 3D 448^3 total with weighted domain-to-GPU assignment "
                 "(paper's load-balance rule)",
}
METRIC = "zone-cycles/sec fp64 at 1/2/4/8 B200; % of HBM peak per kernel (ncu)"
UNIT = "zone-cycles/s"


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def hier(n, ngpu, dpg):
    from paper_conf_icppw_pearce18_b200 import decompose_hierarchical
    return decompose_hierarchical(n, ngpu, dpg)


def workload(name: str, ngpu: int):
    """Return (HydroConfig kwargs, scaling, description, zone size h)."""
    if name in ("sedov128", "sedov32"):
        base = 128 if name == "sedov128" else 32
        if ngpu == 1:
            return dict(n=(base,) * 3), "weak", CONFIGS[name], 1.2 / base
        ndom, cuts, d2r = hier((base, base, base), ngpu, 1)
        n = tuple(base * ndom[a] for a in range(3))
        ndom, cuts, d2r = hier(n, ngpu, 1)
        hb = 1.2 / base
        return (dict(n=n, extent=tuple(hb * v for v in n), ndom=ndom, cuts=cuts, dom_to_rank=d2r),
                "weak", f"Sedov blast 3D {base}^3 zones per GPU (weak), global {n}, {ngpu} domains",
                hb)
    if name == "sedov512":
        n = (512, 512, 512)
        ndom, cuts, d2r = hier(n, ngpu, 8 // ngpu) if ngpu in (1, 2, 4, 8) else hier(n, ngpu, 1)
        return dict(n=n, ndom=ndom, cuts=cuts, dom_to_rank=d2r), "strong", CONFIGS[name], 1.2 / 512
    if name == "weak384":
        gshape = {1: (1, 1, 1), 2: (2, 1, 1), 4: (2, 2, 1), 8: (2, 2, 2)}.get(ngpu)
        if gshape is None:
            raise SystemExit("weak384 is defined for 1/2/4/8 GPUs")
        n = tuple(384 * g for g in gshape)
        ndom, cuts, d2r = hier(n, ngpu, 4)
        hb = 1.2 / 384
        return (dict(n=n, extent=tuple(hb * v for v in n), ndom=ndom, cuts=cuts, dom_to_rank=d2r),
                "weak", CONFIGS[name], hb)
    if name == "uneven448":
        c = [0, 64, 160, 288, 448]
        return (dict(n=(448,) * 3, ndom=(4, 4, 4), cuts=[c, c, c]), "strong", CONFIGS[name],
                1.2 / 448)
    raise SystemExit(f"unknown config {name}")


class ClockSampler:
    """Samples SM clock and throttle reasons with NVML during the timed region."""

    def __init__(self, device: int):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml as N
            N.nvmlInit()
            self.N = N
            self.hdl = N.nvmlDeviceGetHandleByIndex(device)
            self.max_mhz = N.nvmlDeviceGetMaxClockInfo(self.hdl, N.NVML_CLOCK_SM)
        except Exception:
            self.N = None

    def _run(self):
        N = self.N
        names = {
            "gpu_idle": 0x1, "applications_clocks_setting": 0x2, "sw_power_cap": 0x4,
            "hw_slowdown": 0x8, "sync_boost": 0x10, "sw_thermal_slowdown": 0x20,
            "hw_thermal_slowdown": 0x40, "hw_power_brake_slowdown": 0x80,
        }
        while not self._stop.is_set():
            try:
                self.samples.append(N.nvmlDeviceGetClockInfo(self.hdl, N.NVML_CLOCK_SM))
                r = N.nvmlDeviceGetCurrentClocksEventReasons(self.hdl)
                for k, bit in names.items():
                    if r & bit and k != "gpu_idle":
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.N:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.N:
            self.t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                "samples": len(self.samples)}


def measured_peak_hbm():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return 6650.0, "fallback"


def fp64_peak():
    """Measured DFMA lane-op rate (profiles/r01_fp64_peak.txt, tools/fp64_peak.cu)."""
    return 1.708e13


def kernel_counters():
    """Per-kernel ncu counters at the headline config, 512^3 in 8 domains
    (profiles/kernel_counters.json, written by tools/ncu_summary.py from `ncu --set full`
    captures): DRAM bytes per owned zone and executed fp64 pipe instructions
    (DADD+DMUL+DFMA, thread level) per owned zone."""
    try:
        with open(os.path.join(ROOT, "profiles", "kernel_counters.json")) as f:
            return json.load(f)["kernels"]
    except Exception:
        return {}


KC = kernel_counters()
FP64_PER_ZONE = {"k_zone_stage": KC.get("k_zone_stage", {}).get("fp64_inst_per_zone")}
TRAFFIC_PER_ZONE = {k: v.get("dram_bytes_per_zone") for k, v in KC.items()}


def oracle_baseline(h, budget_s=12.0):
    """Time the oracle (as it stands) on a bounded sample of the workload on this host: a
    Sedov corner box of the workload's zone size (the per-zone cost is data-independent)."""
    import oracle
    from oracle import OracleConfig
    s = 96
    o = oracle.Oracle(OracleConfig(n=(s, s, s), extent=(h * s,) * 3))
    o.step(1)  # warm
    t0 = time.perf_counter()
    cycles = 0
    while True:
        o.step(1)
        cycles += 1
        el = time.perf_counter() - t0
        if el > budget_s or cycles >= 100:
            break
    o.close()
    return {"value": s ** 3 * cycles / el, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"Sedov {s}^3 corner box at the workload's zone size, {cycles} cycles "
                      f"single-threaded after 1 warm-up cycle ({el:.1f} s)"}


def _oracle_worker(h, seconds, q):
    import oracle
    from oracle import OracleConfig
    s = 64
    o = oracle.Oracle(OracleConfig(n=(s, s, s), extent=(h * s,) * 3))
    o.step(1)
    t0, cyc = time.perf_counter(), 0
    while time.perf_counter() - t0 < seconds:
        o.step(1)
        cyc += 1
    q.put(s ** 3 * cyc / (time.perf_counter() - t0))
    o.close()


def hetero_model(h, gpu_value, seconds=6.0):
    """SURVEY §8f row f3 (host cores computing thin slabs
    beside the GPUs, "up to 18 %"), not built; measured instead of modelled: one oracle process
    per host core runs concurrently (the paper's CPU-only mode, one domain per core), and the
    aggregate is what the host could add in the ideal case (no halo cost, perfect split)."""
    import multiprocessing as mp
    cores = len(os.sched_getaffinity(0))
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_oracle_worker, args=(h, seconds, q)) for _ in range(cores)]
    for p in ps:
        p.start()
    rates = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join()
    agg = sum(rates)
    return {"host_cores": cores, "all_cores_zone_cycles_per_s": agg,
            "per_core_mean": agg / cores, "gpu_value": gpu_value,
            "ideal_gain_frac": agg / gpu_value,
            "note": "row f3 not built: the paper's cooperative mode gains up to 18 percent on "
                    "K80/P100 nodes; here all host cores running the CPU reference concurrently "
                    f"(one 64^3 Sedov box per core, {seconds:.0f} s) could add this fraction of "
                    "the GPU's rate before any host<->device halo cost"}


def run_reference(args):
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    ngpu = max(ws, args.gpus)
    kw, scaling, desc, h = workload(args.config, ngpu)
    import oracle
    from oracle import OracleConfig
    n = kw["n"]
    zones = n[0] * n[1] * n[2]
    # bounded sample: the whole mesh if a step is cheap, else a 64^3 Sedov corner box of the
    # workload's zone size per step
    per_cycle_s = zones / 3.0e6
    # (the whole mesh only up to configs[1]'s 128^3: the oracle needs ~350 B of host memory per
    # zone, ~47 GB at 512^3)
    whole = zones <= 2_200_000 and per_cycle_s * (args.steps + args.warmup) < 150
    sample_n = n if whole else (64, 64, 64)
    sz = sample_n[0] * sample_n[1] * sample_n[2]
    o = oracle.Oracle(OracleConfig(n=sample_n, extent=kw.get("extent", (1.2,) * 3) if whole
                                   else (h * 64,) * 3))
    o.step(args.warmup)
    t0 = time.perf_counter()
    o.step(args.steps)
    el = time.perf_counter() - t0
    o.close()
    v = sz * args.steps / el
    line = {"metric": METRIC, "value": v, "unit": UNIT, "impl": "reference",
            # n_gpus: the N of this launch (the driver pairs the arms by N); the oracle itself
            # runs on rank 0's host cores only, as cpu_baseline / "device" say
            "n_gpus": ngpu, "device": "host cpu (oracle, rank 0 only)",
            "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1e3 * el / args.steps, "higher_is_better": True, "scaling": scaling,
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": desc, "sample": list(sample_n)},
            "cpu_baseline": {"value": v, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"Sedov {list(sample_n)} at the workload's zone size, "
                                       f"{args.steps} cycles per run"},
            "e2e": {"value": v, "unit": UNIT, "h2d_bytes_per_step": 0,
                    "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


class Run:
    """One benchmarked configuration on this rank (collective over ranks)."""

    def __init__(self, args, name, ngpu, rank, local, dist, share):
        from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
        self.args, self.name, self.ngpu, self.rank, self.dist, self.share = (
            args, name, ngpu, rank, dist, share)
        self.kw, self.scaling, self.desc, self.h = workload(name, ngpu)
        self.cfg = HydroConfig(rank=rank, nranks=ngpu, device=local, path=args.path,
                               transport=args.transport, hg_coef=args.hg, halo=args.halo,
                               q=args.q, **self.kw)
        self.Hydro, self.HydroConfig = Hydro, HydroConfig
        self.hyd = Hydro(self.cfg)
        n = self.kw["n"]
        self.zones = n[0] * n[1] * n[2]
        self.local = local

    def barrier(self):
        import torch
        if self.dist:
            self.dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(self, v, op="max"):
        if not self.dist:
            return v
        import torch
        t = torch.tensor([float(v)], dtype=torch.float64,
                         device="cpu" if self.share else "cuda")
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MAX if op == "max"
                             else self.dist.ReduceOp.SUM)
        return float(t.item())

    def timed(self):
        import torch
        args, hyd = self.args, self.hyd
        stream = torch.cuda.current_stream()
        sp = stream.cuda_stream
        hyd.step(args.warmup, stream=sp)
        self.barrier()
        start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ClockSampler(self.local) as clk:
            start.record(stream)
            info = hyd.step(args.steps, stream=sp)
            end.record(stream)
            torch.cuda.synchronize()
        ms = self.max_over_ranks(start.elapsed_time(end))
        self.barrier()
        if info["status"] != 0:
            raise SystemExit(f"{self.name}: run failed: {info}")
        self.ms = ms
        self.value = self.zones * args.steps / (ms * 1e-3)
        self.clocks = clk.summary()
        self.info = info
        return self.value

    def roofline(self):
        """Dominant kernel's algorithmic bytes per launch / its event-timed mean duration
        (DESIGN.md §9); exact per-domain node and zone counts of this rank."""
        from paper_conf_icppw_pearce18_b200 import layout_export
        args, rank = self.args, self.rank
        kt = self.hyd.time_kernels(min(args.steps, 50))
        self.kt = kt
        launches = self.hyd.kernels_per_cycle() * args.steps
        self.launches = int(self.max_over_ranks(launches, op="sum"))
        lay = layout_export(self.cfg)
        nd_all, nper = int(lay[1]), []
        for d in range(nd_all):
            w = lay[7 + 7 * d: 14 + 7 * d]
            if int(w[6]) == rank:
                nper.append((int(w[3]), int(w[4]), int(w[5])))
        nd_local = max(len(nper), 1)
        Nz = sum(a * b * c for a, b, c in nper) / nd_local
        Nn = sum((a + 1) * (b + 1) * (c + 1) for a, b, c in nper) / nd_local
        peak, peak_kind = measured_peak_hbm()
        kern = []
        if args.path == "two":
            zf = FP64_PER_ZONE.get("k_zone_stage")
            # the zone stage is one grouped launch over all local domains: per-domain mean
            kern.append(("k_zone_stage", kt["zone_stage_ms"], 48.0 * Nn + 24.0 * Nz,
                         zf * Nz if zf else None))
            kern.append(("k_node_energy", kt["node_stage_ms"], 96.0 * Nn + 32.0 * Nz, None))
        elif args.path == "one":
            kern.append(("k_cycle_fused", kt["cycle_kernel_ms"], 96.0 * Nn + 24.0 * Nz, None))
        else:
            kern.append((f"{args.path} zone+node+energy", kt["cycle_kernel_ms"],
                         96.0 * Nn + 24.0 * Nz, None))
        rows = []
        for name, kms, byts, flops in kern:
            hbm = byts / (kms * 1e-3) / 1e9
            r = {"kernel": name, "ms": kms, "alg_bytes": byts, "hbm_gbs": hbm,
                 "hbm_frac": hbm / peak}
            if flops:
                alu = flops / (kms * 1e-3)
                r.update({"fp64_inst_per_s": alu, "fp64_frac": alu / fp64_peak()})
            c = KC.get(name)
            if c:  # the same kernel under ncu at 512^3 (profiles/kernel_counters.json)
                r["ncu"] = {k: c.get(k) for k in ("fp64_pipe_pct", "smem_wavefronts_pct",
                                                  "issue_active", "dram_bytes_per_zone")}
            rows.append(r)
        dom = max(rows, key=lambda r: r["ms"])
        alu_bound = dom.get("fp64_frac", 0.0) > dom["hbm_frac"]
        return {"bound": "alu" if alu_bound else "hbm",
                "achieved": dom["fp64_inst_per_s"] / 1e12 if alu_bound else dom["hbm_gbs"],
                "peak": fp64_peak() / 1e12 if alu_bound else peak,
                "unit": "T fp64-inst/s" if alu_bound else "GB/s",
                "frac": dom["fp64_frac"] if alu_bound else dom["hbm_frac"],
                "traffic": (TRAFFIC_PER_ZONE[dom["kernel"]] * Nz
                            if TRAFFIC_PER_ZONE.get(dom["kernel"]) else None),
                "traffic_source": "ncu dram__bytes_read+write per zone at 512^3 / 8 domains "
                                  "(profiles/kernel_counters.json) x this launch's zones",
                "peak_source": ("measured DFMA rate (profiles/r01_fp64_peak.txt)" if alu_bound
                                else f"{peak_kind} MEASURED_PEAKS.json hbm_gbs"),
                "kernel": dom["kernel"], "kernel_ms": dom["ms"],
                "kernel_share_of_cycle": (dom["ms"] * nd_local / kt["cycle_ms"]
                                          if kt["cycle_ms"] else None),
                "domains_on_rank": nd_local,
                "alg_bytes_per_launch": dom["alg_bytes"], "kernels": rows}

    def e2e_single(self):
        """N=1: hydro_run_batch, one e2e step = H2D of the state from pinned host memory +
        e2e_cycles cycles + D2H of the result into pinned host memory; the copies of
        neighbouring steps overlap the cycles on two copy streams (wall clock around the call).
        Two output sets alternate (step b and b+2 share one: their copies are ordered on the
        same copy stream), so the pinned footprint is three copies of the state."""
        import torch
        args, hyd = self.args, self.hyd
        names = ("x", "y", "z", "u", "v", "w", "e")
        cur = hyd.fields(names)
        pin = lambda a: torch.from_numpy(a).pin_memory().numpy()  # noqa: E731
        pinned = {k: pin(v) for k, v in cur.items()}
        del cur
        outs = [{k: torch.empty(v.shape, dtype=torch.float64).pin_memory().numpy()
                 for k, v in pinned.items()} for _ in range(2)]
        inf0 = hyd.info()
        reps = args.e2e_steps
        hyd.run_batch([pinned] * 2, args.e2e_cycles, [inf0["t"]] * 2, [inf0["dt"]] * 2,
                      out=outs)  # untimed: staging allocation, first DMA into fresh pages
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        _, binfo = hyd.run_batch([pinned] * reps, args.e2e_cycles, [inf0["t"]] * reps,
                                 [inf0["dt"]] * reps, out=[outs[b % 2] for b in range(reps)])
        el = time.perf_counter() - t0
        if any(i["status"] != 0 for i in binfo):
            raise SystemExit(f"e2e run failed: {binfo}")
        h2d = sum(v.nbytes for v in pinned.values())
        d2h = sum(v.nbytes for v in outs[0].values())
        return {"value": self.zones * args.e2e_cycles * reps / el, "unit": UNIT,
                "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
                "cycles_per_step": args.e2e_cycles, "steps": reps,
                "api": "hydro_run_batch (C ABI) from / into pinned host arrays",
                "note": "per step: H2D of the global state x,y,z,u,v,w,e + cycles + D2H of "
                        "the result; copies of neighbouring steps overlapped with the cycles "
                        "(wall clock around the call)"}

    def e2e_ranks(self):
        """N>1: every rank moves exactly its own domains through the C ABI
        (hydro_domain_unpack from pinned host memory, e2e_cycles cycles, hydro_domain_pack into
        pinned host memory), synchronously, wall clock max over ranks."""
        import torch
        args, hyd = self.args, self.hyd
        from paper_conf_icppw_pearce18_b200 import dom_to_rank
        mine = [d for d, r in enumerate(dom_to_rank(self.cfg)) if r == self.rank]
        bufs = {d: torch.empty(hyd.domain_bytes(d), dtype=torch.uint8).pin_memory()
                for d in mine}
        outs = {d: torch.empty_like(b).pin_memory() for d, b in bufs.items()}
        for d in mine:
            hyd.pack_domain(d, out=bufs[d])  # the current state as the step input
        inf0 = hyd.info()
        reps = args.e2e_steps
        self.barrier()
        t0 = time.perf_counter()
        for _ in range(reps):
            for d in mine:
                hyd.unpack_domain(d, bufs[d])
            hyd.set_clock(inf0["t"], inf0["dt"], inf0["cycle"])
            info = hyd.step(args.e2e_cycles)
            for d in mine:
                hyd.pack_domain(d, out=outs[d])
        el = self.max_over_ranks(time.perf_counter() - t0)
        if info["status"] != 0:
            raise SystemExit(f"e2e run failed: {info}")
        nbytes = int(self.max_over_ranks(sum(b.numel() for b in bufs.values()), op="sum"))
        return {"value": self.zones * args.e2e_cycles * reps / el, "unit": UNIT,
                "h2d_bytes_per_step": nbytes, "d2h_bytes_per_step": nbytes,
                "cycles_per_step": args.e2e_cycles, "steps": reps,
                "api": "hydro_domain_unpack / hydro_step / hydro_domain_pack (C ABI), per rank",
                "note": "per step and rank: H2D of the rank's own domains (6 node arrays + e + m "
                        "incl. ghost layer) from pinned host memory, cycles, D2H into pinned "
                        "host memory; bytes summed over ranks; wall clock max over ranks"}

    def close(self):
        self.hyd.close()


def selfcheck(args, name, ngpu, rank, local, dist):
    """Correctness of the benchmarked configuration, in the same run: a fresh context, 40
    cycles, corner window [0,48)^3 against the oracle on a 48^3 Sedov box of the same zone size
    (the window evolves exactly like that box while the blast is inside it; the oracle never
    sees GPU output), plus a far box that must stay exactly at rest (tests/test_gpu_parity.py
    test_full_size_512_eight_domains_corner_window)."""
    import numpy as np
    from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig
    kw, _, _, h = workload(name, ngpu)
    cyc, w = 40, 48
    n = kw["n"]
    if min(n) < 2 * w:
        return None
    cfg = HydroConfig(rank=rank, nranks=ngpu, device=local, path=args.path,
                      transport=args.transport, hg_coef=args.hg, halo=args.halo, q=args.q, **kw)
    hyd = Hydro(cfg)
    info = hyd.step(cyc)
    win = hyd.box((0, 0, 0), (w, w, w))
    far = hyd.box((n[0] - 24, n[1] - 24, n[2] - 24), (n[0] - 8, n[1] - 8, n[2] - 8),
                  names=("u", "v", "w", "e"))
    hyd.close()
    if rank != 0:
        return None
    import oracle
    from oracle import OracleConfig
    fo, io = oracle.run(OracleConfig(n=(w, w, w), extent=(h * w,) * 3, hg_coef=args.hg, q=args.q),
                        cyc)
    inside = (np.abs(fo["u"][:, :, -4:]).max() == 0.0 and np.abs(fo["e"][:, :, -4:]).max() == 0.0)
    errs = {}
    for k in ("x", "y", "z", "u", "v", "w", "rho", "e", "p", "q", "c", "vol", "mass"):
        den = max(float(np.abs(fo[k]).max()), 1e-300)
        errs[k] = float(np.abs(win[k] - fo[k]).max()) / den
    worst = max(errs.values())
    rest = all(float(np.abs(far[k]).max()) == 0.0 for k in far)
    dt_err = abs(info["dt"] - io["dt"]) / io["dt"]
    ok = bool(inside and rest and worst <= 1e-10 and dt_err <= 1e-10 and info["status"] == 0)
    return {"pass": ok, "cycles": cyc, "window": [w, w, w], "max_rel_err": worst,
            "dt_rel_err": dt_err, "far_box_at_rest": rest, "blast_inside_window": bool(inside),
            "tolerance": 1e-10,
            "how": "fresh context of this configuration, 40 cycles; corner window vs the oracle "
                   "on a 48^3 box of the same zone size (R15 norm per field)"}


def nccl_leg(args, name, ngpu, rank, local, dist, share):
    """N>1 with the peer transport: 10 cycles of the same configuration with the NCCL transport
    (grouped send/recv halo + allreduce), compared bitwise with the peer run per local domain
    (hydro_domain_pack), so a multi-GPU driver run executes comm.cu.  A failure is reported in
    the line (the timed numbers stand); a stalled NCCL leg ends in HYDRO_ENCCL after
    HYDRO_NCCL_TIMEOUT_S (set to 120 s here; comm_wait polls ncclCommGetAsyncError)."""
    if ngpu < 2 or args.transport != "peer":
        return None
    if share:
        return {"ran": False, "why": "ranks share one GPU (HYDRO_SHARE_GPU): NCCL refuses"}
    os.environ.setdefault("HYDRO_NCCL_TIMEOUT_S", "120")
    try:
        return _nccl_vs_peer(args, workload(name, ngpu)[0], ngpu, rank, local, dist)
    except Exception as exc:
        return {"ran": True, "error": f"{type(exc).__name__}: {exc}"[:300]}


def _nccl_vs_peer(args, kw, ngpu, rank, local, dist):
    import torch
    from paper_conf_icppw_pearce18_b200 import Hydro, HydroConfig, dom_to_rank
    packs, infos, ms = {}, {}, {}
    for tr in ("peer", "nccl"):
        cfg = HydroConfig(rank=rank, nranks=ngpu, device=local, path=args.path, transport=tr,
                          hg_coef=args.hg, halo=args.halo, **kw)
        hyd = Hydro(cfg)
        hyd.step(2)
        torch.cuda.synchronize()
        dist.barrier()
        t0 = time.perf_counter()
        infos[tr] = hyd.step(10)
        ms[tr] = (time.perf_counter() - t0) * 1e3 / 10
        mine = [d for d, r in enumerate(dom_to_rank(cfg)) if r == rank]
        packs[tr] = {d: hyd.pack_domain(d).cpu() for d in mine}
        hyd.close()
    same = all(torch.equal(packs["peer"][d], packs["nccl"][d]) for d in packs["peer"])
    same = same and infos["peer"]["t"] == infos["nccl"]["t"]
    flag = torch.tensor([1.0 if same else 0.0], device="cuda")
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    return {"ran": True, "cycles": 12, "bitwise_equal_to_peer": bool(flag.item() == 1.0),
            "wall_ms_per_cycle": ms, "transport": "nccl (ncclSend/ncclRecv group + allreduce)"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="sedov512", choices=sorted(CONFIGS))
    ap.add_argument("--second", default="weak384",
                    help="second configuration timed in the same run ('' = none)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--path", default="two", choices=["two", "one", "split", "strict"],
                    help="two: zone + node/energy kernels; one: one fused kernel; split: plain; "
                         "strict: the split pipeline in the oracle's order without FMA (bitwise)")
    ap.add_argument("--transport", default="peer", choices=["peer", "nccl"],
                    help="N>1 halo/dt transport: CUDA IPC peer stores or NCCL send/recv + "
                         "allreduce (the other one is run as a 10-cycle bitwise check)")
    ap.add_argument("--hg", type=float, default=0.0,
                    help="viscous hourglass coefficient (SURVEY f1, reading R17)")
    ap.add_argument("--q", default="scalar", choices=["scalar", "monotone"],
                    help="artificial viscosity (reading R7 / R24; monotone: split kernels)")
    ap.add_argument("--halo", default="kernel", choices=["kernel", "fused"],
                    help="ghost-slab exchange: from the node/energy stage's epilogue (fused) or "
                         "separate copy / peer-push kernels after it")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-selfcheck", action="store_true")
    ap.add_argument("--e2e-cycles", type=int, default=100)
    ap.add_argument("--e2e-steps", type=int, default=5)
    args = ap.parse_args()
    if args.impl == "reference":
        return run_reference(args)
    args.warmup = max(args.warmup, 3)

    import torch

    ws, rank, local = dist_env()
    ngpu = max(ws, 1)
    # HYDRO_SHARE_GPU=1 (testing only): every rank on device 0, gloo for the host collectives
    share = os.environ.get("HYDRO_SHARE_GPU") == "1"
    if share:
        local = 0
    torch.cuda.set_device(local)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("gloo" if share else "nccl")

    run = Run(args, args.config, ngpu, rank, local, dist, share)
    value = run.timed()
    roof = run.roofline()
    e2e = run.e2e_single() if ngpu == 1 else run.e2e_ranks()
    line_cfg = {"workload": run.desc, "mesh": list(run.kw["n"]), "domains": list(run.cfg.ndom),
                "zones": run.zones, "path": args.path, "hg_coef": args.hg, "q": args.q,
                "halo": args.halo,
                "l2": "state > 126 MB L2 (inputs larger than L2; no flush)"
                if run.zones * 120 > 126e6 else "state fits L2",
                "parallelism": f"dp{ngpu} (spatial domains)",
                "transport": args.transport if ngpu > 1 else None}
    main_run = {"ms": run.ms, "clocks": run.clocks, "launches": run.launches, "kt": run.kt,
                "scaling": run.scaling}
    run.close()
    del run

    second = None
    if args.second and args.second != args.config:
        r2 = Run(args, args.second, ngpu, rank, local, dist, share)
        v2 = r2.timed()
        roof2 = r2.roofline()
        second = {"workload": r2.desc, "value": v2, "unit": UNIT,
                  "ms_per_step": r2.ms / args.steps,
                  "steps": args.steps, "warmup": args.warmup, "scaling": r2.scaling,
                  "mesh": list(r2.kw["n"]), "domains": list(r2.cfg.ndom), "zones": r2.zones,
                  "roofline": {k: roof2[k] for k in ("bound", "achieved", "peak", "unit", "frac",
                                                     "kernel", "kernel_ms")},
                  "clocks": r2.clocks, "gpu_launches": r2.launches, "kernel_ms": r2.kt}
        r2.close()
        del r2

    check = None if args.no_selfcheck else selfcheck(args, args.config, ngpu, rank, local, dist)
    nccl = nccl_leg(args, args.config, ngpu, rank, local, dist, share)
    cpu = hetero = None
    if rank == 0 and not args.no_cpu_baseline:
        cpu = oracle_baseline(workload(args.config, ngpu)[3])
        if ngpu == 1:
            hetero = hetero_model(workload(args.config, ngpu)[3], value)
    if dist:
        dist.barrier()
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ngpu,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": main_run["ms"] / args.steps,
            "higher_is_better": True, "scaling": main_run["scaling"], "vs_baseline": None,
            "dtype": "f64", "data": "synthetic", "config": line_cfg,
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "clocks": main_run["clocks"],
            "gpu_launches": main_run["launches"], "kernel_ms": main_run["kt"],
            "selfcheck": check, "nccl_check": nccl, "hetero_host_cpu": hetero,
            args.second or "second": second,
        }
        print(json.dumps(line), flush=True)
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
