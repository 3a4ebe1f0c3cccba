#!/usr/bin/env python
"""Benchmark of the GSAP hot path on B200 (driver contract: one JSON line on rank 0).

A step is one complete SBP partition of the synthetic graph (every row of
SURVEY.md 8(a): Philox proposals, dS + Hastings + MH accept, merge proposals,
merge selection, blockmodel rebuilds, MDL reductions, golden-section driver)
on a context whose graph is already resident in HBM.  The metric is proposals
per second (vertex-move + block-merge proposals generated) over the timed
steps; partition seconds are reported beside it.  Between timed steps L2 is
flushed (a 512 MiB write) outside the timed region.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config 20k|1k|200k|1m|2m]
    python bench.py --impl reference ...   # the CPU oracle on a bounded sample

N > 1 (torchrun, one rank per GPU): independent problems (one graph per rank,
seed offset by rank), no data-path collective: weak scaling.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIG_KEYS = {"1k": "1k", "20k": "20k", "200k": "200k", "1m": "1m", "2m": "2m"}
METRIC = "proposals_per_sec (end-to-end SBP partition)"


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="20k", choices=sorted(CONFIG_KEYS))
    ap.add_argument("--impl", default="gsap", choices=["gsap", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--shard", action="store_true",
                    help="N > 1: partition ONE graph with the sharded path (NCCL all-gathers); "
                         "default: one independent graph per GPU")
    return ap.parse_args()


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled during the timed region."""

    def __init__(self, index):
        self.index = index
        self.samples = []
        self.proc = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 8:
                self.samples.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"]}
        sm = sorted(float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit())
        mx = max((float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()), default=None)
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[4 + i] == "Active"})
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": mx, "reasons": reasons,
                "samples": len(self.samples)}


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except (OSError, ValueError):
        return {}


def cpu_info():
    model = ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return model, os.cpu_count()


def oracle_sample(rowptr, col, seed, max_rounds=1):
    """The oracle as it stands, single-threaded, on the first `max_rounds` SBP rounds."""
    from oracle import oracle
    o = oracle.Oracle(rowptr, col)
    t0 = time.perf_counter()
    res = o.partition_run(oracle.default_params(seed=seed, max_rounds=max_rounds))
    dt = time.perf_counter() - t0
    st = res["stats"]
    props = st.n_move_prop + st.n_merge_prop
    return props, dt, res


def traffic_for(kernel_class):
    """DRAM bytes per launch of the dominant kernel from a committed ncu --set full summary."""
    path = os.path.join(ROOT, "profiles", "traffic.json")
    try:
        d = json.load(open(path))
        return d.get(kernel_class)
    except (OSError, ValueError):
        return None


def run_reference(args, rank, world):
    from gen import dcsbm
    if rank != 0:
        return 0
    rowptr, col, truth, cfg = dcsbm.make(CONFIG_KEYS[args.config])
    vals, times = [], []
    for i in range(args.warmup + args.steps):
        props, dt, _ = oracle_sample(rowptr, col, dcsbm.RUN_SEED + i)
        if i >= args.warmup:
            vals.append(props)
            times.append(dt)
    value = sum(vals) / sum(times)
    model, ncpu = cpu_info()
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "proposals/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sum(times) / len(times),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic DC-SBM (GraphChallenge-shaped, gen/dcsbm.py)",
        "config": {"workload": cfg.name, "V": cfg.V, "E": cfg.E, "sample": "first SBP round per step"},
        "cpu_baseline": {"value": value, "unit": "proposals/s", "cores": 1, "kind": "oracle",
                         "sample": f"oracle (single-thread C) first SBP round of {cfg.name} per step; {model}, "
                                   f"{ncpu} host cpus"},
        "e2e": {"value": value, "unit": "proposals/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        return run_reference(args, rank, world)

    import numpy as np
    import torch
    import torch.distributed as dist

    from gen import dcsbm
    from paper_conf_icpp_changzh24_b200 import gsap

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    rowptr, col, truth, cfg = dcsbm.make(CONFIG_KEYS[args.config])
    shard = args.shard and world > 1
    seed = dcsbm.RUN_SEED + (0 if shard else rank)
    stream = torch.cuda.Stream()
    # the timed steps run without per-kernel events (profile = 0); the roofline
    # numbers come from a second, profiled pass of the same steps below
    params = gsap.gsap_default_params(seed=seed, profile=0)
    gdist = gsap.dist_from_torch() if shard else None
    ctx = gsap.Context(rowptr, col, params=params, stream=stream.cuda_stream, dist=gdist)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    # warm-up
    for _ in range(args.warmup):
        ctx.gsap_run()
    barrier()
    ctx.gsap_reset_stats()
    step_ms, props, results = [], 0, None
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            with torch.cuda.stream(stream):
                flush.fill_(1)                       # L2 flush, outside the timed region
            barrier()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            results = ctx.gsap_run()
            e1.record(stream)
            e1.synchronize()
            step_ms.append(e0.elapsed_time(e1))
    barrier()
    st = ctx.gsap_get_stats()
    props = st["n_move_prop"] + st["n_merge_prop"]
    launches_timed = int(st["gpu_launches"])
    ctx.close()
    # profiled pass (CUDA events around every kernel class on the context
    # stream): same steps, same seed, not part of `value`
    pctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=seed, profile=1),
                        stream=stream.cuda_stream, dist=gsap.dist_from_torch() if shard else None)
    pctx.gsap_run()
    barrier()
    pctx.gsap_reset_stats()
    pms = []
    for _ in range(args.steps):
        with torch.cuda.stream(stream):
            flush.fill_(1)
        barrier()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        pctx.gsap_run()
        e1.record(stream)
        e1.synchronize()
        pms.append(e0.elapsed_time(e1))
    barrier()
    pst = pctx.gsap_get_stats()
    pctx.close()
    total_ms = sum(step_ms)
    if world > 1:
        t = torch.tensor([total_ms, float(props)], dtype=torch.float64, device="cuda")
        tmax = t.clone()
        dist.all_reduce(tmax[:1], op=dist.ReduceOp.MAX)
        dist.all_reduce(t[1:], op=dist.ReduceOp.SUM)
        total_ms, props_all = float(tmax[0]), float(t[1])
    else:
        props_all = float(props)
    value = props_all / (total_ms / 1e3)

    # roofline of the dominant kernel class (device time via CUDA events on the ctx stream)
    pk = peaks()
    classes = {"move": (pst["k_move_ms"], pst["k_move_bytes"], pst["k_move_launches"]),
               "rebuild": (pst["k_rebuild_ms"], pst["k_rebuild_bytes"], pst["k_rebuild_launches"]),
               "merge": (pst["k_merge_ms"], pst["k_merge_bytes"], pst["k_merge_launches"])}
    prof_ms = sum(pms)
    # the dominant kernel of the step is the fused move kernel (proposal + dS +
    # Hastings + MH accept: k_move, with k_move_groups beside it on a second
    # stream for vertices of > 128 neighbour blocks): profiles/r01_bench20k_launches.txt.
    # The rebuild class (more device time in total) is three different
    # algorithms by regime (persistent sparse, persistent dense B <= 221,
    # multi-kernel dense), reported beside it in classes_ms.
    dom = "move"
    ms, byts, launches = classes[dom]
    hbm = pk.get("hbm_gbs", 6650.0)
    achieved = (byts / launches) / (ms / launches / 1e3) / 1e9 if ms > 0 and launches else 0.0
    roofline = {"bound": "hbm", "achieved": achieved, "peak": hbm, "unit": "GB/s",
                "frac": achieved / hbm, "traffic": traffic_for(dom),
                "kernel": "k_move (+ k_move_groups beside it): fused proposal, dS, Hastings, MH accept; "
                          "one MOVE batch per launch",
                "peak_source": "MEASURED_PEAKS.json hbm_gbs" if "hbm_gbs" in pk else "fallback 6650",
                "timing": "CUDA events on the context stream around every launch, in a profiled pass of "
                          "the same steps (profiled ms_per_step %.2f)" % (prof_ms / args.steps),
                "share_of_step": (ms / prof_ms) if prof_ms else None,
                "launches": launches, "ms_per_launch": ms / max(launches, 1),
                "bytes_per_launch": byts / max(launches, 1),
                "classes_ms": {k: v[0] for k, v in classes.items()}}

    # end to end through the public API with host buffers (H2D of the CSR, D2H of the result)
    e2e = None
    if not args.no_e2e:
        rp_pin = torch.from_numpy(rowptr).pin_memory()
        col_pin = torch.from_numpy(col).pin_memory()
        barrier()
        t0 = time.perf_counter()
        out = gsap.gsap_partition(rp_pin, col_pin, params=gsap.gsap_default_params(seed=seed),
                                  dist=gsap.dist_from_torch() if shard else None)
        t1 = time.perf_counter()
        e_props = out["stats"]["n_move_prop"] + out["stats"]["n_merge_prop"]
        e2e = {"value": e_props / (t1 - t0), "unit": "proposals/s",
               "h2d_bytes_per_step": int(rowptr.nbytes + col.nbytes),
               "d2h_bytes_per_step": int(4 * cfg.V + 12), "partition_sec": t1 - t0,
               "setup_sec": out["stats"]["t_setup"]}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        o_props, o_dt, _ = oracle_sample(rowptr, col, seed)
        model, ncpu = cpu_info()
        cpu = {"value": o_props / o_dt, "unit": "proposals/s", "cores": 1, "kind": "oracle",
               "sample": f"first SBP round of {cfg.name} ({o_props} proposals in {o_dt:.1f} s, "
                         f"single-thread C oracle); host: {model}, {ncpu} cpus"}

    if rank == 0:
        from sklearn.metrics import normalized_mutual_info_score as nmi
        line = {
            "metric": METRIC, "value": value, "unit": "proposals/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": total_ms / args.steps, "higher_is_better": True,
            "scaling": "strong" if shard else "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic DC-SBM (GraphChallenge-shaped, gen/dcsbm.py), resident in HBM",
            "config": {"workload": cfg.name, "V": cfg.V, "E": cfg.E, "B_planted": cfg.B_planted,
                       "parallelism": (f"one graph, vertex/block slices over {world} GPUs (NCCL all-gather)"
                                       if shard else f"independent graph per GPU x{world}"),
                       "l2": "flushed (512 MiB write) between timed steps",
                       "partition_sec": total_ms / args.steps / 1e3,
                       "B_found": results["B"], "mdl": results["mdl"],
                       "nmi_vs_planted": float(nmi(truth, results["b"])),
                       "rounds": results["rounds"],
                       "paper_partition_sec_context": "GSAP on 1x A4000, real SBPC graph (Table 3): "
                                                      "1K-LL 0.4 s, 20K-HH 2.0 s, 200K-HL 96 s, 1M-LL 816 s"},
            "roofline": roofline,
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches_timed,
            "clocks": clk.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
