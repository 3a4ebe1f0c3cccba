"""A/B of whole SBP partitions (gsap_run on a resident graph) under gsap_params
variants: per variant, W warm-up runs then K timed runs (CUDA events on the
context stream); prints the mean and min seconds and the partition found.

    python tools/partition_ab.py --config 20k --runs 5 --variant cuda_graphs=1 --variant cuda_graphs=2
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="20k")
ap.add_argument("--runs", type=int, default=5)
ap.add_argument("--warmup", type=int, default=2)
ap.add_argument("--variant", action="append", default=[],
                help="comma-separated gsap_params field=value list (repeatable; '' = defaults)")
a = ap.parse_args()

import torch  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

rowptr, col, truth, cfg = dcsbm.make(a.config)
for var in a.variant or [""]:
    extra = {k: int(v) for k, v in (p.split("=") for p in var.split(",") if p)}
    ctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, **extra))
    times = []
    for i in range(a.warmup + a.runs):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        res = ctx.gsap_run()
        e1.record()
        torch.cuda.synchronize()
        if i >= a.warmup:
            times.append(e0.elapsed_time(e1) * 1e-3)
    print(f"{a.config} [{var or 'defaults'}] mean {sum(times) / len(times):.4f} s min {min(times):.4f} s "
          f"B {res['B']} MDL {res['mdl']:.6e}", flush=True)
    ctx.close()
