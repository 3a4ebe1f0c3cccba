"""Per-launch device time of the move / rebuild kernels on realistic states.

For each requested round count R, a full SBP run is cut after R rounds
(max_rounds = R; the context then holds the best partition so far), and
`--batches` MOVE batches are run through gsap_move_batch with event timing
(profile = 1).  Prints one line per state: B, regime, us per move launch
(k_propose + k_move), us per rebuild, us per batch.

    python tools/bench_kernels.py --config 20k --rounds 1 3 5 8 19
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="20k")
ap.add_argument("--rounds", type=int, nargs="+", default=[1, 3, 5, 8, 19])
ap.add_argument("--batches", type=int, default=16)
ap.add_argument("--json", default=None)
ap.add_argument("--dense-max-B", type=int, default=0)
ap.add_argument("--param", action="append", default=[], help="extra gsap_params field=value (repeatable)")
ap.add_argument("--profile-range", action="store_true",
                help="cudaProfilerStart/Stop around the timed batches (ncu --profile-from-start off)")
a = ap.parse_args()

import torch  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

rowptr, col, truth, cfg = dcsbm.make(a.config)
out = []
for R in a.rounds:
    extra = {k: int(v) for k, v in (p.split("=") for p in a.param)}
    prm = gsap.gsap_default_params(seed=dcsbm.RUN_SEED, profile=1, max_rounds=R, dense_max_B=a.dense_max_B, **extra)
    ctx = gsap.Context(rowptr, col, params=prm)
    ctx.gsap_run()
    B = ctx.B
    nb = 4
    bs = (cfg.V + nb - 1) // nb
    ctx.gsap_reset_stats()
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    if a.profile_range:
        torch.cuda.profiler.start()
    ev0.record()
    for i in range(a.batches):
        k = i % nb
        ctx.gsap_move_batch(1000 + R, i // nb, k * bs, min(cfg.V, (k + 1) * bs) - k * bs, outputs=False)
    ctx.gsap_sync()
    ev1.record()
    torch.cuda.synchronize()
    if a.profile_range:
        torch.cuda.profiler.stop()
    st = ctx.gsap_get_stats()
    mv = 1e3 * st["k_move_ms"] / max(st["k_move_launches"], 1)
    rb = 1e3 * st["k_rebuild_ms"] / max(st["k_rebuild_launches"], 1)
    tot = 1e3 * ev0.elapsed_time(ev1) / a.batches
    row = dict(config=a.config, rounds=R, B=B, move_us=mv, rebuild_us=rb, batch_us=tot,
               accepted=st["n_move_acc"])
    out.append(row)
    print(f"{a.config} R={R:3d} B={B:8d} move {mv:9.1f} us  rebuild {rb:9.1f} us  batch {tot:9.1f} us", flush=True)
    ctx.close()
if a.json:
    json.dump(out, open(a.json, "w"), indent=1)
