"""N2 (incremental blockmodel update, §3.4) measured end to end:
full partitions with params.incremental = 1 (default) and 0, device time
(CUDA events, graph resident, best of 3 after a warm-up), rebuild-class device
time from a profiled run, and a check that both give the same partition.

    python tools/ablation_n2.py 20k 200k 2m
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

for name in sys.argv[1:] or ["20k"]:
    rowptr, col, truth, cfg = dcsbm.make(name)
    out = {}
    for inc in (1, 0):
        ctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, incremental=inc))
        ctx.gsap_run()
        times = []
        for _ in range(3 if cfg.V <= 200000 else 1):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            res = ctx.gsap_run()
            e1.record()
            e1.synchronize()
            times.append(e0.elapsed_time(e1) / 1e3)
        ctx.close()
        pctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, incremental=inc,
                                                                         profile=1))
        pctx.gsap_run()
        st = pctx.gsap_get_stats()
        pctx.close()
        out[inc] = res
        print(json.dumps({"config": cfg.name, "incremental": inc, "partition_sec": min(times),
                          "rebuild_device_sec": st["t_rebuild"], "rebuild_launches": st["k_rebuild_launches"],
                          "B": res["B"], "mdl": res["mdl"]}), flush=True)
    same = out[0]["B"] == out[1]["B"] and out[0]["mdl"] == out[1]["mdl"] and bool((out[0]["b"] == out[1]["b"]).all())
    print(json.dumps({"config": cfg.name, "identical_partition": same}), flush=True)
