"""N4 ablation: the paper-literal lookup-table proposals
(params.proposal_mode = 1; Alg. 1 P:180-200 with the shared tables of
Fig. 4) against fresh Philox draws (mode 0, R:Z6): partition time on the
device (CUDA events, graph resident), MOVE acceptance, found B, MDL, NMI and
pairwise P/R per config.  Prints one JSON line per (config, mode).

    python tools/ablation_n4.py 20k 200k
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import dcsbm, metrics  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

for name in sys.argv[1:] or ["20k"]:
    rowptr, col, truth, cfg = dcsbm.make(name)
    for mode in (0, 1):
        ctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, proposal_mode=mode))
        ctx.gsap_run()                       # warm-up
        ctx.gsap_reset_stats()
        times = []
        for _ in range(3):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            res = ctx.gsap_run()
            e1.record()
            e1.synchronize()
            times.append(e0.elapsed_time(e1) / 1e3)
        st = ctx.gsap_get_stats()
        p, r = metrics.pairwise_precision_recall(truth, res["b"])
        print(json.dumps({"config": cfg.name, "proposal_mode": mode, "partition_sec": min(times),
                          "rounds": res["rounds"], "mcmc_itr_total": st["mcmc_itr_total"] / 3,
                          "move_accept_rate": st["n_move_acc"] / max(st["n_move_prop"], 1),
                          "B": res["B"], "mdl": res["mdl"], "nmi": metrics.nmi(truth, res["b"]),
                          "precision": p, "recall": r}), flush=True)
        ctx.close()
