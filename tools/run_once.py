"""One SBP partition of a named config on cuda:0 (for ncu / nsight captures)."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="20k")
ap.add_argument("--runs", type=int, default=1)
ap.add_argument("--profile", type=int, default=0)
a = ap.parse_args()

import torch  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

rowptr, col, truth, cfg = dcsbm.make(a.config)
ctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, profile=a.profile))
for i in range(a.runs):
    t0 = time.perf_counter()
    res = ctx.gsap_run()
    dt = time.perf_counter() - t0
    st = ctx.gsap_get_stats()
    print(f"run {i}: {dt:.3f} s B={res['B']} rounds={res['rounds']} launches={st['gpu_launches']} "
          f"move_ms={st['k_move_ms']:.1f} rebuild_ms={st['k_rebuild_ms']:.1f} merge_ms={st['k_merge_ms']:.1f} "
          f"itrs={st['mcmc_itr_total']}", flush=True)
    if i == 0:
        for row in res["trace"]:
            print(f"   outer={int(row[0]):3d} B={int(row[1]):8d} itrs={int(row[2]):3d} MDL={row[3]:.6e} sec={row[4]:.4f} acc={int(row[5])} "
                  f"move={row[6]:.2f}ms rebuild={row[7]:.2f}ms merge={row[8]:.2f}ms")
    ctx.gsap_reset_stats()
