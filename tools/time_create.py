"""Time gsap_create (graph copy-in, CSC build, first rebuild) vs a run, for a config."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

cfg = sys.argv[1] if len(sys.argv) > 1 else "20k"
rowptr, col, truth, c = dcsbm.make(cfg)
torch.cuda.synchronize()
for i in range(3):
    t0 = time.perf_counter()
    ctx = gsap.Context(rowptr, col)
    t1 = time.perf_counter()
    res = ctx.gsap_run()
    t2 = time.perf_counter()
    ctx.close()
    t3 = time.perf_counter()
    print(f"create {t1 - t0:.4f} s  run {t2 - t1:.4f} s  destroy {t3 - t2:.4f} s", flush=True)
