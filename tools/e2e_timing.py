"""gsap_partition end to end (pinned host CSR in, host partition out), repeated;
run with GSAP_TIMING=1 for the create / destroy breakdown on stderr."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402

cfg_name = sys.argv[1] if len(sys.argv) > 1 else "20k"
rowptr, col, truth, cfg = dcsbm.make(cfg_name)
rp = torch.from_numpy(rowptr).pin_memory()
cl = torch.from_numpy(col).pin_memory()
for i in range(4):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    out = gsap.gsap_partition(rp, cl, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED))
    t1 = time.perf_counter()
    print(f"{cfg_name} e2e {1e3 * (t1 - t0):.2f} ms setup {1e3 * out['stats']['t_setup']:.2f} ms "
          f"B {out['B']}", flush=True)
