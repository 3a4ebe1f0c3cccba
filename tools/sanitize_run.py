"""A small workload that drives every kernel family once or twice, for
compute-sanitizer (memcheck / racecheck / synccheck / initcheck):
fused MOVE (warp, mid, group, huge roles with shared and global tables),
the sorted two-pass MOVE, every rebuild path (persistent dense, dense
multi-kernel + incremental delta, persistent sparse, multi-kernel sparse),
merge proposals / selection (one-CTA and multi-kernel), MDL, the N4 table.

    compute-sanitizer --tool racecheck python tools/sanitize_run.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np  # noqa: E402

from gen import dcsbm  # noqa: E402
from paper_conf_icpp_changzh24_b200 import gsap  # noqa: E402


def hub_graph():
    rng = np.random.default_rng(0)
    V = 3000
    src = [rng.integers(0, V, 8000)]
    dst = [rng.integers(0, V, 8000)]
    for hub, deg in ((5, 100), (9, 200), (17, 800), (2000, 2600)):
        src.append(np.full(deg, hub))
        dst.append(rng.choice(V, deg, replace=False))
        src.append(rng.choice(V, deg // 2, replace=False))
        dst.append(np.full(deg // 2, hub))
    src = np.concatenate(src)
    dst = np.concatenate(dst)
    order = np.argsort(src, kind="stable")
    rowptr = np.zeros(V + 1, np.int64)
    np.add.at(rowptr, src[order] + 1, 1)
    return np.cumsum(rowptr), dst[order].astype(np.int32)


def drive(rowptr, col, wgt=None, **kw):
    V = len(rowptr) - 1
    ctx = gsap.Context(rowptr, col, wgt, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, cuda_graphs=0, **kw))
    bs = (V + 3) // 4
    for B in (min(V, 31), min(V, 300), min(V, 2500), V):
        b = dcsbm.random_partition(V, B, B)
        ctx.gsap_set_partition(b, B)
        for k in range(2):
            ctx.gsap_move_batch(1, k, k * bs, min(V, (k + 1) * bs) - k * bs)
        if B >= 4:
            ctx.gsap_merge_phase(2, int(0.4 * ctx.B))
        ctx.gsap_mdl()
    ctx.close()


rowptr, col, truth, cfg = dcsbm.make("1k")
drive(rowptr, col)                                            # dense coop / dense mk + delta / sparse coop
drive(rowptr, col, dense_max_B=1, sparse_coop=0)              # multi-kernel sparse
drive(rowptr, col, dense_max_B=1, move_sorted=2)              # sorted two-pass MOVE
drive(rowptr, col, proposal_mode=1, sel_small=0)              # N4 table, multi-kernel selection
hr, hc = hub_graph()
w = np.random.default_rng(1).integers(1, 5, len(hc)).astype(np.int32)
drive(hr, hc, w)                                              # weighted groups / huge (global tables)
drive(hr, hc, None, dense_max_B=1, sparse_coop=0)
print("sanitize workload done")
