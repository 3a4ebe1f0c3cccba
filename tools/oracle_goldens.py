#!/usr/bin/env python
"""Write the oracle's end-to-end results on BASELINE.json configs into tests/golden/.

Calls ONLY oracle/ (the CPU oracle) and gen/ (the seeded input generator); no
value here comes from the CUDA path.  Each file holds the oracle's complete
SBP run (§3 Fig. 2; readings O.7-O.9 in DESIGN.md) of the named
synthetic graph with the default Table 2 parameters and the run
seed: final B, MDL (Eq. 2), pairwise precision / recall and NMI against the
planted partition (§4.4), and the per-round trace
[outer, B after merge, MCMC iterations, MDL, threshold, accepted moves].
The GPU layer-3 tests (north_star: MDL within 1 %, P/R within 0.02) read them.

    python tools/oracle_goldens.py [--threads N] 20k 200k

--threads runs the oracle's per-id loops on N OpenMP threads (identical
results; orc_set_threads).
"""
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from gen import dcsbm, metrics  # noqa: E402
from oracle import oracle  # noqa: E402


def one(name):
    rowptr, col, truth, cfg = dcsbm.make(name)
    o = oracle.Oracle(rowptr, col)
    p = oracle.default_params(seed=dcsbm.RUN_SEED)
    t0 = time.perf_counter()
    res = o.partition_run(p)
    dt = time.perf_counter() - t0
    prec, rec = metrics.pairwise_precision_recall(truth, res["b"])
    st = res["stats"]
    planted = oracle.Oracle(rowptr, col)
    planted.set_partition(truth, cfg.B_planted)
    out = {
        "_cite": "oracle/gsap_oracle.c orc_partition (P:137-141 Fig. 2, Table 2 P:295-305, R:O.7-O.9); "
                 "written by tools/oracle_goldens.py, which calls only oracle/ and gen/",
        "config": cfg.name, "V": cfg.V, "E": cfg.E, "seed": dcsbm.RUN_SEED,
        "B": res["B"], "mdl": res["mdl"], "precision": prec, "recall": rec,
        "nmi": metrics.nmi(truth, res["b"]),
        "mdl_planted": planted.mdl()[0], "B_planted": cfg.B_planted,
        "rounds": res["rounds"], "n_move_prop": st.n_move_prop, "n_move_acc": st.n_move_acc,
        "n_merge_prop": st.n_merge_prop, "mcmc_itr_total": st.mcmc_itr_total,
        "b_sha256": hashlib.sha256(res["b"].astype("<i4").tobytes()).hexdigest(),
        "trace_cols": ["outer", "B", "itrs", "mdl", "thresh", "accepted"],
        "trace": res["trace"].tolist(),
        "oracle_seconds": dt, "oracle_threads": THREADS,
    }
    path = os.path.join(ROOT, "tests", "golden", f"e2e_{name}.json")
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(name, "B", res["B"], "MDL", res["mdl"], "P/R", prec, rec, f"{dt:.1f} s", flush=True)


THREADS = 1

if __name__ == "__main__":
    args = sys.argv[1:]
    if args and args[0] == "--threads":
        THREADS = oracle.set_threads(int(args[1]))
        args = args[2:]
    for n in args or ["20k"]:
        one(n)
