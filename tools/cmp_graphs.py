import sys, time, os
sys.path.insert(0, os.getcwd())
from gen import dcsbm
from paper_conf_icpp_changzh24_b200 import gsap
for cfgname in sys.argv[1:]:
    rowptr, col, truth, cfg = dcsbm.make(cfgname)
    for g in (1, 2, 1, 2):
        ctx = gsap.Context(rowptr, col, params=gsap.gsap_default_params(seed=dcsbm.RUN_SEED, cuda_graphs=g))
        ctx.gsap_run()
        t = time.perf_counter(); r = ctx.gsap_run(); dt = time.perf_counter() - t
        st = ctx.gsap_get_stats()
        print(cfgname, "graphs", g, f"{dt*1e3:.2f} ms", "B", r["B"], "mdl", repr(r["mdl"]), "itrs", st["mcmc_itr_total"], "rounds", r["rounds"], flush=True)
        ctx.close()
