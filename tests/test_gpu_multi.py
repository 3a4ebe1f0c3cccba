"""The multi-GPU data path on ONE GPU: params.sim_ranks = G runs
every MOVE batch and merge phase cut into G ranks' slices exactly as the NCCL
path does (edge-balanced chunk slices, block ranges, slice offsets, per-chunk
dS partials, the gathered apply), each slice computed in rank order, the
in-place all-gathers skipped.  The trajectory must be bit-identical for every
G (randomness keyed by global ids, fixed-chunk sums in chunk order)."""
import numpy as np
import pytest

from gen import dcsbm

pytestmark = pytest.mark.gpu
SEED = dcsbm.RUN_SEED


@pytest.fixture(scope="module")
def G():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_icpp_changzh24_b200 import gsap
    gsap.lib()
    return gsap


def _run(G, rowptr, col, wgt=None, **kw):
    ctx = G.Context(rowptr, col, wgt, params=G.gsap_default_params(seed=SEED, **kw))
    res = ctx.gsap_run()
    st = ctx.gsap_get_stats()
    ctx.close()
    return res, st


@pytest.mark.parametrize("name,extra", [("20k", {}), ("200k", {}), ("200k", {"move_sorted": 2, "dense_max_B": 1}),
                                        ("hubs_w", {})])
def test_sim_ranks_bit_identical(G, name, extra):
    if name == "hubs_w":
        from test_gpu_parity import _hub_graph
        rowptr, col, w = _hub_graph(True)
    else:
        rowptr, col, truth, cfg = dcsbm.make(name)
        w = None
    ref, st_ref = _run(G, rowptr, col, w, **extra)
    for g in (2, 4, 8):
        res, st = _run(G, rowptr, col, w, sim_ranks=g, **extra)
        assert res["B"] == ref["B"] and res["mdl"] == ref["mdl"], (g, res["B"], ref["B"])
        assert np.array_equal(res["b"], ref["b"]), g
        assert np.array_equal(res["trace"][:, [0, 1, 2, 3, 5, 9, 10, 11]],
                              ref["trace"][:, [0, 1, 2, 3, 5, 9, 10, 11]]), g
        # every proposal of every slice was generated exactly once
        assert st["n_move_prop"] == st_ref["n_move_prop"] and st["n_merge_prop"] == st_ref["n_merge_prop"]
        assert st["n_move_acc"] == st_ref["n_move_acc"] and st["n_move_eval"] == st_ref["n_move_eval"]


def test_shard_plan_edge_balanced(G):
    rowptr, col, truth, cfg = dcsbm.make("200k")
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=SEED))
    V = cfg.V
    k = np.diff(rowptr) + np.bincount(col, minlength=V)
    bs = (V + 3) // 4
    for first in (0, bs, 3 * bs):
        count = min(V, first + bs) - first
        for nr in (1, 2, 3, 8):
            f, n = ctx.gsap_shard_plan(first, count, nr)
            assert f[0] == first and np.all(f[1:] == f[:-1] + n[:-1]) and f[-1] + n[-1] == first + count
            assert np.all((f - first) % 1024 == 0)
            work = np.array([k[a:a + c].sum() + 16 * c for a, c in zip(f, n)])
            chunk_max = max(k[a:a + 1024].sum() + 16 * 1024 for a in range(first, first + count, 1024))
            assert work.max() - work.mean() <= chunk_max, (nr, work)
    ctx.close()
