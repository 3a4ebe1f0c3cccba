"""Full-size parity (BASELINE.json configs) on sampled outputs, in the launch
configuration bench.py times: the GPU computes whole batches; the oracle
re-computes a sample of them one by one."""
import numpy as np
import pytest

from gen import dcsbm
from helpers import close, ties

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


@pytest.fixture(scope="module")
def g200k():
    return dcsbm.make("200k")


def _sample_ranges(first, count, n_ranges=8, width=64, seed=0):
    rng = np.random.default_rng(seed)
    starts = np.sort(rng.choice(max(count - width, 1), n_ranges, replace=False)) + first
    return [(int(s), width) for s in starts]


@pytest.mark.parametrize("B", [71, 3000, 20000, 200000])
def test_200k_sampled_move_parity(G, oracle_mod, g200k, B):
    rowptr, col, truth, cfg = g200k
    V = cfg.V
    b = truth.copy() if B == 71 else dcsbm.random_partition(V, B, B)
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=SEED))
    ctx.gsap_set_partition(b, B)
    orc = oracle_mod.Oracle(rowptr, col)
    orc.set_partition(b, B)
    bs = (V + 3) // 4
    first, count = bs, bs                       # the second batch of an iteration
    s = ctx.gsap_propose(G.GSAP_MOVE, 2, 5, first, count)
    dS, H, acc = ctx.gsap_delta_mdl(G.GSAP_MOVE, 2, 5, first, count, s)
    nt = 0
    for (a, w) in _sample_ranges(first, count):
        i = a - first
        s_o = orc.propose(1, SEED, 2, 5, a, w)
        assert np.array_equal(s[i:i + w], s_o)
        dS_o, H_o, p_o, acc_o = orc.delta_move(SEED, 2, 5, a, w, s_o)
        assert np.all(close(dS[i:i + w], dS_o))
        assert np.all(close(H[i:i + w], H_o, floor=1e-300))
        t = ties(oracle_mod, SEED, 2, 5, range(a, a + w), p_o)
        nt += int(t.sum())
        assert np.array_equal(acc[i:i + w][~t], acc_o[~t])
    m_g, _ = ctx.gsap_mdl()
    m_o, _ = orc.mdl()
    assert abs(m_g - m_o) <= 1e-9 * abs(m_o)


@pytest.mark.parametrize("B,move_sorted", [(5000, 1), (5000, 2), (60000, 2)])
def test_200k_fused_batch_and_blockmodel(G, oracle_mod, g200k, B, move_sorted):
    """The fused batch (move + apply + rebuild) equals the oracle's, state compared exactly
    (move_sorted = 2: the sorted two-pass evaluation, sparse regime)."""
    rowptr, col, truth, cfg = g200k
    V = cfg.V
    b = dcsbm.random_partition(V, B, 1)
    extra = {"move_sorted": move_sorted}
    if move_sorted == 2:
        extra["dense_max_B"] = 1
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=SEED, **extra))
    ctx.gsap_set_partition(b, B)
    orc = oracle_mod.Oracle(rowptr, col)
    orc.set_partition(b, B)
    bs = (V + 3) // 4
    s, dS, acc, dsum = ctx.gsap_move_batch(0, 0, 0, bs)
    s_o = orc.propose(1, SEED, 0, 0, 0, bs)
    assert np.array_equal(s, s_o)
    # the fused kernel's dS and MH decisions vs the oracle's on the same
    # snapshot (every vertex of the batch; MH ties counted, not failed)
    dS_o, H_o, p_o, acc_o = orc.delta_move(SEED, 0, 0, 0, bs, s_o)
    assert np.all(close(dS, dS_o)), np.max(np.abs(dS - dS_o))
    t = ties(oracle_mod, SEED, 0, 0, range(bs), p_o)
    assert np.array_equal(acc[~t], acc_o[~t])
    assert abs(dsum - float(np.sum(dS_o[acc == 1]))) <= 1e-9 * max(1.0, abs(dsum))
    orc.apply_moves(0, bs, s, acc)
    orc.rebuild()
    b_g, _ = ctx.gsap_get_partition()
    b_o, _ = orc.partition()
    assert np.array_equal(b_g, b_o)
    g = ctx.gsap_get_blockmodel()
    o = orc.blockmodel()
    for k in ("rowptr", "col", "cnt", "cum", "colptr", "row", "ccnt", "ccum", "dout", "din"):
        assert np.array_equal(g[k].astype(np.int64), o[k].astype(np.int64)), k


def test_200k_merge_phase_sampled(G, oracle_mod, g200k):
    rowptr, col, truth, cfg = g200k
    V = cfg.V
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=SEED))
    orc = oracle_mod.Oracle(rowptr, col)
    B = V
    s = ctx.gsap_propose(G.GSAP_MERGE, 0, 0, 0, B)
    dS = ctx.gsap_delta_mdl(G.GSAP_MERGE, 0, 0, 0, B, s)
    for (a, w) in _sample_ranges(0, B, seed=3):
        s_o = orc.propose(0, SEED, 0, 0, a, w)
        assert np.array_equal(s[a * 10:(a + w) * 10], s_o)
        assert np.all(close(dS[a * 10:(a + w) * 10], orc.delta_merge(a, w, s_o)))
    best, dSb = ctx.gsap_merge_phase(0, int(0.4 * B))
    best_o, dSb_o = orc.best_merges(s, dS)
    assert np.array_equal(best, best_o)
    orc.select_merges(best, dSb, int(0.4 * B))
    b_g, B_g = ctx.gsap_get_partition()
    b_o, B_o = orc.partition()
    assert B_g == B_o and np.array_equal(b_g, b_o)


def test_200k_end_to_end_properties(G, oracle_mod, g200k):
    """Full run: the reported MDL is the oracle's MDL of the returned partition; quality band."""
    from sklearn.metrics import normalized_mutual_info_score as nmi
    rowptr, col, truth, cfg = g200k
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=SEED))
    res = ctx.gsap_run()
    orc = oracle_mod.Oracle(rowptr, col)
    orc.set_partition(res["b"], res["B"])
    assert abs(orc.mdl()[0] - res["mdl"]) <= 1e-9 * res["mdl"]
    # MDL of the planted partition is an upper bound the search should approach
    orc2 = oracle_mod.Oracle(rowptr, col)
    orc2.set_partition(truth, cfg.B_planted)
    print("B", res["B"], "MDL", res["mdl"], "planted MDL", orc2.mdl()[0], "NMI", nmi(truth, res["b"]))
    assert res["mdl"] <= 1.01 * orc2.mdl()[0]


GOLD = __import__("os").path.join(__import__("os").path.dirname(__file__), "golden")


@pytest.mark.parametrize("name", ["20k", "200k"])
def test_layer3_vs_oracle_golden(G, oracle_mod, name):
    """north_star layer 3 at the bench scale: the GPU's end-to-end partition
    of the BASELINE config reaches a final MDL within 1 % of the oracle's run
    and pairwise precision / recall within 0.02 of it (values written by
    tools/oracle_goldens.py, which calls only oracle/).  Trajectories are not
    compared round by round here: the first merge phase at B = V orders
    thousands of blocks by dS values that tie mathematically and differ in
    the last bits between the two independent formulas (parity
    is statistical beyond the first divergence); the GPU driver's decisions
    are replayed through the oracle's bracket logic instead."""
    import json
    import os
    from gen import metrics
    path = os.path.join(GOLD, f"e2e_{name}.json")
    if not os.path.exists(path):
        pytest.skip(f"{path} not generated yet")
    gold = json.load(open(path))
    rowptr, col, truth, cfg = dcsbm.make(name)
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=gold["seed"]))
    res = ctx.gsap_run()
    prec, rec = metrics.pairwise_precision_recall(truth, res["b"])
    print(name, "GPU B", res["B"], "MDL", res["mdl"], "P/R", prec, rec, "| oracle B", gold["B"], "MDL", gold["mdl"],
          "P/R", gold["precision"], gold["recall"])
    assert abs(res["mdl"] - gold["mdl"]) <= 0.01 * gold["mdl"]
    assert abs(prec - gold["precision"]) <= 0.02 and abs(rec - gold["recall"]) <= 0.02
    from test_gpu_parity import assert_driver_replay
    assert_driver_replay(oracle_mod, res, cfg.V)
    # the reported MDL is the oracle's MDL of the returned partition
    orc = oracle_mod.Oracle(rowptr, col)
    orc.set_partition(res["b"], res["B"])
    assert abs(orc.mdl()[0] - res["mdl"]) <= 1e-9 * res["mdl"]


@pytest.mark.parametrize("name", ["1m", "2m"])
def test_1m_2m_end_to_end_properties(G, oracle_mod, name):
    """1M / 2M end to end (the oracle's own run takes hours here): the reported
    MDL is the oracle's Eq. 2 MDL of the returned partition (1e-9), the
    driver's decisions replay through the oracle's bracket logic, and the
    quality lies in the paper's band for GSAP at 1M (Table 4: NMI
    0.69-0.91).  The search is a heuristic: it ends ABOVE the planted
    partition's MDL here (measured round 2: 1M +4.2 %, 2M +9.1 %), i.e. in a
    local optimum with fewer blocks than planted, as the paper's own NMI drop
    at 1M shows for its method; layer 3 proper (vs the oracle's run) is at
    20K / 200K (test_layer3_vs_oracle_golden)."""
    rowptr, col, truth, cfg = dcsbm.make(name)
    ctx = G.Context(rowptr, col, params=G.gsap_default_params(seed=SEED))
    res = ctx.gsap_run()
    ctx.close()
    assert res["rounds"] == len(res["trace"])
    orc = oracle_mod.Oracle(rowptr, col)
    orc.set_partition(res["b"], res["B"])
    m_found = orc.mdl()[0]
    assert abs(m_found - res["mdl"]) <= 1e-9 * m_found
    orc.set_partition(truth, cfg.B_planted)
    m_planted = orc.mdl()[0]
    from gen import metrics
    q = metrics.nmi(truth, res["b"])
    print(name, "found B", res["B"], "MDL", m_found, "| planted B", cfg.B_planted, "MDL", m_planted,
          f"ratio {m_found / m_planted:.4f}", "NMI", q)
    assert q >= 0.69
    from test_gpu_parity import assert_driver_replay
    assert_driver_replay(oracle_mod, res, cfg.V)


def test_bench_tsv_workload(G, tmp_path):
    """N3: bench.py partitions a GraphChallenge TSV graph (1-based ids) with a
    truth file and reports NMI / pairwise P/R in `config`."""
    import json
    import os
    import subprocess
    import sys
    rowptr, col, truth, cfg = dcsbm.make("1k")
    src = np.repeat(np.arange(cfg.V), np.diff(rowptr))
    g = tmp_path / "g.tsv"
    t = tmp_path / "t.tsv"
    np.savetxt(g, np.stack([src + 1, col + 1], 1), fmt="%d", delimiter="\t")
    np.savetxt(t, np.stack([np.arange(cfg.V) + 1, truth + 1], 1), fmt="%d", delimiter="\t")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--tsv", str(g), "--truth", str(t),
                          "--steps", "1", "--warmup", "1", "--no-2m", "--no-cpu-baseline", "--no-e2e"],
                         capture_output=True, text=True, timeout=600, cwd=root)
    assert out.returncode == 0, out.stderr[-2000:]
    line = json.loads([l for l in out.stdout.splitlines() if l.startswith("{")][-1])
    assert line["config"]["V"] == cfg.V and line["config"]["E"] == cfg.E
    assert line["config"]["nmi_vs_planted"] > 0.9 and "pairwise_recall" in line["config"]
