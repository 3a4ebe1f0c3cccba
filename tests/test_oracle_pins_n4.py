"""Pins of the oracle's N4 ablation mode: the paper-literal lookup-table
proposals (§3.2 and Fig. 4: multinomial / uniform / random tables built
once, then Alg. 1).  Reading N4: one weighted
neighbour block per block (the multinomial table), drawn per merge phase /
MOVE batch with its own Philox counter, shared by every proposal that reaches
the block; the uniform and random tables are the per-proposal words; a MERGE
outcome equal to r is redrawn uniformly over the other blocks."""
import numpy as np
import pytest
from scipy import stats

from gen import dcsbm

SEED = dcsbm.RUN_SEED
TABLE_J = 0x40000000


def _state(oracle_mod, seed=3, V=80, E=700, B=9):
    rowptr, col, _ = dcsbm.random_multigraph(V, E, seed)
    o = oracle_mod.Oracle(rowptr, col)
    b = dcsbm.random_partition(V, B, seed)
    o.set_partition(b, B)
    return o, rowptr, col, b, B


def test_table_entries_follow_the_multinomial_law(oracle_mod):
    """mt[x] ~ (M_xt + M_tx) / d_x: the multinomial distribution "derived from
    the weights of connecting edges", self-loop block counted in both
    of x's lines; chi-square over 40 000 tables."""
    o, rowptr, col, b, B = _state(oracle_mod)
    bm = o.blockmodel()
    M = np.zeros((B, B), np.int64)
    for x in range(B):
        for k in range(bm["rowptr"][x], bm["rowptr"][x + 1]):
            M[x, bm["col"][k]] = bm["cnt"][k]
    d = M.sum(0) + M.sum(1)
    n = 40000
    draws = np.array([o.table(SEED, TABLE_J, 0, outer, 0) for outer in range(n)])
    for x in (0, 3, 7):
        law = (M[x, :] + M[:, x]) / d[x]
        obs = np.bincount(draws[:, x], minlength=B)
        keep = law > 0
        assert obs[~keep].sum() == 0
        p = stats.chisquare(obs[keep], law[keep] * n).pvalue
        assert p > 1e-4, (x, p)


def _alg1_merge(mt, deg, B, r, w):
    """Alg. 1 transcribed: lines 2-3 (no neighbours -> random
    table), 5 (u = multi_table[r]), 6-9 (x = uniform table vs B / (B + deg u),
    exact integer form R:Z9), 10 (multi_table[u]); reading N4: r is redrawn."""
    def random_other():
        s = (int(w[2]) * (B - 1)) >> 32
        return s + 1 if s >= r else s
    if deg[r] <= 0:
        return random_other()
    u = mt[r]
    if int(w[1]) * (B + int(deg[u])) <= (B << 32):
        return random_other()
    s = mt[u]
    return s if (s >= 0 and s != r) else random_other()


def test_merge_proposals_are_alg1_with_the_table(oracle_mod):
    o, rowptr, col, b, B = _state(oracle_mod, seed=5)
    bm = o.blockmodel()
    deg = bm["dout"] + bm["din"]
    key = [SEED & 0xffffffff, SEED >> 32]
    for outer in (0, 4):
        mt = o.table(SEED, TABLE_J, 0, outer, 0)
        o.set_proposal_mode(1)
        s = o.propose(0, SEED, outer, 0, 0, B)
        o.set_proposal_mode(0)
        for r in range(B):
            for j in range(10):
                w = oracle_mod.philox([r, j, 0, (outer << 1) | 0], key)
                assert s[r * 10 + j] == _alg1_merge(mt, deg, B, r, w), (outer, r, j)


def test_move_proposals_use_the_table(oracle_mod):
    """MOVE ("the vertex-move phase is similar, but each vertex must
    identify the block ID of its adjacent vertices"): the weighted neighbour n
    from the vertex's own word, u = b[n], the coin, then multi_table[u]."""
    o, rowptr, col, b, B = _state(oracle_mod, seed=7)
    V = len(rowptr) - 1
    bm = o.blockmodel()
    deg = bm["dout"] + bm["din"]
    src = np.repeat(np.arange(V), np.diff(rowptr))
    key = [SEED & 0xffffffff, SEED >> 32]
    first, count, itr, outer = 20, 40, 3, 2
    mt = o.table(SEED, TABLE_J | first, itr, outer, 1)
    o.set_proposal_mode(1)
    s = o.propose(1, SEED, outer, itr, first, count)
    o.set_proposal_mode(0)
    for i in range(count):
        v = first + i
        w = oracle_mod.philox([v, 0, itr, (outer << 1) | 1], key)
        nb = list(col[rowptr[v]:rowptr[v + 1]]) + list(src[col == v])
        K = len(nb)
        if K == 0:
            want = (int(w[2]) * B) >> 32
        else:
            u = b[nb[(int(w[0]) * K) >> 32]]
            if int(w[1]) * (B + int(deg[u])) <= (B << 32):
                want = (int(w[2]) * B) >> 32
            else:
                want = mt[u]
        assert s[i] == want, (v, s[i], want)


def test_table_mode_partition_runs(oracle_mod):
    """The ablation runs end to end and stays in the quality band on an easy graph."""
    from sklearn.metrics import normalized_mutual_info_score as nmi
    rowptr, col, truth = dcsbm.generate(400, 6000, 10.0, 200.0, seed=1, B=4)
    o = oracle_mod.Oracle(rowptr, col)
    o.set_proposal_mode(1)
    res = o.partition_run(oracle_mod.default_params())
    assert nmi(truth, res["b"]) > 0.9
