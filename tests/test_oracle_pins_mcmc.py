"""Pins of the oracle's MCMC driver (R:O.8, Z10, Z19, Z20) against things other
than itself: hand-computed stopping iterations of the GraphChallenge rule, the
batch semantics written out step by step from the per-vertex functions (whose
own pins are in test_oracle_pins.py), and the threshold slot characterised
from the round trace.

Table 2 (§4.1) names only the parameters (max_num_nodal_itr,
delta_entropy_threshold1/2, delta_entropy_moving_avg_window,
num_batches_for_MCMC); the readings are DESIGN.md Z10, Z19, Z20.
"""
import numpy as np
import pytest

from gen import dcsbm

SEED = dcsbm.RUN_SEED


# ------------------------------------------------------------ stopping rule
# Rule (R:Z19): after iteration itr >= w-1, with the GraphChallenge slice
# D[itr-w+1 : itr) (for w = 3: the two iterations BEFORE itr) and the MDL of
# the state after iteration itr, stop iff -mean(slice) < thresh * MDL.
# Each case below is computed by hand in its comment, and each is chosen so
# that a plausible mis-reading gives a different answer (noted per case).
STOP_CASES = [
    # theta*MDL = 0.01 * 1000 = 10.
    # itr2: mean(D0,D1) = -50 -> 50 >= 10 go on;  itr3: mean(D1,D2) = -50 go on;
    # itr4: mean(D2,D3) = -25.5 go on;           itr5: mean(D3,D4) = -1 -> 1 < 10 stop: 6 ran.
    # (3-entry slice incl. D[itr]: itr5 mean(-1,-1,-30) = -10.67 -> goes on;
    #  current-only: stops at itr3 -> 4;  3 entries before itr: itr5 mean(-50,-1,-1) goes on)
    dict(D=[-50, -50, -50, -1, -1, -30, -30, -30], mdl=[1000] * 8, w=3, th=0.01, ran=6),
    # MDL taken AFTER the iteration: itr4: mean(-6,-6) = -6 vs 0.01 * MDL4 = 4 -> go on;
    # itr5: 6 < 10 stop -> 6 ran.  (MDL before the iteration, MDL3 = 1000, stops at itr4 -> 5)
    dict(D=[-50, -50, -6, -6, -6, -6, -6, -6], mdl=[1000, 1000, 1000, 1000, 400, 1000, 1000, 1000],
         w=3, th=0.01, ran=6),
    # strict '<': -mean == theta*MDL (0.5 * 20 = 10) never stops -> all 4 iterations run
    dict(D=[-10, -10, -10, -10], mdl=[20] * 4, w=3, th=0.5, ran=4),
    # no test before itr = w-1 = 2, even when D already says "converged"
    dict(D=[0, 0, 0, 0], mdl=[100] * 4, w=3, th=0.01, ran=3),
    # a worsening phase (positive D) stops at the first test
    dict(D=[5, 5, 5, 5], mdl=[100] * 4, w=3, th=1e-4, ran=3),
    # w = 2: slice [itr-1, itr) = D[itr-1]:  itr1: -50 go on; itr2: D1 = -3 -> 3 < 10 stop: 3 ran
    dict(D=[-50, -3, -50, -50], mdl=[1000] * 4, w=2, th=0.01, ran=3),
    # w = 1: the slice [itr, itr) is empty, mean 0 -> 0 < theta*MDL: stops after the first iteration
    dict(D=[-50, -50, -50], mdl=[1000] * 3, w=1, th=0.01, ran=1),
    # w = 4: slice D[itr-3 : itr) (3 entries): itr3: mean(-30,-30,-3) = -21 go on;
    # itr4: mean(-30,-3,-3) = -12 go on; itr5: mean(-3,-3,-3) = -3 -> stop: 6 ran
    dict(D=[-30, -30, -3, -3, -3, -3, -3], mdl=[1000] * 7, w=4, th=0.01, ran=6),
    # the default thresholds on a 1K-sized MDL: 5e-4 * 24000 = 12; mean(-20,-13) = -16.5 go on,
    # mean(-13,-11.5) = -12.25 go on, mean(-11.5,-2) = -6.75 -> stop at itr4: 5 ran
    dict(D=[-20, -13, -11.5, -2, -1, -1], mdl=[24000] * 6, w=3, th=5e-4, ran=5),
]


@pytest.mark.parametrize("case", range(len(STOP_CASES)))
def test_mcmc_stop_rule_hand_cases(oracle_mod, case):
    c = STOP_CASES[case]
    assert oracle_mod.mcmc_stop_mock(c["D"], c["mdl"], c["w"], c["th"]) == c["ran"]


# ----------------------------------------------------------- batch semantics
def _small_graph():
    rowptr, col, _ = dcsbm.random_multigraph(60, 420, 7)
    b0 = dcsbm.random_partition(60, 8, 3)
    return rowptr, col, b0


def _batches(V, nb):
    bs = (V + nb - 1) // nb
    return [(k * bs, min(V, (k + 1) * bs) - k * bs) for k in range(nb) if k * bs < V]


def test_mcmc_phase_is_the_snapshot_composition(oracle_mod):
    """mcmc_phase == the reading written out (Z10, Z19, Z20): per iteration,
    num_batches contiguous id ranges of ceil(V/4); every vertex of a batch is
    proposed and evaluated on the batch-start state; then all accepted moves
    are applied and M rebuilt; D[itr] = sum of the accepted (stale) dS; the
    GraphChallenge stopping test on the MDL after the iteration."""
    rowptr, col, b0 = _small_graph()
    V = len(rowptr) - 1
    p = oracle_mod.default_params(max_nodal_itr=12, thresh1=2e-3)
    o = oracle_mod.Oracle(rowptr, col)
    o.set_partition(b0, 8)
    ran, st, D = o.mcmc_phase(p, 3, p.thresh1, return_D=True)

    ref = oracle_mod.Oracle(rowptr, col)
    ref.set_partition(b0, 8)
    Dr = []
    for itr in range(p.max_nodal_itr):
        d = 0.0
        for first, count in _batches(V, p.num_batches):
            s = ref.propose(1, SEED, 3, itr, first, count)
            dS, H, pr, acc = ref.delta_move(SEED, 3, itr, first, count, s)
            d += float(np.sum(dS[acc == 1]))
            ref.apply_moves(first, count, s, acc)
            ref.rebuild()
        Dr.append(d)
        if itr >= 2:
            mdl = ref.mdl()[0]
            if -np.mean(Dr[itr - 2:itr]) < p.thresh1 * mdl:
                break
    assert ran == len(Dr) and ran >= 3
    assert np.allclose(D, Dr, rtol=1e-12, atol=1e-12)
    assert np.array_equal(o.partition()[0], ref.partition()[0])


def test_batch_snapshot_differs_from_sequential_gibbs(oracle_mod):
    """The composition above can tell snapshot semantics from immediate
    application: on this graph one batch applied vertex by vertex (each move
    seen by the next proposal, sequential Gibbs) ends in a different b than
    mcmc_batch (batch-start snapshot, P:176 batched parallel MCMC, R:Z10)."""
    rowptr, col, b0 = _small_graph()
    V = len(rowptr) - 1
    p = oracle_mod.default_params()
    first, count = 0, (V + 3) // 4
    o = oracle_mod.Oracle(rowptr, col)
    o.set_partition(b0, 8)
    D = o.mcmc_batch(p, 0, 0, first, count)
    b_snap = o.partition()[0]

    seq = oracle_mod.Oracle(rowptr, col)
    seq.set_partition(b0, 8)
    Dseq = 0.0
    for v in range(first, first + count):
        s = seq.propose(1, SEED, 0, 0, v, 1)
        dS, H, pr, acc = seq.delta_move(SEED, 0, 0, v, 1, s)
        if acc[0]:
            Dseq += dS[0]
        seq.apply_moves(v, 1, s, acc)
        seq.rebuild()
    b_seq = seq.partition()[0]
    assert not np.array_equal(b_snap, b_seq)
    # and the snapshot result is exactly: propose all, evaluate all, then apply
    ref = oracle_mod.Oracle(rowptr, col)
    ref.set_partition(b0, 8)
    s = ref.propose(1, SEED, 0, 0, first, count)
    dS, H, pr, acc = ref.delta_move(SEED, 0, 0, first, count, s)
    ref.apply_moves(first, count, s, acc)
    assert np.array_equal(ref.partition()[0], b_snap)
    assert abs(D - float(np.sum(dS[acc == 1]))) <= 1e-12 * max(1.0, abs(D))


def test_partition_threshold_slot(oracle_mod):
    """thresh1 (5e-4) until the golden-section bracket is established, thresh2
    (1e-4) after (R:Z19).  While B only decreases (merge-down), the bracket's
    low slot is filled by the first round whose MDL is worse than the best so
    far; every round up to and including that one ran with thresh1."""
    rowptr, col, truth, cfg = dcsbm.make("1k")
    o = oracle_mod.Oracle(rowptr, col)
    p = oracle_mod.default_params()
    res = o.partition_run(p)
    tr = res["trace"]
    mdl = tr[:, 3]
    worse = [j for j in range(1, len(tr)) if mdl[j] > mdl[:j].min()]
    assert worse, "the 1K run must establish a bracket"
    k0 = worse[0]
    assert np.all(np.diff(tr[:k0 + 1, 1]) < 0), "merge-down rounds decrease B"
    assert np.all(tr[:k0 + 1, 4] == p.thresh1)
    assert np.all(tr[k0 + 1:, 4] == p.thresh2)
    # and the rounds' accepted-move column adds up to the run's statistic
    assert int(tr[:, 5].sum()) == res["stats"].n_move_acc


def test_bracket_replay_consistent_with_partition_trace(oracle_mod):
    """The replay entry (used to check another driver's trace) on the oracle's
    own 1K run: each round's B after its merge is at most the replayed restart
    B minus K (less only when merged groups held no vertex, R:Z18), the
    threshold slot of every later round matches the replayed bracket state,
    and the search stops after exactly the rounds the run did."""
    rowptr, col, truth, cfg = dcsbm.make("1k")
    p = oracle_mod.default_params()
    res = oracle_mod.Oracle(rowptr, col).partition_run(p)
    tr = res["trace"]
    Bn, Kn, br, stop = oracle_mod.bracket_replay(tr[:, 1].astype(np.int32), tr[:, 3], p.reduction_rate)
    assert stop == len(tr)
    assert tr[0, 1] <= cfg.V - int(cfg.V * p.reduction_rate)
    for k in range(len(tr) - 1):
        assert 0 < tr[k + 1, 1] <= Bn[k] - Kn[k]
        assert tr[k + 1, 4] == (p.thresh2 if br[k] else p.thresh1)
    # mock: a unimodal MDL(B) table replayed round by round ends where golden_mock ends
    V = 500
    mdl = np.array([(B - 77) ** 2 + 0.3 * B for B in range(V + 1)], np.float64)
    vis, Bf = oracle_mod.golden_mock(V, 0.4, mdl)
    Bn, Kn, br, stop = oracle_mod.bracket_replay(vis, mdl[vis], 0.4)
    assert stop == len(vis) and Bf == 77
    assert all(vis[k + 1] == Bn[k] - Kn[k] for k in range(len(vis) - 1))


def test_openmp_mode_gives_identical_results(oracle_mod):
    """The all-core mode changes nothing: same partition, MDL and
    trace as the single-threaded canonical run."""
    rowptr, col, truth, cfg = dcsbm.make("1k")
    p = oracle_mod.default_params()
    try:
        a = oracle_mod.Oracle(rowptr, col).partition_run(p)
        assert oracle_mod.set_threads(4) >= 1
        b = oracle_mod.Oracle(rowptr, col).partition_run(p)
    finally:
        oracle_mod.set_threads(1)
    assert np.array_equal(a["b"], b["b"]) and a["mdl"] == b["mdl"]
    assert np.array_equal(a["trace"], b["trace"])
