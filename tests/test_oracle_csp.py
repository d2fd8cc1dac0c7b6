"""Pins for oracle/csp.py.

* the hand-worked example of SURVEY §8c (fixture tests/golden/csp_worked_example.json);
* special cases: n=1 (every subnet shares everything) degenerates to strictly sequential
  execution; D=1 gives F0 B0 F1 B1 ...;
* the dependency table agrees with Algorithm 2 executed verbatim on every
  decision of random CSP runs;
* every simulated trace satisfies the Table 4 access pattern and the checker
  rejects mutated traces;
* the partition follows its definition on hand cases.
"""
import json
import os

import numpy as np
import pytest

import synth
from oracle import csp

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _unit_costs(choices, sob, D, cf=1, cb=2):
    m, n = len(sob), int(np.max(choices)) + 1
    return csp.task_costs(choices, sob, np.full((m, n), cf), np.full((m, n), cb), D)


def test_worked_example():
    with open(os.path.join(GOLD, "csp_worked_example.json")) as f:
        g = json.load(f)
    choices = np.array(g["choices"])
    sob = np.array(g["stage_of_block"])
    D = g["D"]
    cf, cb = _unit_costs(choices, sob, D, g["cf"], g["cb"])
    for K in range(D):
        got = [sorted(csp.deps(choices, sob, y, K)) for y in range(len(choices))]
        assert got == g["deps"][K]
    res = csp.simulate_csp(choices, sob, D, g["W"], cf, cb, lam=0, policy=0)
    assert res["makespan"] == g["makespan"]
    assert res["stall"] == g["stall"] and res["bubble"] == g["bubble"]
    for K in range(D):
        got = [("F" if k == 0 else "B") + f"{y}@{t}" for (t, KK, k, y) in res["trace"] if KK == K]
        assert got == g["stage_order"][K]
    assert csp.check_trace(res["trace"], choices, sob, D) == []


def test_worked_example_variants():
    sob = np.array([0, 1])
    ch = np.zeros((3, 2), dtype=int)             # every subnet identical: fully serial
    cf, cb = csp.task_costs(ch, sob, np.ones((2, 2)), np.full((2, 2), 2), 2)
    assert csp.simulate_csp(ch, sob, 2, 4, cf, cb)["makespan"] == 18   # = 3 * 2 * 3
    ch4 = np.array([[0, 0], [1, 0], [0, 1], [1, 1]])
    sob1 = np.array([0, 0])
    cf, cb = csp.task_costs(ch4, sob1, np.full((2, 2), 0), np.full((2, 2), 0), 1)
    # D = 1 with a stage cost of 1 / 2 ticks (costs are per stage here)
    cf[:] = 1
    cb[:] = 2
    res = csp.simulate_csp(ch4, sob1, 1, 4, cf, cb)
    assert res["makespan"] == 12
    assert res["order"][0] == [(0, 0), (1, 0), (0, 1), (1, 1), (0, 2), (1, 2), (0, 3), (1, 3)]


@pytest.mark.parametrize("D", [1, 2, 3, 4])
def test_single_choice_is_sequential(D):
    """n = 1: every subnet depends on its predecessor everywhere -> makespan = N*D*(cf+cb)."""
    N, m = 5, 4
    ch = np.zeros((N, m), dtype=int)
    sob = np.array([b * D // m for b in range(m)])
    cf = np.ones((D, N), dtype=int)
    cb = np.full((D, N), 2)
    res = csp.simulate_csp(ch, sob, D, 4 * D, cf, cb)
    assert res["makespan"] == N * D * 3
    # strictly sequential: subnet y+1 starts only after subnet y's last backward
    starts = {(k, y, K): t for t, K, k, y in res["trace"]}
    for y in range(N - 1):
        assert starts[(0, y + 1, 0)] >= starts[(1, y, 0)] + 2


def test_disjoint_subnets_pipeline_fully():
    """No shared candidates: F tasks stream back to back on stage 0 (limited by W)."""
    N, m, D = 6, 2, 2
    ch = np.array([[y, y] for y in range(N)])
    sob = np.array([0, 1])
    cf = np.ones((D, N), dtype=int)
    cb = np.full((D, N), 2)
    res = csp.simulate_csp(ch, sob, D, 8, cf, cb)
    f0 = [t for t, K, k, y in res["trace"] if K == 0 and k == 0]
    assert f0[:2] == [0, 1]
    assert res["makespan"] < N * D * 3


def _alg2_admit(choices, sob):
    L_SN = [[(b, int(c)) for b, c in enumerate(row)] for row in choices]

    def admit(K, inF, fin):
        Lq = sorted(inF)
        _, qval = csp.literal_alg2(Lq, fin, L_SN, K, sob)
        return None if qval < 0 else qval
    return admit


@pytest.mark.parametrize("seed", range(12))
def test_dep_table_equals_literal_alg2(seed):
    rng = np.random.default_rng(seed)
    N = int(rng.integers(4, 14))
    m = int(rng.integers(1, 6))
    n = int(rng.integers(1, 4))
    D = int(rng.integers(1, m + 1))
    W = int(rng.integers(1, 3 * D + 2))
    ch = synth.sample_choices(N, m, n, seed)
    _, sob = np.unique(np.sort(rng.integers(0, D, size=m)), return_inverse=True)
    Dn = int(sob.max()) + 1
    cf = rng.integers(1, 4, size=(Dn, N))
    cb = rng.integers(1, 5, size=(Dn, N))
    lam = int(rng.integers(0, 2))
    ref = csp.simulate_csp(ch, sob, Dn, W, cf, cb, lam=lam)
    alt = csp.simulate_csp(ch, sob, Dn, W, cf, cb, lam=lam, admit=_alg2_admit(ch, sob))
    assert ref["trace"] == alt["trace"]
    assert csp.check_trace(ref["trace"], ch, sob, Dn) == []


@pytest.mark.parametrize("seed", range(8))
def test_idle_accounting_identity(seed):
    """Per stage: busy + stall + bubble = makespan; n = 1 on D = 1 has no idle time."""
    rng = np.random.default_rng(seed)
    N, m, n, D = 9, 4, int(rng.integers(1, 4)), int(rng.integers(1, 5))
    ch = synth.sample_choices(N, m, n, seed)
    sob = np.array([b * D // m for b in range(m)])
    cf = rng.integers(1, 4, size=(D, N))
    cb = rng.integers(1, 5, size=(D, N))
    res = csp.simulate_csp(ch, sob, D, 2 * D, cf, cb, lam=int(rng.integers(0, 2)))
    for K in range(D):
        busy = int(cf[K].sum() + cb[K].sum())
        assert busy + res["stall"][K] + res["bubble"][K] == res["makespan"]
    if D == 1:
        assert res["stall"] == [0] and res["bubble"] == [0]


@pytest.mark.parametrize("policy", [0, 1])
def test_random_traces_are_csp_valid(policy):
    for seed in range(10):
        rng = np.random.default_rng(100 + seed)
        N, m, n, D = 10, 4, int(rng.integers(2, 5)), int(rng.integers(1, 5))
        ch = synth.sample_choices(N, m, n, seed)
        sob = np.array([b * D // m for b in range(m)])
        cf = rng.integers(1, 4, size=(D, N))
        cb = rng.integers(1, 5, size=(D, N))
        res = csp.simulate_csp(ch, sob, D, 2 * D, cf, cb, policy=policy)
        assert csp.check_trace(res["trace"], ch, sob, D) == []
        # the version invariant holds along the trace
        v = csp.expected_versions(ch)
        ver = {}
        for t, K, k, y in res["trace"]:
            for b in csp.stage_blocks(sob, K):
                l = (b, int(ch[y][b]))
                assert ver.get(l, 0) == v[y, b]
                if k == 1:
                    ver[l] = ver.get(l, 0) + 1


def test_checker_rejects_mutations():
    ch = np.array([[0, 0], [1, 0], [0, 1], [1, 1]])
    sob = np.array([0, 1])
    cf, cb = _unit_costs(ch, sob, 2)
    tr = csp.simulate_csp(ch, sob, 2, 4, cf, cb)["trace"]
    assert csp.check_trace(tr, ch, sob, 2) == []
    # move F(2,0) before B(0,0): subnet 2 reads candidate (0,0) before subnet 0 wrote it
    i_f2 = next(i for i, e in enumerate(tr) if e[1] == 0 and e[2] == 0 and e[3] == 2)
    i_b0 = next(i for i, e in enumerate(tr) if e[1] == 0 and e[2] == 1 and e[3] == 0)
    bad = list(tr)
    bad.insert(i_b0, bad.pop(i_f2))
    assert csp.check_trace(bad, ch, sob, 2) != []
    # drop a task
    assert csp.check_trace(tr[:-1], ch, sob, 2) != []


def test_table4_pattern_example():
    """Table 4: a layer used by subnets 2, 5, 7 is accessed 2F-2B-5F-5B-7F-7B."""
    N, m = 8, 3
    ch = np.array([[y, 0 if y in (2, 5, 7) else y + 1, y] for y in range(N)])
    for D in (1, 3):
        sob = np.array([b * D // m for b in range(m)])
        cf = np.ones((D, N), dtype=int)
        cb = np.full((D, N), 2)
        tr = csp.simulate_csp(ch, sob, D, 4 * D, cf, cb)["trace"]
        K1 = sob[1]
        seq = [("F" if k == 0 else "B") + str(y) for t, K, k, y in tr if K == K1 and y in (2, 5, 7)]
        assert seq == ["F2", "B2", "F5", "B5", "F7", "B7"]


def test_partition_hand_cases():
    assert list(csp.balanced_partition([1, 1, 1, 1], 2)) == [0, 0, 1, 1]
    assert list(csp.balanced_partition([3, 1, 1, 1], 2)) == [0, 1, 1, 1]
    assert list(csp.balanced_partition([1, 1, 1], 2)) == [0, 1, 1]          # tie -> earliest
    assert list(csp.balanced_partition([5, 1, 1, 1, 1, 5], 3)) == [0, 1, 1, 1, 1, 2]
    assert list(csp.balanced_partition([2, 2, 2], 3)) == [0, 1, 2]
    assert list(csp.balanced_partition([7], 1)) == [0]


def test_dep_table_small():
    ch = np.array([[0, 1], [0, 0], [1, 1], [0, 1]])
    np.testing.assert_array_equal(csp.dep_table(ch), [[-1, -1], [0, -1], [-1, 0], [1, 2]])
    np.testing.assert_array_equal(csp.expected_versions(ch), [[0, 0], [1, 0], [0, 1], [2, 2]])


# ------------------------------------------------------------------ other sync policies (§8f(1))
def _unit(choices, D, m):
    sob = np.repeat(np.arange(D), m // D)
    ones = np.ones((m, int(np.max(choices)) + 1), dtype=np.int64)
    return sob, csp.task_costs(choices, sob, ones, 2 * ones, D)


def test_bsp_hand_example():
    """D=2, bulk 2, cf=1, cb=2: both forwards before the backwards on each stage, then the
    flush (derived tick by tick: stage 0 F0@0 F1@1 B0@5 B1@7, stage 1 F0@1 F1@2 B0@3 B1@5)."""
    ch = np.array([[0, 0], [0, 0]])
    sob, (tf, tb) = _unit(ch, 2, 2)
    r = csp.simulate_csp(ch, sob, 2, 8, tf, tb, sync="bsp", bulk=2)
    s0 = [("F" if k == 0 else "B") + f"{y}@{t}" for t, K, k, y in r["trace"] if K == 0]
    s1 = [("F" if k == 0 else "B") + f"{y}@{t}" for t, K, k, y in r["trace"] if K == 1]
    assert s0 == ["F0@0", "F1@1", "B0@5", "B1@7"] and s1 == ["F0@1", "F1@2", "B0@3", "B1@5"]
    assert r["makespan"] == 9
    # bulk 1: one subnet at a time, fully serial: N * D * (cf + cb), 2 blocks per stage
    ch4 = synth.sample_choices(4, 4, 3)
    sob, (tf, tb) = _unit(ch4, 2, 4)
    r1 = csp.simulate_csp(ch4, sob, 2, 8, tf, tb, sync="bsp", bulk=1)
    assert r1["makespan"] == 4 * 2 * (2 + 4) and csp.check_trace(r1["trace"], ch4, sob, 2) == []


def test_inorder_is_causal_and_never_overtakes():
    """NASPipe w/o scheduler (Fig.6): forwards start in id order on every stage and the trace
    is still causally valid (so its numerics are the sequential result)."""
    for seed in range(8):
        ch = synth.sample_choices(24, 8, 2, seed)
        sob, (tf, tb) = _unit(ch, 4, 8)
        r = csp.simulate_csp(ch, sob, 4, 16, tf, tb, sync="inorder")
        assert csp.check_trace(r["trace"], ch, sob, 4) == []
        for K in range(4):
            fw = [y for k, y in r["order"][K] if k == 0]
            assert fw == sorted(fw)


def test_serial_is_one_pipeline_at_a_time():
    """NASPipe w/o scheduler as P:L454 words it ("had to finish the execution of a pipeline
    before injecting the next pipeline"; reading A32): one subnet in flight.  Closed form with
    per-stage task costs cf, cb and latency 0: every subnet's F(y, 0..D-1) then B(y, D-1..0)
    runs alone, so makespan = sum_y sum_K (cf + cb) and every stage idles (D - 1) / D of it
    when the costs are uniform; the order is F0..FD-1 B.. per subnet, ascending ids."""
    for seed in range(4):
        ch = synth.sample_choices(12, 8, 3, seed)
        sob, (tf, tb) = _unit(ch, 4, 8)
        r = csp.simulate_csp(ch, sob, 4, 16, tf, tb, sync="serial")
        assert r["makespan"] == int(sum(tf[K][y] + tb[K][y] for K in range(4) for y in range(12)))
        assert csp.check_trace(r["trace"], ch, sob, 4) == []
        ys = [y for _, _, _, y in r["trace"]]
        assert ys == sorted(ys)          # subnet y's 2D tasks all precede y + 1's
    ch = synth.sample_choices(10, 8, 3, 9)
    sob = [b * 4 // 8 for b in range(8)]
    D, N = 4, 10
    tf = [[1] * N for _ in range(D)]
    tb = [[2] * N for _ in range(D)]
    r = csp.simulate_csp(ch, sob, D, 16, tf, tb, sync="serial")
    assert r["makespan"] == N * D * 3
    for K in range(D):
        assert r["stall"][K] + r["bubble"][K] == N * D * 3 - N * 3     # idle (D-1)/D of the time


def test_asp_is_the_no_dependency_schedule():
    ch = synth.sample_choices(20, 8, 2, 3)
    sob, (tf, tb) = _unit(ch, 4, 8)
    a = csp.simulate_csp(ch, sob, 4, 16, tf, tb, sync="asp")
    b = csp.simulate_csp(ch, sob, 4, 16, tf, tb, ignore_deps=True)
    assert a["trace"] == b["trace"]
    # with conflicts it violates the Table 4 access pattern (CSP never does)
    assert csp.check_trace(a["trace"], ch, sob, 4) != []
    assert csp.check_trace(csp.simulate_csp(ch, sob, 4, 16, tf, tb)["trace"], ch, sob, 4) == []


# ---------------------------------------------------------------------- §8f(2) mirroring
def _mirror_golden():
    with open(os.path.join(os.path.dirname(__file__), "golden", "mirror_worked_example.json")) as f:
        return json.load(f)


def test_mirrored_worked_example():
    g = _mirror_golden()
    sob = csp.subnet_partitions(g["choices"], g["cost_f"], g["cost_b"], g["D"])
    assert sob.tolist() == g["stage_of_block"]
    for key, lw in (("lam_w_0", 0), ("lam_w_3", 3)):
        r = csp.simulate_csp_mirrored(g["choices"], sob, g["D"], g["W"], g["cost_f"], g["cost_b"], lam_w=lw)
        assert [list(t) for t in r["trace"]] == g[key]["trace"], key
        assert r["makespan"] == g[key]["makespan"], key
        assert csp.check_trace_mirrored(r["trace"], g["choices"], sob, g["D"], g["cost_b"], lam_w=lw) == []
    r = csp.simulate_csp_mirrored(g["choices"], sob, g["D"], g["W"], g["cost_f"], g["cost_b"])
    assert r["stall"] == g["lam_w_0"]["stall"] and r["bubble"] == g["lam_w_0"]["bubble"]


@pytest.mark.parametrize("seed", range(6))
def test_mirrored_reduces_to_o2_on_a_common_partition(seed):
    """Every subnet on the supernet partition, no mirror latency: exactly simulate_csp."""
    rng = np.random.default_rng(100 + seed)
    m, n, D, N, W, lam = 6, 3, 3, 14, 3, seed % 2
    ch = rng.integers(0, n, (N, m)).tolist()
    cf, cb = rng.integers(0, 5, (m, n)), rng.integers(1, 9, (m, n))
    sob = csp.balanced_partition(csp.block_partition_cost(cf, cb), D)
    a = csp.simulate_csp(ch, sob, D, W, *csp.task_costs(ch, sob, cf, cb, D), lam=lam)
    b = csp.simulate_csp_mirrored(ch, [sob] * N, D, W, cf, cb, lam=lam)
    for k in ("trace", "makespan", "stall", "bubble"):
        assert a[k] == b[k], k


@pytest.mark.parametrize("D", [2, 3])
def test_mirrored_single_choice_is_sequential(D):
    """n = 1: every subnet shares every candidate (and so has the same partition): the
    schedule is strictly sequential, makespan = N * (sum of the subnet's task costs)."""
    m, N = 5, 6
    cf = np.array([[1], [3], [2], [4], [1]])
    cb = 2 * cf
    ch = [[0] * m for _ in range(N)]
    sob = csp.subnet_partitions(ch, cf, cb, D)
    r = csp.simulate_csp_mirrored(ch, sob, D, 4, cf, cb)
    per = sum(max(1, int(sum(cf[b][0] for b in range(m) if sob[0][b] == K))) +
              max(1, int(sum(cb[b][0] for b in range(m) if sob[0][b] == K))) for K in range(D))
    assert r["makespan"] == N * per


@pytest.mark.parametrize("seed", range(8))
def test_mirrored_traces_are_csp_valid_and_idle_adds_up(seed):
    rng = np.random.default_rng(200 + seed)
    m, n, D, N = int(rng.integers(3, 8)), int(rng.integers(2, 5)), int(rng.integers(2, 4)), 16
    ch = rng.integers(0, n, (N, m)).tolist()
    cf, cb = rng.integers(0, 6, (m, n)), rng.integers(0, 12, (m, n))
    sob = csp.subnet_partitions(ch, cf, cb, D)
    for lw in (0, 2):
        r = csp.simulate_csp_mirrored(ch, sob, D, 4, cf, cb, lam_w=lw)
        assert csp.check_trace_mirrored(r["trace"], ch, sob, D, cb, lam_w=lw) == []
        for K in range(D):
            busy = 0
            for (t, KK, kind, y) in r["trace"]:
                if KK == K:
                    bl = [b for b in range(m) if sob[y][b] == K]
                    busy += max(1, int(sum((cf if kind == 0 else cb)[b][ch[y][b]] for b in bl)))
            assert busy + r["stall"][K] + r["bubble"][K] == r["makespan"]


def test_mirrored_checker_rejects_early_read():
    g = _mirror_golden()
    sob = np.array(g["stage_of_block"])
    bad = [list(t) for t in g["lam_w_0"]["trace"]]
    bad[5] = [17, 1, 0, 1]   # F(1, stage 1) one tick before the WRITE of (1,0) lands
    assert csp.check_trace_mirrored(bad, g["choices"], sob, g["D"], g["cost_b"])
    assert csp.check_trace_mirrored(g["lam_w_0"]["trace"], g["choices"], sob, g["D"], g["cost_b"], lam_w=3)


# ---------------------------------------------------------------------- §8f(3) Alg.3
def test_alg3_predictions_on_the_worked_example():
    """Alg.3's backward branch replayed on SURVEY §8c's worked example, derived
    by hand from its stage orders: before B(x,K) the stage pre-finishes x and runs Alg.2 on
    its queue.  Stage 0: B0@4 sees queue {2,3} -> predicts F2 (next: F2@6), B1@7 -> F3 (F3@9).
    Stage 1: B0@2 sees {1} (F1 delivered at tick 2) -> F1 (F1@4); B1@5 and B2@8 see an empty
    queue (F2 / F3 not yet delivered) -> no prediction, although F2@7 / F3@10 follow."""
    with open(os.path.join(GOLD, "csp_worked_example.json")) as f:
        g = json.load(f)
    N, D = len(g["choices"]), g["D"]
    cf = [[g["cf"]] * N for _ in range(D)]
    cb = [[g["cb"]] * N for _ in range(D)]
    got = csp.alg3_backward_predictions(g["choices"], g["stage_of_block"], D, g["W"], cf, cb)
    assert got == [(2, 1, 0, 1, 1), (4, 0, 0, 2, 2), (5, 1, 1, None, 2), (7, 0, 1, 3, 3), (8, 1, 2, None, 3),
                   (10, 0, 2, None, None), (11, 1, 3, None, None), (13, 0, 3, None, None)]


def test_alg3_predictions_are_never_wrong_when_made_at_d1():
    """D = 1: after B(x) the stage runs the lowest admissible queued forward, which is
    exactly Alg.2 on L_f + {x}: every prediction made equals the next forward."""
    rng = np.random.default_rng(3)
    ch = rng.integers(0, 3, (20, 5)).tolist()
    cf, cb = np.ones((1, 20), dtype=np.int64), 2 * np.ones((1, 20), dtype=np.int64)
    preds = csp.alg3_backward_predictions(ch, [0] * 5, 1, 4, cf, cb)
    assert len(preds) == 20
    assert all(p == a for (_, _, _, p, a) in preds if p is not None)
