"""Pins for oracle/residency.py.

* worked example 2 of SURVEY §8c (fixture tests/golden/residency_worked_example.json);
* special cases: budget >= the whole stage loads every candidate exactly once and never
  evicts; budget 0 means everything resident (no traffic); a budget below one task's need
  is an error; Belady is never worse than FIFO-like demand loading on random plans.
"""
import json
import os

import numpy as np
import pytest

import synth
from oracle import csp, residency

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _worked_plan():
    ch = np.array([[0, 0], [1, 0], [0, 1], [1, 1]])
    sob = np.array([0, 0])
    cf = np.ones((1, 4), dtype=int)
    cb = np.full((1, 4), 2)
    order = csp.simulate_csp(ch, sob, 1, 4, cf, cb)["order"][0]
    uses = residency.stage_uses(order, ch, [0, 1], 2)
    kinds = [k for k, _ in order]
    return uses, kinds


def test_worked_example_2():
    with open(os.path.join(GOLD, "residency_worked_example.json")) as f:
        g = json.load(f)
    uses, kinds = _worked_plan()
    nbytes = {u: 1 for u in range(4)}
    for budget, expect in g["traces"].items():
        ev = residency.simulate_residency(uses, kinds, nbytes, int(budget), L=g["L"])["events"]
        got = [f"{op}({i},{u})" for op, i, u in ev]
        assert got == expect, budget


def test_writeback_only_if_dirty():
    uses, kinds = _worked_plan()
    res = residency.simulate_residency(uses, kinds, {u: 1 for u in range(4)}, 3)
    # uid 2 = (block 1, choice 0) is evicted at task 4 after B0 and B1 updated it
    assert res["writebacks"] == [(4, 2)]
    # a read-only plan (no backward) never writes back
    res = residency.simulate_residency(uses, [0] * len(uses), {u: 1 for u in range(4)}, 2)
    assert res["writebacks"] == []


def test_budget_errors_and_special_cases():
    uses, kinds = _worked_plan()
    with pytest.raises(residency.BudgetError):
        residency.simulate_residency(uses, kinds, {u: 1 for u in range(4)}, 1)
    assert residency.simulate_residency(uses, kinds, {u: 1 for u in range(4)}, 0)["events"] == []


@pytest.mark.parametrize("seed", range(6))
def test_large_budget_loads_once(seed):
    rng = np.random.default_rng(seed)
    N, m, n = 12, 3, 3
    ch = synth.sample_choices(N, m, n, seed)
    order = [(k, y) for y in range(N) for k in (0, 1)]
    uses = residency.stage_uses(order, ch, list(range(m)), n)
    nbytes = {u: int(rng.integers(1, 5)) for u in range(m * n)}
    total = sum(nbytes.values())
    ev = residency.simulate_residency(uses, [k for k, _ in order], nbytes, total)["events"]
    loads = [u for op, _, u in ev if op == "LOAD"]
    assert sorted(loads) == sorted(set().union(*uses))
    assert all(op == "LOAD" for op, _, _ in ev)


def test_horizon_reading():
    """A26: a horizon covering the whole plan is the unbounded rule; horizon 1 sees only the
    current task, so every non-needed candidate is 'never used again' and ties go to the
    lowest uid (worked example, budget 3: at task 4 uid 1 is evicted instead of uid 2)."""
    uses, kinds = _worked_plan()
    nbytes = {u: 1 for u in range(4)}
    full = residency.simulate_residency(uses, kinds, nbytes, 3)
    assert residency.simulate_residency(uses, kinds, nbytes, 3, horizon=len(uses)) == full
    short = residency.simulate_residency(uses, kinds, nbytes, 3, L=1, horizon=1)["events"]
    assert [f"{op}({i},{u})" for op, i, u in short] == [
        "LOAD(0,0)", "LOAD(0,2)", "LOAD(2,1)", "EVICT(4,1)", "LOAD(4,3)", "EVICT(6,0)", "LOAD(6,1)"]


@pytest.mark.parametrize("seed", range(6))
def test_belady_optimal_on_unit_sizes(seed):
    """Unit sizes, L=1: Belady's rule minimises loads; compare against exhaustive search
    over eviction choices on a tiny instance."""
    N, m, n = 5, 2, 3
    ch = synth.sample_choices(N, m, n, seed)
    order = [(k, y) for y in range(N) for k in (0, 1)]
    uses = residency.stage_uses(order, ch, list(range(m)), n)
    budget = 3
    ev = residency.simulate_residency(uses, [0] * len(uses), {u: 1 for u in range(m * n)},
                                      budget, L=1)["events"]
    n_loads = sum(op == "LOAD" for op, _, _ in ev)

    best = [10 ** 9]

    def search(i, resident, loads):
        if loads >= best[0]:
            return
        if i == len(uses):
            best[0] = loads
            return
        need = uses[i]
        missing = need - resident
        extra = len(resident | need) - budget
        cands = sorted(resident - need)
        from itertools import combinations
        if extra <= 0:
            search(i + 1, resident | need, loads + len(missing))
            return
        for ev_set in combinations(cands, extra):
            search(i + 1, (resident - set(ev_set)) | need, loads + len(missing))

    search(0, set(), 0)
    assert n_loads == best[0]
