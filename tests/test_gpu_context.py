"""Context switching on the GPU (readings A9, A26).

With an HBM weight budget smaller than the stage's candidates, every candidate starts in the
pinned host stash and is loaded / evicted around the planned tasks.  Checks:
* the executed LOAD/EVICT trace equals the oracle's Belady plan (O6 with horizon H) on the
  oracle's CSP schedule, bit-exactly;
* parameters and losses are bitwise identical to the all-resident run (residency never
  changes numerics), and match the sequential oracle;
* transfer accounting: H2D bytes = loads x candidate bytes (+ batches), write-backs only
  for candidates updated since their load.
"""
import numpy as np
import pytest

import synth
from oracle import csp, residency, train

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _run(cfg, choices, batches, D, budget, horizon=0):
    spec = npipe.Spec(cfg, flags=npipe.FLAG_TRACE | npipe.FLAG_VERSION_CHECK, hbm_weight_budget_bytes=budget,
                      residency_horizon=horizon)
    h = npipe.naspipe_create(spec, D)
    for y, ch in enumerate(choices):
        npipe.naspipe_submit(h, ch, *batches[y])
    npipe.naspipe_drain(h)
    params = {(b, c): npipe.naspipe_get_params(h, b, c)
              for b in range(cfg["n_blocks"]) for c in range(cfg["n_choices"])}
    out = dict(params=params, losses=npipe.naspipe_get_losses(h, len(choices)),
               trace=npipe.naspipe_get_trace(h), res=npipe.naspipe_get_residency_trace(h),
               stats=npipe.naspipe_get_stats(h))
    npipe.naspipe_destroy(h)
    return out


def _oracle_residency(cfg, choices, D, budget, horizon):
    spec = npipe.Spec(cfg)
    sob = npipe.naspipe_partition(spec, D)
    cf, cb = npipe.naspipe_default_costs(spec)
    tf, tb = csp.task_costs(choices, sob, cf, cb, D)
    plan = csp.simulate_csp(choices, sob, D, 4 * D, tf, tb)
    n, m = cfg["n_choices"], cfg["n_blocks"]
    nbytes = {b * n + c: 4 * train.candidate_size(cfg, b, c) for b in range(m) for c in range(n)}
    events = []
    for K in range(D):
        order = plan["order"][K]
        blocks = [b for b in range(m) if sob[b] == K]
        uses = residency.stage_uses(order, choices, blocks, n)
        r = residency.simulate_residency(uses, [k for k, _ in order], nbytes, budget, L=2,
                                         horizon=None if horizon < 0 else horizon)
        events += [(K, i, 0 if op == "LOAD" else 1, u) for op, i, u in r["events"]]
    return events, nbytes


@pytest.mark.parametrize("name,D,N,horizon", [("tiny_transformer", 1, 10, 0), ("tiny_transformer", 2, 10, -1),
                                              ("tiny_transformer", 2, 12, 3), ("toy", 2, 16, 0)])
def test_context_switch_trace_and_bitwise(name, D, N, horizon):
    cfg = synth.get_config(name)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    # budget: 1.5 x the largest possible task need of a stage (forces evictions)
    n = cfg["n_choices"]
    sob = npipe.naspipe_partition(npipe.Spec(cfg), D)
    need = max(sum(max(4 * train.candidate_size(cfg, b, c) for c in range(n))
                   for b in range(cfg["n_blocks"]) if sob[b] == K) for K in range(D))
    budget = int(1.5 * need)
    ref = _run(cfg, choices, batches, D, 0)
    got = _run(cfg, choices, batches, D, budget, horizon)
    H = 64 if horizon == 0 else horizon
    expect, nbytes = _oracle_residency(cfg, choices, D, budget, H)
    assert [tuple(int(v) for v in r) for r in got["res"]] == expect
    assert got["stats"]["res_evicts"] > 0 and got["stats"]["res_loads"] > 0
    assert np.array_equal(got["losses"].view(np.uint32), ref["losses"].view(np.uint32))
    for k in ref["params"]:
        assert np.array_equal(got["params"][k].view(np.uint32), ref["params"][k].view(np.uint32)), k
    assert [tuple(r) for r in got["trace"]] == [tuple(r) for r in ref["trace"]]
    loaded = sum(nbytes[int(u)] for _, _, op, u in got["res"] if op == 0)
    batch_bytes = 2 * 4 * int(np.prod(synth.batch_shape(cfg))) * N
    assert got["stats"]["h2d_bytes"] == loaded + batch_bytes
    assert got["stats"]["writebacks"] <= got["stats"]["res_evicts"]


def test_budget_too_small_is_ebudget():
    cfg = synth.get_config("tiny_transformer")
    spec = npipe.Spec(cfg, hbm_weight_budget_bytes=1024)
    with pytest.raises(npipe.NaspipeError) as e:
        npipe.naspipe_create(spec, 1)
    assert e.value.code == -6


def test_context_switch_matches_oracle_params():
    cfg = synth.get_config("tiny_transformer")
    N = 6
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    theta0 = train.initial_theta(cfg)
    ref, _ = train.train_sequential(cfg, theta0, choices, batches)
    n = cfg["n_choices"]
    need = sum(max(4 * train.candidate_size(cfg, b, c) for c in range(n)) for b in range(cfg["n_blocks"]))
    got = _run(cfg, choices, batches, 1, int(1.2 * need))
    worst = max(np.max(np.abs(got["params"][k] - r)) / np.max(np.abs(r)) for k, r in ref.items())
    assert worst <= 1e-3
