"""Executed layer mirroring (P:L166 per-subnet balanced partitions, P:L298
"Layer Mirroring ... the new parameters are actively pushed to all the other mirrored ones";
DESIGN.md reading A31; include/naspipe.h NASPIPE_FLAG_MIRROR).

Each subnet runs its blocks on the stages of its own balanced partition; a candidate used
on different stages by different subnets lives in a mirror copy per stage, and every WRITE
is pushed to the other copies before a later READ on another stage.  Bars:
* the executed task trace equals the oracle's mirrored CSP plan (oracle/csp.py
  simulate_csp_mirrored) and passes its validity check (Table 4 order, no READ before the
  previous WRITE + push latency);
* the numerics are the sequential result: bitwise equal to the one-stage fixed-partition run
  (itself checked against the oracle in test_gpu_parity.py) and within the A15 / update bars
  of the fp64 oracle;
* at least one candidate was actually mirrored (pushes happened: p2p bytes > 0).
"""
import json
import os

import numpy as np
import pytest

import synth
from oracle import csp, train

import parity_metrics as pm
from test_gpu_parity import FLAGS, run_engine

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _run_mirrored(cfg, choices, batches, D):
    return run_engine(cfg, choices, batches, D=D, flags=FLAGS | npipe.FLAG_MIRROR)


def _check(cfg, choices, batches, D, upd):
    params, losses, trace, stats = _run_mirrored(cfg, choices, batches, D)
    cf, cb = np.asarray(cfg["cost_fwd"]), np.asarray(cfg["cost_bwd"])
    sob = csp.subnet_partitions(np.asarray(choices).tolist(), cf, cb, D)
    lam = int(cfg.get("link_latency", 0))
    plan = csp.simulate_csp_mirrored(np.asarray(choices).tolist(), sob, D, cfg["window"], cf, cb, lam=lam, lam_w=lam)
    assert [tuple(int(v) for v in r) for r in trace] == [tuple(r) for r in plan["trace"]]
    assert csp.check_trace_mirrored(plan["trace"], np.asarray(choices).tolist(), sob, D, cb, lam_w=lam) == []
    mirrored = any(len({int(sob[y][b]) for y in range(len(choices)) if choices[y][b] == c}) > 1
                   for b in range(cfg["n_blocks"]) for c in range(cfg["n_choices"]))
    assert mirrored, "the random costs gave no mirrored candidate"
    assert stats["p2p_bytes"] > 0 and stats["version_checks"] == 2 * len(choices) * cfg["n_blocks"]
    base = dict(cfg)
    p1, l1, _, _ = run_engine(base, choices, batches, D=1)
    assert np.array_equal(losses.view(np.uint32), l1.view(np.uint32))
    for k in p1:
        assert np.array_equal(params[k].view(np.uint32), p1[k].view(np.uint32)), k
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    pm.check(pm.errors(cfg, params, ref, theta0), 1e-3, upd)
    return sob, plan


def test_mirror_worked_example():
    """tests/golden/mirror_worked_example.json (hand-derived): candidate (1, 0) runs on stage 0
    for subnet 0 and on stage 1 for subnet 1; F(1, 1) waits for B(0, 0)'s WRITE."""
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "mirror_worked_example.json")))
    cfg = synth.get_config("toy", n_blocks=3, n_choices=2, cost_fwd=np.array(g["cost_f"], dtype=np.int32),
                           cost_bwd=np.array(g["cost_b"], dtype=np.int32), window=g["W"])
    choices = np.array(g["choices"], dtype=np.int32)
    batches = [synth.make_batch(cfg, y) for y in range(len(choices))]
    sob, plan = _check(cfg, choices, batches, 2, pm.UPD_FP32)
    assert sob.tolist() == g["stage_of_block"]
    assert [list(t) for t in plan["trace"]] == g["lam_w_0"]["trace"]


# seeds whose random cost tables give at least one mirrored candidate (checked in _check);
# toy at D = 4 has one block per stage: every partition is the same, nothing to mirror
@pytest.mark.parametrize("name,D,N,seed,upd", [("toy", 2, 24, 4, "fp32"), ("toy", 3, 20, 2, "fp32"),
                                               ("toy", 3, 20, 3, "fp32"), ("tiny_transformer", 2, 8, 5, "bf16"),
                                               ("tiny_transformer", 3, 6, 5, "bf16")])
def test_mirror_random_costs(name, D, N, seed, upd):
    base = synth.get_config(name)
    m, n = base["n_blocks"], base["n_choices"]
    rng = np.random.default_rng(seed)
    cfg = dict(base, cost_fwd=rng.integers(1, 9, (m, n)).astype(np.int32),
               cost_bwd=rng.integers(2, 18, (m, n)).astype(np.int32), window=4 * D)
    choices = synth.sample_choices(N, m, n)
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    _check(cfg, choices, batches, D, pm.UPD_FP32 if upd == "fp32" else pm.UPD_BF16)


def test_mirror_spos():
    base = synth.get_config("tiny_spos")
    m, n = base["n_blocks"], base["n_choices"]
    rng = np.random.default_rng(9)
    cfg = dict(base, cost_fwd=rng.integers(1, 9, (m, n)).astype(np.int32),
               cost_bwd=rng.integers(2, 18, (m, n)).astype(np.int32), window=8)
    choices = synth.sample_choices(8, m, n)
    batches = [synth.make_batch(cfg, y) for y in range(8)]
    _check(cfg, choices, batches, 2, pm.UPD_SPOS)


def test_mirror_rejects_other_modes():
    cfg = synth.get_config("toy")
    for over in (dict(sync="asp"), dict(bwd_policy=1), dict(hbm_weight_budget_bytes=1 << 20)):
        with pytest.raises(npipe.NaspipeError) as e:
            npipe.naspipe_create(npipe.Spec(dict(cfg, **over), flags=npipe.FLAG_MIRROR), 2)
        assert e.value.code == -1
