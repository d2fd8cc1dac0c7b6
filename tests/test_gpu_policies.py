"""Synchronisation policies on the GPU (include/naspipe.h naspipe_sync).

* ASP (dependencies ignored, PipeDream-style): the executed schedule equals the
  oracle's ASP plan, and the parameters equal the oracle replaying that plan stage by stage
  (oracle/train.py train_replay: stale reads, no weight stashing) — same bars as the CSP
  parity tests.  Its result depends on the stage count while CSP's does not: the
  reproducibility contrast of Table 3, here on B200.
* INORDER ("NASPipe w/o scheduler", Fig.6): a different, still causal schedule with
  bitwise the CSP numerics.
* BSP (GPipe / Retiarii bulks; reading A30): the executed schedule is the
  planner's BSP plan; the parameters equal oracle/train.py train_bsp (each bulk's gradients
  at the bulk-start weights, summed, applied at the flush) within the CSP parity bars;
  bulk = 1 is bitwise the CSP result; a fixed bulk size gives bitwise the same result at
  D = 1, 2, 4 (the bulk, not the stage count, defines the arithmetic).
"""
import numpy as np
import pytest

import synth
from oracle import csp, train

from test_gpu_parity import FLAGS, param_errors, run_engine

import parity_metrics as pm

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _workload(name, N, sync):
    cfg = synth.get_config(name, sync=sync)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    return cfg, choices, batches


def _oracle_plan(cfg, choices, D, sync):
    spec = npipe.Spec(cfg)
    sob = npipe.naspipe_partition(spec, D)
    cf, cb = npipe.naspipe_default_costs(spec)
    tf, tb = csp.task_costs(choices, sob, cf, cb, D)
    return sob, csp.simulate_csp(choices, sob, D, 4 * D, tf, tb, sync=sync)["trace"]


@pytest.mark.parametrize("name,N,D,tol_upd,rtol", [("toy", 24, 2, 1e-5, 1e-5), ("toy", 24, 4, 1e-5, 1e-5),
                                                   ("tiny_transformer", 8, 2, 1e-1, 1e-2)])
def test_asp_matches_oracle_replay(name, N, D, tol_upd, rtol):
    cfg, choices, batches = _workload(name, N, "asp")
    sob, tr = _oracle_plan(cfg, choices, D, "asp")
    params, losses, trace, _ = run_engine(cfg, choices, batches, D)
    assert [tuple(int(v) for v in r) for r in trace] == [tuple(r) for r in tr]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_replay(cfg, theta0, choices, batches, sob, tr)
    pm.check(param_errors(cfg, params, ref, theta0), 1e-3, pm.UPD_FP32 if name == "toy" else pm.UPD_BF16)
    np.testing.assert_allclose(losses, ref_loss, rtol=rtol)


def test_table3_reproducibility_contrast():
    """CSP: bitwise identical parameters at D = 1, 2, 4.  ASP: the stage count changes them."""
    N = 24
    res = {}
    for sync in ("csp", "asp"):
        cfg, choices, batches = _workload("toy", N, sync)
        res[sync] = [run_engine(cfg, choices, batches, D)[0] for D in (1, 2, 4)]
    for p in res["csp"][1:]:
        assert all(np.array_equal(p[k].view(np.uint32), res["csp"][0][k].view(np.uint32)) for k in p)
    a2, a4 = res["asp"][1], res["asp"][2]
    assert any(not np.array_equal(a2[k], a4[k]) for k in a2)


def test_serial_has_csp_numerics():
    """SERIAL (w/o scheduler per P:L454, one subnet in flight): the executed trace is the
    oracle's serial plan and the numerics are bitwise the CSP run's."""
    cfg, choices, batches = _workload("toy", 16, "serial")
    sob, tr = _oracle_plan(cfg, choices, 4, "serial")
    p_s, l_s, trace, _ = run_engine(cfg, choices, batches, 4)
    assert [tuple(int(v) for v in r) for r in trace] == [tuple(r) for r in tr]
    ccfg = synth.get_config("toy")
    p_c, l_c, _, _ = run_engine(ccfg, choices, batches, 4)
    assert np.array_equal(l_s.view(np.uint32), l_c.view(np.uint32))
    for k in p_c:
        assert np.array_equal(p_s[k].view(np.uint32), p_c[k].view(np.uint32)), k


def test_inorder_has_csp_numerics():
    cfg, choices, batches = _workload("toy", 24, "inorder")
    sob, tr = _oracle_plan(cfg, choices, 4, "inorder")
    p_in, l_in, trace, _ = run_engine(cfg, choices, batches, 4)
    assert [tuple(int(v) for v in r) for r in trace] == [tuple(r) for r in tr]
    cfg_c = synth.get_config("toy")
    p_csp, l_csp, _, _ = run_engine(cfg_c, choices, batches, 4)
    assert all(np.array_equal(p_in[k].view(np.uint32), p_csp[k].view(np.uint32)) for k in p_in)
    assert np.array_equal(l_in.view(np.uint32), l_csp.view(np.uint32))


def _run_bsp(name, N, D, bulk, where=None, window=None):
    cfg = synth.get_config(name, sync="bsp", bulk_size=bulk, window=window or 4 * D)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    kw = {} if where is None else dict(where=where)
    return cfg, choices, batches, run_engine(cfg, choices, batches, D, **kw)


@pytest.mark.parametrize("name,N,D,bulk,tol_upd,rtol", [("toy", 24, 2, 4, 1e-5, 1e-5), ("toy", 24, 4, 6, 1e-5, 1e-5),
                                                        ("tiny_transformer", 8, 2, 4, 1e-1, 1e-2)])
def test_bsp_matches_oracle(name, N, D, bulk, tol_upd, rtol):
    cfg, choices, batches, (params, losses, trace, _) = _run_bsp(name, N, D, bulk)
    sob = npipe.naspipe_partition(npipe.Spec(cfg), D)
    cf, cb = npipe.naspipe_default_costs(npipe.Spec(cfg))
    tf, tb = csp.task_costs(choices, sob, cf, cb, D)
    plan = csp.simulate_csp(choices, sob, D, 4 * D, tf, tb, sync="bsp", bulk=bulk)["trace"]
    assert [tuple(int(v) for v in r) for r in trace] == [tuple(r) for r in plan]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_bsp(cfg, theta0, choices, batches, bulk)
    pm.check(param_errors(cfg, params, ref, theta0), 1e-3, pm.UPD_FP32 if name == "toy" else pm.UPD_BF16)
    np.testing.assert_allclose(losses, ref_loss, rtol=rtol)


@pytest.mark.parametrize("name,N,D,bulk,window", [("toy", 24, 1, 8, 4), ("toy", 20, 2, 10, 3),
                                                  ("tiny_transformer", 8, 1, 8, 2)])
def test_bsp_bulk_larger_than_window(name, N, D, bulk, window):
    """A bulk larger than the window W: the planner releases the whole bulk (all its
    forwards before its backwards), so the executor's slot ring must hold G subnets, not W;
    with W slots F(y + W) overwrote y's stashed activations before B(y) read them."""
    cfg, choices, batches, (params, losses, trace, _) = _run_bsp(name, N, D, bulk, window=window)
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_bsp(cfg, theta0, choices, batches, bulk)
    pm.check(param_errors(cfg, params, ref, theta0), 1e-3, pm.UPD_FP32 if name == "toy" else pm.UPD_BF16)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-5 if name == "toy" else 1e-2)


@pytest.mark.parametrize("name,N", [("toy", 12), ("tiny_transformer", 6), ("tiny_spos", 6)])
def test_bsp_bulk1_is_bitwise_csp(name, N):
    """bulk = 1: the accumulator path (WRITE into the copy, flush before the next subnet)
    computes exactly the in-place update: bitwise the CSP parameters and losses."""
    cfg, choices, batches, (p_bsp, l_bsp, _, _) = _run_bsp(name, N, 2, 1)
    ccfg = synth.get_config(name)
    p_csp, l_csp, _, _ = run_engine(ccfg, choices, batches, 2)
    assert np.array_equal(l_bsp.view(np.uint32), l_csp.view(np.uint32))
    for k in p_csp:
        assert np.array_equal(p_bsp[k].view(np.uint32), p_csp[k].view(np.uint32)), k


@pytest.mark.parametrize("name,N", [("toy", 24), ("tiny_spos", 8)])
def test_bsp_fixed_bulk_is_bitwise_across_stage_counts(name, N):
    base = None
    for D in (1, 2, 4):
        _, _, _, (p, l, _, _) = _run_bsp(name, N, D, 4)
        if base is None:
            base = (p, l)
            continue
        assert np.array_equal(l.view(np.uint32), base[1].view(np.uint32)), D
        for k in p:
            assert np.array_equal(p[k].view(np.uint32), base[0][k].view(np.uint32)), (D, k)
