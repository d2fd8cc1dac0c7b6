"""End-to-end parity of the CUDA path against the sequential CPU oracle (SURVEY §4 tier T3),
through the C ABI (naspipe_create / submit / drain / get_params).

Bars (BASELINE.json north_star, reading A15):
* parameters: per tensor max|gpu - ref| / max|ref| <= 1e-3 after 1 step, <= 1e-2 after 100
  steps (tests/parity_metrics.py); the update Delta = theta_t - theta_0 (the params alone are
  dominated by theta_0), normwise per tensor: <= 1e-5 (fp32 MLP); bf16: matrices and biases
  <= 2e-2, LN gamma/beta <= 5e-2 (derivation in DESIGN.md "Tolerances");
* schedule decisions bit-exact: the executed task trace equals the oracle CSP schedule;
* two GPU runs bitwise identical; runs at different stage counts D bitwise identical
  (Table 3, artifact P:L557-561) — all stages of a run share one GPU here.
"""
import numpy as np
import pytest

import synth
from oracle import csp, train

import parity_metrics as pm

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")

FLAGS = npipe.FLAG_TRACE | npipe.FLAG_VERSION_CHECK


def run_engine(cfg, choices, batches, D, where=npipe.BATCH_HOST, flags=FLAGS, theta0=None):
    spec = npipe.Spec(cfg, flags=flags)
    h = npipe.naspipe_create(spec, D)
    if theta0 is not None:
        for (b, c), v in theta0.items():
            npipe.naspipe_set_params(h, b, c, v)
    keep = []
    for y, ch in enumerate(choices):
        x, t = batches[y]
        if where == npipe.BATCH_DEVICE:
            xd = torch.from_numpy(x).cuda()
            td = torch.from_numpy(t).cuda()
            keep += [xd, td]
            npipe.naspipe_submit(h, ch, xd, td, where=where)
        else:
            npipe.naspipe_submit(h, ch, x, t, where=where)
    npipe.naspipe_drain(h)
    params = {(b, c): npipe.naspipe_get_params(h, b, c)
              for b in range(cfg["n_blocks"]) for c in range(cfg["n_choices"])}
    losses = npipe.naspipe_get_losses(h, len(choices))
    trace = npipe.naspipe_get_trace(h)
    stats = npipe.naspipe_get_stats(h)
    npipe.naspipe_destroy(h)
    return params, losses, trace, stats


def param_errors(cfg, got, ref, theta0):
    """Per-tensor A15 and update metrics (tests/parity_metrics.py, A15); printed."""
    sm = pm.errors(cfg, got, ref, theta0)
    print(cfg.get("family"), pm.fmt(sm))
    return sm


def _workload(name, N, **over):
    cfg = synth.get_config(name, **over)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    return cfg, choices, batches


def _oracle(cfg, choices, batches):
    theta0 = train.initial_theta(cfg)
    ref, losses = train.train_sequential(cfg, theta0, choices, batches)
    return theta0, ref, losses


def _check_trace(cfg, choices, D, trace):
    spec = npipe.Spec(cfg)
    sob = npipe.naspipe_partition(spec, D)
    cf, cb = npipe.naspipe_default_costs(spec)
    tf, tb = csp.task_costs(choices, sob, cf, cb, D)
    ref = csp.simulate_csp(choices, sob, D, 4 * D, tf, tb)
    assert [tuple(int(v) for v in r) for r in trace] == [tuple(r) for r in ref["trace"]]
    assert csp.check_trace(ref["trace"], choices, sob, D) == []


@pytest.mark.parametrize("N,tol", [(1, 1e-3), (16, 1e-3), (100, 1e-2)])
def test_toy_mlp_parity(N, tol):
    cfg, choices, batches = _workload("toy", N)
    theta0, ref, ref_loss = _oracle(cfg, choices, batches)
    params, losses, trace, stats = run_engine(cfg, choices, batches, D=2)
    pm.check(param_errors(cfg, params, ref, theta0), tol, pm.UPD_FP32)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-5)
    _check_trace(cfg, choices, 2, trace)
    assert stats["version_checks"] == 2 * N * cfg["n_blocks"]


def test_toy_bitwise_across_runs_and_stage_counts():
    cfg, choices, batches = _workload("toy", 24)
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    for D in (1, 2, 4):
        p, l, tr, _ = run_engine(cfg, choices, batches, D=D)
        assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32)), D
        for k in base:
            assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), (D, k)
        _check_trace(cfg, choices, D, tr)


@pytest.mark.parametrize("N,tol", [(1, 1e-3), (8, 1e-3), (100, 1e-2)])
def test_tiny_transformer_parity(N, tol):
    cfg, choices, batches = _workload("tiny_transformer", N)
    theta0, ref, ref_loss = _oracle(cfg, choices, batches)
    params, losses, trace, _ = run_engine(cfg, choices, batches, D=2)
    sm = param_errors(cfg, params, ref, theta0)
    pm.check(sm, tol, pm.UPD_BF16 if N <= 8 else None)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)
    _check_trace(cfg, choices, 2, trace)


def test_tiny_transformer_bitwise_across_runs_and_stage_counts():
    cfg, choices, batches = _workload("tiny_transformer", 10)
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    for D, where in ((1, npipe.BATCH_HOST), (2, npipe.BATCH_DEVICE), (4, npipe.BATCH_HOST)):
        p, l, _, _ = run_engine(cfg, choices, batches, D=D, where=where)
        assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32)), D
        for k in base:
            assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), (D, k)


@pytest.mark.parametrize("N,tol", [(1, 1e-3), (8, 1e-3), (100, 1e-2)])
def test_tiny_nlp_ops_parity(N, tol):
    """Table 5's NLP ops (Conv 3x1, Sep Conv 7x1, Light Conv 5x1, attention; reading A38) as
    candidates of one supernet: subnets cycle the choices so every (block, op) is trained."""
    cfg = synth.get_config("tiny_nlp")
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = np.array([[(y + b) % n for b in range(m)] for y in range(N)], dtype=np.int32)
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    theta0, ref, ref_loss = _oracle(cfg, choices, batches)
    params, losses, trace, _ = run_engine(cfg, choices, batches, D=2)
    sm = param_errors(cfg, params, ref, theta0)
    pm.check(sm, tol, pm.UPD_BF16 if N <= 8 else None)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)
    _check_trace(cfg, choices, 2, trace)


def test_tiny_nlp_ops_bitwise_across_stage_counts():
    cfg, choices, batches = _workload("tiny_nlp", 10)
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    for D, where in ((1, npipe.BATCH_HOST), (2, npipe.BATCH_DEVICE), (4, npipe.BATCH_HOST)):
        p, l, _, _ = run_engine(cfg, choices, batches, D=D, where=where)
        assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32)), D
        for k in base:
            assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), (D, k)


def test_null_kernels_and_errors():
    cfg, choices, batches = _workload("toy", 6)
    spec = npipe.Spec(cfg, flags=FLAGS | npipe.FLAG_NULL_KERNELS)
    h = npipe.naspipe_create(spec, 2)
    with pytest.raises(npipe.NaspipeError) as e:
        npipe.naspipe_submit(h, np.array([0, 0, 0, 9]), batches[0][0], batches[0][1])
    assert e.value.code == -1
    for y in range(6):
        assert npipe.naspipe_submit(h, choices[y], *batches[y]) == y    # rejected submit kept ids
    npipe.naspipe_drain(h)
    # parameters untouched with null kernels
    for (b, c), v in train.initial_theta(cfg).items():
        assert np.array_equal(npipe.naspipe_get_params(h, b, c), v)
    # a second stream after a drain continues the ids
    assert npipe.naspipe_submit(h, choices[0], *batches[0]) == 6
    with pytest.raises(npipe.NaspipeError) as e:
        npipe.naspipe_get_params(h, 0, 0)
    assert e.value.code == -2
    npipe.naspipe_drain(h)
    npipe.naspipe_destroy(h)


def run_fullsize(name, gold, steps):
    """The first `steps` subnets of a BASELINE.json config at full size, in the bench's launch
    configuration (one stage, DEVICE batches).  Returns (params getter, losses)."""
    cfg = synth.get_config(name)
    ch = gold["choices"][:steps]
    assert np.array_equal(ch, synth.sample_choices(steps, cfg["n_blocks"], cfg["n_choices"]))
    h = npipe.naspipe_create(npipe.Spec(cfg, flags=npipe.FLAG_VERSION_CHECK), 1)
    keep = []
    for y in range(steps):
        x, t = synth.make_batch(cfg, y)
        xd, td = torch.from_numpy(x).cuda(), torch.from_numpy(t).cuda()
        keep += [xd, td]
        npipe.naspipe_submit(h, ch[y], xd, td, where=npipe.BATCH_DEVICE)
    npipe.naspipe_drain(h)
    losses = npipe.naspipe_get_losses(h, steps)
    params = {}

    def got_of(b, c):
        if (b, c) not in params:
            params[(b, c)] = npipe.naspipe_get_params(h, b, c)
        return params[(b, c)]
    return cfg, h, got_of, losses


def load_gold(name):
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", name)
    if not os.path.exists(path):
        pytest.skip(f"{name} not generated (tools/make_multistep_golden.py)")
    return np.load(path)


@pytest.mark.parametrize("steps,tol", [(1, 1e-3), (100, 1e-2)])
def test_transformer_full_size_against_oracle_samples(steps, tol):
    """configs[2] at BASELINE.json's full size (24 blocks x 4 choices, d = 1024, S = 128, B = 32,
    bf16) in the bench's launch configuration, the first `steps` subnets, against sampled
    outputs of the fp64 oracle's sequential training (tests/golden/transformer_fullsize_100steps.npz,
    written by tools/make_multistep_golden.py, which calls only oracle/).  Bars (north_star):
    per-tensor A15 <= 1e-3 after 1 step and <= 1e-2 after 100; after 1 step the update bars of
    tests/parity_metrics.py over the sampled entries; losses rtol 1e-2."""
    gold = load_gold("transformer_fullsize_100steps.npz")
    if f"s{steps}_max_0_{int(gold['choices'][0][0])}_Wqkv" not in gold.files:
        pytest.skip(f"checkpoint {steps} not in the golden yet")
    cfg, h, got_of, losses = run_fullsize("transformer", gold, steps)
    sm = pm.sampled_errors(cfg, gold, steps, got_of)
    npipe.naspipe_destroy(h)
    print(f"configs[2] full size, {steps} steps: {pm.fmt(sm)}; losses {losses[-2:]} vs {gold['losses'][steps - 2:steps]}")
    pm.check(sm, tol, pm.UPD_BF16 if steps == 1 else None)
    np.testing.assert_allclose(losses, gold["losses"][:steps], rtol=1e-2)


def test_nlp_c3_full_size_one_step_against_oracle_samples():
    """The NLP.c3 analog (Table 1: 48 blocks x 24 choices over Table 5's NLP ops,
    reading A38; d = 1024, S = 128, B = 32) at full size in the bench's launch configuration:
    one subnet against sampled outputs of the fp64 oracle (tests/golden/nlp_c3_fullsize_1steps.npz,
    tools/make_multistep_golden.py, oracle/ only): per-tensor A15 <= 1e-3, the update bars,
    loss rtol 1e-2."""
    gold = load_gold("nlp_c3_fullsize_1steps.npz")
    cfg, h, got_of, losses = run_fullsize("nlp_c3", gold, 1)
    sm = pm.sampled_errors(cfg, gold, 1, got_of)
    npipe.naspipe_destroy(h)
    ops = np.asarray(cfg["choice_op"])[gold["choices"][0]]
    print(f"nlp_c3 full size, 1 step (ops used {np.bincount(ops, minlength=4).tolist()}): {pm.fmt(sm)}; "
          f"loss {losses} vs {gold['losses'][:1]}")
    pm.check(sm, 1e-3, pm.UPD_BF16)
    np.testing.assert_allclose(losses, gold["losses"][:1], rtol=1e-2)
