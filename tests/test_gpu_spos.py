"""SPOS CNN family (configs[1]) end to end on the GPU against the sequential CPU oracle
(oracle/spos.py, oracle/train.py), through the C ABI.

Bars (BASELINE.json north_star; A15, A28, A29):
* parameters: A15 metric <= 1e-3 after 1 and 8 steps, <= 1e-2 after 100 steps, against the
  plain fp64 oracle;
* the storage noise floor (A28): the same oracle with its stored tensors rounded the way
  the path stores them (storage="bf16x2": forward hi+lo bf16 pairs, backward bf16) is a
  second, equally valid computation; BatchNorm + ReLU make the result chaotic under
  rounding (one flipped ReLU mask cascades), so the GPU is required to be as close to the
  fp64 definition as that computation is: per-candidate normwise update error <= 2 x the
  emulation's + 0.05, and A15 <= 2 x the emulation's + 1e-4;
* losses rtol 1e-2; schedule trace equal to the oracle's CSP plan;
* bitwise identical across two runs and across D = 1, 2, 4 stages (Table 3).
tiny_spos covers every candidate kind (Shuffle k = 3/5/7, Xception; stride 1 and 2),
ragged BN row blocks (P = 4096, 1024, 256, 64, 16 pixels) and the frozen stem/head.
"""
import numpy as np
import pytest

import synth
from oracle import train

from test_gpu_parity import _check_trace, run_engine

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _errors(got, ref, theta0):
    """(A15, max over candidates of the normwise update error)."""
    a15 = upd = 0.0
    for k, r in ref.items():
        g = got[k].astype(np.float64)
        t0 = theta0[k].astype(np.float64)
        a15 = max(a15, np.max(np.abs(g - r)) / np.max(np.abs(r)))
        if np.any(r != t0):
            upd = max(upd, np.linalg.norm((g - t0) - (r - t0)) / np.linalg.norm(r - t0))
    return a15, upd


def _run(name, choices, D=2, **kw):
    cfg = synth.get_config(name)
    batches = [synth.make_batch(cfg, y) for y in range(len(choices))]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    emu, _ = train.train_sequential(dict(cfg, storage="bf16x2"), theta0, choices, batches)
    params, losses, trace, stats = run_engine(cfg, choices, batches, D=D, **kw)
    gpu = _errors(params, ref, theta0)
    floor = _errors(emu, ref, theta0)
    print(f"{name} N={len(choices)} D={D}: gpu A15={gpu[0]:.2e} upd={gpu[1]:.2e}; "
          f"bf16x2-storage oracle A15={floor[0]:.2e} upd={floor[1]:.2e}")
    return cfg, gpu, floor, losses, ref_loss, trace, stats


@pytest.mark.parametrize("N,tol", [(1, 1e-3), (8, 1e-3), (100, 1e-2)])
def test_tiny_spos_parity(N, tol):
    cfg = synth.get_config("tiny_spos")
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    cfg, gpu, floor, losses, ref_loss, trace, stats = _run("tiny_spos", choices)
    assert gpu[0] <= tol, gpu
    assert gpu[0] <= 2 * floor[0] + 1e-4, (gpu, floor)
    assert gpu[1] <= 2 * floor[1] + 0.05, (gpu, floor)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)
    _check_trace(cfg, choices, 2, trace)
    assert stats["version_checks"] == 2 * N * cfg["n_blocks"]


def test_tiny_spos_every_candidate_kind():
    """Subnets chosen so that every (block, choice) is trained at least once."""
    cfg = synth.get_config("tiny_spos")
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = np.array([[(c + b) % n for b in range(m)] for c in range(n)], dtype=np.int32)
    _, gpu, floor, losses, ref_loss, _, _ = _run("tiny_spos", choices, D=1)
    assert gpu[0] <= 1e-3 and gpu[0] <= 2 * floor[0] + 1e-4, (gpu, floor)
    assert gpu[1] <= 2 * floor[1] + 0.05, (gpu, floor)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)


def test_tiny_spos_bitwise_across_runs_and_stage_counts():
    cfg = synth.get_config("tiny_spos")
    choices = synth.sample_choices(12, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(12)]
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    for D, where in ((1, npipe.BATCH_HOST), (2, npipe.BATCH_DEVICE), (4, npipe.BATCH_HOST)):
        p, l, tr, _ = run_engine(cfg, choices, batches, D=D, where=where)
        assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32)), D
        for k in base:
            assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), (D, k)
        _check_trace(cfg, choices, D, tr)


def test_spos_full_size_one_step():
    """configs[1] at full size (B = 64, 224 x 224, 20 blocks) in the bench's launch
    configuration (one stage), one subnet, against the plain fp64 oracle (A15 <= 1e-3,
    loss rtol 1e-2)."""
    cfg = synth.get_config("spos")
    choices = synth.sample_choices(1, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, 0)]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    params, losses, _, _ = run_engine(cfg, choices, batches, D=1)
    a15, upd = _errors(params, ref, theta0)
    print(f"full-size A15={a15:.3e} upd={upd:.3e} loss {losses[0]:.6f} vs {ref_loss[0]:.6f}")
    assert a15 <= 1e-3, a15
    assert upd <= 0.3, upd   # bf16x2-storage oracle at this size: A15 1.5e-4, update 0.10
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)


def test_spos_full_size_bitwise_across_runs_and_stage_counts():
    """configs[1] at full size: 3 subnets, twice at D = 1 and once at D = 2 and 4 (stages on
    this GPU): parameters and losses bitwise equal (Def.1, Table 3).  At
    this size the weight gradients take the split-K path with ragged k-block counts."""
    cfg = synth.get_config("spos")
    choices = synth.sample_choices(3, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(3)]
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    for D in (1, 2, 4):
        p, l, _, _ = run_engine(cfg, choices, batches, D=D, where=npipe.BATCH_DEVICE)
        assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32)), D
        for k in base:
            assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), (D, k)



def test_spos_full_size_20_steps_against_oracle_samples():
    """configs[1] at full size, 20 subnets trained sequentially by the fp64 oracle
    (tests/golden/spos_fullsize_20steps.npz, written by tools/make_spos_multistep_golden.py
    from oracle/ only) against the GPU in the bench's launch configuration: A15 over 512
    sampled entries of every trained candidate (denominator max |theta| over the whole
    candidate) <= 1e-2 (BJ's multi-step bar), losses rtol 1e-2."""
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "spos_fullsize_20steps.npz")
    if not os.path.exists(path):
        pytest.skip("golden not generated")
    g = np.load(path)
    cfg = synth.get_config("spos")
    choices = g["choices"]
    N = len(choices)
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    params, losses, _, _ = run_engine(cfg, choices, batches, D=1, where=npipe.BATCH_DEVICE)
    worst = 0.0
    for key in g.files:
        if not key.startswith("idx_"):
            continue
        _, b, c = key.split("_")
        got = params[(int(b), int(c))].astype(np.float64)[g[key]]
        ref = g[f"new_{b}_{c}"]
        worst = max(worst, float(np.max(np.abs(got - ref)) / g[f"maxabs_{b}_{c}"]))
    print(f"20-step full-size sampled A15 = {worst:.3e}; losses {losses[-3:]} vs {g['losses'][-3:]}")
    assert worst <= 1e-2, worst
    np.testing.assert_allclose(losses, g["losses"], rtol=1e-2)
