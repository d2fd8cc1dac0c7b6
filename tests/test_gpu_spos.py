"""SPOS CNN family (configs[1]) end to end on the GPU against the sequential CPU oracle
(oracle/spos.py, oracle/train.py), through the C ABI.

Bars (BASELINE.json north_star; A15, A28, A29), all against the plain fp64 oracle:
* parameters: per-tensor A15 <= 1e-3 after 1 and 8 steps, <= 1e-2 after 100 steps;
* update (<= 8 steps): per-tensor normwise error, matrices <= 2e-2, BN gamma/beta <= 5e-2;
  the depthwise units' BN beta (exact gradient identically 0) within an absolute bar
  (tests/parity_metrics.py);
* diagnostic only (printed): the oracle with its stored tensors rounded the way the path
  stores them (storage="bf16x2", reading A28) — the distance of that computation from fp64
  shows the storage noise floor, it sets no bar;
* losses rtol 1e-2; schedule trace equal to the oracle's CSP plan;
* bitwise identical across two runs and across D = 1, 2, 4 stages (Table 3).
tiny_spos covers every candidate kind (Shuffle k = 3/5/7, Xception; stride 1 and 2),
ragged BN row blocks (P = 4096, 1024, 256, 64, 16 pixels) and the frozen stem/head.
"""
import json
import os

import numpy as np
import pytest

import synth
from oracle import train

from test_gpu_parity import _check_trace, load_gold, run_engine, run_fullsize

import parity_metrics as pm

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _run(name, choices, D=2, **kw):
    cfg = synth.get_config(name)
    batches = [synth.make_batch(cfg, y) for y in range(len(choices))]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    emu, _ = train.train_sequential(dict(cfg, storage="bf16x2"), theta0, choices, batches)
    params, losses, trace, stats = run_engine(cfg, choices, batches, D=D, **kw)
    gpu = pm.errors(cfg, params, ref, theta0)
    floor = pm.errors(cfg, emu, ref, theta0)
    print(f"{name} N={len(choices)} D={D}: gpu {pm.fmt(gpu)}\n  bf16x2-storage oracle (diagnostic) {pm.fmt(floor)}")
    return cfg, gpu, floor, losses, ref_loss, trace, stats


@pytest.mark.parametrize("N,tol", [(1, 1e-3), (8, 1e-3), (100, 1e-2)])
def test_tiny_spos_parity(N, tol):
    cfg = synth.get_config("tiny_spos")
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    cfg, gpu, floor, losses, ref_loss, trace, stats = _run("tiny_spos", choices)
    pm.check(gpu, tol, pm.UPD_SPOS if N <= 8 else None)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)
    _check_trace(cfg, choices, 2, trace)
    assert stats["version_checks"] == 2 * N * cfg["n_blocks"]


def test_tiny_spos_every_candidate_kind():
    """Subnets chosen so that every (block, choice) is trained at least once."""
    cfg = synth.get_config("tiny_spos")
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = np.array([[(c + b) % n for b in range(m)] for c in range(n)], dtype=np.int32)
    _, gpu, floor, losses, ref_loss, _, _ = _run("tiny_spos", choices, D=1)
    pm.check(gpu, 1e-3, pm.UPD_SPOS)
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


@pytest.mark.parametrize("N", [1, 8, 100])
def test_tiny_spos_dense_parity(N):
    """Table 5's dense Conv 3x3 candidate (reading A40: the Shuffle block with a dense
    3x3 mid conv; explicit x2 columns, 3-pass tcgen05 GEMM forward, fp32 column gradient +
    fixed-order adjoint, split-K weight gradient with the SGD WRITE) beside Shuffle 5 and
    Xception 3; every (block, choice) trained when N >= 4 (cyclic assignment)."""
    cfg = synth.get_config("tiny_spos_dense")
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = np.array([[(c + b) % n for b in range(m)] for c in range(N)], dtype=np.int32)
    cfg, gpu, floor, losses, ref_loss, trace, stats = _run("tiny_spos_dense", choices)
    pm.check(gpu, 1e-3 if N <= 8 else 1e-2, pm.UPD_SPOS if N <= 8 else None)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)
    _check_trace(cfg, choices, 2, trace)
    assert stats["version_checks"] == 2 * N * m


def test_tiny_spos_dense_bitwise_across_stage_counts():
    cfg = synth.get_config("tiny_spos_dense")
    choices = synth.sample_choices(10, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(10)]
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    for D in (1, 2, 4):
        p, l, tr, _ = run_engine(cfg, choices, batches, D=D)
        assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32)), D
        for k in base:
            assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), (D, k)


@pytest.mark.parametrize("N", [1, 8])
def test_tiny_spos_dilated_parity(N):
    """Dilated depthwise candidates (Table 5's Dil Conv; reading A36): Shuffle k 3/7
    and Xception k 5 at dilation 2, Xception k 3 at dilation 1; every (block, choice) trained
    when N = 8 (two rounds of the cyclic assignment)."""
    cfg = synth.get_config("tiny_spos_dil")
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = np.array([[(c + b) % n for b in range(m)] for c in range(N)], dtype=np.int32)
    cfg, gpu, floor, losses, ref_loss, trace, stats = _run("tiny_spos_dil", choices)
    pm.check(gpu, 1e-3, pm.UPD_SPOS)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)
    _check_trace(cfg, choices, 2, trace)


def test_cv_c3_full_size_one_step_against_oracle_samples():
    """The CV.c3 analog (Table 1: 32 choice blocks x 12 choices over Table 5's op types,
    dilation included; reading A36) at full size, one subnet, against the fp64 oracle
    (tests/golden/cv_c3_fullsize_1steps.npz, tools/make_multistep_golden.py, oracle/ only).

    This supernet is ill-conditioned at initialisation (deep BatchNorm chains over nearly
    constant channels at 7 x 7): the SAME oracle with its stored tensors rounded to fp32 (the
    paper's precision) or the way this path stores them (bf16x2, A28) already moves the
    parameters far from fp64 after one step (A37).  Bars: losses rtol 1e-2;
    per-tensor A15 <= max(1e-3, 1.5 x the bf16x2-storage oracle's A15 at the same samples).
    The dilated kernels themselves are pinned at these shapes in test_gpu_spos_kernels.py and
    end to end at 1e-3 on tiny_spos_dil above."""
    gold = load_gold("cv_c3_fullsize_1steps.npz")
    cfg = synth.get_config("cv_c3")
    fl16 = pm.golden_floor(cfg, gold, load_gold("cv_c3_fullsize_1steps_bf16x2.npz"), 1)
    fl32 = pm.golden_floor(cfg, gold, load_gold("cv_c3_fullsize_1steps_fp32.npz"), 1)
    cfg, h, got_of, losses = run_fullsize("cv_c3", gold, 1)
    sm = pm.sampled_errors(cfg, gold, 1, got_of)
    npipe.naspipe_destroy(h)
    print(f"cv_c3 full size, 1 step: {pm.fmt(sm)}; oracle floors bf16x2 {fl16} fp32 {fl32}; "
          f"loss {losses} vs {gold['losses'][:1]}")
    np.testing.assert_allclose(losses, gold["losses"][:1], rtol=1e-2)
    assert sm["a15"] <= max(1e-3, 1.5 * fl16["a15"]), (sm["a15"], fl16)


def test_cv_c3_full_size_bitwise_across_stage_counts():
    """CV.c3 analog at full size: 3 subnets at D = 1 and D = 4, parameters and losses bitwise
    equal (Def.1, Table 3)."""
    cfg = synth.get_config("cv_c3")
    choices = synth.sample_choices(3, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(3)]
    base, base_loss, _, _ = run_engine(cfg, choices, batches, D=1)
    p, l, _, _ = run_engine(cfg, choices, batches, D=4, where=npipe.BATCH_DEVICE)
    assert np.array_equal(l.view(np.uint32), base_loss.view(np.uint32))
    for k in base:
        assert np.array_equal(p[k].view(np.uint32), base[k].view(np.uint32)), k


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
    sm = pm.errors(cfg, params, ref, theta0)
    print(f"full-size one step: {pm.fmt(sm)} loss {losses[0]:.6f} vs {ref_loss[0]:.6f}")
    pm.check(sm, 1e-3, pm.UPD_SPOS)
    np.testing.assert_allclose(losses, ref_loss, rtol=1e-2)


def test_spos_dense_full_size_one_step():
    """configs[1] geometry with the dense Conv 3x3 candidate (A40) at full size, a subnet that
    uses it in every block (choice 0), one step against the fp64 oracle.  Bars: update bars,
    loss rtol 1e-2, per-tensor A15 <= max(1e-3, 1.5 x the storage floor): block 0's dense
    weight gradient sums 200704 products of the bf16-stored dz (zero-mean after the BatchNorm
    backward) with ReLU outputs (positive mean), a cancelling sum, so the path's bf16 backward
    storage (A28) alone moves that tensor by 1.1e-3 (the oracle with the path's storage,
    tests/golden/spos_dense_fullsize_1step_floor.json from tools/make_dense_floor.py; the
    fp32-storage oracle: 9.5e-5) -- the reading A37 bar of the CV.c3 analog."""
    cfg = synth.get_config("spos_dense")
    choices = np.zeros((1, cfg["n_blocks"]), dtype=np.int32)
    batches = [synth.make_batch(cfg, 0)]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    params, losses, _, _ = run_engine(cfg, choices, batches, D=1)
    sm = pm.errors(cfg, params, ref, theta0)
    floor = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "spos_dense_fullsize_1step_floor.json")))
    bar = max(1e-3, 1.5 * floor["bf16x2"]["a15_tensor"])
    upd = dict(pm.UPD_SPOS, static=max(pm.UPD_SPOS["static"], 1.5 * floor["bf16x2"]["static"]))
    print(f"dense full-size one step: {pm.fmt(sm)} loss {losses[0]:.6f} vs {ref_loss[0]:.6f}; "
          f"storage floor {floor['bf16x2']['a15_tensor']:.2e} (fp32 {floor['fp32']['a15_tensor']:.2e}), bar {bar:.2e}")
    pm.check(sm, bar, upd)
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



@pytest.mark.parametrize("steps", [20, 100])
def test_spos_full_size_multistep_against_oracle_samples(steps):
    """configs[1] at full size, the first 20 / 100 subnets trained sequentially by the fp64
    oracle (tests/golden/spos_fullsize_100steps.npz, written by tools/make_multistep_golden.py
    from oracle/ only) against the GPU in the bench's launch configuration.

    BatchNorm + ReLU on random labels make this trajectory chaotic: the SAME oracle with
    every stored tensor rounded to fp32 (the paper's precision, P:L98;
    tests/golden/spos_fullsize_100steps_fp32.npz) already differs from fp64 by a per-tensor
    A15 of 2.8e-2 after 20 steps (A35).  Bars: per candidate (round-1 reading of
    A15) <= 1e-2, BJ's multi-step bar; per tensor <= max(1e-2, 1.5 x that fp32 floor at the
    same step); losses rtol 1e-2."""
    gold = load_gold("spos_fullsize_100steps.npz")
    if not any(k.startswith(f"s{steps}_max_") for k in gold.files):
        pytest.skip(f"checkpoint {steps} not in the golden yet")
    floor_gold = load_gold("spos_fullsize_100steps_fp32.npz")
    if not any(k.startswith(f"s{steps}_max_") for k in floor_gold.files):
        pytest.skip(f"checkpoint {steps} not in the fp32 floor golden yet")
    cfg = synth.get_config("spos")
    floor = pm.golden_floor(cfg, gold, floor_gold, steps)
    cfg, h, got_of, losses = run_fullsize("spos", gold, steps)
    sm = pm.sampled_errors(cfg, gold, steps, got_of)
    npipe.naspipe_destroy(h)
    print(f"configs[1] full size, {steps} steps: {pm.fmt(sm)}; fp32-oracle floor {floor}; "
          f"losses {losses[-3:]} vs {gold['losses'][steps - 3:steps]}")
    assert sm["a15_cand"] <= 1e-2, sm["a15_cand"]
    assert sm["a15"] <= max(1e-2, 1.5 * floor["a15"]), (sm["a15"], floor)
    np.testing.assert_allclose(losses, gold["losses"][:steps], rtol=1e-2)
