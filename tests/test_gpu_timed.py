"""Timing-driven execution (Alg.1 + Alg.2 P:L170-221 on observed completions,
Alg.3's predictor P:L239-273 evaluated online; reading A39; include/naspipe.h
NASPIPE_FLAG_TIMED).

The host decides each stage's next task when it sees the stage free, from the queues and
finished sets it observes, so the schedule depends on kernel timing.  Bars:
* the executed trace is a valid CSP schedule (oracle csp.check_trace: every task once, the
  stage order of a subnet, the Table 4 access pattern F(x1) B(x1) F(x2) B(x2) ... per candidate);
* at D = 1 it is F0 B0 F1 B1 ... (the only CSP order with backward-first);
* the numerics are the sequential result: parameters and losses BITWISE equal to the planned
  executor's one-stage run, and the version invariant holds at every task;
* Alg.3's counters are consistent (hits <= predictions <= backward starts = N D).
"""
import numpy as np
import pytest

import synth
from oracle import csp

from test_gpu_parity import FLAGS, run_engine

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _run_timed(cfg, choices, batches, D):
    spec = npipe.Spec(cfg, flags=FLAGS | npipe.FLAG_TIMED)
    h = npipe.naspipe_create(spec, D)
    for y, ch in enumerate(choices):
        npipe.naspipe_submit(h, ch, *batches[y])
    npipe.naspipe_drain(h)
    params = {(b, c): npipe.naspipe_get_params(h, b, c)
              for b in range(cfg["n_blocks"]) for c in range(cfg["n_choices"])}
    out = (params, npipe.naspipe_get_losses(h, len(choices)), npipe.naspipe_get_trace(h),
           npipe.naspipe_get_stats(h), npipe.naspipe_get_timed_stats(h))
    npipe.naspipe_destroy(h)
    return out


@pytest.mark.parametrize("name,N,D", [("toy", 12, 1), ("toy", 16, 2), ("toy", 16, 4), ("tiny_transformer", 6, 2),
                                      ("tiny_transformer", 6, 3), ("tiny_spos", 5, 2)])
def test_timed_execution_is_csp_and_bitwise_the_planned_result(name, N, D):
    cfg = synth.get_config(name)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    params, losses, trace, stats, ts = _run_timed(cfg, choices, batches, D)
    sob = npipe.naspipe_partition(npipe.Spec(cfg), D)
    tr = [tuple(int(v) for v in r) for r in trace]
    assert len(tr) == 2 * N * D
    assert csp.check_trace(tr, np.asarray(choices).tolist(), sob, D) == []
    if D == 1:
        assert [(k, y) for _, _, k, y in tr] == [(k, y) for y in range(N) for k in (0, 1)]
    assert stats["version_checks"] == 2 * N * cfg["n_blocks"]
    assert ts["tasks"] == 2 * N * D and ts["backwards"] == N * D
    assert 0 <= ts["hits"] <= ts["predictions"] <= ts["backwards"]
    print(f"{name} D={D}: Alg.3 predictions {ts['predictions']:.0f}/{ts['backwards']:.0f}, "
          f"right {ts['hits']:.0f}; host loop {ts['host_ms']:.1f} ms")
    p1, l1, _, _ = run_engine(cfg, choices, batches, D=1)
    assert np.array_equal(losses.view(np.uint32), l1.view(np.uint32))
    for k in p1:
        assert np.array_equal(params[k].view(np.uint32), p1[k].view(np.uint32)), k


def test_timed_rejects_unsupported_modes():
    cfg = synth.get_config("toy")
    for over in ({"sync": "asp"}, {"hbm_weight_budget_bytes": 1 << 20}):
        with pytest.raises(npipe.NaspipeError):
            npipe.naspipe_create(npipe.Spec(dict(cfg, **over), flags=npipe.FLAG_TIMED), 2)


def test_timed_drains_twice():
    """A second submit / drain after the first continues the id sequence (reading A23)."""
    cfg = synth.get_config("toy")
    N = 8
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    spec = npipe.Spec(cfg, flags=FLAGS | npipe.FLAG_TIMED)
    h = npipe.naspipe_create(spec, 2)
    for y in range(N):
        npipe.naspipe_submit(h, choices[y], *batches[y])
        if y == 3:
            npipe.naspipe_drain(h)
    npipe.naspipe_drain(h)
    params = {(b, c): npipe.naspipe_get_params(h, b, c) for b in range(cfg["n_blocks"]) for c in range(cfg["n_choices"])}
    losses = npipe.naspipe_get_losses(h, N)
    npipe.naspipe_destroy(h)
    p1, l1, _, _ = run_engine(cfg, choices, batches, D=1)
    assert np.array_equal(losses.view(np.uint32), l1.view(np.uint32))
    for k in p1:
        assert np.array_equal(params[k].view(np.uint32), p1[k].view(np.uint32)), k
