"""Pins for oracle/train.py (the sequential trainer).

* closed form: MLP with zero weights is the identity, so one SGD step is textbook
  least-squares gradient descent (loss scaling 2/(B d), lr, only active candidates change);
* invariant: any causally valid reordering (a linear extension of the conflict order)
  gives bitwise identical parameters and losses (Def.1);
* mutation: swapping two conflicting subnets changes the result.
"""
import numpy as np

import synth
from oracle import train


def _toy(N=10, seed=0):
    cfg = synth.get_config("toy")
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"], seed)
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    return cfg, choices, batches


def test_init_is_the_spec_hash():
    cfg = synth.get_config("toy")
    th = train.initial_theta(cfg)
    assert len(th) == 16
    v = th[(1, 2)]
    d = cfg["width"]
    assert v.dtype == np.float32 and v.size == d * d + d
    bound = np.float32(1) / np.sqrt(np.float32(d))
    assert np.all(np.abs(v) <= bound)
    # distinct candidates get distinct streams; values are not all equal
    assert not np.array_equal(th[(0, 0)], th[(0, 1)])
    # splitmix64 reference value (Vigna's splitmix64 with state 0 -> first output)
    z = synth._splitmix64(np.array([0], dtype=np.uint64))[0]
    assert int(z) == 0xE220A8397B1DCDAF


def test_zero_mlp_step_is_least_squares_gd():
    cfg, choices, batches = _toy(N=1)
    d, B, lr = cfg["width"], cfg["batch"], cfg["lr"]
    theta0 = {k: np.zeros_like(v) for k, v in train.initial_theta(cfg).items()}
    theta, losses = train.train_sequential(cfg, theta0, choices[:1], batches[:1])
    X, T = (a.astype(np.float64) for a in batches[0])
    # all four blocks are identity at zero weights: y = x
    assert losses[0] == np.mean((X - T) ** 2)
    G = 2.0 / (B * d) * (X - T)                  # dL/dy, identical at every block
    W_expect = -lr * (G.T @ X)
    b_expect = -lr * G.sum(axis=0)
    for b in range(cfg["n_blocks"]):
        c = int(choices[0][b])
        v = theta[(b, c)]
        np.testing.assert_allclose(v[: d * d].reshape(d, d), W_expect, rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(v[d * d:], b_expect, rtol=1e-12, atol=1e-15)
        for c2 in range(cfg["n_choices"]):
            if c2 != c:
                assert not np.any(theta[(b, c2)]), "inactive candidate changed"


def _random_linear_extension(choices, rng):
    N = len(choices)
    preds = [{x for x in range(y) if np.any(choices[x] == choices[y])} for y in range(N)]
    done, order = set(), []
    while len(order) < N:
        ready = [y for y in range(N) if y not in done and preds[y] <= done]
        y = int(rng.choice(ready))
        order.append(y)
        done.add(y)
    return order


def test_reordering_invariance_bitwise():
    # n large relative to m so that many reorderings exist
    cfg = synth.get_config("toy", n_choices=6, n_blocks=2)
    N = 12
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"], 5)
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    rng = np.random.default_rng(0)
    n_distinct = 0
    for _ in range(6):
        order = _random_linear_extension(choices, rng)
        n_distinct += order != list(range(N))
        th, ls = train.train_sequential(cfg, theta0, choices, batches, order=order)
        assert np.array_equal(ls, ref_loss)
        for k in ref:
            assert np.array_equal(th[k], ref[k]), k
    assert n_distinct > 0


def test_causally_invalid_swap_changes_result():
    cfg, choices, batches = _toy(N=6)
    theta0 = train.initial_theta(cfg)
    ref, _ = train.train_sequential(cfg, theta0, choices, batches)
    # find x < y sharing a candidate, adjacent in the order
    y = next(y for y in range(1, 6) if np.any(choices[y - 1] == choices[y]))
    order = list(range(6))
    order[y - 1], order[y] = order[y], order[y - 1]
    th, _ = train.train_sequential(cfg, theta0, choices, batches, order=order)
    assert any(not np.array_equal(th[k], ref[k]) for k in ref)


# ------------------------------------------------------------------ other sync policies
def test_bsp_bulk_is_gd_on_the_summed_gradient():
    """BSP (GPipe bulk update): a bulk of two subnets with the same candidates, from
    zero weights (every block the identity), updates by -lr (G0^T X0 + G1^T X1) — both
    gradients at the bulk's start weights — where sequential training would not."""
    cfg, choices, batches = _toy(N=2)
    choices = np.array([choices[0], choices[0]])
    d, B, lr = cfg["width"], cfg["batch"], cfg["lr"]
    theta0 = {k: np.zeros_like(v) for k, v in train.initial_theta(cfg).items()}
    theta, losses = train.train_bsp(cfg, theta0, choices, batches, bulk=2)
    W_expect = np.zeros((d, d))
    b_expect = np.zeros(d)
    for y in range(2):
        X, T = (a.astype(np.float64) for a in batches[y])
        assert losses[y] == np.mean((X - T) ** 2)
        G = 2.0 / (B * d) * (X - T)
        W_expect -= lr * (G.T @ X)
        b_expect -= lr * G.sum(axis=0)
    for b in range(cfg["n_blocks"]):
        v = theta[(b, int(choices[0][b]))]
        np.testing.assert_allclose(v[: d * d].reshape(d, d), W_expect, rtol=1e-12, atol=1e-15)
        np.testing.assert_allclose(v[d * d:], b_expect, rtol=1e-12, atol=1e-15)
    seq, _ = train.train_sequential(cfg, theta0, choices, batches)
    assert any(not np.array_equal(seq[k], theta[k]) for k in seq)


def test_bsp_bulk_one_is_sequential():
    cfg, choices, batches = _toy(N=6)
    th0 = train.initial_theta(cfg)
    a, la = train.train_bsp(cfg, th0, choices, batches, bulk=1)
    b, lb = train.train_sequential(cfg, th0, choices, batches)
    assert all(np.array_equal(a[k], b[k]) for k in a) and np.array_equal(la, lb)


def _replay_case(name, N, D, sync):
    from oracle import csp
    cfg = synth.get_config(name)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    sob = np.repeat(np.arange(D), cfg["n_blocks"] // D)
    ones = np.ones((cfg["n_blocks"], cfg["n_choices"]), dtype=np.int64)
    tf, tb = csp.task_costs(choices, sob, ones, 2 * ones, D)
    tr = csp.simulate_csp(choices, sob, D, 4 * D, tf, tb, sync=sync)["trace"]
    return cfg, choices, batches, sob, tr


def test_replay_of_csp_trace_is_sequential():
    """Executing a CSP schedule stage by stage is bitwise the sequential result."""
    for name, N, D in (("toy", 12, 2), ("toy", 12, 4), ("tiny_transformer", 4, 2)):
        cfg, choices, batches, sob, tr = _replay_case(name, N, D, "csp")
        th0 = train.initial_theta(cfg)
        a, la = train.train_replay(cfg, th0, choices, batches, sob, tr)
        b, lb = train.train_sequential(cfg, th0, choices, batches)
        assert all(np.array_equal(a[k], b[k]) for k in a), (name, D)
        assert np.array_equal(la, lb)


def test_replay_of_asp_trace_breaks_causality():
    """ASP (dependencies ignored): at one stage it is sequential; on a pipeline, subnets read
    weights their predecessors have not written yet, so the result changes (Table 3)."""
    cfg, choices, batches, sob, tr = _replay_case("toy", 12, 1, "asp")
    th0 = train.initial_theta(cfg)
    a, _ = train.train_replay(cfg, th0, choices, batches, np.zeros(cfg["n_blocks"], dtype=int), tr)
    b, _ = train.train_sequential(cfg, th0, choices, batches)
    assert all(np.array_equal(a[k], b[k]) for k in a)
    cfg, choices, batches, sob, tr = _replay_case("toy", 12, 2, "asp")
    c, _ = train.train_replay(cfg, th0, choices, batches, sob, tr)
    assert any(not np.array_equal(c[k], b[k]) for k in c)
