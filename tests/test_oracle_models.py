"""Pins for the oracle's block families (oracle/mlp.py, oracle/transformer.py).

* Brute-force central finite differences in float64 (SURVEY §8c "What pins each part").
* Closed forms: LayerNorm output statistics, softmax rows, GELU special values.
"""
import numpy as np
import pytest

from oracle import mlp, transformer


def _num_grad(f, arr, idx, eps):
    old = arr[idx]
    arr[idx] = old + eps
    fp = f()
    arr[idx] = old - eps
    fm = f()
    arr[idx] = old
    return (fp - fm) / (2 * eps)


def _check_all(loss_fn, analytic, tensors, rng, eps=1e-6, n_coords=10, tol=1e-6):
    for name, arr in tensors.items():
        g = analytic[name]
        assert g.shape == arr.shape, name
        flat_idx = rng.choice(arr.size, size=min(n_coords, arr.size), replace=False)
        for fi in flat_idx:
            idx = np.unravel_index(fi, arr.shape)
            num = _num_grad(loss_fn, arr, idx, eps)
            # relative 1e-6, plus an absolute floor for the FD round-off (~1e-16 |L| / eps)
            err = abs(num - g[idx])
            assert err <= tol * max(abs(num), abs(g[idx])) + 1e-7, (name, idx, num, g[idx], err)


def test_mlp_fd():
    rng = np.random.default_rng(0)
    d, B = 8, 5
    p = {"W": rng.standard_normal((d, d)) * 0.4, "b": rng.standard_normal(d) * 0.3}
    x = rng.standard_normal((B, d))
    R = rng.standard_normal((B, d))
    y, tape = mlp.forward(p, x)
    dx, gr = mlp.backward(p, tape, R)
    loss = lambda: float(np.sum(mlp.forward(p, x)[0] * R))          # noqa: E731
    _check_all(loss, gr, p, rng)
    _check_all(loss, {"x": dx}, {"x": x}, rng)


def _tiny_tf_params(rng, d, f, scale=0.3):
    p = {"Wqkv": rng.standard_normal((3 * d, d)) * scale, "bqkv": rng.standard_normal(3 * d) * scale,
         "Wo": rng.standard_normal((d, d)) * scale, "bo": rng.standard_normal(d) * scale,
         "ln1_g": 1 + 0.2 * rng.standard_normal(d), "ln1_b": 0.2 * rng.standard_normal(d),
         "W1": rng.standard_normal((f, d)) * scale, "b1": rng.standard_normal(f) * scale,
         "W2": rng.standard_normal((d, f)) * scale, "b2": rng.standard_normal(d) * scale,
         "ln2_g": 1 + 0.2 * rng.standard_normal(d), "ln2_b": 0.2 * rng.standard_normal(d)}
    return p


@pytest.mark.parametrize("h", [1, 2])
def test_transformer_fd(h):
    rng = np.random.default_rng(1)
    d, f, B, S = 16, 32, 2, 4
    p = _tiny_tf_params(rng, d, f)
    x = rng.standard_normal((B, S, d))
    R = rng.standard_normal((B, S, d))
    y, tape = transformer.forward(p, x, h)
    dx, gr = transformer.backward(p, tape, R)
    loss = lambda: float(np.sum(transformer.forward(p, x, h)[0] * R))  # noqa: E731
    _check_all(loss, gr, p, rng, n_coords=8)
    _check_all(loss, {"x": dx}, {"x": x}, rng, n_coords=16)


def test_layernorm_closed_form():
    rng = np.random.default_rng(2)
    x = rng.standard_normal((7, 33)) * 3 + 5
    y, _ = transformer.ln_fwd(x, np.ones(33), np.zeros(33))
    # normalised rows: mean 0, biased variance var/(var+eps)
    var = x.var(axis=-1)
    np.testing.assert_allclose(y.mean(axis=-1), 0, atol=1e-12)
    np.testing.assert_allclose(y.var(axis=-1), var / (var + 1e-5), rtol=1e-12)


def test_gelu_special_values():
    assert transformer.gelu(np.array(0.0)) == 0.0
    assert transformer.gelu_grad(np.array(0.0)) == 0.5
    # large |z|: GELU -> relu
    np.testing.assert_allclose(transformer.gelu(np.array([30.0, -30.0])), [30.0, 0.0], atol=1e-12)
    # published value of the tanh approximation at z = 1 (0.5*(1+tanh(sqrt(2/pi)*1.044715)))
    np.testing.assert_allclose(transformer.gelu(np.array(1.0)), 0.8411919906082768, rtol=1e-12)


def test_attention_uniform_keys_average_values():
    """Identical keys -> softmax uniform -> each query gets the mean of the values."""
    rng = np.random.default_rng(3)
    B, S, d, h = 2, 5, 8, 2
    q = rng.standard_normal((B, S, d))
    k = np.broadcast_to(rng.standard_normal((B, 1, d)), (B, S, d)).copy()
    v = rng.standard_normal((B, S, d))
    o, _ = transformer.attn_fwd(q, k, v, h)
    np.testing.assert_allclose(o, np.broadcast_to(v.mean(axis=1, keepdims=True), o.shape), rtol=1e-12)
