"""Pins for the NLP op families of oracle/transformer.py (Table 5 P:L443-446 "Conv 3x1, Sep
Conv 7x1, Light Conv 5x1"; reading A38):

* Conv 3x1 and the depthwise sequence conv against torch.nn.functional.conv1d (an independent
  library implementation: zero padding, cross-correlation, groups) and their gradients against
  torch autograd; explicit per-position loops on a tiny case;
* LightConv closed forms: equal kernel weights -> taps 1/k (a moving average; a constant
  sequence far from the ends is returned unchanged), a dominant weight -> a pure shift, taps
  shared inside a head, softmax rows sum to 1; its gradient against torch autograd of the
  softmax + grouped conv1d;
* central finite differences (fp64) of whole blocks of every op for the input and every
  parameter;
* sequences do not mix: changing sample 1 leaves sample 0's output unchanged.
"""
import numpy as np
import pytest

from oracle import transformer as T

torch = pytest.importorskip("torch")


def _t(a):
    return torch.tensor(a, dtype=torch.float64)


def test_seq_dwconv_matches_loops_and_torch():
    rng = np.random.default_rng(0)
    B, S, d, k = 2, 9, 5, 7
    x = rng.standard_normal((B, S, d))
    w = rng.standard_normal((d, k))
    y = T.seq_dwconv(x, w)
    ref = np.zeros_like(y)
    for b in range(B):
        for t in range(S):
            for i in range(d):
                ref[b, t, i] = sum(w[i, u] * x[b, t + u - k // 2, i] for u in range(k) if 0 <= t + u - k // 2 < S)
    np.testing.assert_allclose(y, ref, rtol=1e-13, atol=1e-13)
    X = _t(x).permute(0, 2, 1).requires_grad_()
    W = _t(w)[:, None].requires_grad_()
    Y = torch.nn.functional.conv1d(X, W, padding=k // 2, groups=d)
    np.testing.assert_allclose(Y.detach().permute(0, 2, 1).numpy(), y, rtol=1e-12, atol=1e-12)
    dy = rng.standard_normal(y.shape)
    Y.backward(_t(dy).permute(0, 2, 1))
    dx, dw = T.seq_dwconv_bwd(x, w, dy)
    np.testing.assert_allclose(X.grad.permute(0, 2, 1).numpy(), dx, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(W.grad[:, 0].numpy(), dw, rtol=1e-12, atol=1e-12)


def test_conv3_matches_torch_conv1d():
    """M = cols(a) Wc^T + bc with Wc[o, u*d + i] = tap u of input i equals conv1d(k=3, pad 1)."""
    rng = np.random.default_rng(1)
    B, S, d = 2, 7, 4
    a = rng.standard_normal((B, S, d))
    Wc = rng.standard_normal((d, 3 * d))
    bc = rng.standard_normal(d)
    p = {"Wc": Wc, "bc": bc}
    m, mt = T.mixer_fwd("conv3", p, a, 1)
    Wt = _t(Wc.reshape(d, 3, d).transpose(0, 2, 1).copy()).requires_grad_()     # [out, in, k]
    A = _t(a).permute(0, 2, 1).requires_grad_()
    M = torch.nn.functional.conv1d(A, Wt, _t(bc), padding=1)
    np.testing.assert_allclose(M.detach().permute(0, 2, 1).numpy(), m, rtol=1e-12, atol=1e-12)
    dm = rng.standard_normal(m.shape)
    M.backward(_t(dm).permute(0, 2, 1))
    gr = {}
    da = T.mixer_bwd("conv3", p, a, mt, dm, gr)
    np.testing.assert_allclose(A.grad.permute(0, 2, 1).numpy(), da, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(Wt.grad.numpy().transpose(0, 2, 1).reshape(d, 3 * d), gr["Wc"], rtol=1e-12,
                               atol=1e-12)
    np.testing.assert_allclose(gr["bc"], dm.sum(axis=(0, 1)), rtol=1e-12)


def test_lightconv_closed_forms():
    rng = np.random.default_rng(2)
    d, H, k = 8, 2, 5
    # equal weights: every tap 1/k; a constant sequence stays constant away from the ends
    taps, pr = T.light_taps(np.full((H, k), 0.7), d)
    np.testing.assert_allclose(taps, 1.0 / k, rtol=1e-15)
    x = np.full((1, 11, d), 3.0)
    y = T.seq_dwconv(x, taps)
    np.testing.assert_allclose(y[0, 2:-2], 3.0, rtol=1e-14)
    np.testing.assert_allclose(y[0, 0], 3.0 * 3 / 5, rtol=1e-14)          # 2 of 5 taps fall off the start
    # one dominant weight per head: taps -> one-hot, the conv becomes a shift by u - 2
    Wl = np.full((H, k), -1e3)
    Wl[0, 4] = Wl[1, 0] = 0.0
    taps, _ = T.light_taps(Wl, d)
    x = rng.standard_normal((2, 9, d))
    y = T.seq_dwconv(x, taps)
    np.testing.assert_allclose(y[:, :-2, :4], x[:, 2:, :4], rtol=1e-14)    # head 0 reads t + 2
    np.testing.assert_allclose(y[:, 2:, 4:], x[:, :-2, 4:], rtol=1e-14)    # head 1 reads t - 2
    # random weights: rows sum to 1, channels of a head share their taps
    taps, pr = T.light_taps(rng.standard_normal((H, k)), d)
    np.testing.assert_allclose(pr.sum(axis=1), 1.0, rtol=1e-14)
    assert np.array_equal(taps[:4], np.repeat(pr[:1], 4, axis=0)) and np.array_equal(taps[4:], np.repeat(pr[1:], 4, 0))


def test_lightconv_gradient_matches_torch_autograd():
    rng = np.random.default_rng(3)
    B, S, d, H, k = 2, 8, 6, 3, 5
    v = rng.standard_normal((B, S, d))
    Wl = rng.standard_normal((H, k))
    taps, pr = T.light_taps(Wl, d)
    dy = rng.standard_normal((B, S, d))
    dv, dtaps = T.seq_dwconv_bwd(v, taps, dy)
    dWl = T.light_taps_bwd(pr, dtaps)
    V = _t(v).permute(0, 2, 1).requires_grad_()
    W = _t(Wl).requires_grad_()
    P = torch.softmax(W, dim=1).repeat_interleave(d // H, dim=0)[:, None]
    Y = torch.nn.functional.conv1d(V, P, padding=k // 2, groups=d)
    Y.backward(_t(dy).permute(0, 2, 1))
    np.testing.assert_allclose(V.grad.permute(0, 2, 1).numpy(), dv, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(W.grad.numpy(), dWl, rtol=1e-11, atol=1e-12)


def _params(rng, op, d, h, f, scale=0.3):
    p = {}
    for name, shape, kind, _ in T.mixer_layout(op, d, h):
        p[name] = rng.standard_normal(shape) * scale
    p.update({"ln1_g": 1 + 0.2 * rng.standard_normal(d), "ln1_b": 0.2 * rng.standard_normal(d),
              "W1": rng.standard_normal((f, d)) * scale, "b1": rng.standard_normal(f) * scale,
              "W2": rng.standard_normal((d, f)) * scale, "b2": rng.standard_normal(d) * scale,
              "ln2_g": 1 + 0.2 * rng.standard_normal(d), "ln2_b": 0.2 * rng.standard_normal(d)})
    return p


def _fd(f, analytic, arr, rng, n):
    for fi in rng.choice(arr.size, size=min(n, arr.size), replace=False):
        i = np.unravel_index(fi, arr.shape)
        old = arr[i]
        arr[i] = old + 1e-6
        fp = f()
        arr[i] = old - 1e-6
        fm = f()
        arr[i] = old
        num = (fp - fm) / 2e-6
        assert abs(num - analytic[i]) <= 1e-6 * max(abs(num), abs(analytic[i])) + 1e-8, (i, num, analytic[i])


@pytest.mark.parametrize("op", ["conv3", "sepconv7", "lightconv5", "attn"])
def test_block_fd_every_op(op):
    rng = np.random.default_rng(4)
    d, h, f, B, S = 8, 2, 12, 2, 9
    p = _params(rng, op, d, h, f)
    x = rng.standard_normal((B, S, d))
    R = rng.standard_normal((B, S, d))
    y, tape = T.forward(p, x, h, op)
    dx, gr = T.backward(p, tape, R)
    assert set(gr) == set(p)
    loss = lambda: float(np.sum(T.forward(p, x, h, op)[0] * R))   # noqa: E731
    _fd(loss, dx, x, rng, 12)
    for name in p:
        _fd(loss, gr[name], p[name], rng, 6)


@pytest.mark.parametrize("op", ["conv3", "sepconv7", "lightconv5"])
def test_sequences_do_not_mix(op):
    rng = np.random.default_rng(5)
    d, h, f = 8, 2, 12
    p = _params(rng, op, d, h, f)
    x = rng.standard_normal((2, 6, d))
    y0, _ = T.forward(p, x, h, op)
    x[1] += 5 * rng.standard_normal((6, d))
    y1, _ = T.forward(p, x, h, op)
    assert np.array_equal(y0[0], y1[0]) and not np.allclose(y0[1], y1[1])
