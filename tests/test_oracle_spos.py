"""Pins for oracle/spos.py (configs[1] SPOS CNN family).

* depthwise and dense convolutions against their definition written as explicit loops, and
  special cases (1x1 depthwise = per-channel scaling, centred delta kernel = identity);
* BatchNorm output statistics (closed form);
* central finite differences (fp64) of every block variant (stride 1/2 x Shuffle 3/5/7 and
  Xception) for the input and every parameter, and of the frozen head's cross-entropy;
* the trainer's SGD step on a tiny SPOS supernet changes exactly the active candidates.
"""
import numpy as np
import pytest

import synth
from oracle import spos, train


def _dw_loops(x, w, s, d=1):
    B, H, W, C = x.shape
    k = w.shape[1]
    p = d * (k // 2)
    Ho, Wo = (H + 2 * p - d * (k - 1) - 1) // s + 1, (W + 2 * p - d * (k - 1) - 1) // s + 1
    y = np.zeros((B, Ho, Wo, C))
    for b in range(B):
        for i in range(Ho):
            for j in range(Wo):
                for c in range(C):
                    acc = 0.0
                    for u in range(k):
                        for v in range(k):
                            ii, jj = i * s + u * d - p, j * s + v * d - p
                            if 0 <= ii < H and 0 <= jj < W:
                                acc += x[b, ii, jj, c] * w[c, u, v]
                    y[b, i, j, c] = acc
    return y


@pytest.mark.parametrize("k,s,d", [(3, 1, 1), (5, 2, 1), (7, 1, 1), (3, 2, 1), (3, 1, 2), (5, 2, 2), (7, 1, 2)])
def test_depthwise_matches_loops(k, s, d):
    rng = np.random.default_rng(k * 10 + s + 100 * d)
    x = rng.standard_normal((2, 7, 7, 3))
    w = rng.standard_normal((3, k, k))
    y = spos.dw_fwd(x, w, s, d)
    assert y.shape == (2, (7 - 1) // s + 1, (7 - 1) // s + 1, 3)   # "same" padding for every dilation
    np.testing.assert_allclose(y, _dw_loops(x, w, s, d), rtol=1e-12, atol=1e-12)


def test_dilated_depthwise_special_cases():
    """Dilation 2 of a k x k kernel = the (2k-1) x (2k-1) kernel with zeros between the taps;
    a kernel whose only nonzero tap is the centre is the identity for every dilation."""
    rng = np.random.default_rng(3)
    x = rng.standard_normal((2, 9, 9, 4))
    w = rng.standard_normal((4, 3, 3))
    wz = np.zeros((4, 5, 5))
    wz[:, ::2, ::2] = w
    for s in (1, 2):
        np.testing.assert_allclose(spos.dw_fwd(x, w, s, 2), spos.dw_fwd(x, wz, s, 1), rtol=1e-13, atol=1e-13)
    delta = np.zeros((4, 5, 5))
    delta[:, 2, 2] = 1.0
    np.testing.assert_allclose(spos.dw_fwd(x, delta, 1, 2), x, rtol=1e-14)


def test_depthwise_special_cases():
    rng = np.random.default_rng(0)
    x = rng.standard_normal((2, 5, 5, 4))
    w1 = rng.standard_normal((4, 1, 1))
    np.testing.assert_allclose(spos.dw_fwd(x, w1, 1), x * w1[:, 0, 0], rtol=1e-14)
    delta = np.zeros((4, 3, 3))
    delta[:, 1, 1] = 1.0
    np.testing.assert_allclose(spos.dw_fwd(x, delta, 1), x, rtol=1e-14)
    np.testing.assert_allclose(spos.dw_fwd(x, delta, 2), x[:, ::2, ::2, :], rtol=1e-14)


def test_dense_conv_matches_loops():
    rng = np.random.default_rng(1)
    x = rng.standard_normal((1, 6, 6, 3))
    w = rng.standard_normal((4, 3, 3, 3))
    y = spos.conv_fwd(x, w, 2)
    ref = np.zeros_like(y)
    for i in range(3):
        for j in range(3):
            for o in range(4):
                for u in range(3):
                    for v in range(3):
                        ii, jj = 2 * i + u - 1, 2 * j + v - 1
                        if 0 <= ii < 6 and 0 <= jj < 6:
                            ref[0, i, j, o] += x[0, ii, jj, :] @ w[o, u, v, :]
    np.testing.assert_allclose(y, ref, rtol=1e-12)


@pytest.mark.parametrize("k,s", [(3, 1), (3, 2), (5, 1), (5, 2)])
def test_dense_conv_fwd_bwd_match_torch(k, s):
    """conv_fwd / conv_bwd (the dense Conv 3x3 candidate, reading A40) against PyTorch's
    conv2d (NCHW, padding k // 2) and its autograd gradients, fp64."""
    torch = pytest.importorskip("torch")
    rng = np.random.default_rng(10 * k + s)
    x = rng.standard_normal((2, 10, 10, 8))
    w = rng.standard_normal((6, k, k, 8))
    y = spos.conv_fwd(x, w, s)
    xt = torch.tensor(x.transpose(0, 3, 1, 2), requires_grad=True)
    wt = torch.tensor(w.transpose(0, 3, 1, 2), requires_grad=True)
    yt = torch.nn.functional.conv2d(xt, wt, stride=s, padding=k // 2)
    np.testing.assert_allclose(y, yt.detach().numpy().transpose(0, 2, 3, 1), rtol=1e-12, atol=1e-12)
    dy = rng.standard_normal(y.shape)
    yt.backward(torch.tensor(dy.transpose(0, 3, 1, 2)))
    dx, dw = spos.conv_bwd(x, w, s, dy)
    np.testing.assert_allclose(dx, xt.grad.numpy().transpose(0, 2, 3, 1), rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(dw, wt.grad.numpy().transpose(0, 2, 3, 1), rtol=1e-12, atol=1e-12)


def test_dense_candidate_structure():
    """The dense candidate is the Shuffle block with its depthwise conv replaced: same units,
    the mid conv dense [mid, k, k, mid] (fan-in k k mid); a centred identity kernel (w[o, 1, 1, i]
    = delta_oi) makes it reproduce the Shuffle block with a centred-delta depthwise kernel."""
    b, c_dense, c_shuf = 1, 0, 2          # MINI_DENSE: c 0 = dense k 3, c 2 = Shuffle k 3
    ld = spos.layout(MINI_DENSE, b, c_dense)
    ls = spos.layout(MINI_DENSE, b, c_shuf)
    assert [n for n, *_ in ld] == [n.replace("m_dw", "m_cv") for n, *_ in ls]
    s, inp, mid, out, cout, H = spos.block_dims(MINI_DENSE, b)
    assert dict((n, (sh, f)) for n, sh, _, f in ld)["m_cv"] == ((mid, 3, 3, mid), 9 * mid)
    rng = np.random.default_rng(3)
    ps = {n: (rng.standard_normal(sh) if kind == "uniform" else (np.ones(sh) if kind == "ones" else np.zeros(sh)))
          for n, sh, kind, _ in ls}
    ps["m_dw"] = np.zeros((mid, 3, 3))
    ps["m_dw"][:, 1, 1] = 1.0
    pd = {n.replace("m_dw", "m_cv"): v for n, v in ps.items()}
    pd["m_cv"] = np.zeros((mid, 3, 3, mid))
    pd["m_cv"][:, 1, 1, :] = np.eye(mid)
    x = rng.standard_normal((2, H, H, cout))
    ys, _ = spos.block_fwd(MINI_DENSE, b, c_shuf, ps, x)
    yd, _ = spos.block_fwd(MINI_DENSE, b, c_dense, pd, x)
    np.testing.assert_allclose(yd, ys, rtol=1e-12, atol=1e-12)


def test_batchnorm_closed_form():
    rng = np.random.default_rng(2)
    x = rng.standard_normal((3, 4, 4, 5)) * 3 + 2
    y, _ = spos.bn_fwd(x, np.ones(5), np.zeros(5))
    var = x.var(axis=(0, 1, 2))
    np.testing.assert_allclose(y.mean(axis=(0, 1, 2)), 0, atol=1e-12)
    np.testing.assert_allclose(y.var(axis=(0, 1, 2)), var / (var + 1e-5), rtol=1e-10)


MINI = dict(family="spos", n_blocks=2, n_choices=4, batch=2, image_hw=16, num_classes=5,
            stage_repeats=[2], stage_channels=[8], stem_channels=4, head_channels=6,
            choice_kernel=[3, 5, 7, 3], choice_xception=[0, 0, 0, 1], lr=0.01, init_seed=2)
# the dilated choices of Table 5 (reading A36): Shuffle 3/5 and Xception 3/5 at dilation 2
MINI_DIL = dict(MINI, choice_kernel=[3, 5, 3, 5], choice_xception=[0, 0, 1, 1], choice_dilation=[2, 2, 2, 2])
# Table 5's dense "Conv 3x3" (reading A40): the Shuffle block with a dense k x k mid conv
MINI_DENSE = dict(MINI, choice_kernel=[3, 5, 3, 3], choice_xception=[2, 2, 0, 1])


def _check_fd(f, analytic, arr, rng, n=6, eps=1e-6):
    idxs = rng.choice(arr.size, size=min(n, arr.size), replace=False)
    for fi in idxs:
        i = np.unravel_index(fi, arr.shape)
        old = arr[i]
        arr[i] = old + eps
        fp = f()
        arr[i] = old - eps
        fm = f()
        arr[i] = old
        num = (fp - fm) / (2 * eps)
        assert abs(num - analytic[i]) <= 1e-5 * max(abs(num), abs(analytic[i])) + 1e-7, (i, num, analytic[i])


@pytest.mark.parametrize("cfg", [MINI, MINI_DIL, MINI_DENSE], ids=["plain", "dilated", "dense"])
@pytest.mark.parametrize("b", [0, 1])          # block 0: stride 2 (proj branch), block 1: stride 1
@pytest.mark.parametrize("c", [0, 1, 2, 3])    # Shuffle 3/5/7, Xception (MINI_DIL: dilated Shuffle/Xception 3/5)
def test_block_fd(b, c, cfg):
    MINI = cfg
    rng = np.random.default_rng(10 * b + c)
    s, inp, mid, out, cout, H = spos.block_dims(MINI, b)
    p = {}
    for name, shape, kind, _ in spos.layout(MINI, b, c):
        if kind == "uniform":
            p[name] = rng.standard_normal(shape) * 0.5
        else:
            p[name] = (1.0 if kind == "ones" else 0.0) + 0.2 * rng.standard_normal(shape)
    cin = inp if s == 2 else cout
    x = rng.standard_normal((2, H, H, cin))
    y, tapes = spos.block_fwd(MINI, b, c, p, x)
    assert y.shape == (2, H // s, H // s, cout)
    R = rng.standard_normal(y.shape)
    dx, g = spos.block_bwd(MINI, b, c, p, tapes, R)
    loss = lambda: float(np.sum(spos.block_fwd(MINI, b, c, p, x)[0] * R))   # noqa: E731
    _check_fd(loss, dx, x, rng)
    for name in p:
        _check_fd(loss, g[name], p[name], rng, n=3)


def test_head_loss_fd():
    rng = np.random.default_rng(5)
    fz = train.frozen_theta(MINI)
    x = rng.standard_normal((2, 4, 4, 8))
    labels = np.array([1, 3])
    _, dx = spos.head_loss(fz, x, labels)
    _check_fd(lambda: spos.head_loss(fz, x, labels)[0], dx, x, rng, n=10)


def test_tiny_spos_training_updates_only_active():
    cfg = synth.get_config("tiny_spos")
    ch = synth.sample_choices(2, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(2)]
    th0 = train.initial_theta(cfg)
    th, losses = train.train_sequential(cfg, th0, ch, batches)
    assert np.all(np.isfinite(losses)) and abs(losses[0] - np.log(cfg["num_classes"])) < 1.0
    used = {(b, int(ch[y][b])) for y in range(2) for b in range(cfg["n_blocks"])}
    for k in th:
        changed = not np.array_equal(th[k], th0[k].astype(np.float64))
        assert changed == (k in used), k


def test_storage_rounding_pins():
    """spos.to_bf16 is round-to-nearest-even to bfloat16 (ties, carries, sign, against torch's
    independent conversion); to_bf16x2 keeps 16 mantissa bits; PLAIN storage is the identity."""
    torch = pytest.importorskip("torch")
    assert spos.to_bf16(1 + 2.0 ** -8) == 1.0                     # tie -> even (down)
    assert spos.to_bf16(1 + 3 * 2.0 ** -8) == 1 + 2.0 ** -6       # tie -> even (up)
    assert spos.to_bf16(-(1 + 2.0 ** -7 + 2.0 ** -9)) == -(1 + 2.0 ** -7)
    assert spos.to_bf16(2.0 - 2.0 ** -9) == 2.0                   # carry into the exponent
    x = np.random.default_rng(0).standard_normal(10000) * 10.0 ** np.random.default_rng(1).integers(-20, 20, 10000)
    ref = torch.from_numpy(x.astype(np.float32)).to(torch.bfloat16).to(torch.float64).numpy()
    np.testing.assert_array_equal(spos.to_bf16(x), ref)
    x2 = spos.to_bf16x2(x)
    assert np.all(np.abs(x2 - x.astype(np.float32)) <= 2.0 ** -16 * np.abs(x))
    assert spos.PLAIN.f(x) is x and spos.STORAGE[None] is spos.PLAIN


def test_storage_modes_only_round():
    """The storage modes change the result only by rounding: one tiny_spos step in BF16X2
    storage stays within 1e-3 of the plain loss and differs from it (the rounding is applied)."""
    cfg = synth.get_config("tiny_spos")
    ch = synth.sample_choices(1, cfg["n_blocks"], cfg["n_choices"])
    b = [synth.make_batch(cfg, 0)]
    th0 = train.initial_theta(cfg)
    _, l0 = train.train_sequential(cfg, th0, ch, b)
    _, l1 = train.train_sequential(dict(cfg, storage="bf16x2"), th0, ch, b)
    assert l0[0] != l1[0] and abs(l1[0] - l0[0]) <= 1e-3 * l0[0]
    # FP32 storage (the paper's precision): fp32 rounding of every stored tensor
    x = np.random.default_rng(3).standard_normal(1000) * 3
    np.testing.assert_array_equal(spos.to_fp32(x), x.astype(np.float32).astype(np.float64))
    _, l2 = train.train_sequential(dict(cfg, storage="fp32"), th0, ch, b)
    assert l0[0] != l2[0] and abs(l2[0] - l0[0]) <= 1e-6 * l0[0]
