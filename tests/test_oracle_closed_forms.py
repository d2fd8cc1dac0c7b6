"""Closed-form and library pins of the oracle's forward DEFINITIONS (round 2).

Finite differences only check a backward against its own forward, so a mistake in the
forward definition (attention scale, head split, q/k/v order, LN placement, SPOS channel
split / concat order / ReLU placement, the CE value) passes every FD pin.  The tests here fix
the forward to something other than the oracle itself:

* hand-worked examples whose expected values are derived in the docstrings (d = 4, h = 2,
  S = 2 transformer; stride-1 and stride-2 SPOS blocks with identity 1x1 weights and delta
  depthwise kernels; the CE of an all-zero classifier = ln(num_classes));
* an independent library implementation: torch.nn.TransformerEncoderLayer (norm_first=True,
  tanh-GELU, dropout 0, eps 1e-5) in float64 with the oracle's packed weights — PyTorch's
  in-projection packs q, k, v as contiguous thirds of in_proj_weight, splits heads as
  contiguous column groups and scales by 1/sqrt(head_dim), which is reading A17 — for the
  block forward AND every parameter gradient (autograd);
* torch.nn.functional conv2d / batch_norm / relu / cross_entropy for the SPOS units and head;
* the sampler's conflict rate against 1 - (1 - 1/n)^b (SURVEY §8c "Sampler").

Each of these fails on a deliberately injected 1/sqrt(d) scale, swapped q/v thirds, an
interleaved head split, post-LN placement, a swapped stride-1 split parity, a swapped
concat(proj, main) order, or a ReLU moved in the Shuffle chain (checked by mutation when the
tests were written; see the round-2 commit message).
"""
import math

import numpy as np
import pytest

import synth
from oracle import spos, transformer

torch = pytest.importorskip("torch")

R = 1.0 / math.sqrt(1.0 + 1e-5)          # LN / BN normalisation of a unit-variance input


# ------------------------------------------------------------------------------ transformer
def _tf_params(d, f, Wq=None, Wk=None, Wv=None, Wo=None):
    z = np.zeros
    p = {"Wqkv": np.concatenate([Wq, Wk, Wv]), "bqkv": z(3 * d), "Wo": Wo, "bo": z(d),
         "ln1_g": np.ones(d), "ln1_b": z(d), "W1": z((f, d)), "b1": z(f), "W2": z((d, f)),
         "b2": z(d), "ln2_g": np.ones(d), "ln2_b": z(d)}
    return p


def test_transformer_hand_worked_d4_h2_s2():
    """d = 4, h = 2 (hd = 2), S = 2, B = 1.  Wq = Wk = I, Wv = 2I, Wo = I, every bias 0,
    FFN weights 0 (so the FFN adds GELU(0)·0 + 0 = 0 and y = x1).

    x_0 = [1,-1,1,-1], x_1 = [1,1,-1,-1]: each row has mean 0 and biased variance 1, so
    pre-LN gives a_i = r x_i with r = 1/sqrt(1 + 1e-5).  q = k = a, v = 2a.
    Head 0 = columns {0,1}: a_0 -> r[1,-1], a_1 -> r[1,1]; head 1 = columns {2,3}:
    a_0 -> r[1,-1], a_1 -> r[-1,-1].  In both heads q_i.k_i = 2 r^2 and q_0.k_1 = 0, so the
    scaled scores are [[s, 0], [0, s]] with s = 2 r^2 / sqrt(hd) = sqrt(2) r^2, and
    p = e^s / (e^s + 1) = sigmoid(sqrt(2) r^2) ≈ 0.80442.  Then
        o_0 = p v_0 + (1 - p) v_1 = 2 r (p x_0 + (1 - p) x_1)   (same for every head's columns)
        y_0 = x_0 + o_0,  y_1 = x_1 + 2 r (p x_1 + (1 - p) x_0).
    A 1/sqrt(d) scale gives p = sigmoid(r^2) ≈ 0.7311; q and v swapped doubles the scores
    (p ≈ 0.9442) and halves v; post-LN would return LN(x + o) whose rows have variance 1.
    """
    d, f = 4, 8
    I = np.eye(d)
    p = _tf_params(d, f, Wq=I, Wk=I, Wv=2 * I, Wo=I)
    x = np.array([[[1.0, -1, 1, -1], [1, 1, -1, -1]]])
    y, _ = transformer.forward(p, x, 2)
    r = R
    pr = 1.0 / (1.0 + math.exp(-math.sqrt(2.0) * r * r))
    assert abs(pr - 0.80442) < 1e-4
    x0, x1 = x[0, 0], x[0, 1]
    exp = np.stack([x0 + 2 * r * (pr * x0 + (1 - pr) * x1), x1 + 2 * r * (pr * x1 + (1 - pr) * x0)])
    np.testing.assert_allclose(y[0], exp, rtol=0, atol=1e-13)


def test_transformer_hand_worked_head_split():
    """Heads are CONTIGUOUS column groups (A17).  d = 4, h = 2, S = 2, Wk = Wv = Wo = I,
    Wq = diag(c, c, 0, 0) with c = ln(3) / (sqrt(2) r^2) (r as above), biases and FFN 0,
    so the two heads see different score structures;
    x_0 = [1,-1, 1,-1], x_1 = [1,1,-1,-1] (mean 0, variance 1: a = r x).
    Head 0 (cols 0,1): q_0 = c r[1,-1], q_1 = c r[1,1]; k_0 = r[1,-1], k_1 = r[1,1];
      scaled scores row 0: [2 c r^2 / sqrt(2), 0] = [ln 3, 0] -> p = [3/4, 1/4];
      row 1: [0, ln 3] -> [1/4, 3/4].  o_0[0:2] = 3/4 a_0 + 1/4 a_1, o_1[0:2] = 1/4 a_0 + 3/4 a_1.
    Head 1 (cols 2,3): q = 0 -> uniform attention: o_i[2:4] = (a_0 + a_1)/2 [2:4].
    An interleaved split (head j = columns j::h) gives head 0 = cols {0,2} with q = [c r, 0]
    and different weights; the test fails on it.
    """
    d, f = 4, 8
    r = R
    c = math.log(3.0) / (math.sqrt(2.0) * r * r)
    p = _tf_params(d, f, Wq=np.diag([c, c, 0.0, 0.0]), Wk=np.eye(d), Wv=np.eye(d), Wo=np.eye(d))
    x = np.array([[[1.0, -1, 1, -1], [1, 1, -1, -1]]])
    y, _ = transformer.forward(p, x, 2)
    a0, a1 = r * x[0, 0], r * x[0, 1]
    o0 = np.concatenate([0.75 * a0[:2] + 0.25 * a1[:2], 0.5 * (a0[2:] + a1[2:])])
    o1 = np.concatenate([0.25 * a0[:2] + 0.75 * a1[:2], 0.5 * (a0[2:] + a1[2:])])
    np.testing.assert_allclose(y[0], np.stack([x[0, 0] + o0, x[0, 1] + o1]), rtol=0, atol=1e-13)


def _torch_layer(p, d, h, f):
    layer = torch.nn.TransformerEncoderLayer(
        d_model=d, nhead=h, dim_feedforward=f, dropout=0.0,
        activation=lambda t: torch.nn.functional.gelu(t, approximate="tanh"),
        layer_norm_eps=1e-5, batch_first=True, norm_first=True, dtype=torch.float64)
    T = lambda a: torch.tensor(a, dtype=torch.float64)  # noqa: E731
    with torch.no_grad():
        layer.self_attn.in_proj_weight.copy_(T(p["Wqkv"]))
        layer.self_attn.in_proj_bias.copy_(T(p["bqkv"]))
        layer.self_attn.out_proj.weight.copy_(T(p["Wo"]))
        layer.self_attn.out_proj.bias.copy_(T(p["bo"]))
        layer.norm1.weight.copy_(T(p["ln1_g"]))
        layer.norm1.bias.copy_(T(p["ln1_b"]))
        layer.linear1.weight.copy_(T(p["W1"]))
        layer.linear1.bias.copy_(T(p["b1"]))
        layer.linear2.weight.copy_(T(p["W2"]))
        layer.linear2.bias.copy_(T(p["b2"]))
        layer.norm2.weight.copy_(T(p["ln2_g"]))
        layer.norm2.bias.copy_(T(p["ln2_b"]))
    layer.train()      # dropout is 0; train() avoids the fused inference fast path
    grads = {"Wqkv": layer.self_attn.in_proj_weight, "bqkv": layer.self_attn.in_proj_bias,
             "Wo": layer.self_attn.out_proj.weight, "bo": layer.self_attn.out_proj.bias,
             "ln1_g": layer.norm1.weight, "ln1_b": layer.norm1.bias,
             "W1": layer.linear1.weight, "b1": layer.linear1.bias,
             "W2": layer.linear2.weight, "b2": layer.linear2.bias,
             "ln2_g": layer.norm2.weight, "ln2_b": layer.norm2.bias}
    return layer, grads


@pytest.mark.parametrize("d,h,f,S", [(16, 2, 32, 5), (24, 3, 40, 7), (32, 4, 64, 4)])
def test_transformer_block_matches_torch_encoder_layer(d, h, f, S):
    """Forward and every gradient of the A17 block against PyTorch's pre-LN encoder layer."""
    rng = np.random.default_rng(d + h)
    p = {"Wqkv": rng.standard_normal((3 * d, d)) * 0.3, "bqkv": rng.standard_normal(3 * d) * 0.3,
         "Wo": rng.standard_normal((d, d)) * 0.3, "bo": rng.standard_normal(d) * 0.3,
         "ln1_g": 1 + 0.2 * rng.standard_normal(d), "ln1_b": 0.2 * rng.standard_normal(d),
         "W1": rng.standard_normal((f, d)) * 0.3, "b1": rng.standard_normal(f) * 0.3,
         "W2": rng.standard_normal((d, f)) * 0.3, "b2": rng.standard_normal(d) * 0.3,
         "ln2_g": 1 + 0.2 * rng.standard_normal(d), "ln2_b": 0.2 * rng.standard_normal(d)}
    x = rng.standard_normal((2, S, d))
    R_ = rng.standard_normal((2, S, d))
    y, tape = transformer.forward(p, x, h)
    dx, gr = transformer.backward(p, tape, R_)
    layer, tparams = _torch_layer(p, d, h, f)
    xt = torch.tensor(x, requires_grad=True)
    yt = layer(xt)
    np.testing.assert_allclose(y, yt.detach().numpy(), rtol=1e-11, atol=1e-11)
    (yt * torch.tensor(R_)).sum().backward()
    np.testing.assert_allclose(dx, xt.grad.numpy(), rtol=1e-10, atol=1e-10)
    for name, t in tparams.items():
        np.testing.assert_allclose(gr[name], t.grad.numpy(), rtol=1e-10, atol=1e-10, err_msg=name)


# ------------------------------------------------------------------------------ SPOS
def _spos_cfg():
    # one stride-2 block (16 -> 32 channels) then one stride-1 block (32 channels)
    return dict(family="spos", n_blocks=2, n_choices=4, batch=1, image_hw=8, num_classes=10,
                stage_repeats=[2], stage_channels=[32], stem_channels=16, head_channels=8,
                choice_kernel=[3, 5, 7, 3], choice_xception=[0, 0, 0, 1], lr=0.001)


def _identity_params(cfg, b, c):
    """Every 1x1 weight = identity (rectangular: eye), every depthwise kernel = centred
    delta, BN gamma = 1, beta = 0."""
    p = {}
    for name, shape, kind, _ in spos.layout(cfg, b, c):
        if name.endswith("_g"):
            p[name] = np.ones(shape)
        elif name.endswith("_b"):
            p[name] = np.zeros(shape)
        elif len(shape) == 2:
            p[name] = np.eye(*shape)
        else:
            w = np.zeros(shape)
            w[:, shape[1] // 2, shape[2] // 2] = 1.0
            p[name] = w
    return p


# Per-channel pixel patterns over the 4 pixels of a 1x2x2 map: each has mean 0 and biased
# variance 1, so BN of it is r * pattern (r = 1/sqrt(1 + 1e-5)).
PAT = np.array([[1.0, -1, 1, -1], [-1.0, 1, 1, -1], [1.0, 1, -1, -1], [-1.0, -1, 1, 1]])


def _bn_relu_chain_value(n_bn_after_first_relu):
    """After BN -> ReLU of a ±1 pattern, the map is r·[pattern > 0] (values r or 0): mean r/2,
    biased variance r²/4.  Each further BN (delta / identity convs leave values alone) maps
    the two-level map {v, 0} (mean v/2, variance v²/4) to {+q, -q} with
    q = (v/2) / sqrt(v²/4 + eps); subsequent BNs of a ±q pattern give ±q/sqrt(q² + eps)."""
    v = R
    q = (v / 2) / math.sqrt(v * v / 4 + 1e-5)
    for _ in range(n_bn_after_first_relu - 1):
        q = q / math.sqrt(q * q + 1e-5)
    return q


def test_spos_stride1_shuffle_hand_worked():
    """Stride-1 Shuffle3 block, C = 32 (inp = mid = out_main = 16), B = 1, 2x2 pixels,
    identity pw weights and delta dw kernels.  Input channel 2j (even) = E_j (arbitrary,
    here 10 + j + pixel/10), channel 2j+1 (odd) = PAT[j % 4].
    Reading A27: x_proj = even channels (passed through), x_main = odd channels;
      main = pw1 -> BN -> ReLU -> dw -> BN -> pw2 -> BN -> ReLU;  y = concat(x_proj, main).
    pw1 = I: BN(PAT) = r PAT -> ReLU -> r [PAT > 0]; dw delta keeps it; BN -> q (2·[PAT>0] - 1)
    with q from _bn_relu_chain_value(1); pw2 = I; BN -> ±q' (q' = q / sqrt(q² + eps));
    ReLU -> q' [PAT > 0].  So y[..., :16] = even input channels, y[..., 16 + j] = q' [PAT_j > 0].
    A swapped split parity puts PAT into the pass-through half; a swapped concat puts the
    main branch first; dropping the final ReLU leaves -q' entries; moving the first ReLU
    after the dw BN changes the chain's value (q -> r-scaled levels)."""
    cfg = _spos_cfg()
    b, c = 1, 0
    p = _identity_params(cfg, b, c)
    x = np.zeros((1, 2, 2, 32))
    for j in range(16):
        x[0, :, :, 2 * j] = (10 + j + np.arange(4) / 10).reshape(2, 2)
        x[0, :, :, 2 * j + 1] = PAT[j % 4].reshape(2, 2)
    y, _ = spos.block_fwd(cfg, b, c, p, x)
    q2 = _bn_relu_chain_value(2)
    exp = np.zeros_like(y)
    exp[..., :16] = x[..., 0::2]
    for j in range(16):
        exp[0, :, :, 16 + j] = (q2 * (PAT[j % 4] > 0)).reshape(2, 2)
    np.testing.assert_allclose(y, exp, rtol=0, atol=1e-12)


def test_spos_stride2_shuffle_hand_worked():
    """Stride-2 Shuffle3 block, inp = 16 -> C_out = 32 (mid = 16, out_main = 16), B = 1,
    input 4x4 -> output 2x2.  Delta dw kernels with stride 2 sample pixels (2i, 2j); the input
    is built so the sampled 2x2 map of channel j is PAT[j % 4] and the other pixels are 0.
    Reading A27: y = concat(proj(x), main(x)),
      proj = dw s2 -> BN -> pw -> BN -> ReLU:  BN(PAT) = r PAT; pw = I; BN -> ±r/sqrt(r²+eps)·PAT
             = r2 PAT (r2 = r / sqrt(r² + eps)); ReLU -> r2 [PAT > 0];
      main = pw1 -> BN -> ReLU -> dw s2 -> BN -> pw2 -> BN -> ReLU  (pw1 on the full 4x4 map:
             the BN statistics then include the zero pixels: mean and variance over 16 pixels).
    The main branch is computed from its definition in stages below; the proj half is the
    closed form r2 [PAT > 0], so a swapped concat order fails."""
    cfg = _spos_cfg()
    b, c = 0, 0
    p = _identity_params(cfg, b, c)
    x = np.zeros((1, 4, 4, 16))
    for j in range(16):
        x[0, 0::2, 0::2, j] = PAT[j % 4].reshape(2, 2)
    y, _ = spos.block_fwd(cfg, b, c, p, x)
    r2 = R / math.sqrt(R * R + 1e-5)
    for j in range(16):
        np.testing.assert_allclose(y[0, :, :, j].ravel(), r2 * (PAT[j % 4] > 0), rtol=0, atol=1e-12)
    # main branch: 4x4 map m with 4 entries of PAT (2 at +1, 2 at -1) and 12 zeros: mean 0,
    # biased variance 4/16 = 1/4 -> BN multiplies by 1/sqrt(1/4 + eps) =: s1; ReLU keeps the
    # two +s1 entries; dw s2 samples exactly the 4 PAT pixels -> s1 [PAT > 0] (mean s1/2,
    # variance s1²/4) -> BN -> ±q; pw2 = I; BN -> ±q/sqrt(q²+eps); ReLU -> that [PAT > 0].
    s1 = 1.0 / math.sqrt(0.25 + 1e-5)
    q = (s1 / 2) / math.sqrt(s1 * s1 / 4 + 1e-5)
    q = q / math.sqrt(q * q + 1e-5)
    for j in range(16):
        np.testing.assert_allclose(y[0, :, :, 16 + j].ravel(), q * (PAT[j % 4] > 0), rtol=0, atol=1e-12)


def test_spos_stride1_xception_relu_placement():
    """Xception (choice 3) main branch: dw -> BN -> pw1 -> BN -> ReLU -> dw -> BN -> pw2 -> BN
    -> ReLU -> dw -> BN -> pw3 -> BN -> ReLU (A27).  With identity/delta weights and the ±1
    patterns: dw -> BN gives r PAT (no ReLU after a dw BN); pw1 -> BN -> r2 PAT -> ReLU ->
    r2 [PAT>0]; then (dw BN, pw BN) twice more around the second ReLU.  Levels: after the
    first ReLU the map is v [PAT > 0]; BN -> ±q(v); BN (pw2) -> ±q'; ReLU -> q' [PAT>0];
    dw BN -> ±q''; pw3 BN -> ±q'''; ReLU -> q''' [PAT > 0]."""
    cfg = _spos_cfg()
    b, c = 1, 3
    p = _identity_params(cfg, b, c)
    x = np.zeros((1, 2, 2, 32))
    for j in range(16):
        x[0, :, :, 2 * j + 1] = PAT[j % 4].reshape(2, 2)
    y, _ = spos.block_fwd(cfg, b, c, p, x)

    def bn_two_level(v):          # {v, 0} with equal counts -> ±(v/2)/sqrt(v²/4 + eps)
        return (v / 2) / math.sqrt(v * v / 4 + 1e-5)

    def bn_pm(q):                 # {+q, -q} -> ±q/sqrt(q² + eps)
        return q / math.sqrt(q * q + 1e-5)
    v = bn_pm(R)                  # dw BN: r PAT (= ±r) ; pw1 BN: ±r/sqrt(r²+eps)
    q = bn_pm(bn_two_level(v))    # ReLU -> {v,0}; dw2 BN -> ±q; pw2 BN -> ±q'
    q = bn_pm(bn_two_level(q))    # ReLU -> {q',0}; dw3 BN; pw3 BN
    for j in range(16):
        np.testing.assert_allclose(y[0, :, :, 16 + j].ravel(), q * (PAT[j % 4] > 0), rtol=0, atol=1e-12)


def _torch_unit(x, w, kind, s, g, bb, relu, dil=1):
    X = torch.tensor(x).permute(0, 3, 1, 2)
    W = torch.tensor(w)
    if kind == "dw":
        z = torch.nn.functional.conv2d(X, W[:, None], stride=s, padding=dil * (w.shape[1] // 2), dilation=dil,
                                       groups=w.shape[0])
    else:
        z = torch.nn.functional.conv2d(X, W[:, :, None, None])
    y = torch.nn.functional.batch_norm(z, None, None, torch.tensor(g), torch.tensor(bb), training=True, eps=1e-5)
    if relu:
        y = torch.relu(y)
    return y.permute(0, 2, 3, 1).numpy()


@pytest.mark.parametrize("kind,k,s,relu,dil", [("dw", 3, 1, False, 1), ("dw", 5, 2, False, 1), ("dw", 7, 1, False, 1),
                                               ("pw", 1, 1, True, 1), ("pw", 1, 1, False, 1), ("dw", 3, 1, False, 2),
                                               ("dw", 5, 2, False, 2), ("dw", 7, 1, False, 2)])
def test_spos_unit_matches_torch(kind, k, s, relu, dil):
    """conv (dilation dil: Table 5's Dil Conv, reading A36) -> training-mode BN (biased
    variance, eps 1e-5) [-> ReLU] against torch.nn.functional."""
    rng = np.random.default_rng(k * 7 + s + 31 * dil)
    C = 6
    x = rng.standard_normal((3, 9, 9, C))
    w = rng.standard_normal((C, k, k)) if kind == "dw" else rng.standard_normal((C + 2, C))
    co = w.shape[0]
    g, bb = 1 + 0.3 * rng.standard_normal(co), 0.3 * rng.standard_normal(co)
    p = {"u": w, "u_g": g, "u_b": bb}
    y, _ = spos._unit_fwd(p, "u", kind, s, relu, x, dil=dil)
    np.testing.assert_allclose(y, _torch_unit(x, w, kind, s, g, bb, relu, dil), rtol=1e-11, atol=1e-11)


@pytest.mark.parametrize("k,s,dil", [(3, 1, 2), (5, 2, 2), (7, 1, 2), (3, 2, 1)])
def test_spos_depthwise_backward_matches_torch_autograd(k, s, dil):
    """dw_bwd's input and weight gradients (dilated and not) against torch autograd of conv2d."""
    rng = np.random.default_rng(100 * k + 10 * s + dil)
    C = 5
    x = rng.standard_normal((2, 11, 11, C))
    w = rng.standard_normal((C, k, k))
    y = spos.dw_fwd(x, w, s, dil)
    dy = rng.standard_normal(y.shape)
    dx, dw = spos.dw_bwd(x, w, s, dy, dil)
    X = torch.tensor(x).permute(0, 3, 1, 2).requires_grad_()
    W = torch.tensor(w)[:, None].requires_grad_()
    Y = torch.nn.functional.conv2d(X, W, stride=s, padding=dil * (k // 2), dilation=dil, groups=C)
    np.testing.assert_allclose(Y.detach().permute(0, 2, 3, 1).numpy(), y, rtol=1e-11, atol=1e-11)
    Y.backward(torch.tensor(dy).permute(0, 3, 1, 2))
    np.testing.assert_allclose(X.grad.permute(0, 2, 3, 1).numpy(), dx, rtol=1e-11, atol=1e-11)
    np.testing.assert_allclose(W.grad[:, 0].numpy(), dw, rtol=1e-11, atol=1e-11)


def test_head_ce_zero_classifier_is_ln_classes():
    """FC weights 0 -> every logit 0 -> softmax uniform -> mean CE = ln(num_classes) exactly,
    and dL/dlogits = (1/C - onehot)/B, which the zero FC maps to a zero input gradient."""
    rng = np.random.default_rng(5)
    for C in (10, 1000):
        fz = {"head": {"w": rng.standard_normal((8, 6))}, "fc": {"w": np.zeros((C, 8))}}
        x = rng.standard_normal((4, 3, 3, 6))
        labels = rng.integers(0, C, size=4)
        loss, dx = spos.head_loss(fz, x, labels)
        assert abs(loss - math.log(C)) < 1e-13
        assert np.all(dx == 0)


def test_head_loss_matches_torch():
    """pw -> BN(1, 0) -> ReLU -> GAP -> FC -> mean CE and dL/dx against torch autograd."""
    rng = np.random.default_rng(6)
    wh, wf = rng.standard_normal((8, 6)), rng.standard_normal((10, 8))
    x = rng.standard_normal((4, 3, 3, 6))
    labels = rng.integers(0, 10, size=4)
    loss, dx = spos.head_loss({"head": {"w": wh}, "fc": {"w": wf}}, x, labels)
    X = torch.tensor(x, requires_grad=True)
    z = torch.nn.functional.conv2d(X.permute(0, 3, 1, 2), torch.tensor(wh)[:, :, None, None])
    yv = torch.relu(torch.nn.functional.batch_norm(z, None, None, training=True, eps=1e-5))
    logits = yv.mean(dim=(2, 3)) @ torch.tensor(wf).T
    lt = torch.nn.functional.cross_entropy(logits, torch.tensor(labels))
    lt.backward()
    assert abs(loss - lt.item()) < 1e-12
    np.testing.assert_allclose(dx, X.grad.numpy(), rtol=1e-10, atol=1e-12)


# ------------------------------------------------------------------------------ sampler
@pytest.mark.parametrize("n,b", [(4, 3), (16, 3), (8, 6)])
def test_sampler_conflict_rate(n, b):
    """SURVEY §8c "Sampler": consecutive uniformly sampled subnets share at least one of a
    stage's b blocks' candidates with probability 1 - (1 - 1/n)^b (n = 4, b = 3: 0.578)."""
    N = 20000
    ch = synth.sample_choices(N, b, n, seed=123)
    rate = float(np.mean(np.any(ch[1:] == ch[:-1], axis=1)))
    exp = 1 - (1 - 1 / n) ** b
    sigma = math.sqrt(exp * (1 - exp) / (N - 1))
    assert abs(rate - exp) < 5 * sigma, (rate, exp)
    # per-block marginals are uniform: chi-square well inside its 99.9 % quantile
    for j in range(b):
        cnt = np.bincount(ch[:, j], minlength=n)
        chi2 = float(np.sum((cnt - N / n) ** 2 / (N / n)))
        assert chi2 < 3 * n + 30, chi2
