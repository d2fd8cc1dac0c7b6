"""Transformer candidate (configs[2]/[3]: "choices over FFN width/heads, seq 128").

Reading SURVEY §8c A17 (the paper names "8 Head Attention" among its NLP ops, Table 5
P:L446, but gives no block internals): pre-LN, non-causal multi-head attention with bias,
FFN ``W2 GELU_tanh(W1 x + b1) + b2``, LayerNorm eps 1e-5 with biased variance, scale
1/sqrt(hd), no dropout, no final LN.

    a   = LN1(x)
    qkv = a Wqkv^T + bqkv            q, k, v = contiguous thirds; head j = columns [j hd,(j+1) hd)
    o_j = softmax(q_j k_j^T / sqrt(hd)) v_j
    x1  = x + concat_j(o_j) Wo^T + bo
    y   = x1 + GELU_tanh(LN2(x1) W1^T + b1) W2^T + b2

Packing: Wqkv, bqkv, Wo, bo, ln1.g, ln1.b, W1, b1, W2, b2, ln2.g, ln2.b.
"""
import numpy as np

EPS = 1e-5
GELU_C = np.sqrt(2.0 / np.pi)


def dims(cfg, c):
    return cfg["d_model"], cfg["choice_heads"][c], cfg["choice_ffn"][c]


def layout(cfg, c):
    d, h, f = dims(cfg, c)
    return [("Wqkv", (3 * d, d), "uniform", d), ("bqkv", (3 * d,), "uniform", d),
            ("Wo", (d, d), "uniform", d), ("bo", (d,), "uniform", d),
            ("ln1_g", (d,), "ones", 0), ("ln1_b", (d,), "zeros", 0),
            ("W1", (f, d), "uniform", d), ("b1", (f,), "uniform", d),
            ("W2", (d, f), "uniform", f), ("b2", (d,), "uniform", f),
            ("ln2_g", (d,), "ones", 0), ("ln2_b", (d,), "zeros", 0)]


# ---- LayerNorm: textbook definition and its gradient -----------------------------------
def ln_fwd(x, g, b):
    mu = x.mean(axis=-1, keepdims=True)
    var = ((x - mu) ** 2).mean(axis=-1, keepdims=True)      # biased variance
    rstd = 1.0 / np.sqrt(var + EPS)
    xhat = (x - mu) * rstd
    return g * xhat + b, (xhat, rstd)


def ln_bwd(dy, g, cache):
    xhat, rstd = cache
    dxhat = dy * g
    dx = rstd * (dxhat - dxhat.mean(axis=-1, keepdims=True)
                 - xhat * (dxhat * xhat).mean(axis=-1, keepdims=True))
    red = tuple(range(dy.ndim - 1))
    return dx, (dy * xhat).sum(axis=red), dy.sum(axis=red)


# ---- GELU (tanh form) -------------------------------------------------------------------
def gelu(z):
    return 0.5 * z * (1.0 + np.tanh(GELU_C * (z + 0.044715 * z ** 3)))


def gelu_grad(z):
    t = np.tanh(GELU_C * (z + 0.044715 * z ** 3))
    return 0.5 * (1.0 + t) + 0.5 * z * (1.0 - t * t) * GELU_C * (1.0 + 3 * 0.044715 * z * z)


# ---- attention ---------------------------------------------------------------------------
def _heads(t, h):
    B, S, d = t.shape
    return t.reshape(B, S, h, d // h).transpose(0, 2, 1, 3)       # [B,h,S,hd]


def _merge(t):
    B, h, S, hd = t.shape
    return t.transpose(0, 2, 1, 3).reshape(B, S, h * hd)


def attn_fwd(q, k, v, h):
    qh, kh, vh = _heads(q, h), _heads(k, h), _heads(v, h)
    scale = 1.0 / np.sqrt(qh.shape[-1])
    s = (qh @ kh.swapaxes(-1, -2)) * scale              # [B,h,S,S] = q k^T
    s = s - s.max(axis=-1, keepdims=True)
    p = np.exp(s)
    p = p / p.sum(axis=-1, keepdims=True)
    o = p @ vh
    return _merge(o), (qh, kh, vh, p, scale)


def attn_bwd(do, cache):
    qh, kh, vh, p, scale = cache
    h = qh.shape[1]
    doh = _heads(do, h)
    dv = p.swapaxes(-1, -2) @ doh
    dp = doh @ vh.swapaxes(-1, -2)
    ds = p * (dp - (dp * p).sum(axis=-1, keepdims=True))
    dq = (ds @ kh) * scale
    dk = (ds.swapaxes(-1, -2) @ qh) * scale
    return _merge(dq), _merge(dk), _merge(dv)


# ---- block -------------------------------------------------------------------------------
def forward(p, x, h):
    """x: [B,S,d] float64; h = number of heads of this candidate."""
    d = x.shape[-1]
    a, c1 = ln_fwd(x, p["ln1_g"], p["ln1_b"])
    qkv = a @ p["Wqkv"].T + p["bqkv"]
    q, k, v = qkv[..., :d], qkv[..., d:2 * d], qkv[..., 2 * d:]
    o, ca = attn_fwd(q, k, v, h)
    x1 = x + o @ p["Wo"].T + p["bo"]
    a2, c2 = ln_fwd(x1, p["ln2_g"], p["ln2_b"])
    z = a2 @ p["W1"].T + p["b1"]
    g = gelu(z)
    y = x1 + g @ p["W2"].T + p["b2"]
    return y, (a, c1, ca, o, a2, c2, z, g)


def backward(p, tape, dy):
    a, c1, ca, o, a2, c2, z, g = tape
    B, S, d = dy.shape
    f2 = lambda t: t.reshape(-1, t.shape[-1])                     # noqa: E731
    gr = {}
    # FFN half
    gr["W2"] = f2(dy).T @ f2(g)
    gr["b2"] = f2(dy).sum(axis=0)
    dz = (dy @ p["W2"]) * gelu_grad(z)
    gr["W1"] = f2(dz).T @ f2(a2)
    gr["b1"] = f2(dz).sum(axis=0)
    da2 = dz @ p["W1"]
    dx1_ln, gr["ln2_g"], gr["ln2_b"] = ln_bwd(da2, p["ln2_g"], c2)
    dx1 = dy + dx1_ln
    # attention half
    gr["Wo"] = f2(dx1).T @ f2(o)
    gr["bo"] = f2(dx1).sum(axis=0)
    do = dx1 @ p["Wo"]
    dq, dk, dv = attn_bwd(do, ca)
    dqkv = np.concatenate([dq, dk, dv], axis=-1)
    gr["Wqkv"] = f2(dqkv).T @ f2(a)
    gr["bqkv"] = f2(dqkv).sum(axis=0)
    da = dqkv @ p["Wqkv"]
    dx_ln, gr["ln1_g"], gr["ln1_b"] = ln_bwd(da, p["ln1_g"], c1)
    return dx1 + dx_ln, gr
