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

NLP op families (§8f(4); Table 5 P:L443-446 "Conv 3x1, Sep Conv 7x1, Light Conv 5x1, 8 Head
Attention", the Evolved-Transformer space of P:L579; reading A38 — the paper gives no layer
internals): candidate c's token mixer M is cfg["choice_op"][c] (default "attn"), the rest of
the block is unchanged:

    x1 = x + M(LN1(x));   y = x1 + FFN(LN2(x1))
    attn       M(a) = MHA(a) as above (heads = choice_heads[c])
    conv3      M(a) = Conv1d_{k=3}(a) + bc: dense d -> d convolution along the sequence,
               zero "same" padding inside each sequence: M[t] = sum_u Wc_u a[t+u-1] + bc,
               Wc packed [d, 3d] with column u*d + i = tap u, input channel i
    sepconv7   M(a) = DW_{k=7}(a) Wp^T + bp: depthwise conv along the sequence (taps Wd [d, 7],
               no bias, pad 3) then pointwise d -> d
    lightconv5 M(a) = LightConv_{k=5,H}(a Wi^T + bi) Wo^T + bo: Wu et al.'s lightweight conv
               (a depthwise conv whose taps are softmax-normalised over the kernel and shared
               by the d/H channels of each of H = choice_heads[c] heads: channel i uses row
               i // (d/H) of Wl [H, 5]), between input and output projections (no GLU)
"""
import numpy as np

EPS = 1e-5
GELU_C = np.sqrt(2.0 / np.pi)


OPS = ("attn", "conv3", "sepconv7", "lightconv5")


def dims(cfg, c):
    return cfg["d_model"], cfg["choice_heads"][c], cfg["choice_ffn"][c]


def op_of(cfg, c):
    return OPS[int(cfg.get("choice_op", [0] * cfg["n_choices"])[c])]


def mixer_layout(op, d, h):
    if op == "attn":
        return [("Wqkv", (3 * d, d), "uniform", d), ("bqkv", (3 * d,), "uniform", d),
                ("Wo", (d, d), "uniform", d), ("bo", (d,), "uniform", d)]
    if op == "conv3":
        return [("Wc", (d, 3 * d), "uniform", 3 * d), ("bc", (d,), "uniform", 3 * d)]
    if op == "sepconv7":
        return [("Wd", (d, 7), "uniform", 7), ("Wp", (d, d), "uniform", d), ("bp", (d,), "uniform", d)]
    if op == "lightconv5":
        return [("Wi", (d, d), "uniform", d), ("bi", (d,), "uniform", d), ("Wl", (h, 5), "uniform", 5),
                ("Wo", (d, d), "uniform", d), ("bo", (d,), "uniform", d)]
    raise ValueError(op)


def layout(cfg, c):
    d, h, f = dims(cfg, c)
    return mixer_layout(op_of(cfg, c), d, h) + [
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


# ---- sequence convolutions (reading A38) ----------------------------------------------------
def seq_dwconv(x, w):
    """Depthwise conv along the sequence: y[b,t,i] = sum_u w[i,u] x[b, t+u-P, i], P = k//2, zero
    outside [0, S) of each sequence.  x [B,S,d], w [d,k]."""
    B, S, d = x.shape
    k = w.shape[1]
    P = k // 2
    xp = np.zeros((B, S + 2 * P, d))
    xp[:, P:P + S] = x
    y = np.zeros_like(x)
    for u in range(k):
        y += xp[:, u:u + S] * w[:, u]
    return y


def seq_dwconv_bwd(x, w, dy):
    """Gradients of seq_dwconv: (dx, dw)."""
    B, S, d = x.shape
    k = w.shape[1]
    P = k // 2
    xp = np.zeros((B, S + 2 * P, d))
    xp[:, P:P + S] = x
    dxp = np.zeros_like(xp)
    dw = np.zeros_like(w)
    for u in range(k):
        dxp[:, u:u + S] += dy * w[:, u]
        dw[:, u] = np.sum(dy * xp[:, u:u + S], axis=(0, 1))
    return dxp[:, P:P + S], dw


def light_taps(Wl, d):
    """Per-channel taps of LightConv: softmax over the kernel of row i // (d/H) of Wl [H,k]."""
    H = Wl.shape[0]
    e = np.exp(Wl - Wl.max(axis=1, keepdims=True))
    p = e / e.sum(axis=1, keepdims=True)
    return np.repeat(p, d // H, axis=0), p


def light_taps_bwd(p, dtaps):
    """dWl from the per-channel tap gradients dtaps [d,k] (softmax Jacobian, summed per head)."""
    H, k = p.shape
    g = dtaps.reshape(H, -1, k).sum(axis=1)                      # [H,k]: sum over the head's channels
    return p * (g - (g * p).sum(axis=1, keepdims=True))


def conv3_cols(a):
    """im2col of Conv 3x1: cols[b,t, u*d + i] = a[b, t+u-1, i] (zero outside the sequence)."""
    B, S, d = a.shape
    ap = np.zeros((B, S + 2, d))
    ap[:, 1:S + 1] = a
    return np.concatenate([ap[:, u:u + S] for u in range(3)], axis=-1)


def conv3_cols_bwd(dcols):
    B, S, d3 = dcols.shape
    d = d3 // 3
    dap = np.zeros((B, S + 2, d))
    for u in range(3):
        dap[:, u:u + S] += dcols[..., u * d:(u + 1) * d]
    return dap[:, 1:S + 1]


def mixer_fwd(op, p, a, h):
    if op == "attn":
        d = a.shape[-1]
        qkv = a @ p["Wqkv"].T + p["bqkv"]
        q, k, v = qkv[..., :d], qkv[..., d:2 * d], qkv[..., 2 * d:]
        o, ca = attn_fwd(q, k, v, h)
        return o @ p["Wo"].T + p["bo"], (ca, o)
    if op == "conv3":
        cols = conv3_cols(a)
        return cols @ p["Wc"].T + p["bc"], (cols,)
    if op == "sepconv7":
        s = seq_dwconv(a, p["Wd"])
        return s @ p["Wp"].T + p["bp"], (s,)
    if op == "lightconv5":
        v = a @ p["Wi"].T + p["bi"]
        taps, pr = light_taps(p["Wl"], a.shape[-1])
        l_ = seq_dwconv(v, taps)
        return l_ @ p["Wo"].T + p["bo"], (v, taps, pr, l_)
    raise ValueError(op)


def mixer_bwd(op, p, a, mt, dm, gr):
    """dm = gradient of the mixer output; fills gr with the mixer's parameter gradients and
    returns the gradient of its input a."""
    f2 = lambda t: t.reshape(-1, t.shape[-1])                     # noqa: E731
    if op == "attn":
        ca, o = mt
        gr["Wo"] = f2(dm).T @ f2(o)
        gr["bo"] = f2(dm).sum(axis=0)
        dq, dk, dv = attn_bwd(dm @ p["Wo"], ca)
        dqkv = np.concatenate([dq, dk, dv], axis=-1)
        gr["Wqkv"] = f2(dqkv).T @ f2(a)
        gr["bqkv"] = f2(dqkv).sum(axis=0)
        return dqkv @ p["Wqkv"]
    if op == "conv3":
        (cols,) = mt
        gr["Wc"] = f2(dm).T @ f2(cols)
        gr["bc"] = f2(dm).sum(axis=0)
        return conv3_cols_bwd(dm @ p["Wc"])
    if op == "sepconv7":
        (s,) = mt
        gr["Wp"] = f2(dm).T @ f2(s)
        gr["bp"] = f2(dm).sum(axis=0)
        da, gr["Wd"] = seq_dwconv_bwd(a, p["Wd"], dm @ p["Wp"])
        return da
    if op == "lightconv5":
        v, taps, pr, l_ = mt
        gr["Wo"] = f2(dm).T @ f2(l_)
        gr["bo"] = f2(dm).sum(axis=0)
        dv, dtaps = seq_dwconv_bwd(v, taps, dm @ p["Wo"])
        gr["Wl"] = light_taps_bwd(pr, dtaps)
        gr["Wi"] = f2(dv).T @ f2(a)
        gr["bi"] = f2(dv).sum(axis=0)
        return dv @ p["Wi"]
    raise ValueError(op)


# ---- block -------------------------------------------------------------------------------
def forward(p, x, h, op="attn"):
    """x: [B,S,d] float64; h = number of heads of this candidate; op = its token mixer (A38)."""
    a, c1 = ln_fwd(x, p["ln1_g"], p["ln1_b"])
    m, mt = mixer_fwd(op, p, a, h)
    x1 = x + m
    a2, c2 = ln_fwd(x1, p["ln2_g"], p["ln2_b"])
    z = a2 @ p["W1"].T + p["b1"]
    g = gelu(z)
    y = x1 + g @ p["W2"].T + p["b2"]
    return y, (op, a, c1, mt, a2, c2, z, g)


def backward(p, tape, dy):
    op, a, c1, mt, a2, c2, z, g = tape
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
    # mixer half
    da = mixer_bwd(op, p, a, mt, dx1, gr)
    dx_ln, gr["ln1_g"], gr["ln1_b"] = ln_bwd(da, p["ln1_g"], c1)
    return dx1 + dx_ln, gr
