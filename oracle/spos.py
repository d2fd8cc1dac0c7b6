"""SPOS-style CNN supernet (configs[1]: "SPOS-style CNN supernet (20 layers x 4 choices,
synthetic 224x224 images, batch 64)").  TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The paper names the CV candidate ops (Table 5: Conv 3x3, Sep Conv 3x3/5x5, Dil
Conv 3x3) and cites SPOS [9] for the sampling; block internals follow SPOS's
ShuffleNetV2 search space — reading SURVEY §8c "C2 SPOS candidate" (A16/A17):

* NHWC tensors; every conv is bias-free and followed by BatchNorm in training mode (batch
  statistics over N*H*W, biased variance, eps 1e-5, trainable gamma/beta, no running stats).
* Stages: repeats [4,4,8,4], C_out [64,160,320,640]; the first block of a stage has stride 2,
  inp = C_prev, mid = C_out/2, out_main = C_out - inp; other blocks stride 1 with
  inp = mid = out_main = C_out/2.
* Stride 1: x_proj = even channels (passed through), x_main = odd channels;
  y = concat(x_proj, main(x_main)).
* Stride 2: y = concat(proj(x), main(x)), proj = dw k s2 -> BN -> pw inp->inp -> BN -> ReLU.
* Choices 0/1/2 (Shuffle k = 3/5/7): main = pw inp->mid -> BN -> ReLU -> dw k (stride s) -> BN
  -> pw mid->out_main -> BN -> ReLU.
* Choice 3 (Xception, k=3): main = dw3 (s) -> BN -> pw inp->mid -> BN -> ReLU -> dw3 -> BN ->
  pw mid->mid -> BN -> ReLU -> dw3 -> BN -> pw mid->out_main -> BN -> ReLU.
* Frozen stem: conv3x3 s2 pad 1 3->C0 -> BN(gamma=1, beta=0) -> ReLU.  Frozen head: pw ->
  BN(1, 0) -> ReLU -> global average pool -> FC (no bias) -> mean cross-entropy.  Frozen
  parts are never updated (reading A2); their weights use the counter hash with reserved uids.
* Packing of a candidate: the proj branch's convs (stride-2 blocks) then the main branch's, in
  order, each conv weight followed by its BN gamma, beta.  pw weights [out, in]; dw weights
  [C, k, k]; the stem weight [out, kh, kw, in].

Storage precision (reading A28).  Every function takes an optional ``st``, the
rounding applied where a tensor is stored (a ``Storage``): ``st.f`` for forward tensors
(conv outputs z, BN/ReLU outputs y), ``st.w`` for the 1x1-conv weight operand of the
forward, ``st.b`` for backward tensors (dz, dx, the head's dr), ``st.op`` for the operands
the backward contractions read (x in the weight gradients, W in the 1x1 input gradients).
``PLAIN`` (default) is the fp64 definition.  ``BF16`` rounds all of them to bfloat16;
``BF16X2`` is the CUDA path's storage (forward tensors and weights as hi + lo bfloat16
pairs, 16-bit mantissa; backward tensors and operands bfloat16).  These modes exist to
measure the numerical noise floor of a storage format: BatchNorm + ReLU make the result
chaotic under rounding (one flipped ReLU mask cascades), and with BF16 storage the weight
update of configs[1] decorrelates from the fp64 one (A15 2.7e-3 after one step, update
error > 100 %), which is why the path stores the forward in bf16x2.
"""
import numpy as np

EPS = 1e-5


def to_bf16(x):
    """Round to the nearest bfloat16 (ties to even), returned as float64.  fp64 -> fp32 is
    round-to-nearest first (the kernels hold fp32 values when they store bf16)."""
    a = np.ascontiguousarray(x, dtype=np.float32)
    u = a.view(np.uint32).astype(np.uint64)
    r = ((u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))) >> np.uint64(16)) << np.uint64(16)
    out = r.astype(np.uint32).view(np.float32).astype(np.float64)
    nan = np.isnan(a)
    if np.any(nan):
        out[nan] = np.nan
    return out


def _id(x):
    return x


def to_bf16x2(x):
    """hi + lo with hi = bf16(x), lo = bf16(x - hi) (from the fp32 value)."""
    a = np.asarray(x, dtype=np.float32).astype(np.float64)
    hi = to_bf16(a)
    return hi + to_bf16(a - hi)


class Storage:
    def __init__(self, f=_id, w=_id, b=_id, op=_id):
        self.f, self.w, self.b, self.op = f, w, b, op


def to_fp32(x):
    """Round to float32 (nearest), returned as float64: the paper's precision."""
    return np.asarray(x, dtype=np.float32).astype(np.float64)


PLAIN = Storage()
BF16 = Storage(to_bf16, to_bf16, to_bf16, to_bf16)
BF16X2 = Storage(to_bf16x2, to_bf16x2, to_bf16, to_bf16)
FP32 = Storage(to_fp32, to_fp32, to_fp32, to_fp32)   # every stored tensor in fp32 (the paper's)
STORAGE = {None: PLAIN, "fp64": PLAIN, "bf16": BF16, "bf16x2": BF16X2, "fp32": FP32}


# ------------------------------------------------------------------ shapes / layout
def block_dims(cfg, b):
    """(stride, inp, mid, out_main, C_out, H_in) of block b."""
    reps, chans = cfg["stage_repeats"], cfg["stage_channels"]
    c_prev, H = cfg["stem_channels"], cfg["image_hw"] // 2
    k = 0
    for st, (r, co) in enumerate(zip(reps, chans)):
        for i in range(r):
            if k == b:
                if i == 0:
                    return 2, c_prev, co // 2, co - c_prev, co, H
                return 1, co // 2, co // 2, co // 2, co, H
            if i == 0:
                H //= 2
            k += 1
        c_prev = co
    raise IndexError(b)


def dilation(cfg, c):
    """Dilation of candidate c's depthwise convs (Table 5's "Dil Conv 3x3"; reading
    A36): cfg["choice_dilation"][c], default 1."""
    return int(cfg.get("choice_dilation", [1] * cfg["n_choices"])[c])


def convs(cfg, b, c):
    """Ordered conv list of candidate (b, c): (name, kind 'pw'|'dw'|'cv', cin, cout, k, stride).
    Every depthwise conv of the candidate uses its kernel size k = choice_kernel[c] (the
    Xception choice of the default configs has k = 3) and its dilation (dilation()).
    choice_xception[c] == 2 is Table 5's dense "Conv 3x3" (reading A40): the Shuffle
    block with its depthwise k x k conv replaced by a DENSE k x k conv over the mid channels
    ('cv': mid -> mid, stride s, pad k // 2, no bias, BN, no ReLU, dilation 1); the stride-2
    proj branch stays depthwise."""
    s, inp, mid, out, _, _ = block_dims(cfg, b)
    k = cfg["choice_kernel"][c]
    L = []
    if s == 2:
        L += [("p_dw", "dw", inp, inp, k, 2), ("p_pw", "pw", inp, inp, 1, 1)]
    if cfg["choice_xception"][c] == 2:
        L += [("m_pw1", "pw", inp, mid, 1, 1), ("m_cv", "cv", mid, mid, k, s), ("m_pw2", "pw", mid, out, 1, 1)]
    elif not cfg["choice_xception"][c]:
        L += [("m_pw1", "pw", inp, mid, 1, 1), ("m_dw", "dw", mid, mid, k, s), ("m_pw2", "pw", mid, out, 1, 1)]
    else:
        L += [("x_dw1", "dw", inp, inp, k, s), ("x_pw1", "pw", inp, mid, 1, 1), ("x_dw2", "dw", mid, mid, k, 1),
              ("x_pw2", "pw", mid, mid, 1, 1), ("x_dw3", "dw", mid, mid, k, 1), ("x_pw3", "pw", mid, out, 1, 1)]
    return L


def layout(cfg, b, c):
    out = []
    for name, kind, cin, cout, k, _ in convs(cfg, b, c):
        if kind == "pw":
            out.append((name, (cout, cin), "uniform", cin))
        elif kind == "cv":
            out.append((name, (cout, k, k, cin), "uniform", k * k * cin))
        else:
            out.append((name, (cout, k, k), "uniform", k * k))
        out.append((name + "_g", (cout,), "ones", 0))
        out.append((name + "_b", (cout,), "zeros", 0))
    return out


def frozen_layout(cfg):
    C0, Ch = cfg["stem_channels"], cfg["head_channels"]
    Clast = cfg["stage_channels"][-1]
    return {"stem": [("w", (C0, 3, 3, 3), "uniform", 27)],
            "head": [("w", (Ch, Clast), "uniform", Clast)],
            "fc": [("w", (cfg["num_classes"], Ch), "uniform", Ch)]}


# ------------------------------------------------------------------ primitive ops
def pad_hw(x, p):
    return np.pad(x, ((0, 0), (p, p), (p, p), (0, 0)))


def dw_fwd(x, w, s, dil=1):
    """Depthwise conv, pad dil*(k//2): y[b,i,j,c] = sum_{u,v} xpad[b, i*s+u*dil, j*s+v*dil, c] w[c,u,v]."""
    k = w.shape[1]
    p = dil * (k // 2)
    xp = pad_hw(x, p)
    B, H, W, C = x.shape
    Ho, Wo = (H + 2 * p - dil * (k - 1) - 1) // s + 1, (W + 2 * p - dil * (k - 1) - 1) // s + 1
    y = np.zeros((B, Ho, Wo, C))
    for u in range(k):
        for v in range(k):
            y += xp[:, u * dil:u * dil + s * (Ho - 1) + 1:s, v * dil:v * dil + s * (Wo - 1) + 1:s, :] * w[:, u, v]
    return y


def dw_bwd(x, w, s, dy, dil=1):
    k = w.shape[1]
    p = dil * (k // 2)
    xp = pad_hw(x, p)
    B, Ho, Wo, C = dy.shape
    dxp = np.zeros_like(xp)
    dw = np.zeros_like(w)
    for u in range(k):
        for v in range(k):
            sl = (slice(None), slice(u * dil, u * dil + s * (Ho - 1) + 1, s),
                  slice(v * dil, v * dil + s * (Wo - 1) + 1, s), slice(None))
            dxp[sl] += dy * w[:, u, v]
            dw[:, u, v] = np.sum(dy * xp[sl], axis=(0, 1, 2))
    return dxp[:, p:p + x.shape[1], p:p + x.shape[2], :], dw


def conv_fwd(x, w, s):
    """Dense conv (stem): w [Cout, k, k, Cin], pad k//2."""
    k = w.shape[1]
    p = k // 2
    xp = pad_hw(x, p)
    B, H, W, _ = x.shape
    Ho, Wo = (H + 2 * p - k) // s + 1, (W + 2 * p - k) // s + 1
    y = np.zeros((B, Ho, Wo, w.shape[0]))
    for u in range(k):
        for v in range(k):
            y += xp[:, u:u + s * (Ho - 1) + 1:s, v:v + s * (Wo - 1) + 1:s, :] @ w[:, u, v, :].T
    return y


def conv_bwd(x, w, s, dy):
    """Gradients of conv_fwd (pad k // 2, stride s): dx = sum over taps of the transposed
    correlation of dy with w, dw[o, u, v, i] = sum over (b, oh, ow) of dy[.., o] xpad[.., i]."""
    k = w.shape[1]
    p = k // 2
    xp = pad_hw(x, p)
    B, Ho, Wo, _ = dy.shape
    dxp = np.zeros_like(xp)
    dw = np.zeros_like(w)
    for u in range(k):
        for v in range(k):
            sl = (slice(None), slice(u, u + s * (Ho - 1) + 1, s), slice(v, v + s * (Wo - 1) + 1, s), slice(None))
            dxp[sl] += dy @ w[:, u, v, :]
            dw[:, u, v, :] = np.einsum("bhwo,bhwi->oi", dy, xp[sl])
    return dxp[:, p:p + x.shape[1], p:p + x.shape[2], :], dw


def bn_fwd(x, g, b):
    mu = x.mean(axis=(0, 1, 2))
    var = ((x - mu) ** 2).mean(axis=(0, 1, 2))
    rstd = 1.0 / np.sqrt(var + EPS)
    xh = (x - mu) * rstd
    return g * xh + b, (xh, rstd)


def bn_bwd(dy, g, cache):
    xh, rstd = cache
    dxh = dy * g
    dx = rstd * (dxh - dxh.mean(axis=(0, 1, 2)) - xh * (dxh * xh).mean(axis=(0, 1, 2)))
    return dx, (dy * xh).sum(axis=(0, 1, 2)), dy.sum(axis=(0, 1, 2))


# ------------------------------------------------------------------ conv -> BN [-> ReLU] unit
def _unit_fwd(p, name, kind, s, relu, x, st=PLAIN, dil=1):
    w = p[name]
    if kind == "dw":
        z = dw_fwd(x, w, s, dil)
    elif kind == "cv":
        z = conv_fwd(x, st.w(w), s)
    else:
        z = x @ st.w(w).T
    z = st.f(z)
    y, cb = bn_fwd(z, p[name + "_g"], p[name + "_b"])
    if relu:
        y = np.maximum(y, 0.0)
    y = st.f(y)
    return y, (x, cb, y if relu else None)


def _unit_bwd(p, name, kind, s, dy, tape, grads, st=PLAIN, add=None, dil=1):
    """dx of the unit (+ add, the other branch's gradient of the same input, before the
    storage rounding), accumulating the parameter gradients into grads."""
    x, cb, yr = tape
    if yr is not None:
        dy = dy * (yr > 0)
    dz, grads[name + "_g"], grads[name + "_b"] = bn_bwd(dy, p[name + "_g"], cb)
    dz = st.b(dz)
    if kind == "dw":
        dx, _ = dw_bwd(x, p[name], s, dz, dil)
        _, grads[name] = dw_bwd(st.op(x), p[name], s, dz, dil)
    elif kind == "cv":
        dx, _ = conv_bwd(x, st.op(p[name]), s, dz)
        _, grads[name] = conv_bwd(st.op(x), p[name], s, dz)
    else:
        grads[name] = np.einsum("bhwo,bhwi->oi", dz, st.op(x))
        dx = dz @ st.op(p[name])
    return st.b(dx if add is None else dx + add)


def _chain(cfg, b, c, which):
    """Units of the proj ('p') or main branch: (name, kind, stride, relu, dilation)."""
    out = []
    d = dilation(cfg, c)
    cl = [u for u in convs(cfg, b, c) if u[0].startswith(which)]
    for i, (name, kind, _, _, _, s) in enumerate(cl):
        relu = kind == "pw" and (which == "p" or i == len(cl) - 1 or name in ("m_pw1", "x_pw1", "x_pw2"))
        out.append((name, kind, s, relu, d if kind == "dw" else 1))
    return out


def block_fwd(cfg, b, c, p, x, st=PLAIN):
    s = block_dims(cfg, b)[0]
    main_key = "x" if cfg["choice_xception"][c] == 1 else "m"
    if s == 1:
        xp, xm = x[..., 0::2], x[..., 1::2]
    else:
        xp = xm = x
    tapes = {"p": [], main_key: []}
    h = xm
    for name, kind, stride, relu, dil in _chain(cfg, b, c, main_key):
        h, t = _unit_fwd(p, name, kind, stride, relu, h, st, dil)
        tapes[main_key].append(t)
    main = h
    if s == 2:
        h = xp
        for name, kind, stride, relu, dil in _chain(cfg, b, c, "p"):
            h, t = _unit_fwd(p, name, kind, stride, relu, h, st, dil)
            tapes["p"].append(t)
        xp = h
    return np.concatenate([xp, main], axis=-1), tapes


def block_bwd(cfg, b, c, p, tapes, dy, st=PLAIN):
    s, inp = block_dims(cfg, b)[:2]
    main_key = "x" if cfg["choice_xception"][c] == 1 else "m"
    cp = inp if s == 2 else dy.shape[-1] // 2
    d_proj, d_main = dy[..., :cp], dy[..., cp:]
    grads = {}
    h = d_main
    chain = _chain(cfg, b, c, main_key)
    for (name, kind, stride, relu, dil), t in zip(reversed(chain), reversed(tapes[main_key])):
        h = _unit_bwd(p, name, kind, stride, h, t, grads, st, dil=dil)
    if s == 1:
        dx = np.zeros(d_proj.shape[:-1] + (2 * cp,))
        dx[..., 0::2] = d_proj
        dx[..., 1::2] = h
        return dx, grads
    g = d_proj
    pchain = list(zip(reversed(_chain(cfg, b, c, "p")), reversed(tapes["p"])))
    for i, ((name, kind, stride, relu, dil), t) in enumerate(pchain):
        last = i == len(pchain) - 1     # the proj branch's first unit: add the main branch's dx
        g = _unit_bwd(p, name, kind, stride, g, t, grads, st, add=h if last else None, dil=dil)
    return g, grads


# ------------------------------------------------------------------ frozen stem / head
def stem_fwd(fz, x, st=PLAIN):
    z = st.f(conv_fwd(x, fz["stem"]["w"], 2))
    C = z.shape[-1]
    y, _ = bn_fwd(z, np.ones(C), np.zeros(C))
    return st.f(np.maximum(y, 0.0))


def head_loss(fz, x, labels, st=PLAIN):
    """Returns (loss, dL/dx) through pw -> BN -> ReLU -> GAP -> FC -> mean CE (frozen)."""
    wh, wf = fz["head"]["w"], fz["fc"]["w"]
    z = st.f(x @ st.w(wh).T)
    C = z.shape[-1]
    y, cb = bn_fwd(z, np.ones(C), np.zeros(C))
    r = st.f(np.maximum(y, 0.0))
    gap = r.mean(axis=(1, 2))
    logits = gap @ wf.T
    mx = logits.max(axis=1, keepdims=True)
    lse = mx[:, 0] + np.log(np.exp(logits - mx).sum(axis=1))
    B = x.shape[0]
    loss = float(np.mean(lse - logits[np.arange(B), labels]))
    prob = np.exp(logits - lse[:, None])
    dlog = prob
    dlog[np.arange(B), labels] -= 1.0
    dlog /= B
    dgap = dlog @ wf
    dr = st.b(np.broadcast_to(dgap[:, None, None, :] / (r.shape[1] * r.shape[2]), r.shape))
    dy = dr * (r > 0)
    dz, _, _ = bn_bwd(dy, np.ones(C), cb)
    return loss, st.b(st.b(dz) @ st.op(wh))
