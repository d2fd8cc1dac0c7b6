"""SPOS CNN kernel unit tests on the GPU (SURVEY §4 tier T2) through include/naspipe_debug.h.

Reference: float64 NumPy written here from the textbook definitions (depthwise conv with
zero padding k//2, training-mode BatchNorm, its backward, the channel split of a stride-1
ShuffleNetV2 block), evaluated on the SAME rounded inputs the kernel reads.  Forward
tensors are bf16x2 (hi + lo planes, A28), gradients bf16.  Bars: bf16 outputs
within 2^-8 normwise and >= 99 % of elements within 1 bf16 ulp of the rounded reference;
bf16x2 and fp32 outputs (statistics, weight-gradient sums) normwise <= 1e-5; exact copies
(split / merge) bitwise; every kernel bitwise reproducible across two runs.
Shapes include the full configs[1] block-0 geometry (P = 200704 pixels) and ragged BN row
blocks (P not a multiple of 256).
"""
import ctypes as C

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")
L = npipe.lib
_vp, _i = C.c_void_p, C.c_int
L.naspipe_debug_dw.argtypes = [_vp] * 7 + [_i] * 6 + [_vp]
L.naspipe_debug_bn_fwd.argtypes = [_vp, _i, _i, _vp, _vp, _i, _vp, _i, C.c_size_t, _vp, _vp, _vp]
L.naspipe_debug_bn_bwd.argtypes = [_vp, _i, _vp, _i, _i, _vp, _vp, _vp, _vp, _i, _vp, _vp, _vp, C.c_float, _i, _vp]
L.naspipe_debug_chan_split.argtypes = [_vp, _i, _i, _vp, _i, C.c_size_t, _vp, _vp]
L.naspipe_debug_gemm_x2.argtypes = [_i, _i, _i, _vp, _vp, _i, _vp, _vp, _i, _vp, _vp, _vp]
L.naspipe_debug_chan_merge.argtypes = [_vp, _i, _vp, _i, _i, _vp, _vp]
L.naspipe_debug_stem.argtypes = [_vp, _vp, _vp, _i, _i, _i, _vp]
L.naspipe_debug_dw_bn_fold.argtypes = [_vp, _i, _i, _i, _vp, _vp, _i, _vp, _i, _i, _i] + [_vp] * 9
L.naspipe_debug_dense_cols.argtypes = [_vp] * 5 + [_i] * 5 + [_vp]
L.naspipe_debug_bnb_fused.argtypes = [_i, _vp, _vp, _vp, _vp] + [_i] * 6 + [_vp] * 5 + [_i, _vp, _vp]


def _ok(rc):
    assert rc == 0, L.naspipe_last_error().decode()


def _p(t):
    return None if t is None else t.data_ptr()


def _f64(t):
    return t.detach().to(torch.float64).cpu().numpy()


def _bf(a):
    """bf16 device tensor of a (RNE) and its exact float64 value."""
    t = torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(torch.bfloat16).cuda()
    return t, _f64(t)


def _x2(a):
    """bf16x2 device tensor [2, *shape] (hi plane, lo plane) of a and its exact value."""
    a = np.asarray(a, dtype=np.float32)
    hi = torch.from_numpy(a).to(torch.bfloat16)
    lo = (torch.from_numpy(a) - hi.float()).to(torch.bfloat16)
    t = torch.stack([hi, lo]).cuda()
    return t, _f64(t[0]) + _f64(t[1])


def _v2(t):
    """value of a bf16x2 tensor [2, ...]"""
    return _f64(t[0]) + _f64(t[1])


def _check_x2(got, ref, tol=1e-5):
    assert np.max(np.abs(got - ref)) / max(np.max(np.abs(ref)), 1e-30) <= tol


def _check_bf16(got, ref):
    scale = max(np.max(np.abs(ref)), 1e-30)
    assert np.max(np.abs(got - ref)) / scale <= 2.0 ** -8
    r16 = _f64(torch.from_numpy(ref.astype(np.float32)).to(torch.bfloat16))
    ulp = np.maximum(np.abs(r16), 1e-30) * 2.0 ** -7
    assert np.mean(np.abs(got - r16) <= ulp + 1e-30) >= 0.99


def _dw_ref(x, w, s, d=1):
    B, H, _, Cc = x.shape
    k = w.shape[1]
    p = d * (k // 2)
    Ho = (H + 2 * p - d * (k - 1) - 1) // s + 1
    xp = np.pad(x, ((0, 0), (p, p), (p, p), (0, 0)))
    y = np.zeros((B, Ho, Ho, Cc))
    for u in range(k):
        for v in range(k):
            y += xp[:, u * d:u * d + s * (Ho - 1) + 1:s, v * d:v * d + s * (Ho - 1) + 1:s, :] * w[:, u, v]
    return y


def _dw_bwd_ref(x, w, s, dz, d=1):
    k = w.shape[1]
    p = d * (k // 2)
    B, Ho, _, Cc = dz.shape
    xp = np.pad(x, ((0, 0), (p, p), (p, p), (0, 0)))
    dxp = np.zeros_like(xp)
    dw = np.zeros_like(w)
    for u in range(k):
        for v in range(k):
            sl = (slice(None), slice(u * d, u * d + s * (Ho - 1) + 1, s), slice(v * d, v * d + s * (Ho - 1) + 1, s),
                  slice(None))
            dxp[sl] += dz * w[:, u, v]
            dw[:, u, v] = np.sum(dz * xp[sl], axis=(0, 1, 2))
    H = x.shape[1]
    return dxp[:, p:p + H, p:p + H, :], dw


@pytest.mark.parametrize("B,H,Cc,k,s,d", [(2, 9, 16, 3, 1, 1), (3, 8, 48, 5, 2, 1), (2, 14, 32, 7, 1, 1),
                                          (1, 7, 640, 3, 1, 1), (4, 6, 320, 7, 2, 1), (64, 112, 16, 3, 2, 1),
                                          (2, 9, 16, 3, 1, 2), (3, 8, 48, 5, 2, 2), (2, 14, 32, 7, 1, 2),
                                          (4, 6, 320, 7, 2, 2), (2, 37, 24, 5, 1, 2), (2, 40, 64, 3, 2, 2),
                                          # the CV.c3 analog's full-size dilated shapes (synth cv_c3)
                                          (64, 112, 16, 5, 2, 2), (64, 112, 16, 7, 2, 2), (64, 56, 32, 7, 1, 2),
                                          (64, 28, 80, 5, 1, 2), (64, 14, 160, 3, 1, 2), (64, 7, 320, 7, 1, 2)])
def test_depthwise_fwd_dgrad_wgrad(B, H, Cc, k, s, d):
    """Depthwise conv kernels (dilation d: Table 5's Dil Conv, reading A36) vs explicit tap loops."""
    rng = np.random.default_rng(B * 100 + H + Cc + k + 7 * d)
    xd, x = _x2(rng.standard_normal((B, H, H, Cc)))
    x_hi = _f64(xd[0])
    w = (rng.standard_normal((Cc, k, k)) / k).astype(np.float32)
    wd = torch.from_numpy(w).cuda()
    Ho = (H - 1) // s + 1
    dzd, dz = _bf(rng.standard_normal((B, Ho, Ho, Cc)))
    addd, add = _bf(rng.standard_normal((B, H, H, Cc)))
    z = torch.empty((2, B, Ho, Ho, Cc), dtype=torch.bfloat16, device="cuda")
    dx = torch.empty((B, H, H, Cc), dtype=torch.bfloat16, device="cuda")
    dws = torch.empty((Cc, k, k), dtype=torch.float32, device="cuda")
    outs = []
    for _ in range(2):
        _ok(L.naspipe_debug_dw(_p(xd), _p(wd), _p(z), _p(dzd), _p(addd), _p(dx), _p(dws), B, H, Cc, k, s, d, None))
        torch.cuda.synchronize()
        outs.append((z.clone(), dx.clone(), dws.clone()))
    for a, b in zip(outs[0], outs[1]):
        assert torch.equal(a, b)
    if B * H * H > 100000:   # full-size block 0: check the reductions on a sample of channels
        ch = [0, 7, 15, Cc - 1]
        x, x_hi, dz, add, w64 = x[..., ch], x_hi[..., ch], dz[..., ch], add[..., ch], w[ch].astype(np.float64)
        got_z, got_dx, got_dw = _v2(z)[..., ch], _f64(dx)[..., ch], _f64(dws)[ch]
    else:
        w64 = w.astype(np.float64)
        got_z, got_dx, got_dw = _v2(z), _f64(dx), _f64(dws)
    _check_x2(got_z, _dw_ref(x, w64, s, d))
    rdx, _ = _dw_bwd_ref(x, w64, s, dz, d)
    _, rdw = _dw_bwd_ref(x_hi, w64, s, dz, d)     # the weight gradient reads the hi plane
    _check_bf16(got_dx, rdx + add)
    assert np.max(np.abs(got_dw - rdw)) / np.max(np.abs(rdw)) <= 1e-5


def _bn_ref(z, g, b, relu):
    mu = z.mean(axis=0)
    var = ((z - mu) ** 2).mean(axis=0)
    rstd = 1.0 / np.sqrt(var + 1e-5)
    xh = (z - mu) * rstd
    y = g * xh + b
    return (np.maximum(y, 0) if relu else y), mu, rstd, xh


@pytest.mark.parametrize("P,Cc,relu", [(16, 64, 1), (4096, 16, 0), (1000, 48, 1), (3136, 1024, 1), (50176, 160, 1),
                                       (200704, 32, 0)])
def test_batchnorm_fwd_bwd(P, Cc, relu):
    rng = np.random.default_rng(P + Cc)
    zd, z = _x2(rng.standard_normal((P, Cc)) * rng.uniform(0.5, 2.0, Cc) + rng.uniform(-1, 1, Cc))
    g = rng.uniform(0.5, 1.5, Cc).astype(np.float32)
    b = rng.uniform(-0.3, 0.3, Cc).astype(np.float32)
    gd, bd = torch.from_numpy(g).cuda(), torch.from_numpy(b).cuda()
    ld = Cc + 16   # the output is a column slice of a wider tensor (block-output concat)
    y = torch.zeros((2, P, ld), dtype=torch.bfloat16, device="cuda")
    mean = torch.empty(Cc, device="cuda")
    rstd = torch.empty(Cc, device="cuda")
    _ok(L.naspipe_debug_bn_fwd(_p(zd), P, Cc, _p(gd), _p(bd), relu, _p(y[0, :, 8:]), ld, P * ld, _p(mean), _p(rstd),
                               None))
    torch.cuda.synchronize()
    ry, mu, rs, xh = _bn_ref(z, g.astype(np.float64), b.astype(np.float64), relu)
    assert np.max(np.abs(_f64(mean) - mu)) <= 1e-5 * max(1.0, np.max(np.abs(mu)))
    assert np.max(np.abs(_f64(rstd) / rs - 1)) <= 1e-5
    yy = _v2(y)
    _check_x2(yy[:, 8:8 + Cc], ry)
    assert not yy[:, :8].any() and not yy[:, 8 + Cc:].any()
    # backward with a strided incoming gradient
    dyfull_d, dyfull = _bf(rng.standard_normal((P, ld)))
    dy = dyfull[:, 8:8 + Cc]
    dz = torch.empty((P, Cc), dtype=torch.bfloat16, device="cuda")
    sums = torch.empty(2 * Cc, device="cuda")
    old = torch.empty(2 * Cc, device="cuda")
    lr = 0.01
    g2, b2 = gd.clone(), bd.clone()
    _ok(L.naspipe_debug_bn_bwd(_p(dyfull_d[:, 8:]), ld, _p(zd), P, Cc, _p(mean), _p(rstd), _p(g2), _p(b2), relu,
                               _p(dz), _p(sums), _p(old), lr, 1, None))
    torch.cuda.synchronize()
    # reference with the kernel's own statistics (the statistics were checked above)
    mu32, rs32 = _f64(mean), _f64(rstd)
    xh = (z - mu32) * rs32
    yv = g.astype(np.float64) * xh + b
    d = dy * (yv > 0) if relu else dy
    s1, s2 = d.sum(axis=0), (d * xh).sum(axis=0)
    rdz = rs32 * g * (d - s1 / P - xh * s2 / P)
    s = _f64(sums)
    assert np.max(np.abs(s[:Cc] - s1)) <= 1e-5 * np.max(np.abs(s1)) + 1e-6 * np.sqrt(P)
    assert np.max(np.abs(s[Cc:] - s2)) <= 1e-5 * np.max(np.abs(s2)) + 1e-6 * np.sqrt(P)
    np.testing.assert_array_equal(_f64(old), np.concatenate([g, b]).astype(np.float64))
    np.testing.assert_allclose(_f64(g2), g - lr * s[Cc:].astype(np.float32), rtol=1e-6, atol=1e-7)
    np.testing.assert_allclose(_f64(b2), b - lr * s[:Cc].astype(np.float32), rtol=1e-6, atol=1e-7)
    _check_bf16(_f64(dz), rdz)


@pytest.mark.parametrize("B,H,Cc,k,s,d,relu", [(2, 9, 16, 3, 1, 1, 1), (3, 8, 48, 5, 2, 1, 1), (2, 14, 32, 7, 1, 2, 0),
                                             (64, 56, 32, 3, 1, 1, 1), (64, 112, 32, 5, 2, 1, 1),
                                             (64, 7, 320, 7, 1, 1, 1), (64, 14, 160, 3, 2, 2, 1)])
def test_bn_apply_folded_into_depthwise_is_bitwise_the_stored_path(B, H, Cc, k, s, d, relu):
    """conv -> BN -> ReLU -> depthwise with bn_apply folded into the depthwise conv's load
    (BnApplyIn): the conv output, the weight gradient (BN recomputed on load) and the
    published mean / rstd are BITWISE those of the stored path (bn_apply -> y -> dw_fwd); the
    published g, b snapshots are the forward's; and the result matches explicit loops."""
    rng = np.random.default_rng(B + H + Cc + k + s + d)
    zd, z = _x2(rng.standard_normal((B, H, H, Cc)) * rng.uniform(0.5, 2.0, Cc) + rng.uniform(-1, 1, Cc))
    g = rng.uniform(0.5, 1.5, Cc).astype(np.float32)
    b = rng.uniform(-0.3, 0.3, Cc).astype(np.float32)
    gd, bd = torch.from_numpy(g).cuda(), torch.from_numpy(b).cuda()
    w = (rng.standard_normal((Cc, k, k)) / k).astype(np.float32)
    wd = torch.from_numpy(w).cuda()
    Ho = (H - 1) // s + 1
    dzd, dz = _bf(rng.standard_normal((B, Ho, Ho, Cc)))
    out_ref = torch.empty((2, B, Ho, Ho, Cc), dtype=torch.bfloat16, device="cuda")
    out = torch.empty_like(out_ref)
    dws_ref = torch.empty((Cc, k, k), device="cuda")
    dws = torch.empty_like(dws_ref)
    meta = torch.empty(4 * Cc, device="cuda")
    mean_ref, rstd_ref = torch.empty(Cc, device="cuda"), torch.empty(Cc, device="cuda")
    _ok(L.naspipe_debug_dw_bn_fold(_p(zd), B, H, Cc, _p(gd), _p(bd), relu, _p(wd), k, s, d, _p(dzd), _p(out_ref),
                                   _p(out), _p(dws_ref), _p(dws), _p(meta), _p(mean_ref), _p(rstd_ref), None))
    torch.cuda.synchronize()
    assert torch.equal(out, out_ref)
    assert torch.equal(dws, dws_ref)
    assert torch.equal(meta[:Cc], mean_ref) and torch.equal(meta[Cc:2 * Cc], rstd_ref)
    assert torch.equal(meta[2 * Cc:3 * Cc], gd) and torch.equal(meta[3 * Cc:], bd)
    if B * H * H <= 20000:  # and the composition against explicit loops (fp64 on the stored y)
        ry, _, _, _ = _bn_ref(z.reshape(-1, Cc), g.astype(np.float64), b.astype(np.float64), relu)
        _check_x2(_v2(out), _dw_ref(ry.reshape(z.shape), w.astype(np.float64), s, d), tol=1e-4)


@pytest.mark.parametrize("kind,B,H,Cc,Cout,k,dil,relu", [
    (0, 2, 9, 16, 0, 3, 1, 1), (0, 3, 14, 32, 0, 7, 1, 0), (0, 2, 37, 24, 0, 5, 2, 1), (0, 64, 56, 32, 0, 3, 1, 1),
    (0, 64, 7, 320, 0, 7, 2, 1), (2, 3, 9, 16, 0, 3, 1, 1), (2, 2, 14, 48, 0, 7, 2, 0), (2, 64, 112, 32, 0, 7, 1, 1),
    (2, 64, 14, 160, 0, 5, 1, 1),
    (1, 2, 9, 16, 48, 0, 0, 0), (1, 3, 13, 80, 160, 0, 0, 1), (1, 64, 14, 160, 320, 0, 0, 0),
    (1, 64, 7, 320, 640, 0, 0, 1), (1, 64, 56, 32, 32, 0, 0, 0)])
def test_bn_backward_sums_fused_into_input_gradient(kind, B, H, Cc, Cout, k, dil, relu):
    """bn_bwd_reduce fused into the producer of dy (stride-1 / stride-2 depthwise dgrad, 1x1-conv dgrad
    epilogue EPI_BNBWD): dx as the plain kernels compute it, and (sum dy', sum dy' xh) of the
    STORED dx against an fp64 reference on the same values (unit z -> BN -> ReLU?)."""
    rng = np.random.default_rng(1000 * kind + B + H + Cc + k)
    P = B * H * H
    if kind in (0, 2):
        w = (rng.standard_normal((Cc, k, k)) / k).astype(np.float32)
        wd, w16d = torch.from_numpy(w).cuda(), None
        Ho = H if kind == 0 else (H - 1) // 2 + 1
        dzd, dz = _bf(rng.standard_normal((B, Ho, Ho, Cc)))
    else:
        w16d, w16 = _bf(rng.standard_normal((Cout, Cc)) / np.sqrt(Cout))
        wd = None
        dzd, dz = _bf(rng.standard_normal((P, Cout)))
    zd, z = _x2(rng.standard_normal((P, Cc)) * rng.uniform(0.5, 2.0, Cc) + rng.uniform(-1, 1, Cc))
    mu = z.mean(axis=0).astype(np.float32)
    rs = (1.0 / np.sqrt(z.var(axis=0) + 1e-5)).astype(np.float32)
    g = rng.uniform(0.5, 1.5, Cc).astype(np.float32)
    b = rng.uniform(-0.3, 0.3, Cc).astype(np.float32)
    md, rd, gd, bd = (torch.from_numpy(a).cuda() for a in (mu, rs, g, b))
    dx = torch.empty((P, Cc), dtype=torch.bfloat16, device="cuda")
    sums = torch.empty(2 * Cc, device="cuda")
    outs = []
    for _ in range(2):
        _ok(L.naspipe_debug_bnb_fused(kind, _p(dzd), _p(wd), _p(w16d), _p(dx), B, H, Cc, Cout, k, dil, _p(zd), _p(md),
                                      _p(rd), _p(gd), _p(bd), relu, _p(sums), None))
        torch.cuda.synchronize()
        outs.append((dx.clone(), sums.clone()))
    assert torch.equal(outs[0][0], outs[1][0]) and torch.equal(outs[0][1], outs[1][1])
    if kind in (0, 2):
        rdx, _ = _dw_bwd_ref(np.zeros((B, H, H, Cc)), w.astype(np.float64), 1 if kind == 0 else 2, dz, dil)
        rdx = rdx.reshape(P, Cc)
    else:
        rdx = dz @ w16
    got = _f64(dx)
    _check_bf16(got, rdx)
    # the sums are taken over the stored dx (bf16); xh and the ReLU mask as the kernel forms
    # them (fp32 xh = (z - mean) rstd, y = fma(g, xh, b): the sign of the exact g xh + b)
    xh32 = ((z.astype(np.float32) - mu) * rs).astype(np.float32)
    xh = xh32.astype(np.float64)
    d = got * ((g.astype(np.float64) * xh + b) > 0) if relu else got
    s1, s2 = d.sum(axis=0), (d * xh).sum(axis=0)
    s = _f64(sums)
    a1, a2 = np.abs(d).sum(axis=0), np.abs(d * xh).sum(axis=0)
    assert np.all(np.abs(s[:Cc] - s1) <= 1e-5 * a1 + 1e-9)
    assert np.all(np.abs(s[Cc:] - s2) <= 1e-5 * a2 + 1e-9)


@pytest.mark.parametrize("B,H,Cc,k,s", [(2, 9, 16, 3, 1), (3, 8, 24, 3, 2), (2, 12, 8, 5, 2), (64, 56, 32, 3, 1),
                                        (64, 112, 32, 3, 2)])
def test_dense_conv_columns_and_adjoint(B, H, Cc, k, s):
    """The dense Conv 3x3 columns (A40): im2col of the x2 planes bitwise equal to the
    definition (exact copies, zero padding), and col2im = the exact adjoint of im2col on the
    fp32 column gradient (the sum over the taps that read an input, fp64 reference) + add,
    rounded to bf16."""
    rng = np.random.default_rng(B + H + Cc + k + s)
    xd, _ = _x2(rng.standard_normal((B, H, H, Cc)))
    Ho = (H - 1) // s + 1
    K = k * k * Cc
    cols = torch.empty((2, B * Ho * Ho, K), dtype=torch.bfloat16, device="cuda")
    dcols_h = rng.standard_normal((B * Ho * Ho, K)).astype(np.float32)
    dcols = torch.from_numpy(dcols_h).cuda()
    addd, add = _bf(rng.standard_normal((B, H, H, Cc)))
    dx = torch.empty((B, H, H, Cc), dtype=torch.bfloat16, device="cuda")
    _ok(L.naspipe_debug_dense_cols(_p(xd), _p(cols), _p(dcols), _p(addd), _p(dx), B, H, Cc, k, s, None))
    torch.cuda.synchronize()
    p = k // 2
    xp = torch.nn.functional.pad(xd.float().permute(0, 1, 4, 2, 3), (p, p, p, p))  # [2, B, C, H+2p, H+2p]
    ref = torch.empty((2, B, Ho, Ho, k, k, Cc), device="cuda")
    for u in range(k):
        for v in range(k):
            ref[:, :, :, :, u, v, :] = xp[:, :, :, u:u + s * (Ho - 1) + 1:s, v:v + s * (Ho - 1) + 1:s].permute(0, 1, 3, 4, 2)
    assert torch.equal(cols.float().reshape(2, B, Ho, Ho, k, k, Cc), ref)
    if B * H * H * Cc > 2_000_000:
        return  # the adjoint on the small shapes (fp64 reference below)
    dc = dcols_h.astype(np.float64).reshape(B, Ho, Ho, k, k, Cc)
    rdx = np.zeros((B, H + 2 * p, H + 2 * p, Cc))
    for u in range(k):
        for v in range(k):
            rdx[:, u:u + s * (Ho - 1) + 1:s, v:v + s * (Ho - 1) + 1:s, :] += dc[:, :, :, u, v, :]
    rdx = rdx[:, p:p + H, p:p + H, :] + add
    _check_bf16(_f64(dx), rdx)


@pytest.mark.parametrize("P,Ch", [(7, 16), (3136, 320), (1000, 80)])
def test_channel_split_merge_exact(P, Ch):
    rng = np.random.default_rng(P)
    xd, _ = _x2(rng.standard_normal((P, 2 * Ch)))
    out = torch.zeros((2, P, 2 * Ch), dtype=torch.bfloat16, device="cuda")
    xm = torch.empty((2, P, Ch), dtype=torch.bfloat16, device="cuda")
    _ok(L.naspipe_debug_chan_split(_p(xd), P, Ch, _p(out), 2 * Ch, P * 2 * Ch, _p(xm), None))
    gd, g = _bf(rng.standard_normal((P, 2 * Ch)))
    dmd, dm = _bf(rng.standard_normal((P, Ch)))
    dx = torch.empty((P, 2 * Ch), dtype=torch.bfloat16, device="cuda")
    _ok(L.naspipe_debug_chan_merge(_p(gd), 2 * Ch, _p(dmd), P, Ch, _p(dx), None))
    torch.cuda.synchronize()
    for pl in range(2):   # both planes are exact copies
        x = _f64(xd[pl])
        o = _f64(out[pl])
        np.testing.assert_array_equal(o[:, :Ch], x[:, 0::2])
        assert not o[:, Ch:].any()
        np.testing.assert_array_equal(_f64(xm[pl]), x[:, 1::2])
    r = np.empty((P, 2 * Ch))
    r[:, 0::2] = g[:, :Ch]
    r[:, 1::2] = dm
    np.testing.assert_array_equal(_f64(dx), r)


def test_stem_conv():
    rng = np.random.default_rng(3)
    B, H, C0 = 2, 32, 16
    x = rng.standard_normal((B, H, H, 3)).astype(np.float32)
    w = (rng.standard_normal((C0, 3, 3, 3)) / 5).astype(np.float32)
    z = torch.empty((2, B, H // 2, H // 2, C0), dtype=torch.bfloat16, device="cuda")
    xd, wd = torch.from_numpy(x).cuda(), torch.from_numpy(w).cuda()   # keep both alive during the launch
    _ok(L.naspipe_debug_stem(_p(xd), _p(wd), _p(z), B, H, C0, None))
    torch.cuda.synchronize()
    xp = np.pad(x.astype(np.float64), ((0, 0), (1, 1), (1, 1), (0, 0)))
    ref = np.zeros((B, H // 2, H // 2, C0))
    for u in range(3):
        for v in range(3):
            ref += xp[:, u:u + H - 1:2, v:v + H - 1:2, :] @ w[:, u, v, :].T.astype(np.float64)
    _check_x2(_v2(z), ref)


@pytest.mark.parametrize("M,N,K", [(128, 64, 64), (200, 48, 16), (3136, 1024, 640), (1000, 320, 160), (512, 144, 96)])
def test_gemm_bf16x2_three_pass(M, N, K):
    """z = x W^T on bf16x2 planes: error of the dropped lo*lo term and fp32 accumulation only."""
    rng = np.random.default_rng(M + N + K)
    ad, a = _x2(np.maximum(rng.standard_normal((M, K)), 0))
    bd, b = _x2(rng.standard_normal((N, K)) / np.sqrt(K))
    out = torch.empty((2, M, N), dtype=torch.bfloat16, device="cuda")
    res = []
    for _ in range(2):
        _ok(L.naspipe_debug_gemm_x2(M, N, K, _p(ad[0]), _p(ad[1]), K, _p(bd[0]), _p(bd[1]), K, _p(out[0]),
                                    _p(out[1]), None))
        torch.cuda.synchronize()
        res.append(out.clone())
    assert torch.equal(res[0], res[1])
    _check_x2(_v2(out), a @ b.T)
