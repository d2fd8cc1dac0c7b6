"""Kernel unit tests on the GPU (SURVEY §4 tier T2), through include/naspipe_debug.h.

Reference: float64 NumPy on the SAME bf16-rounded operands (plain matmul / softmax /
LayerNorm definitions).  bf16 outputs must lie within 1 bf16 ulp-scale normwise error of
the exact result; fp32 outputs normwise <= 1e-5 (fp32 accumulation).  Every kernel is run
twice and must be bitwise identical (fixed reduction order, no atomics).
"""
import ctypes as C

import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")
L = npipe.lib
_vp = C.c_void_p
L.naspipe_debug_gemm.argtypes = [C.c_int] * 3 + [_vp, C.c_int, C.c_int, _vp, C.c_int, C.c_int, C.c_int,
                                                 _vp, _vp, _vp, _vp, _vp, _vp, _vp, C.c_float, _vp]
L.naspipe_debug_attn_fwd.argtypes = [_vp, _vp, _vp] + [C.c_int] * 4 + [_vp]
L.naspipe_debug_attn_bwd.argtypes = [_vp] * 5 + [C.c_int] * 4 + [_vp]
L.naspipe_debug_ln_fwd.argtypes = [_vp] * 6 + [C.c_int] * 2 + [_vp]
L.naspipe_debug_ln_bwd.argtypes = [_vp] * 11 + [C.c_int] * 2 + [_vp]


def _ok(rc):
    assert rc == 0, L.naspipe_last_error().decode()


def _p(t):
    return None if t is None else t.data_ptr()


def _dev(a, dtype):
    return torch.from_numpy(np.ascontiguousarray(a)).to(device="cuda", dtype=dtype)


def _f64(t):
    return t.detach().to(torch.float64).cpu().numpy()


def _bf16_round(a):
    return _f64(torch.from_numpy(np.ascontiguousarray(a, dtype=np.float32)).to(torch.bfloat16))


def _normwise(got, ref):
    return float(np.max(np.abs(got - ref)) / max(np.max(np.abs(ref)), 1e-30))


def _gemm(M, N, K, A, a_mn, B, b_mn, epi, **kw):
    out = kw.get("out")
    _ok(L.naspipe_debug_gemm(M, N, K, _p(A), int(a_mn), A.shape[1], _p(B), int(b_mn), B.shape[1], epi,
                             _p(kw.get("bias")), _p(kw.get("resid")), _p(kw.get("aux")), _p(out),
                             _p(kw.get("out2")), _p(kw.get("w32")), _p(kw.get("w16")), kw.get("lr", 0.0), None))
    torch.cuda.synchronize()


SHAPES = [(128, 128, 64), (256, 384, 512), (304, 208, 200), (304, 272, 192), (4096, 1024, 1024),
          (256, 512, 4096),   # M, N >= 256: CTA-pair kernel (ragged: 304 x 272); split-K
          (1000, 32, 640), (520, 80, 96), (4096, 160, 200), (96, 64, 20000)]  # 64 / 128-wide N tiles; split-K


@pytest.mark.parametrize("M,N,K", SHAPES)
@pytest.mark.parametrize("a_mn,b_mn", [(False, False), (False, True), (True, True), (True, False)])
def test_gemm_f32_all_majors(M, N, K, a_mn, b_mn):
    rng = np.random.default_rng(M + N + K)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((N, K)).astype(np.float32)
    Ad = _dev(A.T if a_mn else A, torch.bfloat16)          # MN-major: stored [K][M]
    Bd = _dev(B.T if b_mn else B, torch.bfloat16)
    ref = _bf16_round(A) @ _bf16_round(B).T
    out = torch.empty((M, N), device="cuda", dtype=torch.float32)
    _gemm(M, N, K, Ad, a_mn, Bd, b_mn, 1, out=out)
    got = _f64(out)
    assert _normwise(got, ref) <= 1e-5 * max(1.0, np.sqrt(K / 1024))
    out2 = torch.empty_like(out)
    _gemm(M, N, K, Ad, a_mn, Bd, b_mn, 1, out=out2)
    assert torch.equal(out, out2), "GEMM not bitwise deterministic"


@pytest.mark.parametrize("M,N,K", [(256, 384, 320), (4096, 3072, 1024)])
def test_gemm_epilogues(M, N, K):
    rng = np.random.default_rng(7)
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = (rng.standard_normal((N, K)) / np.sqrt(K)).astype(np.float32)
    bias = rng.standard_normal(N).astype(np.float32)
    resid = rng.standard_normal((M, N)).astype(np.float32)
    Ad, Bd = _dev(A, torch.bfloat16), _dev(B, torch.bfloat16)
    C0 = _bf16_round(A) @ _bf16_round(B).T
    # bias + bf16
    out = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    _gemm(M, N, K, Ad, False, Bd, False, 2, out=out, bias=_dev(bias, torch.float32))
    assert _normwise(_f64(out), C0 + bias) <= 2 ** -8
    # bias + residual f32
    o32 = torch.empty((M, N), device="cuda", dtype=torch.float32)
    _gemm(M, N, K, Ad, False, Bd, False, 3, out=o32, bias=_dev(bias, torch.float32), resid=_dev(resid, torch.float32))
    assert _normwise(_f64(o32), C0 + bias + resid) <= 1e-5
    # bias + GELU (z and g)
    z = torch.empty((M, N), device="cuda", dtype=torch.bfloat16)
    g = torch.empty_like(z)
    _gemm(M, N, K, Ad, False, Bd, False, 4, out=z, out2=g, bias=_dev(bias, torch.float32))
    zr = C0 + bias
    gr = 0.5 * zr * (1 + np.tanh(np.sqrt(2 / np.pi) * (zr + 0.044715 * zr ** 3)))
    assert _normwise(_f64(z), zr) <= 2 ** -8
    assert _normwise(_f64(g), gr) <= 2 ** -8
    # GELU' with aux = z
    dz = torch.empty_like(z)
    _gemm(M, N, K, Ad, False, Bd, False, 5, out=dz, aux=z)
    zz = _f64(z)
    t = np.tanh(np.sqrt(2 / np.pi) * (zz + 0.044715 * zz ** 3))
    gp = 0.5 * (1 + t) + 0.5 * zz * (1 - t * t) * np.sqrt(2 / np.pi) * (1 + 3 * 0.044715 * zz * zz)
    assert _normwise(_f64(dz), C0 * gp) <= 2 ** -7


@pytest.mark.parametrize("M,N,K", [(32, 32, 64 * 56 * 56), (80, 80, 64 * 28 * 28 + 64)])
def test_gemm_splitk_ragged_k(M, N, K):
    """Split-K with a k-block count the split factor does not divide (the SPOS weight
    gradients: K = B*H*W pixels).  Every split must own >= 1 k-block: an empty split would
    leave its workspace slice stale (here: filled with another GEMM's partials first), and
    the result would depend on what ran before it."""
    rng = np.random.default_rng(K)
    junk = rng.standard_normal((512, 4096)).astype(np.float32)
    jd = _dev(junk, torch.bfloat16)
    _gemm(512, 512, 4096, jd, False, jd, False, 1, out=torch.empty((512, 512), device="cuda"))  # dirty workspace
    A = rng.standard_normal((M, K)).astype(np.float32)
    B = rng.standard_normal((N, K)).astype(np.float32)
    Ad, Bd = _dev(A.T, torch.bfloat16), _dev(B.T, torch.bfloat16)   # MN-major, as the wgrad reads them
    out = torch.empty((M, N), device="cuda", dtype=torch.float32)
    _gemm(M, N, K, Ad, True, Bd, True, 1, out=out)
    ref = _bf16_round(A) @ _bf16_round(B).T
    assert _normwise(_f64(out), ref) <= 1e-5 * np.sqrt(K / 1024)
    _gemm(512, 512, 4096, jd, False, jd, False, 1, out=torch.empty((512, 512), device="cuda"))
    out2 = torch.empty_like(out)
    _gemm(M, N, K, Ad, True, Bd, True, 1, out=out2)
    assert torch.equal(out, out2), "split-K result depends on the workspace's previous contents"


def test_gemm_sgd_epilogue():
    rng = np.random.default_rng(9)
    T, N, K = 4096, 1024, 768         # dW[N,K] = dY^T X : MN-major operands, K = T
    dY = rng.standard_normal((T, N)).astype(np.float32)
    X = rng.standard_normal((T, K)).astype(np.float32)
    W = rng.standard_normal((N, K)).astype(np.float32)
    w32 = _dev(W, torch.float32)
    w16 = torch.empty((N, K), device="cuda", dtype=torch.bfloat16)
    lr = 1e-3
    _gemm(N, K, T, _dev(dY, torch.bfloat16), True, _dev(X, torch.bfloat16), True, 6, w32=w32, w16=w16, lr=lr)
    dW = _bf16_round(dY).T @ _bf16_round(X)
    ref = W.astype(np.float64) - lr * dW
    assert _normwise(_f64(w32) - W, ref - W) <= 1e-5
    assert torch.equal(w16, w32.to(torch.bfloat16))


def _attn_ref(qkv, B, S, d, h):
    hd = d // h
    x = qkv.reshape(B, S, 3, h, hd)
    q, k, v = x[:, :, 0].transpose(0, 2, 1, 3), x[:, :, 1].transpose(0, 2, 1, 3), x[:, :, 2].transpose(0, 2, 1, 3)
    s = np.einsum("bhqe,bhke->bhqk", q, k) / np.sqrt(hd)
    mx = s.max(-1, keepdims=True)
    p = np.exp(s - mx)
    den = p.sum(-1, keepdims=True)
    p = p / den
    o = np.einsum("bhqk,bhke->bhqe", p, v)
    return o.transpose(0, 2, 1, 3).reshape(B * S, d), (mx + np.log(den))[..., 0], (q, k, v, p)


@pytest.mark.parametrize("B,S,d,h", [(2, 128, 192, 3), (2, 128, 192, 2), (3, 64, 128, 2), (4, 128, 1024, 8),
                                     (2, 128, 1024, 16)])
def test_attention_fwd_bwd(B, S, d, h):
    rng = np.random.default_rng(B * S + d + h)
    qkv = rng.standard_normal((B * S, 3 * d)).astype(np.float32)
    qkv_d = _dev(qkv, torch.bfloat16)
    qkv_r = _f64(qkv_d)
    o = torch.empty((B * S, d), device="cuda", dtype=torch.bfloat16)
    lse = torch.empty((B * h * S,), device="cuda", dtype=torch.float32)
    _ok(L.naspipe_debug_attn_fwd(_p(qkv_d), _p(o), _p(lse), B, S, d, h, None))
    torch.cuda.synchronize()
    o_ref, lse_ref, (q, k, v, p) = _attn_ref(qkv_r, B, S, d, h)
    assert _normwise(_f64(o), o_ref) <= 1e-2
    np.testing.assert_allclose(_f64(lse).reshape(B, h, S), lse_ref, rtol=1e-4, atol=1e-4)
    # backward
    do = rng.standard_normal((B * S, d)).astype(np.float32)
    do_d = _dev(do, torch.bfloat16)
    dqkv = torch.empty((B * S, 3 * d), device="cuda", dtype=torch.bfloat16)
    _ok(L.naspipe_debug_attn_bwd(_p(qkv_d), _p(o), _p(lse), _p(do_d), _p(dqkv), B, S, d, h, None))
    torch.cuda.synchronize()
    hd = d // h
    doh = _f64(do_d).reshape(B, S, h, hd).transpose(0, 2, 1, 3)
    dv = np.einsum("bhqk,bhqe->bhke", p, doh)
    dp = np.einsum("bhqe,bhke->bhqk", doh, v)
    ds = p * (dp - (dp * p).sum(-1, keepdims=True))
    dq = np.einsum("bhqk,bhke->bhqe", ds, k) / np.sqrt(hd)
    dk = np.einsum("bhqk,bhqe->bhke", ds, q) / np.sqrt(hd)
    m = lambda t: t.transpose(0, 2, 1, 3).reshape(B * S, d)   # noqa: E731
    got = _f64(dqkv)
    for i, ref in enumerate([m(dq), m(dk), m(dv)]):
        assert _normwise(got[:, i * d:(i + 1) * d], ref) <= 2e-2, ("qkv"[i], _normwise(got[:, i * d:(i + 1) * d], ref))
    dqkv2 = torch.empty_like(dqkv)
    _ok(L.naspipe_debug_attn_bwd(_p(qkv_d), _p(o), _p(lse), _p(do_d), _p(dqkv2), B, S, d, h, None))
    torch.cuda.synchronize()
    assert torch.equal(dqkv, dqkv2)


@pytest.mark.parametrize("T,d", [(256, 192), (4096, 1024), (100, 64)])
def test_layernorm_fwd_bwd(T, d):
    rng = np.random.default_rng(T + d)
    x = (rng.standard_normal((T, d)) * 2 + 0.5).astype(np.float32)
    g = (1 + 0.1 * rng.standard_normal(d)).astype(np.float32)
    b = (0.1 * rng.standard_normal(d)).astype(np.float32)
    xd, gd, bd = _dev(x, torch.float32), _dev(g, torch.float32), _dev(b, torch.float32)
    y = torch.empty((T, d), device="cuda", dtype=torch.bfloat16)
    mean = torch.empty(T, device="cuda")
    rstd = torch.empty(T, device="cuda")
    _ok(L.naspipe_debug_ln_fwd(_p(xd), _p(gd), _p(bd), _p(y), _p(mean), _p(rstd), T, d, None))
    torch.cuda.synchronize()
    x64 = x.astype(np.float64)
    mu = x64.mean(-1, keepdims=True)
    rs = 1 / np.sqrt(x64.var(-1, keepdims=True) + 1e-5)
    xh = (x64 - mu) * rs
    assert _normwise(_f64(y), g * xh + b) <= 2 ** -8
    dy = rng.standard_normal((T, d)).astype(np.float32)
    resid = rng.standard_normal((T, d)).astype(np.float32)
    dx = torch.empty((T, d), device="cuda")
    dx16 = torch.empty((T, d), device="cuda", dtype=torch.bfloat16)
    dg, db, cs = (torch.empty(d, device="cuda") for _ in range(3))
    dyd, rd = _dev(dy, torch.float32), _dev(resid, torch.float32)   # keep alive across the call
    _ok(L.naspipe_debug_ln_bwd(_p(dyd), _p(xd), _p(mean), _p(rstd), _p(gd), _p(rd), _p(dx), _p(dx16), _p(dg),
                               _p(db), _p(cs), T, d, None))
    torch.cuda.synchronize()
    dxh = dy * g
    dx_ref = resid + rs * (dxh - dxh.mean(-1, keepdims=True) - xh * (dxh * xh).mean(-1, keepdims=True))
    assert _normwise(_f64(dx), dx_ref) <= 1e-5
    assert _normwise(_f64(dg), (dy * xh).sum(0)) <= 1e-5
    assert _normwise(_f64(db), dy.astype(np.float64).sum(0)) <= 1e-5
    assert _normwise(_f64(cs), dx_ref.sum(0)) <= 1e-5
    assert torch.equal(dx16, dx.to(torch.bfloat16))
