"""Noise floors of the parity bars, measured with the ORACLE only (no GPU): the same fp64
oracle run with stored tensors rounded to a format, against the plain fp64 oracle, with the
per-tensor metrics of tests/parity_metrics.py (DESIGN.md §3 "Tolerances", A35;
profiles/r2_numerics.md).

    python tools/numerics_floor.py spos-step  [--storage fp32|bf16x2|bf16x2-bwd]  # configs[1], 1 step
    python tools/numerics_floor.py spos-steps --steps 20 --storage fp32           # vs the 100-step golden
    python tools/numerics_floor.py ln-gamma                                        # configs[2] block 0 ln1.g
"""
import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import synth  # noqa: E402
from oracle import spos, train  # noqa: E402
from oracle import transformer as T  # noqa: E402
import parity_metrics as pm  # noqa: E402

STORAGES = {"fp32": spos.FP32, "bf16x2": spos.BF16X2,
            "bf16x2-bwd": spos.Storage(spos.to_bf16x2, spos.to_bf16x2, spos.to_bf16x2, spos.to_bf16)}


def spos_step(storage):
    cfg = synth.get_config("spos")
    ch = synth.sample_choices(1, cfg["n_blocks"], cfg["n_choices"])
    b = [synth.make_batch(cfg, 0)]
    th0 = train.initial_theta(cfg)
    ref, _ = train.train_sequential(cfg, th0, ch, b)
    spos.STORAGE["_floor"] = STORAGES[storage]
    emu, _ = train.train_sequential(dict(cfg, storage="_floor"), th0, ch, b)
    print(f"configs[1] one step, {storage} storage vs fp64:", pm.fmt(pm.errors(cfg, emu, ref, th0)))


def spos_steps(storage, steps):
    gold = np.load(os.path.join(ROOT, "tests", "golden", "spos_fullsize_100steps.npz"))
    cfg = synth.get_config("spos")
    spos.STORAGE["_floor"] = STORAGES[storage]
    c = dict(cfg, storage="_floor")
    th = {k: train.unpack(cfg, k[0], k[1], v) for k, v in train.initial_theta(cfg).items()}
    t0 = time.time()
    for y in range(steps):
        x, t = synth.make_batch(cfg, y)
        loss, g = train.subnet_step(c, th, gold["choices"][y], x, t)
        train.sgd_apply(th, g, cfg["lr"])
        print(y, loss, f"{time.time() - t0:.0f} s", flush=True)
    packed = {k: train.pack(cfg, k[0], k[1], v) for k, v in th.items()}
    sm = pm.sampled_errors(cfg, gold, steps, lambda b, cc: packed[(b, cc)])
    print(f"configs[1] {steps} steps, {storage} storage vs fp64:", pm.fmt(sm))


def ln_gamma():
    """ln1.gamma of configs[2] block 0 with the real gradient of subnet 0's loss: the
    cancellation ratio of d gamma = sum_t da_t xhat_t and the error bf16 roundings of the
    block's own backward (dqkv, W, dO, P, dS) cause."""
    bf = spos.to_bf16
    cfg = synth.get_config("transformer")
    ch = synth.sample_choices(1, 24, 4)[0]
    th = {}
    for b in range(24):
        c = int(ch[b])
        segs = [(int(np.prod(s)), k, f) for _, s, k, f in train.candidate_layout(cfg, b, c)]
        th[b] = train.unpack(cfg, b, c, synth.init_packed(2, b * 4 + c, segs))
    x, t = synth.make_batch(cfg, 0)
    h = x.astype(np.float64)
    tapes = []
    for b in range(24):
        y, tp = T.forward(th[b], h, cfg["choice_heads"][int(ch[b])])
        tapes.append(tp)
        h = y
    _, dy = train.mse_loss(h, t.astype(np.float64))
    for b in reversed(range(1, 24)):
        dy, _ = T.backward(th[b], tapes[b], dy)
    p, tape = th[0], tapes[0]
    _, g = T.backward(p, tape, dy)
    a, c1, ca, o, a2, c2, z, gg = tape
    dz = (dy @ p["W2"]) * T.gelu_grad(z)
    dx1 = dy + T.ln_bwd(dz @ p["W1"], p["ln2_g"], c2)[0]
    do = dx1 @ p["Wo"]
    qh, kh, vh, pp, scale = ca
    doh = T._heads(bf(do), qh.shape[1])
    P = bf(pp)
    dv = P.swapaxes(-1, -2) @ doh
    dp = doh @ vh.swapaxes(-1, -2)
    dS = bf(pp * (dp - (dp * pp).sum(axis=-1, keepdims=True)))
    dqkv = np.concatenate([T._merge((dS @ kh) * scale), T._merge((dS.swapaxes(-1, -2) @ qh) * scale), T._merge(dv)],
                          axis=-1)
    da = bf(dqkv) @ bf(p["Wqkv"])
    _, dg, _ = T.ln_bwd(da, p["ln1_g"], c1)
    f2 = lambda q: q.reshape(-1, q.shape[-1])  # noqa: E731
    da_exact = np.concatenate(T.attn_bwd(do, ca), axis=-1) @ p["Wqkv"]
    terms = f2(da_exact) * f2(c1[0])
    print("ln1.g of configs[2] block 0: block-local bf16 roundings give a normwise error of "
          f"{np.linalg.norm(dg - g['ln1_g']) / np.linalg.norm(g['ln1_g']):.2e}; cancellation "
          f"sum|terms| / |sum| (median over channels) = {np.median(np.abs(terms).sum(0) / np.abs(terms.sum(0))):.1f}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("what", choices=["spos-step", "spos-steps", "ln-gamma"])
    ap.add_argument("--storage", default="fp32", choices=sorted(STORAGES))
    ap.add_argument("--steps", type=int, default=20)
    a = ap.parse_args()
    if a.what == "spos-step":
        spos_step(a.storage)
    elif a.what == "spos-steps":
        spos_steps(a.storage, a.steps)
    else:
        ln_gamma()


if __name__ == "__main__":
    main()
