"""Write tests/golden/transformer_fullsize_step1.npz: the fp64 ORACLE's result of training
subnet 0 of configs[2] (24 blocks x 4 choices, d = 1024, S = 128, B = 32; synth recipe)
for one step, reduced to sampled outputs the GPU parity test can compare against.

Calls only oracle/ (and synth/ for the seeded inputs); nothing here comes from the CUDA
path.  Stored per active candidate (b, c_0[b]) and per tensor of the packed layout:
  idx_<b>_<name>   sampled flat indices (default_rng(7), 256 per tensor, or all if smaller)
  new_<b>_<name>   theta_1 at those indices
  dnorm_<b>_<name> ||theta_1 - theta_0||_2 over the whole tensor
  dsamp_<b>_<name> (theta_1 - theta_0) at those indices
plus maxabs_<b> = max |theta_1| over the packed candidate (the A15 denominator) and loss.

    python tools/make_fullsize_golden.py      # ~5 min on 8 cores
"""
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from oracle import train  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "transformer_fullsize_step1.npz")


def main():
    cfg = synth.get_config("transformer")
    ch = synth.sample_choices(1, cfg["n_blocks"], cfg["n_choices"])[0]
    x, t = synth.make_batch(cfg, 0)
    n = cfg["n_choices"]
    theta0, theta = {}, {}
    for b in range(cfg["n_blocks"]):
        c = int(ch[b])
        segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in train.candidate_layout(cfg, b, c)]
        theta0[(b, c)] = synth.init_packed(cfg["init_seed"], b * n + c, segs).astype(np.float64)
        theta[(b, c)] = train.unpack(cfg, b, c, theta0[(b, c)])
    t0 = time.time()
    loss, grads = train.subnet_step(cfg, theta, ch, x, t)
    train.sgd_apply(theta, grads, cfg["lr"])
    print(f"oracle step: {time.time() - t0:.1f} s, loss {loss:.8f}")
    rng = np.random.default_rng(7)
    out = {"loss": np.float64(loss), "choices": np.asarray(ch, dtype=np.int32)}
    for b in range(cfg["n_blocks"]):
        c = int(ch[b])
        new = train.pack(cfg, b, c, theta[(b, c)])
        out[f"maxabs_{b}"] = np.float64(np.max(np.abs(new)))
        off = 0
        for name, shape, _, _ in train.candidate_layout(cfg, b, c):
            k = int(np.prod(shape))
            seg_new, seg_old = new[off:off + k], theta0[(b, c)][off:off + k]
            off += k
            idx = np.arange(k) if k <= 256 else np.sort(rng.choice(k, 256, replace=False))
            out[f"idx_{b}_{name}"] = idx.astype(np.int64)
            out[f"new_{b}_{name}"] = seg_new[idx]
            out[f"dsamp_{b}_{name}"] = (seg_new - seg_old)[idx]
            out[f"dnorm_{b}_{name}"] = np.float64(np.linalg.norm(seg_new - seg_old))
    np.savez_compressed(OUT, **out)
    print("wrote", OUT, os.path.getsize(OUT), "bytes")


if __name__ == "__main__":
    main()
