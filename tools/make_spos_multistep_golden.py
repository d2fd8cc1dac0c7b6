"""Write tests/golden/spos_fullsize_20steps.npz: the fp64 ORACLE's sequential training of the
first 20 subnets of configs[1] at full size (SPOS CNN, 20 blocks x 4 choices, 224x224,
B = 64; synth recipe: choices default_rng(0), batch y from default_rng([1, y]), A21 init),
reduced to sampled outputs the GPU parity test can compare against.

Calls only oracle/ (and synth/ for the seeded inputs); nothing here comes from the CUDA
path.  Stored per trained candidate (b, c): idx_<b>_<c> (512 flat indices of the packed
vector, default_rng(11)), new_<b>_<c> (theta_20 there), maxabs_<b>_<c> (max |theta_20| over the
packed vector: the A15 denominator); plus the 20 losses and the choices.

    python tools/make_spos_multistep_golden.py [--steps 20]     # ~1 h on 8 cores
"""
import argparse
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from oracle import train  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    a = ap.parse_args()
    out_path = os.path.join(ROOT, "tests", "golden", f"spos_fullsize_{a.steps}steps.npz")
    cfg = synth.get_config("spos")
    N = a.steps
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    theta0 = train.initial_theta(cfg)
    t0 = time.time()
    ref, losses = train.train_sequential(cfg, theta0, choices, batches)
    print(f"oracle: {N} subnets in {time.time() - t0:.0f} s, losses {losses}", flush=True)
    rng = np.random.default_rng(11)
    out = {"losses": np.asarray(losses, dtype=np.float64), "choices": np.asarray(choices, dtype=np.int32)}
    trained = sorted({(b, int(choices[y][b])) for y in range(N) for b in range(cfg["n_blocks"])})
    for (b, c) in trained:
        v = np.asarray(ref[(b, c)], dtype=np.float64)
        idx = np.sort(rng.choice(v.size, min(512, v.size), replace=False))
        out[f"idx_{b}_{c}"] = idx.astype(np.int64)
        out[f"new_{b}_{c}"] = v[idx]
        out[f"maxabs_{b}_{c}"] = np.float64(np.max(np.abs(v)))
    np.savez_compressed(out_path, **out)
    print("wrote", out_path, os.path.getsize(out_path), "bytes")


if __name__ == "__main__":
    main()
