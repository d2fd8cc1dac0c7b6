"""Write tests/golden/<workload>_fullsize_<N>steps.npz: the fp64 ORACLE's sequential training
of the first N subnets of a BASELINE.json config at full size (synth recipe: choices
default_rng(0), batch y from default_rng([1, y]), A21 init), reduced to per-tensor sampled
outputs at several checkpoints, for the north_star bar "within 1e-3 max relative error after
1 step and within 1e-2 after 100 steps" (A15, per tensor).

Calls only oracle/ (and synth/ for the seeded inputs); nothing here comes from the CUDA
path.  Stored, for every candidate (b, c) trained by the last checkpoint and every tensor
``name`` of its packed layout (oracle.train.candidate_layout):

  idx_<b>_<c>_<name>            sampled flat indices into the tensor (default_rng(13), <= 256)
  init_<b>_<c>_<name>           theta_0 at those indices
  s<k>_<b>_<c>_<name>           theta_k at those indices (checkpoint k; only if trained by k)
  s<k>_max_<b>_<c>_<name>       max |theta_k| over the whole tensor   (the A15 denominator)
  s<k>_dmax_<b>_<c>_<name>      max |theta_k - theta_0| over the whole tensor (update bar)
plus losses (all N), choices [N, m], checkpoints.

    python tools/make_multistep_golden.py --workload transformer --steps 100 --checkpoints 1,100
    python tools/make_multistep_golden.py --workload spos --steps 100 --checkpoints 1,20,100
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
    ap.add_argument("--workload", default="transformer")
    ap.add_argument("--steps", type=int, default=100)
    ap.add_argument("--checkpoints", default="1,100")
    ap.add_argument("--samples", type=int, default=256)
    ap.add_argument("--storage", default=None,
                    help="SPOS: run the oracle with this storage rounding (oracle/spos.py STORAGE, e.g. fp32 = the "
                         "paper's precision P:L98) -- the precision floor of the multi-step bar (DESIGN.md A35)")
    a = ap.parse_args()
    cks = sorted({int(s) for s in a.checkpoints.split(",")} | {a.steps})
    suffix = f"_{a.storage}" if a.storage else ""
    out_path = os.path.join(ROOT, "tests", "golden", f"{a.workload}_fullsize_{a.steps}steps{suffix}.npz")
    cfg = synth.get_config(a.workload)
    run_cfg = dict(cfg, storage=a.storage) if a.storage else cfg
    N, n = a.steps, cfg["n_choices"]
    choices = synth.sample_choices(N, cfg["n_blocks"], n)
    used = sorted({(b, int(choices[y][b])) for y in range(N) for b in range(cfg["n_blocks"])})
    # theta_0 of the candidates the run touches (the others never change)
    theta0 = {}
    for (b, c) in used:
        segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in train.candidate_layout(cfg, b, c)]
        theta0[(b, c)] = synth.init_packed(cfg["init_seed"], b * n + c, segs)
    theta = {k: train.unpack(cfg, k[0], k[1], v) for k, v in theta0.items()}
    offs = {}
    for k in used:      # offsets of each tensor in the packed theta_0 vector
        off = 0
        for name, shape, _, _ in train.candidate_layout(cfg, *k):
            offs[(k, name)] = (off, off + int(np.prod(shape)))
            off += int(np.prod(shape))

    def init_of(k, name):
        lo, hi = offs[(k, name)]
        return np.asarray(theta0[k][lo:hi], dtype=np.float64)
    rng = np.random.default_rng(13)
    out = {"choices": np.asarray(choices, dtype=np.int32), "checkpoints": np.asarray(cks, dtype=np.int64)}
    idx = {}
    for k in used:
        for name, shape, _, _ in train.candidate_layout(cfg, *k):
            size = int(np.prod(shape))
            ii = np.arange(size) if size <= a.samples else np.sort(rng.choice(size, a.samples, replace=False))
            idx[(k, name)] = ii
            out[f"idx_{k[0]}_{k[1]}_{name}"] = ii.astype(np.int64)
            out[f"init_{k[0]}_{k[1]}_{name}"] = init_of(k, name)[ii]
    losses = np.zeros(N)
    trained = set()
    t0 = time.time()
    for y in range(N):
        x, t = synth.make_batch(cfg, y)
        loss, grads = train.subnet_step(run_cfg, theta, choices[y], x, t)
        train.sgd_apply(theta, grads, cfg["lr"])
        losses[y] = loss
        trained |= set(grads)
        print(f"step {y + 1}/{N}: loss {loss:.8f}  ({time.time() - t0:.0f} s)", flush=True)
        if y + 1 in cks:
            for k in sorted(trained):
                for name, _, _, _ in train.candidate_layout(cfg, *k):
                    v, v0 = theta[k][name].ravel(), init_of(k, name)
                    tag = f"{k[0]}_{k[1]}_{name}"
                    out[f"s{y + 1}_{tag}"] = v[idx[(k, name)]]
                    out[f"s{y + 1}_max_{tag}"] = np.float64(np.max(np.abs(v)))
                    out[f"s{y + 1}_dmax_{tag}"] = np.float64(np.max(np.abs(v - v0)))
            out["losses"] = losses.copy()
            np.savez_compressed(out_path, **out)      # partial file after every checkpoint
            print(f"checkpoint {y + 1}: wrote {out_path}", flush=True)
    print("wrote", out_path, os.path.getsize(out_path), "bytes")


if __name__ == "__main__":
    main()
