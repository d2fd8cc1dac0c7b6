"""Storage-precision floors of the spos_dense full-size one-step check (reading A40): the fp64
oracle against itself with every stored tensor rounded to fp32 (the paper's precision) and
to the path's storage (bf16x2 forward, bf16 backward; reading A28).  Calls only oracle/ and
synth; writes tests/golden/spos_dense_fullsize_1step_floor.json.

    python tools/make_dense_floor.py        # ~10 min on 16 host cores (three full-size oracle runs)
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402

import parity_metrics as pm  # noqa: E402
import synth  # noqa: E402
from oracle import train  # noqa: E402


def main():
    cfg = synth.get_config("spos_dense")
    choices = np.zeros((1, cfg["n_blocks"]), dtype=np.int32)   # the dense candidate in every block
    batches = [synth.make_batch(cfg, 0)]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    out = {"config": "spos_dense", "choices": "all 0 (dense Conv 3x3)", "steps": 1,
           "source": "tools/make_dense_floor.py (oracle/ only)", "loss_fp64": float(ref_loss[0])}
    for st in ("fp32", "bf16x2"):
        got, _ = train.train_sequential(dict(cfg, storage=st), theta0, choices, batches)
        e = pm.errors(cfg, got, ref, theta0)
        out[st] = {"a15_tensor": float(e["a15"]), "a15_candidate": float(e["a15_cand"]), "upd": {k: float(v) for k, v in e["upd"].items()},
                   "static": float(e["static"]), "fmt": pm.fmt(e)}
        print(st, pm.fmt(e), flush=True)
    with open(os.path.join(ROOT, "tests", "golden", "spos_dense_fullsize_1step_floor.json"), "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
