"""Bisect a cv_c3 parity failure (GPU box): one step at batch 4 of several variants."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402
from oracle import train  # noqa: E402
import parity_metrics as pm  # noqa: E402
from test_gpu_parity import run_engine  # noqa: E402


def one(label, cfg, choices):
    batches = [synth.make_batch(cfg, y) for y in range(len(choices))]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, choices, batches)
    params, losses, _, _ = run_engine(cfg, choices, batches, D=1)
    sm = pm.errors(cfg, params, ref, theta0)
    print(f"{label}: {pm.fmt(sm)} loss {losses} vs {ref_loss}", flush=True)


base = synth.get_config("cv_c3", batch=int(sys.argv[1]) if len(sys.argv) > 1 else 4)
m, n = base["n_blocks"], base["n_choices"]
for c in range(n):
    one(f"all choice {c}", base, np.full((1, m), c, dtype=np.int32))
one("sampled", base, synth.sample_choices(1, m, n))
sp = synth.get_config("spos", batch=4)
one("spos b4", sp, synth.sample_choices(1, sp["n_blocks"], sp["n_choices"]))
