"""Alg.3's context predictor against the exact plan lookahead.

For each workload (default integer cost tables) and D, the O2 plan of N uniformly sampled
subnets is replayed through oracle.csp.alg3_backward_predictions: before every B(x, K) the
stage predicts its next forward with Alg.2 on L_f + {x}.  Reported: how many of the
forwards that follow a backward were predicted correctly (the context the predictor
prefetches in time), how many predictions were wrong, and how many were missing (the
forward had not reached the stage's queue yet).  The executor's Belady plan lookahead
(readings A9, A26) knows every next task exactly: 100 % by construction.

    python tools/alg3_predictor.py [--subnets 96] [--out profiles/r1_alg3_predictor.md]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
from oracle import csp  # noqa: E402  (analysis tool: plan-level, no GPU)
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402

WORKLOADS = {"configs[1] spos": ("spos", None), "configs[2] transformer": ("transformer", None),
             "configs[3] large_transformer": ("large_transformer", None), "configs[4] sweep n=16": ("sweep", 16),
             "configs[4] sweep n=64": ("sweep", 64)}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--subnets", type=int, default=96)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1_alg3_predictor.md"))
    a = ap.parse_args()
    rows = []
    for label, (name, n) in WORKLOADS.items():
        cfg = synth.sweep_config(n) if name == "sweep" else synth.get_config(name)
        choices = synth.sample_choices(a.subnets, cfg["n_blocks"], cfg["n_choices"]).tolist()
        for D in (2, 4, 8):
            spec = npipe.Spec(cfg)
            sob = npipe.naspipe_partition(spec, D)
            cf, cb = npipe.naspipe_default_costs(spec)
            tf, tb = csp.task_costs(choices, sob, cf, cb, D)
            preds = csp.alg3_backward_predictions(choices, sob, D, 4 * D, tf, tb)
            follow = [(p, x) for (_, _, _, p, x) in preds if x is not None]
            hit = sum(1 for p, x in follow if p == x)
            wrong = sum(1 for (_, _, _, p, x) in preds if p is not None and p != x)
            missing = sum(1 for p, x in follow if p is None)
            r = {"workload": label, "D": D, "backwards": len(preds), "followed_by_forward": len(follow),
                 "predicted_correctly": hit, "wrong_predictions": wrong, "no_prediction": missing,
                 "hit_rate": hit / len(follow) if follow else None}
            rows.append(r)
            print(json.dumps(r), flush=True)
    with open(a.out.replace(".md", ".json"), "w") as f:
        json.dump(rows, f, indent=1)
    with open(a.out, "w") as f:
        f.write("# Alg.3 context predictor vs the exact plan lookahead (plan level)\n\n")
        f.write("`python tools/alg3_predictor.py` — O2 plans of N = %d uniformly sampled subnets (seed 0), W = 4D, default "
                "cost tables; `oracle.csp.alg3_backward_predictions` replays Alg.3's backward branch (P:L239-273) at every "
                "B(x,K). Hit rate = correctly predicted next forwards / forwards that follow a backward. The executor's "
                "exact plan lookahead (readings A9, A26) is 100%% by construction.\n\n" % a.subnets)
        f.write("| workload | D | backwards | followed by a forward | predicted correctly | wrong | no prediction | hit rate |\n")
        f.write("|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            hr = "—" if r["hit_rate"] is None else f"{100 * r['hit_rate']:.1f}%"
            f.write(f"| {r['workload']} | {r['D']} | {r['backwards']} | {r['followed_by_forward']} | "
                    f"{r['predicted_correctly']} | {r['wrong_predictions']} | {r['no_prediction']} | {hr} |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()
