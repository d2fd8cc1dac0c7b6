"""configs[4]: search-space sweep — dependency stalls vs throughput at D = 1/2/4/8 stages.

For n choices per block (uniform candidate shape h=16, f=3072, so cost does not vary with the
choice) the C++ planner (the schedule the executor runs) is driven with integer task costs in
microseconds taken from a measured single-GPU step (--step-ms, one subnet = m blocks, backward
= 2x forward by default).  Reported per (n, D): plan makespan, predicted samples/s =
N*B / makespan, dependency-stall and bubble fractions of stage time, the speed-up over D=1 and
the two brackets of SURVEY §8d: no dependencies (upper bound) and n=1 (fully serial).  The
closed-form conflict probability of consecutive subnets on a stage, 1-(1-1/n)^(m/D), is shown
beside the stall fraction.

    python tools/sweep.py --step-ms 13.2 [--out profiles/r1_sweep_c5.md]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402


def run(n, D, N, step_us, m=24, B=32, ignore_deps=False):
    cfg = synth.sweep_config(max(n, 1))
    cfg["n_choices"] = n
    cfg["choice_heads"], cfg["choice_ffn"] = [16] * n, [3072] * n
    per_block = step_us / m
    cf = np.full((m, n), max(1, int(round(per_block / 3))), dtype=np.int32)
    cb = np.full((m, n), max(1, int(round(2 * per_block / 3))), dtype=np.int32)
    cfg.update(cost_fwd=cf, cost_bwd=cb, window=4 * D)
    spec = npipe.Spec(cfg)
    choices = synth.sample_choices(N, m, n)
    if ignore_deps:  # every subnet gets private candidates: no dependencies at all
        choices = np.zeros((N, m), dtype=np.int32)
        cfg2 = dict(cfg, n_choices=N, choice_heads=[16] * N, choice_ffn=[3072] * N,
                    cost_fwd=np.full((m, N), cf[0, 0], np.int32), cost_bwd=np.full((m, N), cb[0, 0], np.int32))
        spec = npipe.Spec(cfg2)
        choices = np.tile(np.arange(N, dtype=np.int32)[:, None], (1, m))
    plan = npipe.naspipe_plan(spec, D, choices)
    mk = plan.makespan()
    st, bu = plan.idle(D)
    return dict(makespan_us=mk, samples_per_s=N * B / (mk / 1e6), stall=float(st.sum()) / (D * mk),
                bubble=float(bu.sum()) / (D * mk))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--step-ms", type=float, required=True, help="measured single-GPU time of one subnet")
    ap.add_argument("--subnets", type=int, default=256)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1_sweep_c5.md"))
    args = ap.parse_args()
    step_us = args.step_ms * 1000
    rows = []
    for n in (2, 4, 8, 16, 32, 64, 128):
        base = None
        for D in (1, 2, 4, 8):
            r = run(n, D, args.subnets, step_us)
            base = base or r["samples_per_s"]
            r.update(n=n, D=D, speedup=r["samples_per_s"] / base, conflict=1 - (1 - 1 / n) ** (24 / D))
            rows.append(r)
    bounds = {}
    for D in (1, 2, 4, 8):
        bounds[D] = dict(no_deps=run(1, D, args.subnets, step_us, ignore_deps=True)["samples_per_s"],
                         serial=run(1, D, args.subnets, step_us)["samples_per_s"])
    lines = ["# configs[4] search-space sweep (plan level, measured per-block cost)", "",
             f"Single-GPU step (one subnet, 24 blocks, uniform h=16 f=3072): {args.step_ms:.2f} ms "
             f"(measured on B200); N = {args.subnets} subnets, B = 32, W = 4D, strict backward-first.", "",
             "| n | D | samples/s (plan) | speed-up vs D=1 | stall frac | bubble frac | P(conflict) |",
             "|---|---|---|---|---|---|---|"]
    for r in rows:
        lines.append(f"| {r['n']} | {r['D']} | {r['samples_per_s']:.0f} | {r['speedup']:.2f} | "
                     f"{r['stall']:.3f} | {r['bubble']:.3f} | {r['conflict']:.3f} |")
    lines += ["", "Brackets (same costs): D | no dependencies (upper bound) | n = 1 (fully serial)", ""]
    for D, b in bounds.items():
        lines.append(f"- D={D}: {b['no_deps']:.0f} / {b['serial']:.0f} samples/s")
    lines += ["", "Throughput rises with n at every D > 1 (P:L350, P:L567); with n = 4-8 CSP is nearly "
              "serial (SURVEY §8d 'CSP-plan bound').", ""]
    with open(args.out, "w") as f:
        f.write("\n".join(lines))
    with open(args.out.replace(".md", ".json"), "w") as f:
        json.dump(dict(rows=rows, bounds=bounds, step_ms=args.step_ms), f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
