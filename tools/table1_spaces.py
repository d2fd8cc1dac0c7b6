"""The paper's search spaces at plan level (Table 1; SURVEY §8f(4) "at Table 1
scales"): NLP.c0-c3 = 48 blocks x 96/72/48/24 candidates, CV.c1-c3 = 32 blocks x 48/24/12,
uniform per-block sampling, D = 8 stages (the paper's default), N = 256
subnets, W = 4D, unit per-block costs (cf = 1, cb = 2: a uniform candidate cost, so the
bubble comes from the schedule alone).  The C++ planner (the schedule the executor runs)
gives, per space and policy: makespan, speed-up over one stage, bubble ratio (idle stage
time), and throughput relative to BSP (GPipe's bulk-synchronous schedule) -- the
paper's headline comparison ("1.1X ~ 7.8X" over GPipe; NLP.c1 7.8X) on the
same cost model, plus the paper's Table 2 bubble ratios as context.

    python tools/table1_spaces.py [--out profiles/r2_table1_spaces.md]
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

SPACES = [("NLP.c0", 48, 96, None), ("NLP.c1", 48, 72, 0.39), ("NLP.c2", 48, 48, 0.57), ("NLP.c3", 48, 24, 0.68),
          ("CV.c1", 32, 48, 0.43), ("CV.c2", 32, 24, 0.58), ("CV.c3", 32, 12, 0.68)]
POLICIES = ["csp", "serial", "inorder", "bsp", "asp"]


def plan(m, n, D, N, sync, seed=0):
    cfg = dict(synth.get_config("toy"), n_blocks=m, n_choices=n, window=4 * D, bulk_size=4 * D, sync=sync,
               cost_fwd=np.ones((m, n), np.int32), cost_bwd=np.full((m, n), 2, np.int32))
    ch = synth.sample_choices(N, m, n, seed)
    p = npipe.naspipe_plan(npipe.Spec(cfg), D, ch)
    mk = p.makespan()
    st, bu = p.idle(D)
    return mk, float(st.sum() + bu.sum()) / (D * mk)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--subnets", type=int, default=256)
    ap.add_argument("--stages", type=int, default=8)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2_table1_spaces.md"))
    a = ap.parse_args()
    D, N = a.stages, a.subnets
    rows = []
    for name, m, n, paper_bubble in SPACES:
        one, _ = plan(m, n, 1, N, "csp")
        r = dict(space=name, m=m, n=n, paper_bubble=paper_bubble)
        for sync in POLICIES:
            mk, idle = plan(m, n, D, N, sync)
            r[sync] = dict(makespan=mk, speedup=one / mk, bubble=idle)
        r["csp_over_bsp"] = r["bsp"]["makespan"] / r["csp"]["makespan"]
        r["csp_over_serial"] = r["serial"]["makespan"] / r["csp"]["makespan"]
        rows.append(r)
    lines = [f"# The paper's search spaces (Table 1) at plan level, D = {D}, N = {N}", "",
             "Unit per-block costs (cf = 1, cb = 2), W = 4D, BSP bulk = 4D, strict backward-first, uniform per-block "
             "sampling.  Speed-up = one-stage makespan / D-stage makespan; bubble = idle fraction of stage time.  "
             "BSP executes more subnets concurrently than CSP allows but computes a different (non-sequential) "
             "result (Table 3); SERIAL is 'w/o scheduler' (P:L454, reading A32).", "",
             "| space | m x n | CSP speed-up | CSP bubble (paper, Table 2) | CSP / BSP (GPipe) | CSP / SERIAL | "
             "SERIAL bubble | BSP speed-up | ASP speed-up |", "|---|---|---|---|---|---|---|---|---|"]
    for r in rows:
        pb = f"{r['paper_bubble']:.2f}" if r["paper_bubble"] is not None else "n/a"
        lines.append(f"| {r['space']} | {r['m']} x {r['n']} | {r['csp']['speedup']:.2f}x | {r['csp']['bubble']:.2f} "
                     f"({pb}) | {r['csp_over_bsp']:.2f}x | {r['csp_over_serial']:.2f}x | {r['serial']['bubble']:.2f} | "
                     f"{r['bsp']['speedup']:.2f}x | {r['asp']['speedup']:.2f}x |")
    lines += ["", "Ordering checks: CSP throughput rises with the number of candidates (Artifact Exp.2, P:L563-567: "
              "T(NLP.c0) > c1 > c2 > c3) and its bubble falls (Table 2, P:L350).  The bubble LEVELS are higher "
              "than the paper's (SURVEY §8d: the paper does not say how it measured bubble; parameter-free "
              "candidates, which create no dependencies, are a plausible unstated cause).  With uniform costs "
              "BSP (GPipe) fills the pipeline better than CSP at these scales: the paper's 1.1-7.8x over GPipe "
              "comes from GPipe's smaller batch / recomputation and memory limits on 11 GB GPUs (Table 2 "
              "batch sizes), which a plan-level model with equal batches does not contain.", ""]
    with open(a.out, "w") as f:
        f.write("\n".join(lines))
    with open(a.out.replace(".md", ".json"), "w") as f:
        json.dump(rows, f, indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
