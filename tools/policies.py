"""CSP against the other synchronisation policies, at plan level.

For a workload (its default integer cost table, or uniform costs scaled to a measured
single-GPU step) the C++ planner — the schedule the executor runs — is driven with each
policy of include/naspipe.h naspipe_sync:
  CSP      the method (Def.2)
  INORDER  NASPipe w/o scheduler (Fig.6 ablation): no overtaking of a blocked head
  ASP      dependencies ignored (PipeDream): the no-dependency bound
  BSP      GPipe / Retiarii bulks of 4D subnets with a flush
Reported per (policy, D): plan speed-up over one stage (N * sum of costs / makespan) and the
idle fraction of stage time.  A second table replays Table 4: the order in
which the stage owning one candidate READs (F) and WRITEs (B) it, at D = 4 and D = 8 — CSP's
is the same at both and follows the sequential order; ASP's and BSP's change with D (and
break the F-B alternation), which is why their results are not reproducible (Table 3).

    python tools/policies.py [--workload transformer] [--out profiles/r1_policies.md]
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

POLICIES = ["csp", "serial", "inorder", "asp", "bsp"]


def plan(cfg, choices, D, sync):
    spec = npipe.Spec(dict(cfg, sync=sync, window=4 * D, bulk_size=4 * D))
    p = npipe.naspipe_plan(spec, D, choices)
    return spec, p


def speedup(cfg, choices, D, sync):
    spec, p = plan(cfg, choices, D, sync)
    cf, cb = npipe.naspipe_default_costs(spec)
    serial = sum(int(max(1, cf[b, c]) + max(1, cb[b, c])) for row in choices for b, c in enumerate(row))
    # the serial reference is the D=1 plan (one stage task per subnet and kind)
    _, p1 = plan(cfg, choices, 1, "csp")
    mk = p.makespan()
    st, bu = p.idle(D)
    return dict(speedup=p1.makespan() / mk, idle=float(st.sum() + bu.sum()) / (D * mk), makespan=mk,
                serial_sum=serial)


def access_order(cfg, choices, D, sync, cand):
    b, c = cand
    spec, p = plan(cfg, choices, D, sync)
    sob = npipe.naspipe_partition(spec, D)
    seq = []
    for t, K, kind, y in p.trace():
        if K == sob[b] and choices[y][b] == c:
            seq.append(f"{y}{'F' if kind == 0 else 'B'}")
    return seq


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="transformer")
    ap.add_argument("--subnets", type=int, default=256)
    ap.add_argument("--n-choices", type=int, default=0, help="override n (sweep-style uniform candidates)")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2_policies.md"))
    args = ap.parse_args()
    if args.n_choices:
        cfg = synth.sweep_config(args.n_choices)
        name = f"configs[4] uniform candidates, n={args.n_choices}"
    else:
        cfg = synth.get_config(args.workload)
        name = args.workload
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = synth.sample_choices(args.subnets, m, n)
    rows = []
    for D in (2, 4, 8):
        for sync in POLICIES:
            r = speedup(cfg, choices, D, sync)
            r.update(D=D, sync=sync)
            rows.append(r)
    lines = [f"# Synchronisation policies at plan level — {name} (m={m}, n={n}), N={args.subnets}", "",
             "Default integer cost table of the library (naspipe_default_costs), W = 4D, BSP bulk = 4D, strict "
             "backward-first.  Speed-up = makespan of the one-stage plan / makespan at D.", "",
             "| D | CSP | w/o scheduler (SERIAL, P:L454) | in-order admission (INORDER) | ASP (no deps) | BSP (GPipe) "
             "| idle CSP / SERIAL / INORDER / ASP / BSP |",
             "|---|---|---|---|---|---|---|"]
    for D in (2, 4, 8):
        rr = {r["sync"]: r for r in rows if r["D"] == D}
        lines.append(f"| {D} | {rr['csp']['speedup']:.2f}x | {rr['serial']['speedup']:.2f}x | {rr['inorder']['speedup']:.2f}x | "
                     f"{rr['asp']['speedup']:.2f}x | {rr['bsp']['speedup']:.2f}x | "
                     + " / ".join(f"{rr[s]['idle']:.2f}" for s in POLICIES) + " |")
    # Table 4: the access order of one candidate used by several early subnets
    b = 0
    users = {}
    for y, row in enumerate(choices[:64]):
        users.setdefault((b, int(row[b])), []).append(y)
    cand = max(users, key=lambda k: len(users[k]))
    lines += ["", f"Table 4 replay (P:L435): READ (F) / WRITE (B) order of candidate (block {cand[0]}, choice "
              f"{cand[1]}) on its stage, first 8 accesses:", "",
              "| policy | D = 4 | D = 8 | same at both |", "|---|---|---|---|"]
    t4 = {}
    for sync in POLICIES:
        a4 = access_order(cfg, choices, 4, sync, cand)[:8]
        a8 = access_order(cfg, choices, 8, sync, cand)[:8]
        t4[sync] = (a4, a8)
        lines.append(f"| {sync} | {'-'.join(a4)} | {'-'.join(a8)} | {'yes' if a4 == a8 else 'no'} |")
    lines += ["", "CSP's order is the sequential F-B alternation in id order at every D (reading A20: "
              "numerics unique); ASP/BSP let later subnets READ before earlier ones WRITE.", ""]
    text = "\n".join(lines)
    with open(args.out, "w") as f:
        f.write(text)
    with open(args.out.replace(".md", ".json"), "w") as f:
        json.dump(dict(rows=rows, table4=t4, candidate=cand), f, indent=1)
    print(text)


if __name__ == "__main__":
    main()
