"""per-subnet balanced partitions with layer mirroring, at plan level.

For each workload (its default integer cost table, include/naspipe.h naspipe_default_costs)
and D, the CSP plan of N uniformly sampled subnets is computed twice by the C++ planners:
  fixed      the supernet partition every stage owns (reading A12; what the executor runs)
  mirrored   each subnet's own balanced partition, candidates mirrored across
             stages, a WRITE reaching a mirror after `mirror_latency` ticks (A31)
Reported: plan speed-up over one stage (D=1 makespan / makespan), bottleneck balance
(max over subnets of its largest stage cost / its mean stage cost), the fraction of a
subnet's blocks placed off the supernet partition, and the mirror latency used (the
candidate's fp32 bytes over NVLink, 900 GB/s, in 1-us ticks).

    python tools/mirroring.py [--subnets 128] [--out profiles/r1_mirroring.md]
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

WORKLOADS = {"configs[1] spos": ("spos", None), "configs[2] transformer": ("transformer", None),
             "configs[3] large_transformer": ("large_transformer", None),
             "configs[4] sweep n=16": ("sweep", 16), "configs[4] sweep n=64": ("sweep", 64)}


def cfg_of(name, n):
    return synth.sweep_config(n) if name == "sweep" else synth.get_config(name)


def row(label, cfg, N, D, seed):
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    if seed:
        choices = np.random.default_rng(seed).integers(0, cfg["n_choices"], choices.shape).astype(np.int32)
    spec = npipe.Spec(dict(cfg, window=4 * D))
    cf, cb = npipe.naspipe_default_costs(spec)
    m, n = cfg["n_blocks"], cfg["n_choices"]
    # mirror push latency: mean candidate fp32 bytes at 900 GB/s, in 1-us ticks
    mean_bytes = np.mean([4 * npipe.naspipe_param_count(spec, b, c) for b in range(m) for c in range(n)])
    lam_w = int(np.ceil(mean_bytes / 900e9 * 1e6))
    one = npipe.naspipe_plan(npipe.Spec(dict(cfg, window=4)), 1, choices).makespan()
    fixed = npipe.naspipe_plan(spec, D, choices)
    mir = npipe.naspipe_plan_mirrored(spec, D, choices, lam_w)
    sob = npipe.naspipe_partition(spec, D)
    off = float(np.mean(mir["stage_of_block"] != sob[None, :]))

    def balance(stage_of):
        worst = []
        for y in range(N):
            st = np.zeros(D)
            for b in range(m):
                st[stage_of[y][b]] += cf[b, choices[y][b]] + cb[b, choices[y][b]]
            worst.append(st.max() / st.mean())
        return float(np.mean(worst))

    fst, fbu = fixed.idle(D)
    return {"workload": label, "D": D, "subnets": N, "mirror_latency_ticks": lam_w,
            "fixed_speedup": one / fixed.makespan(), "mirrored_speedup": one / mir["makespan"],
            "fixed_balance": balance([sob] * N), "mirrored_balance": balance(mir["stage_of_block"]),
            "blocks_off_supernet_partition": off,
            "fixed_idle": float(fst.sum() + fbu.sum()) / (D * fixed.makespan()),
            "mirrored_idle": float(mir["stall"].sum() + mir["bubble"].sum()) / (D * mir["makespan"])}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--subnets", type=int, default=128)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1_mirroring.md"))
    a = ap.parse_args()
    rows = []
    for label, (name, n) in WORKLOADS.items():
        cfg = cfg_of(name, n)
        for D in (2, 4, 8):
            r = row(label, cfg, a.subnets, D, 0)
            rows.append(r)
            print(json.dumps(r), flush=True)
    with open(a.out.replace(".md", ".json"), "w") as f:
        json.dump(rows, f, indent=1)
    with open(a.out, "w") as f:
        f.write("# Per-subnet partitions with layer mirroring vs the fixed supernet partition (plan level)\n\n")
        f.write("`python tools/mirroring.py` — C++ planners (`naspipe_plan`, `naspipe_plan_mirrored`), default "
                f"integer cost tables, N = {a.subnets} uniformly sampled subnets (seed 0), W = 4D. Speed-up = "
                "D=1 makespan / makespan. Balance = mean over subnets of (largest stage cost / mean stage cost) "
                "of that subnet's tasks (1 = perfectly balanced). Mirror latency = mean candidate fp32 bytes "
                "over 900 GB/s NVLink in 1-us ticks (P:L298's push of updated parameters).\n\n")
        f.write("| workload | D | fixed speed-up | mirrored speed-up | fixed balance | mirrored balance | "
                "blocks off the supernet partition | fixed idle | mirrored idle | mirror latency (ticks) |\n")
        f.write("|---|---|---|---|---|---|---|---|---|---|\n")
        for r in rows:
            f.write(f"| {r['workload']} | {r['D']} | {r['fixed_speedup']:.2f}x | {r['mirrored_speedup']:.2f}x | "
                    f"{r['fixed_balance']:.3f} | {r['mirrored_balance']:.3f} | {100 * r['blocks_off_supernet_partition']:.1f}% | "
                    f"{100 * r['fixed_idle']:.1f}% | {100 * r['mirrored_idle']:.1f}% | {r['mirror_latency_ticks']} |\n")
    print("wrote", a.out)


if __name__ == "__main__":
    main()
