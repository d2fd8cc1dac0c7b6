"""Projected samples/s at 2/4/8 stages for BJ's configs from the measured one-GPU step.

This round's boxes have one GPU, so the multi-stage throughput is projected with the C++
planner (the schedule the executor runs): the analytic per-(block, choice) cost table
(naspipe_default_costs) is rescaled so that the mean subnet costs the MEASURED one-stage
step (bench.py's ms_per_step); every stage boundary adds lambda = one boundary tensor over
900 GB/s NVLink (+ 5 us launch/sync latency) in 1-us ticks; N = 256 subnets, W = 4D, strict
backward-first.  projected samples/s = N * B / makespan.  This is the CSP-plan bound with
measured costs (SURVEY §8d fraction 3's denominator), not a measurement.

    python tools/projection.py [--bench profiles/r1_bench_v12_default_spos.json]
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


def boundary_bytes(cfg):
    """bytes of the largest stage-boundary tensor (activation in, gradient back)."""
    if cfg["family"] == "spos":   # bf16x2 block outputs: 2 planes x 2 B x B*H*W*C at 56x56x64
        return 2 * 2 * cfg["batch"] * (cfg["image_hw"] // 4) ** 2 * cfg["stage_channels"][0]
    return 4 * cfg["batch"] * cfg["seq_len"] * cfg["d_model"]   # fp32 [T, d]


def project(cfg, step_ms, N=256):
    spec = npipe.Spec(cfg)
    cf, cb = npipe.naspipe_default_costs(spec)
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = synth.sample_choices(N, m, n)
    mean_sub = np.mean([sum(int(cf[b, c]) + int(cb[b, c]) for b, c in enumerate(row)) for row in choices])
    scale = step_ms * 1000.0 / mean_sub
    cfs = np.maximum(1, np.round(cf * scale)).astype(np.int32)
    cbs = np.maximum(1, np.round(cb * scale)).astype(np.int32)
    lam = int(np.ceil(boundary_bytes(cfg) / 900e9 * 1e6 + 5))
    rows = []
    for D in (1, 2, 4, 8):
        s = npipe.Spec(dict(cfg, cost_fwd=cfs, cost_bwd=cbs, window=4 * D, link_latency=lam if D > 1 else 0))
        p = npipe.naspipe_plan(s, D, choices)
        st, bu = p.idle(D)
        mk = p.makespan()
        rows.append({"D": D, "makespan_ms": mk / 1000.0, "samples_per_s": N * cfg["batch"] / (mk / 1e6),
                     "stall_frac": float(st.sum()) / (D * mk), "bubble_frac": float(bu.sum()) / (D * mk),
                     "link_latency_us": lam if D > 1 else 0})
    for r in rows:
        r["speedup_vs_1"] = r["samples_per_s"] / rows[0]["samples_per_s"]
    return rows


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--bench", default=os.path.join(ROOT, "profiles", "r1_bench_v12_default_spos.json"))
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r1_projection.md"))
    a = ap.parse_args()
    d = json.loads(open(a.bench).read().strip().splitlines()[-1])
    cases = [("configs[1] SPOS CNN", synth.get_config("spos"), d["ms_per_step"])]
    sec = d.get("secondary", {}).get("configs[2] transformer")
    if sec and "ms_per_step" in sec:
        cases.append(("configs[2] transformer", synth.get_config("transformer"), sec["ms_per_step"]))
    out = {}
    with open(a.out, "w") as f:
        f.write("# Projected throughput at 1/2/4/8 stages (CSP plan with measured step cost)\n\n")
        f.write(f"`python tools/projection.py` from `{os.path.relpath(a.bench, ROOT)}`: analytic cost table rescaled "
                "to the measured one-stage step, boundary latency = one boundary tensor over 900 GB/s NVLink + 5 us, "
                "N = 256 uniformly sampled subnets, W = 4D. A projection (this round's boxes have one GPU), not a "
                "measurement.\n\n")
        for label, cfg, ms in cases:
            rows = project(cfg, ms)
            out[label] = rows
            f.write(f"## {label} (measured one-stage step {ms:.2f} ms)\n\n")
            f.write("| D | projected samples/s | speed-up vs D=1 | stall frac | bubble frac | link latency (us) |\n")
            f.write("|---|---|---|---|---|---|\n")
            for r in rows:
                f.write(f"| {r['D']} | {r['samples_per_s']:.0f} | {r['speedup_vs_1']:.2f}x | {r['stall_frac']:.3f} | "
                        f"{r['bubble_frac']:.3f} | {r['link_latency_us']} |\n")
            f.write("\n")
            print(label, json.dumps(rows))
    with open(a.out.replace(".md", ".json"), "w") as f:
        json.dump(out, f, indent=1)
    print("wrote", a.out)


if __name__ == "__main__":
    main()
