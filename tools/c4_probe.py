"""configs[3] context-switch probe: per-subnet device time with the bench's budget (diagnostics).

    python tools/c4_probe.py [--budget-x 3] [--subnets 6]"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402
import synth  # noqa: E402
import bench  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--budget-x", type=float, default=3.0)
ap.add_argument("--subnets", type=int, default=6)
ap.add_argument("--no-drain", action="store_true", help="submit all subnets, drain once at the end")
a = ap.parse_args()
cfg = synth.get_config("large_transformer")
t0 = time.time()
budget = bench.stage_budget(cfg, 1, a.budget_x, npipe)
h = npipe.naspipe_create(npipe.Spec(cfg, hbm_weight_budget_bytes=budget), 1)
print(f"create {time.time() - t0:.1f}s budget {budget / 1e9:.2f} GB", flush=True)
choices = synth.sample_choices(a.subnets, cfg["n_blocks"], cfg["n_choices"])
x, t = synth.make_batch(cfg, 0)
xd, td = torch.from_numpy(x).cuda(), torch.from_numpy(t).cuda()
for y in range(a.subnets):
    t1 = time.time()
    npipe.naspipe_submit(h, choices[y], xd, td, where=npipe.BATCH_DEVICE)
    if a.no_drain:
        print(f"submitted {y} in {1e3 * (time.time() - t1):.1f} ms", flush=True)
        continue
    npipe.naspipe_drain(h)
    s = npipe.naspipe_get_stats(h)
    print(f"subnet {y}: {1e3 * (time.time() - t1):.1f} ms  loads {s['res_loads']:.0f} evicts {s['res_evicts']:.0f} "
          f"h2d {s['h2d_bytes'] / 1e9:.1f} GB d2h {s['d2h_bytes'] / 1e9:.1f} GB", flush=True)
if a.no_drain:
    t1 = time.time()
    npipe.naspipe_drain(h)
    print(f"drain {1e3 * (time.time() - t1):.1f} ms", flush=True)
npipe.naspipe_destroy(h)
