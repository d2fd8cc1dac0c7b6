"""Which outputs differ between two identical runs (diagnostics for bench.bit_repro).

    python tools/repro_diag.py [--workload spos] [--subnets 1]"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if "--pkg" in sys.argv:   # another build of the package first on the path
    sys.path.insert(0, os.path.abspath(sys.argv[sys.argv.index("--pkg") + 1]))
import torch  # noqa: E402
import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="spos")
ap.add_argument("--subnets", type=int, default=1)
ap.add_argument("--batch", type=int, default=0)
ap.add_argument("--hw", type=int, default=0)
ap.add_argument("--pkg", default=None)
a = ap.parse_args()
cfg = synth.get_config(a.workload)
if a.batch:
    cfg = dict(cfg, batch=a.batch)
if a.hw:
    cfg = dict(cfg, image_hw=a.hw)
m, n = cfg["n_blocks"], cfg["n_choices"]
choices = synth.sample_choices(a.subnets, m, n)
batches = [synth.make_batch(cfg, y) for y in range(a.subnets)]
dev = [(torch.from_numpy(x).cuda(), torch.from_numpy(t).cuda()) for x, t in batches]
runs = []
for rep in range(3):
    h = npipe.naspipe_create(npipe.Spec(cfg), 1)
    for y in range(a.subnets):
        npipe.naspipe_submit(h, choices[y], *dev[y], where=npipe.BATCH_DEVICE)
    npipe.naspipe_drain(h)
    p = {(b, int(choices[y][b])): npipe.naspipe_get_params(h, b, int(choices[y][b]))
         for y in range(a.subnets) for b in range(m)}
    runs.append((npipe.naspipe_get_losses(h, a.subnets), p))
    npipe.naspipe_destroy(h)
print("package", npipe.__file__, "choices", choices.tolist())
for rep in (1, 2):
    l0, p0 = runs[0]
    l1, p1 = runs[rep]
    print(f"run0 vs run{rep}: losses equal {np.array_equal(l0.view(np.uint32), l1.view(np.uint32))} {l0} {l1}")
    for k in sorted(p0):
        d = np.nonzero(p0[k].view(np.uint32) != p1[k].view(np.uint32))[0]
        if len(d):
            print(f"  cand {k}: {len(d)} of {len(p0[k])} differ, first idx {d[:5].tolist()} "
                  f"maxabs {np.max(np.abs(p0[k][d] - p1[k][d])):.3e}")
