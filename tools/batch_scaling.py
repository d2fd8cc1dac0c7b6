"""Step time vs batch size (diagnostics: a step time that does not shrink with the batch is
launch/latency-bound, one that scales linearly is bandwidth/compute-bound).

    python tools/batch_scaling.py [--workload spos] [--batches 64,32,16,8] [--steps 20]"""
import argparse
import json
import time
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
if "--pkg" in sys.argv:   # another build of the package first on the path (A/B runs)
    sys.path.insert(0, os.path.abspath(sys.argv[sys.argv.index("--pkg") + 1]))
import torch  # noqa: E402
import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--workload", default="spos")
ap.add_argument("--batches", default="64,32,16,8")
ap.add_argument("--steps", type=int, default=20)
ap.add_argument("--pkg", default=None)
a = ap.parse_args()
for B in (int(b) for b in a.batches.split(",")):
    cfg = dict(synth.get_config(a.workload), batch=B)
    choices = synth.sample_choices(3 + a.steps, cfg["n_blocks"], cfg["n_choices"])
    pool = [synth.make_batch(cfg, y) for y in range(2)]
    dev = [(torch.from_numpy(x).cuda(), torch.from_numpy(t).cuda()) for x, t in pool]
    h = npipe.naspipe_create(npipe.Spec(cfg), 1)
    for y in range(3):
        npipe.naspipe_submit(h, choices[y], *dev[y % 2], where=npipe.BATCH_DEVICE)
    npipe.naspipe_drain(h)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    t0 = time.perf_counter()
    for y in range(3, 3 + a.steps):
        npipe.naspipe_submit(h, choices[y], *dev[y % 2], where=npipe.BATCH_DEVICE)
    t1 = time.perf_counter()
    npipe.naspipe_drain(h)
    e1.record()
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    ms = e0.elapsed_time(e1) / a.steps
    npipe.naspipe_destroy(h)
    print(json.dumps({"pkg": a.pkg, "workload": a.workload, "batch": B, "ms_per_step": ms, "samples_per_s": B / ms * 1e3,
                      "host_submit_ms_per_step": (t1 - t0) * 1e3 / a.steps, "host_total_ms_per_step": (t2 - t0) * 1e3 / a.steps}))
