"""Per-stream busy time of a bench-like run (GPU box): CUPTI kernel records via torch.profiler's
chrome trace, grouped by CUDA stream, plus the wall span.  Shows which stream bounds the step.

    python tools/stream_timeline.py [workload] [steps]
"""
import json
import os
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402


def union(iv):
    iv.sort()
    tot, cur_s, cur_e = 0.0, None, None
    for s, e in iv:
        if cur_e is None or s > cur_e:
            if cur_e is not None:
                tot += cur_e - cur_s
            cur_s, cur_e = s, e
        else:
            cur_e = max(cur_e, e)
    if cur_e is not None:
        tot += cur_e - cur_s
    return tot


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "spos"
    K = int(sys.argv[2]) if len(sys.argv) > 2 else 10
    cfg = synth.get_config(name)
    torch.cuda.set_device(0)
    npipe.naspipe_set_pdl(False)
    h = npipe.naspipe_create(npipe.Spec(cfg), 1)
    ch = synth.sample_choices(3 + K, cfg["n_blocks"], cfg["n_choices"])
    pool = [tuple(torch.from_numpy(a).cuda() for a in synth.make_batch(cfg, y)) for y in range(4)]
    for y in range(3):
        npipe.naspipe_submit(h, ch[y], *pool[y % 4], where=npipe.BATCH_DEVICE)
    npipe.naspipe_drain(h)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for y in range(3, 3 + K):
            npipe.naspipe_submit(h, ch[y], *pool[y % 4], where=npipe.BATCH_DEVICE)
        npipe.naspipe_drain(h)
        torch.cuda.synchronize()
    path = os.path.join(tempfile.mkdtemp(), "t.json")
    prof.export_chrome_trace(path)
    ev = json.load(open(path))["traceEvents"]
    ks = [e for e in ev if e.get("cat") == "kernel"]
    by = {}
    for e in ks:
        st = e.get("args", {}).get("stream", e.get("tid"))
        by.setdefault(st, []).append((e["ts"], e["ts"] + e["dur"], e["name"]))
    t0 = min(e["ts"] for e in ks)
    t1 = max(e["ts"] + e["dur"] for e in ks)
    print(f"{name}: {K} steps, kernel span {(t1 - t0) / 1e3:.2f} ms ({(t1 - t0) / K / 1e3:.3f} ms/step), "
          f"all-stream union {union([(a, b) for v in by.values() for a, b, _ in v]) / K / 1e3:.3f} ms/step")
    for st, v in sorted(by.items(), key=lambda kv: -len(kv[1])):
        busy = union([(a, b) for a, b, _ in v])
        names = {}
        for a, b, n in v:
            names[n[:60]] = names.get(n[:60], 0.0) + (b - a)
        top = sorted(names.items(), key=lambda kv: -kv[1])[:5]
        print(f"  stream {st}: {len(v) / K:.1f} launches/step, busy {busy / K / 1e3:.3f} ms/step "
              f"({busy / (t1 - t0):.2f} of span); top: " + "; ".join(f"{n.split('(')[0][-40:]} {t / K:.0f}us" for n, t in top))
    npipe.naspipe_destroy(h)


if __name__ == "__main__":
    main()
