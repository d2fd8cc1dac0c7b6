"""Per-kernel device time per step of a bench-like run (GPU box), CUPTI records via
torch.profiler, PDL off (a kernel's interval then excludes its wait for the predecessor),
grouped by (stream, kernel name).  Used for the A/B of kernel fusions:

    NASPIPE_SPOS_FUSE_BNB=0 python tools/kernel_table.py [workload] [steps]
"""
import json
import os
import sys
import tempfile

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from torch.profiler import ProfilerActivity, profile  # noqa: E402

import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402
from tools.stream_timeline import union  # noqa: E402


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
    ks = [e for e in json.load(open(path))["traceEvents"] if e.get("cat") == "kernel"]
    t0 = min(e["ts"] for e in ks)
    t1 = max(e["ts"] + e["dur"] for e in ks)
    env = {k: v for k, v in os.environ.items() if k.startswith("NASPIPE_")}
    print(f"{name} {env}: span {(t1 - t0) / K / 1e3:.3f} ms/step")
    by = {}
    for e in ks:
        st = e.get("args", {}).get("stream", e.get("tid"))
        by.setdefault(st, []).append(e)
    for st, v in sorted(by.items(), key=lambda kv: -len(kv[1])):
        busy = union([(e["ts"], e["ts"] + e["dur"]) for e in v])
        print(f"  stream {st}: {len(v) / K:.1f} launches/step busy {busy / K:.0f} us/step")
        agg = {}
        for e in v:
            n = e["name"].replace("(anonymous namespace)::", "").replace("void ", "").split("(")[0][-70:]
            a = agg.setdefault(n, [0, 0.0])
            a[0] += 1
            a[1] += e["dur"]
        durs = {}
        for e in v:
            n = e["name"].replace("(anonymous namespace)::", "").replace("void ", "").split("(")[0][-70:]
            durs.setdefault(n, []).append((e["dur"], str(e.get("args", {}).get("grid", ""))))
        for n, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            d = sorted(x for x, _ in durs[n])
            q = lambda f: d[min(len(d) - 1, int(f * len(d)))]  # noqa: E731
            print(f"    {t / K:8.1f} us {c / K:6.1f}x  {t / c:7.2f} us/launch  [min {d[0]:.1f} p50 {q(0.5):.1f} "
                  f"p90 {q(0.9):.1f} max {d[-1]:.1f}]  {n}")
            if os.environ.get("KT_GRIDS") and ("bn_" in n or "dw_" in n):
                by = {}
                for x, g in durs[n]:
                    by.setdefault(g, []).append(x)
                for g, xs in sorted(by.items(), key=lambda kv: -sum(kv[1])):
                    print(f"        grid {g}: {len(xs) / K:.1f}x  mean {sum(xs) / len(xs):.1f} us")
    npipe.naspipe_destroy(h)


if __name__ == "__main__":
    main()
