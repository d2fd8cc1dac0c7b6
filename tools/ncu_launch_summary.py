"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list by kernel."""
import collections
import csv
import io
import re
import sys


def load(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    return list(csv.DictReader(io.StringIO("\n".join(lines[start:]))))


def key_of(name):
    m = re.search(r"gemm_tc_kernel<(.*?)>", name)
    if m:
        return "gemm_tc<" + m.group(1).replace("(naspipe::GemmEpi)", "") + ">"
    return re.sub(r"\(.*", "", name).replace("void ", "").replace("naspipe::", "")[:80]


def main(path):
    rows = load(path)
    agg = collections.defaultdict(lambda: [0, 0.0])
    for r in rows:
        v = float(r["Metric Value"])
        u = r["Metric Unit"]
        v = v / 1000 if u in ("ns", "nsecond") else v * 1000 if u in ("ms", "msecond") else v
        k = key_of(r["Kernel Name"])
        agg[k][0] += 1
        agg[k][1] += v
    tot = sum(v[1] for v in agg.values())
    print(f"{len(rows)} launches, {tot:.1f} us total (serialised, cold-cache)")
    for k, (n, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"{t:10.1f} us {100 * t / tot:5.1f}%  n={n:4d}  {k}")


if __name__ == "__main__":
    main(sys.argv[1])
