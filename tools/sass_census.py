"""SASS census of libnaspipe.so: per kernel, the count of the instructions that prove the
Blackwell-native paths (B200_PROFILING.md "What proves a Blackwell-native kernel"):
UTC*MMA (tcgen05.mma), UTCBAR (tcgen05.commit), LDTM (tcgen05.ld), UTMALDG (TMA loads),
HMMA (legacy mma.sync).  A regression of a GEMM to a non-tcgen05 path shows up here.

    python tools/sass_census.py [--out profiles/r2_sass_census.md]
"""
import argparse
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SO = os.path.join(ROOT, "paper_conf_asplos_zhaolcscwzlc22_b200", "libnaspipe.so")
OPS = ["UTCHMMA", "UTCQMMA", "UTCBAR", "LDTM", "UTMALDG", "UTMASTG", "HMMA", "REDG", "ATOMG", "BAR.SYNC"]


def census(so=SO):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", so], capture_output=True, text=True).stdout
    kernels, cur = {}, None
    for line in out.splitlines():
        m = re.match(r"\s+Function : (\S+)", line)
        if m:
            cur = m.group(1)
            kernels[cur] = {k: 0 for k in OPS}
            continue
        if cur is None:
            continue
        for k in OPS:
            if re.search(r"\b" + re.escape(k) + r"\b", line):
                kernels[cur][k] += 1
    names = {}
    if kernels:
        dem = subprocess.run(["c++filt"], input="\n".join(kernels), capture_output=True, text=True).stdout.split("\n")
        names = dict(zip(kernels, dem))
    return kernels, names


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "r2_sass_census.md"))
    a = ap.parse_args()
    kernels, names = census()
    lines = ["# SASS census of libnaspipe.so (cuobjdump -sass, sm_100a)", "",
             "Counts of instruction mnemonics per kernel (static, not executed counts).  UTCHMMA = tcgen05.mma, "
             "UTCBAR = tcgen05.commit, LDTM = tcgen05.ld, UTMALDG = TMA tensor load, HMMA = legacy mma.sync.", "",
             "| kernel | " + " | ".join(OPS) + " |", "|---|" + "---|" * len(OPS)]
    for k in sorted(kernels, key=lambda k: names.get(k, k)):
        c = kernels[k]
        if not any(c[o] for o in OPS[:7]):
            continue
        lines.append(f"| `{names.get(k, k)[:110]}` | " + " | ".join(str(c[o]) for o in OPS) + " |")
    text = "\n".join(lines) + "\n"
    with open(a.out, "w") as f:
        f.write(text)
    print(text)


if __name__ == "__main__":
    sys.exit(main())
