"""Build profiles/dominant_traffic.json (read by bench.py's roofline `traffic`) from the raw
ncu --set full CSVs of the bench's timed region (tools/gpu_r2b_final.sh):

    python tools/make_dominant_traffic.py <spos_bn_raw.csv> <tf_raw.csv> [tag]

spos: the BatchNorm kernel family (bn_apply, bn_bwd_reduce, bn_bwd_apply) -- DRAM read +
write bytes per launch, mean over every captured launch.  transformer: the tcgen05 GEMMs --
bytes per launch and the tensor-pipe utilisation, time-weighted."""
import csv
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "us": 1.0, "ms": 1e3, "%": 1.0, "": 1.0,
         "register/thread": 1.0}


def rows(path):
    r = list(csv.reader(open(path)))
    h, units = r[0], r[1]
    out = []
    for x in r[2:]:
        d = {}
        for i, k in enumerate(h):
            v = x[i]
            try:
                d[k] = float(v.replace(",", "")) * SCALE.get(units[i], 1.0)
            except ValueError:
                d[k] = v
        out.append(d)
    return out


def short(name):
    n = re.sub(r"\(anonymous namespace\)::|unnamed>::|void |naspipe::", "", name)
    return n.split("(")[0]


def entry(d):
    return {"kernel": short(d["Kernel Name"]), "us": d["gpu__time_duration.sum"],
            "dram_read": d["dram__bytes_read.sum"], "dram_write": d["dram__bytes_write.sum"],
            "grid": d.get("launch__grid_size"), "regs": d.get("launch__registers_per_thread"),
            "tensor_pipe_pct": d.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"),
            "warps_active_pct": d.get("sm__warps_active.avg.pct_of_peak_sustained_active")}


def main():
    spos_csv, tf_csv = sys.argv[1], sys.argv[2]
    tag = sys.argv[3] if len(sys.argv) > 3 else "r2b"
    bn = [entry(d) for d in rows(spos_csv) if re.search(r"bn_(apply|bwd_apply|bwd_reduce)_kernel", d["Kernel Name"])]
    tf = [entry(d) for d in rows(tf_csv)]
    gemm = [e for e in tf if "gemm" in e["kernel"]]
    tw = sum(e["us"] for e in gemm)
    out = {"source": f"{tag}: ncu --set full --clock-control none --profile-from-start off (NASPIPE_PROFILE_RANGE=1: "
                     "the bench's timed region only), tools/gpu_r2b_final.sh; raw CSV in profiles/"
                     f"{tag}_ncu_*_raw.csv.  DRAM writes that stay in L2 when the kernel ends are not counted.",
           "spos": {"kernel": "BatchNorm kernel family (bn_apply, bn_bwd_reduce, bn_bwd_apply; every launch captured)",
                    "dram_bytes_per_launch_mean": sum(e["dram_read"] + e["dram_write"] for e in bn) / max(1, len(bn)),
                    "launches": bn},
           "transformer": {"kernel": "tcgen05 GEMMs (gemm_pair_kernel / gemm_tc_kernel)",
                           "dram_bytes_per_launch_mean": sum(e["dram_read"] + e["dram_write"] for e in gemm) / max(1, len(gemm)),
                           "tensor_pipe_pct_mean": sum((e["tensor_pipe_pct"] or 0) * e["us"] for e in gemm) / max(tw, 1e-9),
                           "launches": gemm, "other_kernels": [e for e in tf if "gemm" not in e["kernel"]]}}
    with open(os.path.join(ROOT, "profiles", "dominant_traffic.json"), "w") as f:
        json.dump(out, f, indent=1)
    print(len(bn), out["spos"]["dram_bytes_per_launch_mean"], len(gemm), out["transformer"]["tensor_pipe_pct_mean"])


if __name__ == "__main__":
    main()
