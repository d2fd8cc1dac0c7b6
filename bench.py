#!/usr/bin/env python
"""Benchmark of the NASPipe hot path on B200 (contract: see DESIGN.md "Measurement").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload NAME]

One step = one subnet trained through the whole pipeline (forward, loss, backward and the
SGD WRITE of every active candidate on every stage) on one synthetic batch.  N = 1 runs the
whole supernet as one stage on one GPU; N > 1 (torchrun, one process per GPU) runs an
N-stage CSP pipeline, stage r on GPU r, the stage boundaries crossing NVLink through the
peer-memory transport (--transport peer, default: the producing kernels store straight into
the next GPU's receive ring) or NCCL send/recv (--transport nccl).

Default workload: configs[1] (SPOS CNN supernet, 20 blocks x 4 choices, 224x224, batch 64).
Printed by rank 0 as ONE JSON line:
* value = samples/s of the whole job with the inputs already resident in HBM (device
  batches), CUDA events on the default stream around the K steps (the drain waits for every
  stage stream), max over ranks;
* e2e = the same through the C ABI with pinned HOST buffers (H2D of input + target inside
  the timed region, D2H of the step losses);
* roofline = the dominant kernel family's algorithmic work (counted by the library per
  launch) over its device time from CUPTI activity records (torch.profiler) of a SEPARATE
  run of the same K steps (no events between kernels, so the kernels run as in `value`);
  SPOS: the BatchNorm kernels against HBM bandwidth; transformer: the tcgen05 GEMMs against
  the sustained bf16 peak;
* fractions = SURVEY §8d's three: kernel, end to end vs the hardware roofline, end to end
  vs the CSP-plan bound (the planner's makespan with per-stage costs calibrated to the
  measured busy time);
* cpu_baseline = the fp64 NumPy oracle on a bounded sample, on this host's cores (and on one);
* secondary = configs[2] (transformer, the tensor-core path) and configs[3] (context
  switching at a 3x budget) measured the same way in child processes.
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import synth  # noqa: E402


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="spos")
    ap.add_argument("--transport", default="peer", choices=["peer", "nccl"],
                    help="stage-boundary transport at N > 1 (include/naspipe.h)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-profile", action="store_true", help="skip the CUPTI kernel-time run (roofline)")
    ap.add_argument("--no-secondary", action="store_true", help="skip the configs[2]/[3] lines embedded in the output")
    ap.add_argument("--no-repro", action="store_true", help="skip the bit-reproducibility digests")
    ap.add_argument("--sync", default="csp", choices=["csp", "inorder", "asp", "bsp"],
                    help="synchronisation policy (include/naspipe.h naspipe_sync; SURVEY §8f(1))")
    ap.add_argument("--recompute", action="store_true",
                    help="activation recomputation (transformer family; P:L282, reading A13)")
    ap.add_argument("--budget-x", type=float, default=0.0,
                    help="HBM weight budget per stage as a multiple of one subnet's mean stage slice "
                         "(0 = all candidates resident; P:L337 uses ~3)")
    ap.add_argument("--n-choices", type=int, default=0, help="override n (search-space sweep, configs[4])")
    ap.add_argument("--virtual-stages", type=int, default=1,
                    help="N = 1: pipeline stages on the one GPU (CSP across concurrently running stage streams)")
    ap.add_argument("--lookahead", type=int, default=0, help="residency prefetch depth L in tasks (0 = 2, P:L156)")
    ap.add_argument("--timed", action="store_true",
                    help="N = 1: the timing-driven executor (NASPIPE_FLAG_TIMED: Alg.1 on observed completions, "
                         "Alg.3's predictor scored) instead of the planned one")
    return ap.parse_args()


def stage_budget(cfg, D, x, npipe):
    """x times the mean fp32 bytes of one subnet's slice on the largest stage."""
    spec = npipe.Spec(cfg)
    sob = npipe.naspipe_partition(spec, D)
    n = cfg["n_choices"]
    per_stage = [0.0] * D
    for b in range(cfg["n_blocks"]):
        per_stage[sob[b]] += np.mean([4 * npipe.naspipe_param_count(spec, b, c) for c in range(n)])
    return int(x * max(per_stage))


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return dict(bf16=d["bf16_tflops"], bf16_sustained=d.get("bf16_tflops_sustained", d["bf16_tflops"]),
                    hbm=d["hbm_gbs"], source="MEASURED_PEAKS.json")
    return dict(bf16=1590.0, bf16_sustained=1400.0, hbm=6650.0, source="fallback (B200_PROFILING.md)")


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 100 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device, self.rows, self.proc = device, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([v.strip() for v in line.split(",")])

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            self.proc.wait()

    def summary(self):
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        sm = [float(r[0]) for r in self.rows if len(r) >= 6 and r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if len(r) >= 6 and r[1].replace(".", "").isdigit()]
        reasons = sorted({names[i] for r in self.rows if len(r) >= 6 for i in range(4)
                          if r[2 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(sm)}


# ------------------------------------------------------------------------------ CPU oracle
def oracle_sample(cfg, k, n_images=None):
    """Time the fp64 oracle (test infrastructure, timing only) on a bounded sample of subnet
    0's step at the FULL batch: sample k = block (k mod m) of subnet 0, forward + backward +
    SGD of that candidate; SPOS adds the frozen stem to block 0's sample and the frozen head
    + cross-entropy to block m-1's, so m consecutive samples are exactly one subnet's work.
    Returns seconds."""
    from oracle import spos, train, transformer, mlp   # noqa: F401
    m = cfg["n_blocks"]
    ch = synth.sample_choices(1, m, cfg["n_choices"])[0]
    x, t = synth.make_batch(cfg, 0)
    b = k % m
    c = int(ch[b])
    segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in train.candidate_layout(cfg, b, c)]
    p = train.unpack(cfg, b, c, synth.init_packed(cfg["init_seed"], b * cfg["n_choices"] + c, segs))
    rng = np.random.default_rng(k)
    if cfg["family"] == "spos":
        s_, inp, _, _, _, H = spos.block_dims(cfg, b)
        cin = inp if s_ == 2 else 2 * inp
        h = rng.standard_normal((cfg["batch"], H, H, cin))
        fz = train.frozen_theta(cfg) if b in (0, m - 1) else None
        t0 = time.perf_counter()
        if b == 0:
            h = spos.stem_fwd(fz, np.asarray(x, dtype=np.float64))
        y, tapes = spos.block_fwd(cfg, b, c, p, h)
        if b == m - 1:
            _, dy = spos.head_loss(fz, y, np.asarray(t, dtype=np.int64))
        else:
            dy = rng.standard_normal(y.shape)
        _, g = spos.block_bwd(cfg, b, c, p, tapes, dy)
        train.sgd_apply({(b, c): p}, {(b, c): g}, cfg["lr"])
        return time.perf_counter() - t0
    h = np.asarray(x, dtype=np.float64) if b == 0 else rng.standard_normal(np.shape(x))
    t0 = time.perf_counter()
    sub = dict(cfg, n_blocks=1)
    loss, grads = train.subnet_step(sub, {(0, c): p}, [c], h, t)
    train.sgd_apply({(0, c): p}, grads, cfg["lr"])
    return time.perf_counter() - t0


def cpu_threads():
    try:
        from threadpoolctl import threadpool_info
        return max((i.get("num_threads", 1) for i in threadpool_info()), default=os.cpu_count())
    except Exception:
        return os.cpu_count()


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def cpu_baseline(cfg):
    """The oracle on a bounded, evenly spaced sample of block positions of subnet 0 at the
    full batch (SPOS: every 2nd block plus the last, stem/head included; transformer: blocks
    0 and m-1), on all host threads, scaled to a whole subnet by m / #sampled; plus block 0
    on ONE thread, scaled to a subnet by the all-thread subnet / block-0 ratio."""
    m = cfg["n_blocks"]
    stride = {"spos": 2, "transformer": max(1, m - 1)}.get(cfg["family"], 1)
    pos = sorted(set(range(0, m, stride)) | {m - 1})
    ts = [oracle_sample(cfg, k) for k in pos]
    per_subnet = float(np.mean(ts)) * m
    one = None
    try:
        from threadpoolctl import threadpool_limits
        with threadpool_limits(limits=1):
            t1 = oracle_sample(cfg, 0)
        one = cfg["batch"] / (t1 * per_subnet / max(ts[0], 1e-9))
    except Exception:
        pass
    return {"value": cfg["batch"] / per_subnet, "unit": "samples/s", "cores": cpu_threads(), "kind": "oracle",
            "cpu_model": cpu_model(), "value_1_thread": one,
            "sample": f"fp64 NumPy oracle, block positions {pos} of subnet 0 at B={cfg['batch']} (fwd+bwd+SGD of "
                      f"the candidate{'; stem at block 0, head + CE at block m-1' if cfg['family'] == 'spos' else ''}),"
                      f" {sum(ts):.1f} s, scaled x{m / len(pos):.2f} to one subnet; 1-thread: block 0 on one thread "
                      f"scaled by the all-thread subnet / block-0 time ratio"}


def run_reference(args, cfg, rank, world):
    """--impl reference: the oracle as it stands, on host cores, rank 0 only.  Step k = block
    (k mod m) of subnet 0 at the full batch (SPOS: + stem at block 0, + head/CE at block m-1),
    so every m consecutive steps are one whole subnet: value = B / (m x mean step time), and
    ms_per_step is the real mean step time (steps x ms_per_step = the timed run)."""
    if rank != 0:
        return
    m = cfg["n_blocks"]
    for k in range(args.warmup):
        oracle_sample(cfg, k)
    ts = [oracle_sample(cfg, args.warmup + k) for k in range(args.steps)]
    # whole-subnet rate from the mean time per block position (every position sampled when K >= m)
    by_pos = {}
    for k, t in enumerate(ts):
        by_pos.setdefault((args.warmup + k) % m, []).append(t)
    per_subnet = sum(np.mean(v) for v in by_pos.values()) * m / len(by_pos)
    value = cfg["batch"] / per_subnet
    cores = cpu_threads()
    sample = (f"step k = block (k mod {m}) of subnet 0 at B={cfg['batch']}, fwd+bwd+SGD in the fp64 oracle "
              f"({'stem/head included at blocks 0/m-1; ' if cfg['family'] == 'spos' else ''}{len(by_pos)} of {m} "
              f"block positions sampled); value = B / (m x mean time per position)")
    print(json.dumps({
        "impl": "reference", "metric": "supernet samples/sec", "value": value, "unit": "samples/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * float(np.mean(ts)),
        "higher_is_better": True, "scaling": "weak" if world > 1 else "strong", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": workload_config(args, cfg, world),
        "cpu_baseline": {"kind": "oracle", "cores": cores, "cpu_model": cpu_model(), "sample": sample, "value": value,
                         "unit": "samples/s"},
        "e2e": {"value": value, "unit": "samples/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}))


def _traffic(family):
    """dram bytes per launch of the dominant kernel from the committed ncu --set full summary."""
    p = os.path.join(ROOT, "profiles", "dominant_traffic.json")
    if not os.path.exists(p):
        return None
    with open(p) as f:
        d = json.load(f).get(family)
    if d is None:
        return None
    out = {"dram_bytes_per_launch": d["dram_bytes_per_launch_mean"],
           "source": d.get("source", "profiles/dominant_traffic.json (ncu --set full capture)")}
    if "tensor_pipe_pct_mean" in d:   # sm__pipe_tensor_cycles_active, time-weighted over the captured GEMMs
        out["tensor_pipe_pct"] = d["tensor_pipe_pct_mean"]
    return out


def secondary(args, workload, extra=(), steps=None):
    """Another config measured by this script in a child process (started before this
    process touches the GPU), reported beside the headline line."""
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--workload", workload, "--steps", str(steps or args.steps),
           "--warmup", str(args.warmup), "--no-cpu", "--no-e2e", "--no-secondary"] + list(extra)
    try:
        out = subprocess.run(cmd, capture_output=True, text=True, timeout=600).stdout.strip().splitlines()
        d = json.loads(out[-1])
        return {k: d.get(k) for k in ("value", "unit", "ms_per_step", "config", "roofline", "fractions", "clocks",
                                      "gpu_launches", "bit_repro", "context_switch")}
    except Exception as e:  # reported, never fatal for the headline line
        return {"error": repr(e)[:200]}


# ------------------------------------------------------------------------------ CUPTI kernel times
KERNEL_FAMILIES = {"spos": ("bn_stats", "bn_apply", "bn_bwd_reduce", "bn_bwd_apply", "bn_write"),
                   "transformer": ("gemm_tc", "gemm_pair")}


def profile_kernels(run):
    """Run `run()` under torch.profiler with CUDA activity only (CUPTI activity records of
    every kernel of the process, including libnaspipe.so's).  Returns ({name: [count, us]},
    busy_us = union of the kernel intervals)."""
    import torch
    from torch.profiler import ProfilerActivity, profile
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        run()
        torch.cuda.synchronize()
    per, iv = {}, []
    for e in prof.events():
        if "cuda" not in str(getattr(e, "device_type", "")).lower():
            continue
        name = e.name
        if name.startswith(("Memcpy", "Memset", "cudaMemcpy", "cudaMemset")) or "memcpy" in name.lower():
            continue
        t0, t1 = e.time_range.start, e.time_range.end
        c = per.setdefault(name, [0, 0.0])
        c[0] += 1
        c[1] += float(t1 - t0)
        iv.append((t0, t1))
    iv.sort()
    busy, cur0, cur1 = 0.0, None, None
    for a, b in iv:
        if cur1 is None or a > cur1:
            if cur1 is not None:
                busy += cur1 - cur0
            cur0, cur1 = a, b
        else:
            cur1 = max(cur1, b)
    if cur1 is not None:
        busy += cur1 - cur0
    return per, float(busy)


def family_time(per, family):
    keys = KERNEL_FAMILIES[family]
    n = us = 0
    for name, (c, t) in per.items():
        if any(k in name for k in keys):
            n += c
            us += t
    return n, us


def plan_bound_ms(cfg, npipe, choices, D, busy_us):
    """SURVEY §8d fraction 3's denominator: the CSP planner's makespan for these subnets with
    the analytic per-(block, choice) cost table rescaled per stage so that stage r's planned
    busy time equals rank r's measured kernel busy time; boundary latency = one boundary
    tensor over 900 GB/s + 2 us."""
    spec = npipe.Spec(cfg)
    sob = np.asarray(npipe.naspipe_partition(spec, D))
    cf, cb = npipe.naspipe_default_costs(spec)
    m = cfg["n_blocks"]
    planned = np.zeros(D)
    for row in choices:
        for b in range(m):
            planned[sob[b]] += int(cf[b, row[b]]) + int(cb[b, row[b]])
    scale = np.asarray(busy_us, dtype=np.float64) / np.maximum(planned, 1)
    sc = scale[sob][:, None]
    cfs = np.maximum(1, np.round(cf * sc)).astype(np.int32)
    cbs = np.maximum(1, np.round(cb * sc)).astype(np.int32)
    if cfg["family"] == "spos":
        bb = 2 * 2 * cfg["batch"] * (cfg["image_hw"] // 4) ** 2 * cfg["stage_channels"][0]
    elif cfg["family"] == "transformer":
        bb = 4 * cfg["batch"] * cfg["seq_len"] * cfg["d_model"]
    else:
        bb = 4 * cfg["batch"] * cfg["width"]
    lam = int(np.ceil(bb / 900e9 * 1e6 + 2)) if D > 1 else 0
    s = npipe.Spec(dict(cfg, cost_fwd=cfs, cost_bwd=cbs, stage_of_block=sob.astype(np.int32), link_latency=lam))
    return npipe.naspipe_plan(s, D, choices).makespan() / 1000.0


def algorithmic_work(cfg, st, steps, choices=None):
    """(work per step, unit, peak key) of the whole step for fraction 2: transformer = GEMM
    flops (library counter) + attention flops (12 B S^2 d per attention block, fwd + bwd; the
    NLP conv ops of A38 count their GEMMs only); SPOS = none beyond the counted BatchNorm
    bytes (its other kernels' bytes are not counted: the fraction is then a lower bound)."""
    if cfg["family"] == "transformer":
        ops = np.asarray(cfg.get("choice_op", [0] * cfg["n_choices"]))
        n_att = (float(np.mean(np.sum(ops[np.asarray(choices)] == 0, axis=1))) if choices is not None
                 else float(np.sum(ops == 0)) / len(ops) * cfg["n_blocks"])
        att = 12.0 * cfg["batch"] * cfg["seq_len"] ** 2 * cfg["d_model"] * n_att
        return st["gemm_flops"] / steps + att, "flop", "bf16_sustained"
    return None, None, None


def workload_config(args, cfg, world):
    names = {"transformer": "configs[2] transformer", "large_transformer": "configs[3] large_transformer",
             "toy": "configs[0] toy", "spos": "configs[1] SPOS CNN",
             "cv_c3": "CV.c3 analog (Table 1: 32 blocks x 12 choices, Table 5 ops incl. dilated)",
             "nlp_c3": "NLP.c3 analog (Table 1: 48 blocks x 24 choices, Table 5 NLP ops)",
             "nlp_c2": "NLP.c2 analog (Table 1: 48 blocks x 48 choices, Table 5 NLP ops)",
             "nlp_c1": "NLP.c1 analog (Table 1: 48 blocks x 72 choices, Table 5 NLP ops)",
             "nlp_c0": "NLP.c0 analog (Table 1: 48 blocks x 96 choices, Table 5 NLP ops)",
             "cv_c2": "CV.c2 analog (Table 1: 32 blocks x 24 choices, Table 5 ops incl. dilated)",
             "cv_c1": "CV.c1 analog (Table 1: 32 blocks x 48 choices, Table 5 ops incl. dilated)",
             "spos_dense": "configs[1] geometry with Table 5's dense Conv 3x3 candidate (A40)"}
    c = {"workload": names.get(args.workload, args.workload) if not args.n_choices
         else f"configs[4] sweep n={args.n_choices}",
         "n_blocks": cfg["n_blocks"], "n_choices": cfg["n_choices"], "batch": cfg["batch"],
         "stages": world, "parallelism": f"pp{world}" if world > 1 else "single stage",
         "activation_recompute": bool(getattr(args, "recompute", False)),
         "sync_policy": getattr(args, "sync", "csp"),
         "executor": "timing-driven (Alg.1 on observed completions)" if getattr(args, "timed", False) else "planned",
         "virtual_stages": getattr(args, "virtual_stages", 1),
         "l2": "working set > L2 (active weights + activations per step >> 126 MB)",
         # reduction-order / launch tuning knobs in effect (empty = the library defaults):
         # bitwise comparisons carry their reduction configuration
         "env_knobs": {k: v for k, v in sorted(os.environ.items()) if k.startswith("NASPIPE_")}}
    if cfg["family"] == "transformer":
        c.update(seq_len=cfg["seq_len"], d_model=cfg["d_model"], heads=cfg["choice_heads"], ffn=cfg["choice_ffn"])
        if "choice_op" in cfg:
            c["op"] = cfg["choice_op"]
    if cfg["family"] == "spos":
        c.update(image_hw=cfg["image_hw"], stage_repeats=cfg["stage_repeats"], stage_channels=cfg["stage_channels"],
                 choice_kernel=cfg["choice_kernel"], choice_xception=cfg["choice_xception"],
                 choice_dilation=cfg.get("choice_dilation", [1] * cfg["n_choices"]),
                 num_classes=cfg["num_classes"])
    return c


def bit_repro_digests(cfg, npipe, dev_pool, n_sub, make_handle, blocks):
    """Train n_sub subnets with a fresh handle; SHA-256 per trained candidate of `blocks`
    (fp32 masters) and of the losses (if this handle has them)."""
    import hashlib
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = synth.sample_choices(n_sub, m, n)
    used = sorted({(b, int(choices[y][b])) for y in range(n_sub) for b in range(m) if b in blocks})
    h, has_loss = make_handle()
    for y in range(n_sub):
        x, t = dev_pool[y % len(dev_pool)]
        npipe.naspipe_submit(h, choices[y], x, t, where=npipe.BATCH_DEVICE)
    npipe.naspipe_drain(h)
    out = {f"{b},{c}": hashlib.sha256(np.ascontiguousarray(npipe.naspipe_get_params(h, b, c),
                                                            dtype=np.float32).tobytes()).hexdigest()
           for b, c in used}
    if has_loss:
        out["losses"] = hashlib.sha256(np.ascontiguousarray(npipe.naspipe_get_losses(h, n_sub),
                                                            dtype=np.float32).tobytes()).hexdigest()
    npipe.naspipe_destroy(h)
    return out


def combine(d):
    import hashlib
    sha = hashlib.sha256()
    for k in sorted(d):
        sha.update(f"{k}={d[k]};".encode())
    return sha.hexdigest()


# ------------------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if os.environ.get("NASPIPE_BENCH_SHARE_GPU"):  # test only: every rank on GPU 0 (1-GPU boxes)
        local = 0
    cfg = synth.get_config(args.workload) if args.n_choices == 0 else synth.sweep_config(args.n_choices)
    if args.impl == "reference":
        run_reference(args, cfg, rank, world)
        return
    # the embedded lines run in child processes BEFORE this process touches the GPU (a child
    # started while the parent holds a CUDA context stalled on the box)
    sec = None
    if world == 1 and args.workload == "spos" and not args.no_secondary and not args.n_choices:
        sec = {"configs[2] transformer": secondary(args, "transformer"),
               "configs[3] large_transformer (budget 3x, context switching)":
                   secondary(args, "large_transformer", ["--budget-x", "3", "--no-repro"], steps=min(args.steps, 12)),
               "CV.c3 analog (32 x 12, dilated candidates)": secondary(args, "cv_c3", ["--no-repro"]),
               "NLP.c3 analog (48 x 24, Table 5 NLP ops)": secondary(args, "nlp_c3", ["--no-repro"])}

    import torch
    import torch.distributed as dist
    import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe

    torch.cuda.set_device(local)
    if world > 1:
        if os.environ.get("NASPIPE_BENCH_SHARE_GPU"):  # NCCL refuses two ranks on one GPU
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    D = world
    m, n, B = cfg["n_blocks"], cfg["n_choices"], cfg["batch"]
    total = args.warmup + 4 * args.steps
    choices = synth.sample_choices(total, m, n)
    # device-resident input pool (value run) and pinned host pool (e2e run)
    pool = [synth.make_batch(cfg, y) for y in range(4)]
    dev_pool = [(torch.from_numpy(x).cuda(), torch.from_numpy(t).cuda()) for x, t in pool]
    host_pool = [(torch.from_numpy(x).pin_memory(), torch.from_numpy(t).pin_memory()) for x, t in pool]
    budget = stage_budget(cfg, D, args.budget_x, npipe) if args.budget_x > 0 else 0
    assert not (args.timed and world > 1), "--timed: one process (stages on this GPU via --virtual-stages)"
    spec = npipe.Spec(cfg, hbm_weight_budget_bytes=budget, lookahead=args.lookahead, sync=args.sync,
                      flags=(npipe.FLAG_RECOMPUTE if args.recompute else 0) | (npipe.FLAG_TIMED if args.timed else 0))

    def create(sp):
        if world == 1:
            return npipe.naspipe_create(sp, args.virtual_stages)
        if args.transport == "nccl":
            ids = [None]
            if rank == 0:
                ids[0] = b"".join(npipe.naspipe_nccl_unique_id() for _ in range(2 * (D - 1)))
            dist.broadcast_object_list(ids, src=0)
            return npipe.naspipe_create_rank(sp, D, rank, local, ids[0])
        hh = npipe.naspipe_create_rank_peer(sp, D, rank, local)
        blobs = [None] * D
        dist.all_gather_object(blobs, npipe.naspipe_peer_export(hh))
        npipe.naspipe_peer_connect(hh, blobs[rank - 1] if rank > 0 else None, blobs[rank + 1] if rank < D - 1 else None)
        return hh

    h = create(spec)

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def reduce(v, op="max"):
        if world == 1:
            return v
        t = torch.tensor([v], device="cpu" if dist.get_backend() == "gloo" else "cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX if op == "max" else dist.ReduceOp.SUM)
        return float(t.item())

    def gather(obj):
        if world == 1:
            return [obj]
        out = [None] * world
        dist.all_gather_object(out, obj)
        return out

    state = {"y": 0}

    def steps(where=npipe.BATCH_DEVICE):
        p = dev_pool if where == npipe.BATCH_DEVICE else host_pool
        for _ in range(args.steps):
            x, t = p[state["y"] % 4]
            npipe.naspipe_submit(h, choices[state["y"]], x, t, where=where)
            state["y"] += 1
        npipe.naspipe_drain(h)

    for _ in range(args.warmup):
        x, t = dev_pool[state["y"] % 4]
        npipe.naspipe_submit(h, choices[state["y"]], x, t, where=npipe.BATCH_DEVICE)
        state["y"] += 1
    npipe.naspipe_drain(h)

    # ---- timed region 1: inputs resident in HBM
    s0 = npipe.naspipe_get_stats(h)
    y0 = state["y"]
    barrier()
    prof = os.environ.get("NASPIPE_PROFILE_RANGE") == "1"   # ncu --profile-from-start off
    if prof:
        torch.cuda.profiler.start()
    with ClockSampler(local) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        steps()
        e1.record()
        torch.cuda.synchronize()
    if prof:
        torch.cuda.profiler.stop()
    s1 = npipe.naspipe_get_stats(h)
    # the default-stream events bracket the drain (host waits for every stage stream), so
    # the elapsed time covers all device work of the K steps
    ms = reduce(e0.elapsed_time(e1))
    value = args.steps * B / (ms / 1000)
    launches = reduce(s1["kernel_launches"] - s0["kernel_launches"], "sum")
    timed_choices = choices[y0:y0 + args.steps]

    # ---- kernel times: the same K steps again under CUPTI activity tracing (not used for
    # `value`); the library counts the dominant family's algorithmic work per launch
    pk = peaks()
    roofline = fractions = kernels_top = None
    if not args.no_profile:
        barrier()
        s2 = npipe.naspipe_get_stats(h)
        npipe.naspipe_set_pdl(False)   # each kernel's CUPTI interval = its own execution (no PDL overlap)
        per, busy_us = profile_kernels(steps)
        npipe.naspipe_set_pdl(True)
        s3 = npipe.naspipe_get_stats(h)
        fam = "spos" if cfg["family"] == "spos" else "transformer"
        fn, fus = family_time(per, fam)
        work = s3["dominant_flops"] - s2["dominant_flops"]
        if fam == "transformer":   # GEMM flops are counted by the GEMM launcher itself
            work = s3["gemm_flops"] - s2["gemm_flops"]
        dominant_us = reduce(fus, "sum")
        work = reduce(work, "sum")
        kern_total_us = reduce(sum(t for _, t in per.values()), "sum")
        if fam == "spos":
            achieved = work / (dominant_us * 1e-6) / 1e9 if dominant_us else None
            roofline = {"bound": "hbm", "kernel": "BatchNorm kernel family (" + ", ".join(KERNEL_FAMILIES[fam]) + ")",
                        "achieved": achieved, "peak": pk["hbm"], "unit": "GB/s",
                        "peak_source": pk["source"] + " hbm_gbs (copy bandwidth)",
                        "algorithmic_bytes_per_step": work / args.steps}
        else:
            achieved = work / (dominant_us * 1e-6) / 1e12 if dominant_us else None
            roofline = {"bound": "tensor", "kernel": "tcgen05 GEMMs (gemm_pair_kernel / gemm_tc_kernel, all shapes)",
                        "achieved": achieved, "peak": pk["bf16_sustained"], "unit": "TFLOP/s",
                        "peak_source": pk["source"] + " bf16_tflops_sustained (kernels inside a long step)",
                        "algorithmic_flops_per_step": work / args.steps}
        roofline.update({"frac": achieved / roofline["peak"] if achieved else None, "traffic": _traffic(fam),
                         "timing": "CUPTI activity records (torch.profiler, CUDA activity only) of a separate run "
                                   "of the same K steps, no events between kernels, PDL off in that run so a "
                                   "kernel's interval excludes its wait for the predecessor",
                         "launches": reduce(fn, "sum"), "device_us": dominant_us,
                         "share_of_kernel_time": dominant_us / kern_total_us if kern_total_us else None})
        # GEMM tensor utilisation in this run (algorithmic flops / GEMM device time / peak)
        gn, gus = family_time(per, "transformer")
        gflops = reduce(s3["gemm_flops"] - s2["gemm_flops"], "sum")
        gus = reduce(gus, "sum")
        roofline["gemm_tensor_util"] = {
            "value": (gflops / (gus * 1e-6) / 1e12) / pk["bf16_sustained"] if gus else None,
            "tflops": gflops / (gus * 1e-6) / 1e12 if gus else None, "launches": reduce(gn, "sum"),
            "note": "algorithmic GEMM flops / GEMM device time (CUPTI) / sustained bf16 peak; SPOS counts one "
                    "bf16 product per 3-pass bf16x2 GEMM"}
        busy = gather(busy_us)
        w_step, w_unit, w_peak = algorithmic_work(cfg, {"gemm_flops": gflops}, args.steps, timed_choices)
        e2e_hw = None
        if w_step is not None:
            e2e_hw = (w_step * 1e-12) / (D * pk[w_peak] * (ms / args.steps / 1000))
        elif fam == "spos":
            e2e_hw = (roofline["algorithmic_bytes_per_step"] * 1e-9) / (D * pk["hbm"] * (ms / args.steps / 1000))
        # every kernel's algorithmic HBM bytes (stats all_bytes, counted by the library at each
        # launch) over the value region: the whole step against the HBM roofline
        all_b = reduce(s1["all_bytes"] - s0["all_bytes"], "sum") / args.steps
        e2e_all = (all_b / (D * pk["hbm"] * 1e9 * (ms / args.steps / 1000))) if all_b > 0 else None
        plan_ms = (plan_bound_ms(cfg, npipe, timed_choices, D, [b for b in busy])
                   if args.sync == "csp" and args.virtual_stages == 1 else None)
        fractions = {"kernel": roofline["frac"],
                     "end_to_end_vs_hardware": e2e_hw,
                     "end_to_end_vs_hardware_note": ("(GEMM + attention flops) / (D x sustained bf16 peak x step time)"
                                                     if fam == "transformer" else
                                                     "BatchNorm algorithmic bytes only / (D x HBM peak x step time): "
                                                     "a lower bound (the conv kernels' bytes are not counted)"),
                     "end_to_end_all_kernels_vs_hbm": e2e_all,
                     "all_kernels_bytes_per_step": all_b if all_b > 0 else None,
                     "end_to_end_all_kernels_note": ("every SPOS kernel's algorithmic HBM bytes (each tensor read / "
                                                     "written once per launch at its stored width) / (D x HBM peak x "
                                                     "step time)") if e2e_all else None,
                     "end_to_end_vs_csp_plan": (plan_ms / ms) if plan_ms else None,
                     "csp_plan_ms": plan_ms, "measured_ms": ms, "busy_ms_per_rank": [b / 1000 for b in busy]}
        top = sorted(per.items(), key=lambda kv: -kv[1][1])[:14]
        kernels_top = [{"name": k[:90], "launches": c, "us": round(t, 1)} for k, (c, t) in top]

    # ---- timed region 3: end to end through the C ABI with pinned host buffers
    e2e = None
    if not args.no_e2e:
        barrier()
        e0.record()
        steps(npipe.BATCH_HOST)
        if rank == world - 1:
            npipe.naspipe_get_losses(h, state["y"])[-args.steps:]   # D2H of the step results
        e1.record()
        torch.cuda.synchronize()
        ms2 = reduce(e0.elapsed_time(e1))
        x, t = host_pool[0]
        e2e = {"value": args.steps * B / (ms2 / 1000), "unit": "samples/s",
               "h2d_bytes_per_step": x.numel() * x.element_size() + t.numel() * t.element_size(),
               "d2h_bytes_per_step": 4}
    timed_stats = npipe.naspipe_get_timed_stats(h) if args.timed else None
    losses = npipe.naspipe_get_losses(h, state["y"]) if rank == world - 1 else None
    loss_ok = bool(losses is None or np.all(np.isfinite(losses)))
    loss_ok = reduce(0.0 if loss_ok else 1.0) == 0.0
    npipe.naspipe_destroy(h)

    # ---- bit reproducibility (Def.1; Table 3; artifact P:L557-561)
    repro = None
    if not args.no_repro and not args.budget_x:
        n_sub = 8
        if world == 1:
            runs = []
            for Dr in (1, 1, 2, 4):
                if Dr > m:
                    continue
                dg = bit_repro_digests(cfg, npipe, dev_pool, n_sub,
                                       lambda: (npipe.naspipe_create(npipe.Spec(cfg), Dr), True), set(range(m)))
                runs.append({"stages": Dr, "sha256": combine(dg)})
            repro = {"policy": "csp", "subnets": n_sub, "runs": runs,
                     "bitwise_equal": len({r["sha256"] for r in runs}) == 1}
        else:
            sob = npipe.naspipe_partition(npipe.Spec(cfg), D)
            mine = bit_repro_digests(cfg, npipe, dev_pool, n_sub, lambda: (create(npipe.Spec(cfg)), rank == D - 1),
                                     {b for b in range(m) if sob[b] == rank})
            parts = gather(mine)
            ref = None
            if rank == 0:   # the same subnets as ONE stage on this GPU
                ref = bit_repro_digests(cfg, npipe, dev_pool, n_sub,
                                        lambda: (npipe.naspipe_create(npipe.Spec(cfg), 1), True), set(range(m)))
            if rank == 0:
                merged = {}
                for p in parts:
                    merged.update(p)
                repro = {"policy": "csp", "subnets": n_sub,
                         "runs": [{"stages": 1, "processes": 1, "sha256": combine(ref)},
                                  {"stages": D, "processes": D, "transport": args.transport, "sha256": combine(merged)}],
                         "bitwise_equal": combine(ref) == combine(merged)}
            barrier()

    if rank != 0:
        return
    cpu = None
    if world == 1 and not args.no_cpu:
        cpu = cpu_baseline(cfg)
    out = {"metric": "supernet samples/sec", "value": value, "unit": "samples/s", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f32" if cfg["family"] == "mlp" else "bf16",
           "data": "synthetic (N(0,1) inputs/targets, counter-hash init, uniform per-block choices)",
           "config": dict(workload_config(args, cfg, world), transport=args.transport if world > 1 else None),
           "clocks": clk.summary(), "e2e": e2e,
           "gpu_launches": int(launches), "roofline": roofline, "fractions": fractions, "kernels_top": kernels_top,
           "cpu_baseline": cpu,
           "context_switch": {"budget_bytes_per_stage": budget, "budget_x": args.budget_x,
                              "lookahead": args.lookahead or 2,
                              "loads": s1["res_loads"] - s0["res_loads"], "evicts": s1["res_evicts"] - s0["res_evicts"],
                              "writebacks": s1["writebacks"] - s0["writebacks"],
                              "h2d_GBps": (s1["h2d_bytes"] - s0["h2d_bytes"]) / (ms / 1000) / 1e9,
                              "d2h_GBps": (s1["d2h_bytes"] - s0["d2h_bytes"]) / (ms / 1000) / 1e9,
                              "pcie_note": "against pinned cudaMemcpyAsync H2D/D2H measured on this box "
                                           "(profiles/*pcie*; tools/pcie_bw.py)"} if budget else None,
           "p2p_GBps": (s1["p2p_bytes"] - s0["p2p_bytes"]) / (ms / 1000) / 1e9 if world > 1 else None,
           "loss_finite": loss_ok, "bit_repro": repro}
    if timed_stats is not None:
        out["timed_executor"] = dict(timed_stats, note="all timed regions of this run (value, CUPTI, e2e); Alg.3 "
                                     "hits = predictions equal to the stage's next forward")
    if sec is not None:
        out["secondary"] = sec
    print(json.dumps(out))


if __name__ == "__main__":
    main()
