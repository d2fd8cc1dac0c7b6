#!/usr/bin/env python
"""Benchmark of the NASPipe hot path on B200 (contract: see DESIGN.md "Measurement").

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference] [--workload NAME]

One step = one subnet trained through the whole pipeline (forward, loss, backward and the
SGD WRITE of every active candidate on every stage) on one synthetic batch.  N = 1 runs the
whole supernet as one stage on one GPU; N > 1 (torchrun, one process per GPU) runs an
N-stage CSP pipeline with NCCL send/recv between stages.

Default workload: configs[1] (SPOS CNN supernet, 20 blocks x 4 choices, 224x224, batch 64).
Printed by rank 0 as ONE JSON line: value = samples/s of the whole job with the inputs
already resident in HBM (device batches); e2e = the same through the C ABI with pinned HOST
buffers (H2D of input+target inside the timed region, D2H of the step losses);
roofline = the dominant kernel timed by CUDA events on its stream (SPOS: the BatchNorm
kernels against HBM bandwidth; transformer: the tcgen05 GEMM against bf16 peak);
cpu_baseline = the fp64 NumPy oracle on a bounded sample, on this host's cores;
secondary = the configs[2] transformer (the tensor-core path) measured the same way.
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
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-secondary", action="store_true", help="skip the configs[2] line embedded in the output")
    ap.add_argument("--no-repro", action="store_true", help="skip the bit-reproducibility digests")
    ap.add_argument("--sync", default="csp", choices=["csp", "inorder", "asp", "bsp"],
                    help="synchronisation policy (include/naspipe.h naspipe_sync; SURVEY §8f(1))")
    ap.add_argument("--recompute", action="store_true",
                    help="activation recomputation (transformer family; P:L282, reading A13)")
    ap.add_argument("--budget-x", type=float, default=0.0,
                    help="HBM weight budget per stage as a multiple of one subnet's mean stage slice "
                         "(0 = all candidates resident; P:L337 uses ~3)")
    ap.add_argument("--n-choices", type=int, default=0, help="override n (search-space sweep, configs[4])")
    ap.add_argument("--lookahead", type=int, default=0, help="residency prefetch depth L in tasks (0 = 2, P:L156)")
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
def oracle_block_sample(cfg, n_blocks_sample):
    """Time the fp64 oracle on a bounded sample of one subnet's step (fwd + bwd + SGD).
    MLP / transformer: `n_blocks_sample` full-size blocks of subnet 0.  SPOS: the whole
    subnet (stem, 20 blocks, head) on `n_blocks_sample` of the batch's images (its BatchNorm
    statistics then cover that sub-batch; the arithmetic per image is the same).
    Returns seconds."""
    from oracle import train, transformer, mlp   # noqa: F401  (test infrastructure, timing only)
    ch = synth.sample_choices(1, cfg["n_blocks"], cfg["n_choices"])[0]
    x, t = synth.make_batch(cfg, 0)
    if cfg["family"] == "spos":
        sub = dict(cfg, batch=n_blocks_sample)
        theta = {(b, int(c)): train.unpack(cfg, b, int(c), v) for (b, c), v in
                 ((k, v) for k, v in train.initial_theta(cfg).items()) if int(ch[b]) == c}
        t0 = time.perf_counter()
        loss, grads = train.subnet_step(sub, theta, ch, x[:n_blocks_sample], t[:n_blocks_sample])
        train.sgd_apply(theta, grads, cfg["lr"])
        return time.perf_counter() - t0
    theta = {}
    for b in range(n_blocks_sample):
        c = int(ch[b])
        segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in train.candidate_layout(cfg, b, c)]
        theta[(b, c)] = train.unpack(cfg, b, c, synth.init_packed(cfg["init_seed"], b * cfg["n_choices"] + c, segs))
    t0 = time.perf_counter()
    sub = dict(cfg, n_blocks=n_blocks_sample)
    loss, grads = train.subnet_step(sub, theta, ch[:n_blocks_sample], x, t)
    train.sgd_apply(theta, grads, cfg["lr"])
    return time.perf_counter() - t0


def sample_size(cfg):
    """(sample units, units per subnet, description) of the bounded oracle sample."""
    if cfg["family"] == "spos":
        return 16, cfg["batch"], "images"
    if cfg["family"] == "transformer":
        return (2 if cfg["d_model"] <= 1024 else 1), cfg["n_blocks"], "blocks"
    return cfg["n_blocks"], cfg["n_blocks"], "blocks"


def cpu_threads():
    try:
        from threadpoolctl import threadpool_info
        return max((i.get("num_threads", 1) for i in threadpool_info()), default=os.cpu_count())
    except Exception:
        return os.cpu_count()


def cpu_baseline(cfg):
    ns, per, unit = sample_size(cfg)
    secs = oracle_block_sample(cfg, ns)
    per_subnet = secs * per / ns
    return {"value": cfg["batch"] / per_subnet, "unit": "samples/s", "cores": cpu_threads(), "kind": "oracle",
            "sample": f"fp64 NumPy oracle, {ns} of {per} {unit} of subnet 0 (fwd+bwd+SGD), "
                      f"{secs:.2f} s, scaled x{per / ns:g} to one subnet of B={cfg['batch']}"}


def run_reference(args, cfg, rank, world):
    """--impl reference: the oracle as it stands, on host cores, rank 0 only."""
    if rank != 0:
        return
    ns, per, unit = sample_size(cfg)
    if cfg["family"] == "transformer":
        ns = 1
    if cfg["family"] == "spos":
        ns = 2   # ~1 s of oracle work per step: the default K/W run ends within a few minutes
    for _ in range(args.warmup):
        oracle_block_sample(cfg, ns)
    ts = [oracle_block_sample(cfg, ns) for _ in range(args.steps)]
    per_subnet = float(np.mean(ts)) * per / ns
    value = cfg["batch"] / per_subnet
    cores = cpu_threads()
    sample = (f"each step = {ns} of {per} {unit} of subnet 0, fwd+bwd+SGD in the fp64 oracle, "
              f"scaled x{per / ns:g} to one subnet")
    print(json.dumps({
        "impl": "reference", "metric": "supernet samples/sec", "value": value, "unit": "samples/s",
        "n_gpus": world, "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * per_subnet,
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": workload_config(args, cfg, world),
        "cpu_baseline": {"kind": "oracle", "cores": cores, "sample": sample, "value": value, "unit": "samples/s"},
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
           "source": "profiles/dominant_traffic.json (ncu --set full capture)"}
    if "tensor_pipe_pct_mean" in d:   # sm__pipe_tensor_cycles_active, time-weighted over the captured GEMMs
        out["tensor_pipe_pct"] = d["tensor_pipe_pct_mean"]
    return out


def secondary(args):
    """configs[2] (transformer, the tensor-core path) measured in a child process, reported
    beside the headline configs[1] line."""
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--workload", "transformer", "--steps", str(args.steps),
           "--warmup", str(args.warmup), "--no-cpu", "--no-e2e", "--no-secondary"]
    try:
        out = subprocess.run(cmd, capture_output=True, text=True, timeout=300).stdout.strip().splitlines()
        d = json.loads(out[-1])
        return {k: d.get(k) for k in ("value", "unit", "ms_per_step", "config", "roofline", "clocks", "gpu_launches",
                                      "bit_repro")}
    except Exception as e:  # reported, never fatal for the headline line
        return {"error": repr(e)[:200]}


def bit_repro(cfg, npipe, dev_pool, n_sub=8, stage_counts=(1, 1, 2, 4)):
    """BJ's "bit-repro check" (Def.1, Table 3): train the same n_sub subnets
    on the same device batches with fresh handles — twice at D=1, then at D=2 and D=4 (all
    stages on this GPU; the stage boundaries then sit in the middle of the supernet) — and
    hash every trained candidate's fp32 master plus the losses with SHA-256.  All digests must
    be equal."""
    import hashlib
    m, n = cfg["n_blocks"], cfg["n_choices"]
    choices = synth.sample_choices(n_sub, m, n)
    used = sorted({(b, int(choices[y][b])) for y in range(n_sub) for b in range(m)})
    digests = []
    for D in stage_counts:
        if D > m:
            continue
        h = npipe.naspipe_create(npipe.Spec(cfg), D)
        for y in range(n_sub):
            x, t = dev_pool[y % len(dev_pool)]
            npipe.naspipe_submit(h, choices[y], x, t, where=npipe.BATCH_DEVICE)
        npipe.naspipe_drain(h)
        sha = hashlib.sha256()
        for b, c in used:
            sha.update(np.ascontiguousarray(npipe.naspipe_get_params(h, b, c), dtype=np.float32).tobytes())
        sha.update(np.ascontiguousarray(npipe.naspipe_get_losses(h, n_sub), dtype=np.float32).tobytes())
        npipe.naspipe_destroy(h)
        digests.append({"stages": D, "sha256": sha.hexdigest()})
    return {"policy": "csp", "subnets": n_sub, "candidates_hashed": len(used), "runs": digests,
            "bitwise_equal": len({d["sha256"] for d in digests}) == 1}


def workload_config(args, cfg, world):
    names = {"transformer": "configs[2] transformer", "large_transformer": "configs[3] large_transformer",
             "toy": "configs[0] toy", "spos": "configs[1] SPOS CNN"}
    c = {"workload": names.get(args.workload, args.workload) if not args.n_choices
         else f"configs[4] sweep n={args.n_choices}",
         "n_blocks": cfg["n_blocks"], "n_choices": cfg["n_choices"], "batch": cfg["batch"],
         "stages": world, "parallelism": f"pp{world}" if world > 1 else "single stage",
         "activation_recompute": bool(getattr(args, "recompute", False)),
         "sync_policy": getattr(args, "sync", "csp"),
         "l2": "working set > L2 (active weights + activations per step >> 126 MB)"}
    if cfg["family"] == "transformer":
        c.update(seq_len=cfg["seq_len"], d_model=cfg["d_model"], heads=cfg["choice_heads"], ffn=cfg["choice_ffn"])
    if cfg["family"] == "spos":
        c.update(image_hw=cfg["image_hw"], stage_repeats=cfg["stage_repeats"], stage_channels=cfg["stage_channels"],
                 choice_kernel=cfg["choice_kernel"], choice_xception=cfg["choice_xception"],
                 num_classes=cfg["num_classes"])
    return c


# ------------------------------------------------------------------------------ GPU arm
def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    cfg = synth.get_config(args.workload) if args.n_choices == 0 else synth.sweep_config(args.n_choices)
    if args.impl == "reference":
        run_reference(args, cfg, rank, world)
        return
    # the configs[2] line runs in a child process BEFORE this process touches the GPU (a
    # child started while the parent holds a CUDA context stalled on the box)
    sec = None
    if world == 1 and args.workload == "spos" and not args.no_secondary and not args.n_choices:
        sec = secondary(args)

    import torch
    import torch.distributed as dist
    import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    D = world
    m, n, B = cfg["n_blocks"], cfg["n_choices"], cfg["batch"]
    total = args.warmup + 3 * args.steps
    choices = synth.sample_choices(total, m, n)
    # device-resident input pool (value run) and pinned host pool (e2e run)
    pool = [synth.make_batch(cfg, y) for y in range(4)]
    dev_pool = [(torch.from_numpy(x).cuda(), torch.from_numpy(t).cuda()) for x, t in pool]
    host_pool = [(torch.from_numpy(x).pin_memory(), torch.from_numpy(t).pin_memory()) for x, t in pool]
    budget = stage_budget(cfg, D, args.budget_x, npipe) if args.budget_x > 0 else 0
    spec = npipe.Spec(cfg, hbm_weight_budget_bytes=budget, lookahead=args.lookahead, sync=args.sync,
                      flags=npipe.FLAG_RECOMPUTE if args.recompute else 0)
    if world == 1:
        h = npipe.naspipe_create(spec, 1)
    else:
        ids = [None]
        if rank == 0:
            ids[0] = b"".join(npipe.naspipe_nccl_unique_id() for _ in range(2 * (D - 1)))
        dist.broadcast_object_list(ids, src=0)
        h = npipe.naspipe_create_rank(spec, D, rank, local, ids[0])

    def barrier():
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()

    def max_over_ranks(v):
        if world == 1:
            return v
        t = torch.tensor([v], device="cuda", dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    y = 0
    for _ in range(args.warmup):
        x, t = dev_pool[y % 4]
        npipe.naspipe_submit(h, choices[y], x, t, where=npipe.BATCH_DEVICE)
        y += 1
    npipe.naspipe_drain(h)

    # ---- timed region 1: inputs resident in HBM
    s0 = npipe.naspipe_get_stats(h)
    barrier()
    prof = os.environ.get("NASPIPE_PROFILE_RANGE") == "1"   # ncu --profile-from-start off
    if prof:
        torch.cuda.profiler.start()
    with ClockSampler(local) as clk:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t_wall = time.perf_counter()
        e0.record()
        for _ in range(args.steps):
            x, t = dev_pool[y % 4]
            npipe.naspipe_submit(h, choices[y], x, t, where=npipe.BATCH_DEVICE)
            y += 1
        npipe.naspipe_drain(h)
        e1.record()
        torch.cuda.synchronize()
        t_wall = time.perf_counter() - t_wall
    if prof:
        torch.cuda.profiler.stop()
    s1 = npipe.naspipe_get_stats(h)
    # the default-stream events bracket the drain (host waits for every stage stream), so
    # the elapsed time covers all device work of the K steps
    ms = max_over_ranks(e0.elapsed_time(e1))
    value = args.steps * B / (ms / 1000)

    launches = (s1["kernel_launches"] - s0["kernel_launches"])

    # ---- roofline of the dominant kernel: a second timed region of the same K steps with
    # CUDA events bracketing each of its launches on its stream (kept out of `value`: the
    # events cost the kernels' PDL overlap)
    npipe.naspipe_set_timing(h, True)
    s2 = npipe.naspipe_get_stats(h)
    barrier()
    e0.record()
    for _ in range(args.steps):
        x, t = dev_pool[y % 4]
        npipe.naspipe_submit(h, choices[y], x, t, where=npipe.BATCH_DEVICE)
        y += 1
    npipe.naspipe_drain(h)
    e1.record()
    torch.cuda.synchronize()
    ms_timed = max_over_ranks(e0.elapsed_time(e1))
    s3 = npipe.naspipe_get_stats(h)
    npipe.naspipe_set_timing(h, False)
    g_flops = s3["dominant_flops"] - s2["dominant_flops"]
    g_ms = s3["dominant_ms"] - s2["dominant_ms"]
    g_n = s3["dominant_launches"] - s2["dominant_launches"]
    ms_r = ms_timed
    pk = peaks()
    if cfg["family"] == "spos":
        # SPOS: the BatchNorm kernels are the step's dominant family (HBM-bound); work = their
        # algorithmic bytes, one timed unit = one BN call (stats/apply/bwd)
        achieved = (g_flops / g_n) / ((g_ms / g_n) / 1000) / 1e9 if g_n else None
        traffic = _traffic("spos")
        roofline = {"bound": "hbm", "kernel": "BatchNorm kernels (bn_stats+finalize, bn_apply, "
                                              "bn_bwd_reduce+finalize, bn_bwd_apply), all units of the step",
                    "achieved": achieved, "peak": pk["hbm"], "unit": "GB/s",
                    "frac": achieved / pk["hbm"] if achieved else None, "traffic": traffic,
                    "peak_source": pk["source"] + " hbm_gbs (copy bandwidth)",
                    "launches": g_n, "share_of_timed_step": g_ms / ms_r if ms_r else None,
                    "algorithmic_bytes_per_step": g_flops / args.steps}
    else:
        achieved = (g_flops / g_n) / ((g_ms / g_n) / 1000) / 1e12 if g_n else None
        traffic = _traffic("transformer")
        roofline = {"bound": "tensor", "kernel": "tcgen05 GEMM (gemm_pair_kernel / gemm_tc_kernel, all shapes)",
                    "achieved": achieved, "peak": pk["bf16_sustained"], "unit": "TFLOP/s",
                    "frac": achieved / pk["bf16_sustained"] if achieved else None, "traffic": traffic,
                    "peak_source": pk["source"] + " bf16_tflops_sustained (kernel timed inside a long step)",
                    "launches": g_n, "share_of_timed_step": g_ms / ms_r if ms_r else None,
                    "algorithmic_flops_per_step": g_flops / args.steps}

    # ---- timed region 3: end to end through the C ABI with pinned host buffers
    e2e = None
    if not args.no_e2e:
        barrier()
        e0.record()
        for k in range(args.steps):
            x, t = host_pool[y % 4]
            npipe.naspipe_submit(h, choices[y], x, t, where=npipe.BATCH_HOST)
            y += 1
        npipe.naspipe_drain(h)
        if rank == world - 1:
            npipe.naspipe_get_losses(h, y)[-args.steps:]   # D2H of the step results
        e1.record()
        torch.cuda.synchronize()
        ms2 = max_over_ranks(e0.elapsed_time(e1))
        e2e = {"value": args.steps * B / (ms2 / 1000), "unit": "samples/s",
               "h2d_bytes_per_step": x.numel() * x.element_size() + t.numel() * t.element_size(),
               "d2h_bytes_per_step": 4}
    losses = npipe.naspipe_get_losses(h, y) if rank == world - 1 else None
    npipe.naspipe_destroy(h)
    repro = None
    if world == 1 and not args.no_repro and not args.budget_x:
        repro = bit_repro(cfg, npipe, dev_pool)

    if rank != 0:
        return
    cpu = None
    if world == 1 and not args.no_cpu:
        cpu = cpu_baseline(cfg)
    out = {"metric": "supernet samples/sec", "value": value, "unit": "samples/s", "n_gpus": world,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": True,
           "scaling": "strong", "vs_baseline": None, "dtype": "f32" if cfg["family"] == "mlp" else "bf16",
           "data": "synthetic (N(0,1) inputs/targets, counter-hash init, uniform per-block choices)",
           "config": workload_config(args, cfg, world), "clocks": clk.summary(), "e2e": e2e,
           "gpu_launches": int(launches), "roofline": roofline, "cpu_baseline": cpu,
           "context_switch": {"budget_bytes_per_stage": budget, "budget_x": args.budget_x,
                              "lookahead": args.lookahead or 2,
                              "loads": s1["res_loads"] - s0["res_loads"], "evicts": s1["res_evicts"] - s0["res_evicts"],
                              "writebacks": s1["writebacks"] - s0["writebacks"],
                              "h2d_GBps": (s1["h2d_bytes"] - s0["h2d_bytes"]) / (ms / 1000) / 1e9,
                              "d2h_GBps": (s1["d2h_bytes"] - s0["d2h_bytes"]) / (ms / 1000) / 1e9} if budget else None,
           "loss_finite": bool(losses is None or np.all(np.isfinite(losses))), "bit_repro": repro}
    if sec is not None:
        out["secondary"] = {"configs[2] transformer": sec}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
