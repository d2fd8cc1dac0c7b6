"""One rank of a multi-process CSP pipeline (peer-memory or NCCL transport), for
tests/test_gpu_multirank.py and bench.py-style checks.  Run as a script:

    python tests/rank_worker.py --workload toy --world 2 --rank R --port P --n 12 --out f.npz

Every rank: create its stage (naspipe_create_rank_peer on device rank % device_count),
exchange the peer blobs over a gloo process group (plumbing only), connect, submit the same
N subnets (synth recipe, HOST batches), drain, and save its blocks' parameters, the losses
(last rank) and its executed trace.
"""
import argparse
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="toy")
    ap.add_argument("--world", type=int, default=2)
    ap.add_argument("--rank", type=int, required=True)
    ap.add_argument("--port", type=int, required=True)
    ap.add_argument("--n", type=int, default=12)
    ap.add_argument("--transport", default="peer", choices=["peer", "nccl"])
    ap.add_argument("--sync", default="csp")
    ap.add_argument("--out", required=True)
    a = ap.parse_args()
    import torch
    import torch.distributed as dist
    import synth
    import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe

    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{a.port}", rank=a.rank, world_size=a.world)
    dev = a.rank % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    cfg = synth.get_config(a.workload, sync=a.sync)
    spec = npipe.Spec(cfg, flags=npipe.FLAG_TRACE | npipe.FLAG_VERSION_CHECK)
    D, r = a.world, a.rank
    if a.transport == "peer":
        h = npipe.naspipe_create_rank_peer(spec, D, r, dev)
        blobs = [None] * D
        dist.all_gather_object(blobs, npipe.naspipe_peer_export(h))
        npipe.naspipe_peer_connect(h, blobs[r - 1] if r > 0 else None, blobs[r + 1] if r < D - 1 else None)
    else:
        ids = [None]
        if r == 0:
            ids = [b"".join(npipe.naspipe_nccl_unique_id() for _ in range(2 * (D - 1)))]
        dist.broadcast_object_list(ids, src=0)
        h = npipe.naspipe_create_rank(spec, D, r, dev, ids[0])
    choices = synth.sample_choices(a.n, cfg["n_blocks"], cfg["n_choices"])
    for y in range(a.n):
        x, t = synth.make_batch(cfg, y)
        npipe.naspipe_submit(h, choices[y], x, t)
    npipe.naspipe_drain(h)
    sob = npipe.naspipe_partition(spec, D)
    out = {"trace": np.asarray(npipe.naspipe_get_trace(h), dtype=np.int64).reshape(-1, 4)}
    for b in range(cfg["n_blocks"]):
        if sob[b] != r:
            continue
        for c in range(cfg["n_choices"]):
            out[f"p_{b}_{c}"] = npipe.naspipe_get_params(h, b, c)
    if r == D - 1:
        out["losses"] = npipe.naspipe_get_losses(h, a.n)
    st = npipe.naspipe_get_stats(h)
    out["p2p_bytes"] = np.float64(st["p2p_bytes"])
    out["version_checks"] = np.float64(st["version_checks"])
    np.savez(a.out, **out)
    dist.barrier()            # every rank drained: no peer still maps or writes our rings
    npipe.naspipe_destroy(h)
    dist.barrier()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()
