"""The one-process-per-GPU path (naspipe_create_rank_peer) executed for real:
2 and 3 rank processes, each running one pipeline stage, exchanging activations and
gradients through the peer-memory transport (CUDA IPC rings + stream-memory flags;
include/naspipe.h).  On a one-GPU box all ranks share the device (IPC mappings of the same
HBM), which exercises the whole rank logic — blob exchange, ring addressing, flag protocol,
per-rank planning — on the hardware available; on a multi-GPU box rank r uses device r.

Bar (Def.1, Table 3, artifact P:L557-561): every candidate's parameters,
the losses and each rank's executed trace are BITWISE those of the single-process run with
the same stages (and hence of D = 1: tests/test_gpu_parity.py), and every task passed the
version check (CSP's race check).
"""
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")

from test_gpu_parity import run_engine  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _run_ranks(tmp_path, workload, world, n, transport="peer", sync="csp"):
    port = _free_port()
    procs, outs = [], []
    for r in range(world):
        out = str(tmp_path / f"rank{r}.npz")
        outs.append(out)
        procs.append(subprocess.Popen([sys.executable, os.path.join(HERE, "rank_worker.py"), "--workload", workload,
                                       "--world", str(world), "--rank", str(r), "--port", str(port), "--n", str(n),
                                       "--transport", transport, "--sync", sync, "--out", out],
                                      stdout=subprocess.PIPE, stderr=subprocess.STDOUT, text=True))
    logs = []
    for p in procs:
        try:
            logs.append(p.communicate(timeout=300)[0])
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
    for p, log in zip(procs, logs):
        assert p.returncode == 0, log[-3000:]
    return [np.load(o) for o in outs]


@pytest.mark.parametrize("workload,world,n", [("toy", 2, 16), ("toy", 3, 12), ("tiny_transformer", 2, 8),
                                              ("tiny_transformer", 3, 6), ("tiny_spos", 2, 6)])
def test_peer_ranks_bitwise_equal_single_process(tmp_path, workload, world, n):
    ranks = _run_ranks(tmp_path, workload, world, n)
    cfg = synth.get_config(workload)
    choices = synth.sample_choices(n, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(n)]
    ref, ref_loss, ref_trace, _ = run_engine(cfg, choices, batches, D=world)
    sob = npipe.naspipe_partition(npipe.Spec(cfg), world)
    for b in range(cfg["n_blocks"]):
        for c in range(cfg["n_choices"]):
            got = ranks[sob[b]][f"p_{b}_{c}"]
            assert np.array_equal(got.view(np.uint32), ref[(b, c)].view(np.uint32)), (b, c)
    assert np.array_equal(ranks[-1]["losses"].view(np.uint32), ref_loss.view(np.uint32))
    ref_trace = np.asarray(ref_trace, dtype=np.int64).reshape(-1, 4)
    for r in range(world):
        assert np.array_equal(ranks[r]["trace"], ref_trace[ref_trace[:, 1] == r]), r
        nb = int(np.sum(np.asarray(sob) == r))
        assert ranks[r]["version_checks"] == 2 * n * nb
        assert ranks[r]["p2p_bytes"] > 0


def test_peer_ranks_asp_and_bsp(tmp_path):
    """The other synchronisation policies run through the same transport (toy, 2 ranks)."""
    for sync in ("asp", "bsp"):
        ranks = _run_ranks(tmp_path, "toy", 2, 12, sync=sync)
        cfg = synth.get_config("toy", sync=sync)
        choices = synth.sample_choices(12, cfg["n_blocks"], cfg["n_choices"])
        batches = [synth.make_batch(cfg, y) for y in range(12)]
        ref, ref_loss, _, _ = run_engine(cfg, choices, batches, D=2)
        assert np.array_equal(ranks[-1]["losses"].view(np.uint32), ref_loss.view(np.uint32)), sync
        sob = npipe.naspipe_partition(npipe.Spec(cfg), 2)
        for (b, c), v in ref.items():
            assert np.array_equal(ranks[sob[b]][f"p_{b}_{c}"].view(np.uint32), v.view(np.uint32)), (sync, b, c)


@pytest.mark.skipif(not torch.cuda.is_available() or torch.cuda.device_count() < 2,
                    reason="NCCL refuses two ranks on one GPU; needs >= 2 GPUs")
def test_nccl_ranks_bitwise_equal_single_process(tmp_path):
    ranks = _run_ranks(tmp_path, "tiny_transformer", 2, 8, transport="nccl")
    cfg = synth.get_config("tiny_transformer")
    choices = synth.sample_choices(8, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(8)]
    ref, ref_loss, _, _ = run_engine(cfg, choices, batches, D=2)
    assert np.array_equal(ranks[-1]["losses"].view(np.uint32), ref_loss.view(np.uint32))
