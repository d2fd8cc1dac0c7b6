"""Multi-process (N > 1) host logic on CPU with torch.distributed gloo, world size 2-4.

In multi-process mode every rank replays the same CSP plan and issues its NCCL
sends/receives in plan order (naspipe_plan_comm_schedule, the same comm_ops() the executor
uses).  Here each rank sends its schedule's messages over gloo (one tag per channel and
direction, like the executor's one communicator per channel) carrying the subnet id, and
checks that every receive gets exactly the subnet id its schedule expects — i.e. sender
order == receiver posting order on every channel, the condition NCCL p2p needs.
"""
import os
import socket
import tempfile

import numpy as np
import pytest

import synth

npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")
torch = pytest.importorskip("torch")

SEND_ACT, RECV_ACT, SEND_GRAD, RECV_GRAD = 0, 1, 2, 3


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _tag(op, rank):
    # activation channel k -> k+1: tag 2k;  gradient channel k+1 -> k: tag 2k+1
    if op == SEND_ACT:
        return 2 * rank
    if op == RECV_ACT:
        return 2 * (rank - 1)
    if op == SEND_GRAD:
        return 2 * (rank - 1) + 1
    return 2 * rank + 1


def _worker(rank, world, port, cfg, n_subnets, out_dir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        choices = synth.sample_choices(n_subnets, cfg["n_blocks"], cfg["n_choices"], seed=7)  # identical on every rank
        plan = npipe.naspipe_plan(npipe.Spec(cfg), world, choices)
        sched = plan.comm_schedule(rank)
        reqs, recvs = [], []
        for op, peer, y in sched:
            if op in (SEND_ACT, SEND_GRAD):
                reqs.append(dist.isend(torch.tensor([int(y)], dtype=torch.int64), int(peer), tag=_tag(op, rank)))
            else:
                buf = torch.zeros(1, dtype=torch.int64)
                reqs.append(dist.irecv(buf, int(peer), tag=_tag(op, rank)))
                recvs.append((int(y), buf))
        for r in reqs:
            r.wait()
        got = [int(b.item()) for _, b in recvs]
        expect = [y for y, _ in recvs]
        ok = got == expect
        n_send = int(np.sum(np.isin(sched[:, 0], [SEND_ACT, SEND_GRAD]))) if len(sched) else 0
        with open(os.path.join(out_dir, f"r{rank}"), "w") as f:
            f.write(f"{int(ok)} {len(recvs)} {n_send}\n")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,m,n", [(2, 4, 4), (3, 6, 3), (4, 8, 2)])
def test_p2p_schedules_match_over_gloo(world, m, n):
    import torch.multiprocessing as mp
    cfg = dict(family="mlp", n_blocks=m, n_choices=n, batch=2, width=8, compute_dtype="fp32", lr=0.05)
    N = 12
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_worker, args=(world, _free_port(), cfg, N, d), nprocs=world, start_method="spawn")
        rows = [open(os.path.join(d, f"r{r}")).read().split() for r in range(world)]
    assert all(r[0] == "1" for r in rows), rows
    # every subnet crosses every boundary once forward and once backward
    assert sum(int(r[1]) for r in rows) == 2 * N * (world - 1)
    assert sum(int(r[2]) for r in rows) == 2 * N * (world - 1)


def test_comm_schedule_structure():
    cfg = dict(family="mlp", n_blocks=4, n_choices=3, batch=2, width=8, compute_dtype="fp32")
    choices = synth.sample_choices(10, 4, 3, seed=3)
    plan = npipe.naspipe_plan(npipe.Spec(cfg), 4, choices)
    for rank in range(4):
        s = plan.comm_schedule(rank)
        ops = set(s[:, 0].tolist())
        assert (RECV_ACT in ops) == (rank > 0) and (SEND_GRAD in ops) == (rank > 0)
        assert (SEND_ACT in ops) == (rank < 3) and (RECV_GRAD in ops) == (rank < 3)
        # activations of subnet y are received before its gradient is sent back
        for y in range(10):
            if rank > 0:
                i_rx = next(i for i, r in enumerate(s) if r[0] == RECV_ACT and r[2] == y)
                i_tx = next(i for i, r in enumerate(s) if r[0] == SEND_GRAD and r[2] == y)
                assert i_rx < i_tx
