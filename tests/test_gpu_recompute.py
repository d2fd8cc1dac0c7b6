"""Activation recomputation ("NASPIPE adopts activation recomputing
techniques"; reading A13; include/naspipe.h NASPIPE_FLAG_RECOMPUTE).

The forward keeps only each block's input and the backward recomputes the block before its
gradient.  The kernels are deterministic and CSP/BSP never update a candidate between F(y)
and B(y), so every parameter and loss must be bitwise those of the run that stores the
activations (which test_gpu_parity.py pins to the oracle)."""
import numpy as np
import pytest

import synth

from test_gpu_parity import FLAGS, run_engine

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")


def _bitwise(a, b):
    pa, la = a[0], a[1]
    pb, lb = b[0], b[1]
    assert np.array_equal(la.view(np.uint32), lb.view(np.uint32))
    for k in pa:
        assert np.array_equal(pa[k].view(np.uint32), pb[k].view(np.uint32)), k


@pytest.mark.parametrize("name,N,D,sync", [("tiny_transformer", 6, 1, "csp"), ("tiny_transformer", 6, 2, "csp"),
                                           ("tiny_transformer", 8, 2, "bsp"), ("transformer", 2, 1, "csp")])
def test_recompute_is_bitwise_equal(name, N, D, sync):
    cfg = synth.get_config(name, sync=sync, bulk_size=4)
    choices = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    ref = run_engine(cfg, choices, batches, D)
    got = run_engine(cfg, choices, batches, D, flags=FLAGS | npipe.FLAG_RECOMPUTE)
    _bitwise(ref, got)
