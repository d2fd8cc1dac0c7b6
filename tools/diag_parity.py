"""Per-tensor parity diagnostic of the CUDA path vs the fp64 oracle (prints a table)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import synth
from oracle import train
from test_gpu_parity import run_engine, _workload, _oracle

name = sys.argv[1] if len(sys.argv) > 1 else "tiny_transformer"
N = int(sys.argv[2]) if len(sys.argv) > 2 else 1
cfg, choices, batches = _workload(name, N)
theta0, ref, ref_loss = _oracle(cfg, choices, batches)
params, losses, trace, _ = run_engine(cfg, choices, batches, D=2)
print("loss rel err", np.max(np.abs(losses - ref_loss) / np.abs(ref_loss)))
rows = {}
for (b, c), r in ref.items():
    g = params[(b, c)].astype(np.float64); t0 = theta0[(b, c)].astype(np.float64)
    off = 0
    for nm, shape, _, _ in train.candidate_layout(cfg, b, c):
        n = int(np.prod(shape)); gs, rs, ts = g[off:off+n], r[off:off+n], t0[off:off+n]; off += n
        dr = rs - ts
        if np.max(np.abs(dr)) == 0: continue
        e = np.max(np.abs(gs - rs)) / np.max(np.abs(rs))
        de = np.max(np.abs((gs - ts) - dr)) / np.max(np.abs(dr))
        ne = np.linalg.norm((gs - ts) - dr) / np.linalg.norm(dr)
        rows.setdefault(nm, []).append((e, de, ne))
for nm, v in rows.items():
    v = np.array(v)
    print(f"{nm:6s} err {v[:,0].max():.2e}  dmax {v[:,1].max():.2e}  dnorm {v[:,2].max():.2e}")
