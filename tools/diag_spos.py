"""Per-tensor parity diagnostic of the SPOS family against the oracle (GPU box only).

    python tools/diag_spos.py [N] [D] [config]
"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
import paper_conf_asplos_zhaolcscwzlc22_b200 as npipe  # noqa: E402
from oracle import train  # noqa: E402


def main():
    N = int(sys.argv[1]) if len(sys.argv) > 1 else 1
    D = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    name = sys.argv[3] if len(sys.argv) > 3 else "tiny_spos"
    storage = sys.argv[4] if len(sys.argv) > 4 else "bf16"
    verbose = len(sys.argv) > 5
    cfg = synth.get_config(name, storage=storage)
    ch = synth.sample_choices(N, cfg["n_blocks"], cfg["n_choices"])
    batches = [synth.make_batch(cfg, y) for y in range(N)]
    theta0 = train.initial_theta(cfg)
    ref, ref_loss = train.train_sequential(cfg, theta0, ch, batches)
    h = npipe.naspipe_create(npipe.Spec(cfg), D)
    for y in range(N):
        npipe.naspipe_submit(h, ch[y], *batches[y])
    npipe.naspipe_drain(h)
    print("choices", ch.tolist())
    print("loss gpu", npipe.naspipe_get_losses(h, N), "ref", ref_loss)
    worst_a15 = worst_cand = 0.0
    for (b, c), r in sorted(ref.items()):
        g = npipe.naspipe_get_params(h, b, c).astype(np.float64)
        worst_a15 = max(worst_a15, np.max(np.abs(g - r)) / np.max(np.abs(r)))
        t0c = theta0[(b, c)].astype(np.float64)
        if np.any(r != t0c):
            worst_cand = max(worst_cand, np.linalg.norm((g - t0c) - (r - t0c)) / np.linalg.norm(r - t0c))
        off = 0
        for nm, shape, _, _ in train.candidate_layout(cfg, b, c):
            n = int(np.prod(shape))
            gs, rs, t0 = g[off:off + n], r[off:off + n], theta0[(b, c)][off:off + n].astype(np.float64)
            off += n
            dr, dg = rs - t0, gs - t0
            if verbose and (np.any(dr != 0) or np.any(dg != 0)):
                e = np.linalg.norm(dg - dr) / max(np.linalg.norm(dr), 1e-300)
                print(f"({b},{c}) {nm:8s} |dref|={np.linalg.norm(dr):.3e} |dgpu|={np.linalg.norm(dg):.3e} "
                      f"rel={e:.3e} cos={np.dot(dg, dr) / max(np.linalg.norm(dg) * np.linalg.norm(dr), 1e-300):.4f}")
    print(f"{name} N={N} D={D} storage={storage}: A15={worst_a15:.3e} candidate update rel={worst_cand:.3e}")
    npipe.naspipe_destroy(h)


if __name__ == "__main__":
    main()
