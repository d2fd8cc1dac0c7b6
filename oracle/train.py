"""Sequential supernet training: the numeric oracle.

PAPER.md Def.1: the result of training is the parameters of all layers, bitwise.
P:L107: inter-subnet reproducibility "requires that the read-write interleaving among
subnets is equivalent to training each subnet sequentially, one at a time, according to the
order provided by the exploration algorithm".  P:L96: a later subnet reads a shared layer
"with the update made in the backward pass (with optimizer step) of the former".  CSP
(Def.2) reaches exactly this sequential result, so the oracle IS the sequential
definition:

    for y in 0..N-1 (chronological order):
        forward SN_y's active candidates in block order, loss, backward,
        theta[b, c_y[b]] -= lr * dL_y/dtheta[b, c_y[b]]   for every block b

Readings: plain SGD, constant lr, no momentum/weight decay, only active candidates change
(A3); dgrad uses pre-update weights (A4); loss = mean((y - t)^2) over all elements (A18);
no stem/head for the MLP/transformer families (A2).
"""
import numpy as np

from . import mlp, spos, transformer

FAMILIES = {"mlp": mlp, "transformer": transformer, "spos": spos}


def candidate_layout(cfg, b, c):
    if cfg["family"] == "mlp":
        return mlp.layout(cfg)
    if cfg["family"] == "transformer":
        return transformer.layout(cfg, c)
    if cfg["family"] == "spos":
        return spos.layout(cfg, b, c)
    raise ValueError(cfg["family"])


def candidate_size(cfg, b, c):
    return sum(int(np.prod(s)) for _, s, _, _ in candidate_layout(cfg, b, c))


def unpack(cfg, b, c, vec):
    """Packed float vector -> dict of float64 arrays (packing order of the layout)."""
    out, off = {}, 0
    for name, shape, _, _ in candidate_layout(cfg, b, c):
        n = int(np.prod(shape))
        out[name] = np.asarray(vec[off:off + n], dtype=np.float64).reshape(shape)
        off += n
    assert off == len(vec)
    return out


def pack(cfg, b, c, params):
    return np.concatenate([np.asarray(params[name], dtype=np.float64).ravel()
                           for name, _, _, _ in candidate_layout(cfg, b, c)])


def mse_loss(y, t):
    """A18: mean((y - t)^2) over all elements, and its gradient."""
    diff = y - t
    return float(np.mean(diff * diff)), 2.0 * diff / diff.size


def _block_fwd(cfg, p, x, c):
    if cfg["family"] == "mlp":
        return mlp.forward(p, x)
    return transformer.forward(p, x, cfg["choice_heads"][c], transformer.op_of(cfg, c))


def _block_bwd(cfg, p, tape, dy):
    if cfg["family"] == "mlp":
        return mlp.backward(p, tape, dy)
    return transformer.backward(p, tape, dy)


def frozen_theta(cfg):
    """SPOS frozen stem / head / FC weights: counter hash with reserved uids m*n + {0,1,2}."""
    from synth import init_packed
    base = cfg["n_blocks"] * cfg["n_choices"]
    out = {}
    for k, (part, segs) in enumerate(spos.frozen_layout(cfg).items()):
        name, shape, kind, fan = segs[0]
        v = init_packed(cfg["init_seed"], base + k, [(int(np.prod(shape)), kind, fan)])
        out[part] = {name: v.astype(np.float64).reshape(shape)}
    return out


def _spos_step(cfg, theta, choice, x, labels):
    """SPOS step; cfg["storage"] in (None, "fp64", "bf16", "bf16x2") selects the storage
    rounding of reading A28 (spos.Storage); default plain fp64."""
    q = spos.STORAGE[cfg.get("storage")]
    fz = frozen_theta(cfg)
    h = spos.stem_fwd(fz, np.asarray(x, dtype=np.float64), q)
    tapes = []
    for b, c in enumerate(choice):
        h, tp = spos.block_fwd(cfg, b, int(c), theta[(b, int(c))], h, q)
        tapes.append(tp)
    loss, dy = spos.head_loss(fz, h, np.asarray(labels, dtype=np.int64), q)
    grads = {}
    for b in reversed(range(len(choice))):
        c = int(choice[b])
        dy, g = spos.block_bwd(cfg, b, c, theta[(b, c)], tapes[b], dy, q)
        grads[(b, c)] = g
    return loss, grads


def subnet_step(cfg, theta, choice, x, t):
    """One subnet's forward + backward.  Returns (loss, grads{(b,c): dict}).

    Does not modify theta.  All gradients are taken at the pre-update parameters.
    SPOS: t is the integer label vector; the loss is the frozen head's mean cross-entropy.
    """
    if cfg["family"] == "spos":
        return _spos_step(cfg, theta, choice, x, t)
    h = np.asarray(x, dtype=np.float64)
    tapes = []
    for b, c in enumerate(choice):
        p = theta[(b, int(c))]
        h, tape = _block_fwd(cfg, p, h, int(c))
        tapes.append(tape)
    loss, dy = mse_loss(h, np.asarray(t, dtype=np.float64))
    grads = {}
    for b in reversed(range(len(choice))):
        c = int(choice[b])
        dy, g = _block_bwd(cfg, theta[(b, c)], tapes[b], dy)
        grads[(b, c)] = g
    return loss, grads


def sgd_apply(theta, grads, lr):
    for key, g in grads.items():
        p = theta[key]
        for name in g:
            p[name] = p[name] - lr * g[name]


def train_sequential(cfg, theta0, choices, batches, order=None):
    """O1.  theta0: {(b,c): packed vector}; choices: int [N, m]; batches: list of (x, t).

    ``order`` (default chronological 0..N-1) exists only for the reordering-invariance
    property test: any linear extension of the conflict order must give identical results.
    Returns (theta {(b,c): packed float64 vector}, losses [N]).
    """
    theta = {k: unpack(cfg, k[0], k[1], v) for k, v in theta0.items()}
    N = len(choices)
    losses = np.zeros(N)
    for y in (range(N) if order is None else order):
        x, t = batches[y]
        loss, grads = subnet_step(cfg, theta, choices[y], x, t)
        sgd_apply(theta, grads, cfg["lr"])
        losses[y] = loss
    return {k: pack(cfg, k[0], k[1], v) for k, v in theta.items()}, losses


def initial_theta(cfg):
    """theta0 from the shared counter hash (synth.init_packed), every candidate."""
    from synth import init_packed
    n = cfg["n_choices"]
    theta = {}
    for b in range(cfg["n_blocks"]):
        for c in range(n):
            segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in candidate_layout(cfg, b, c)]
            theta[(b, c)] = init_packed(cfg["init_seed"], b * n + c, segs)
    return theta


# --------------------------------------------------------------------------------------
# Other synchronisation policies (include/naspipe.h naspipe_sync)
# --------------------------------------------------------------------------------------
def train_bsp(cfg, theta0, choices, batches, bulk):
    """BSP (GPipe / Retiarii bulk update): subnets in bulks of ``bulk``
    consecutive ids; every subnet of a bulk computes its gradient at the bulk's start
    parameters, the bulk's gradients are summed in id order and applied at the flush.
    bulk = 1 is the sequential result (O1)."""
    theta = {k: unpack(cfg, k[0], k[1], v) for k, v in theta0.items()}
    N = len(choices)
    losses = np.zeros(N)
    for y0 in range(0, N, bulk):
        total = {}
        for y in range(y0, min(N, y0 + bulk)):
            x, t = batches[y]
            loss, grads = subnet_step(cfg, theta, choices[y], x, t)
            losses[y] = loss
            for key, g in grads.items():
                if key not in total:
                    total[key] = {name: np.array(v, dtype=np.float64) for name, v in g.items()}
                else:
                    for name in g:
                        total[key][name] = total[key][name] + g[name]
        sgd_apply(theta, total, cfg["lr"])
    return {k: pack(cfg, k[0], k[1], v) for k, v in theta.items()}, losses


def train_replay(cfg, theta0, choices, batches, stage_of_block, trace):
    """Execute a stage-level task trace [(t, K, kind, y)] in its order (MLP / transformer):
    F(y, K) runs stage K's blocks forward with the parameters current at that point, the
    last stage computes the loss and its seed gradient; B(y, K) back-propagates through
    stage K's blocks in reverse with the parameters current at its start (every input
    gradient of the task uses pre-update weights, reading A4), then applies SGD to stage K's
    candidates.  For a CSP trace this is the sequential result (O1); for an ASP trace it
    defines what the asynchronous pipeline computes (stale reads, no weight stashing)."""
    assert cfg["family"] in ("mlp", "transformer")
    theta = {k: unpack(cfg, k[0], k[1], v) for k, v in theta0.items()}
    D = int(max(stage_of_block)) + 1
    blocks = [[b for b in range(len(stage_of_block)) if stage_of_block[b] == K] for K in range(D)]
    act = {}    # (y, K) -> stage input
    tapes = {}  # (y, b) -> block tape
    grad = {}   # (y, K) -> gradient w.r.t. the stage output
    losses = np.zeros(len(choices))
    for (_, K, kind, y) in trace:
        ch = choices[y]
        if kind == 0:
            h = np.asarray(batches[y][0], dtype=np.float64) if K == 0 else act[(y, K)]
            for b in blocks[K]:
                h, tapes[(y, b)] = _block_fwd(cfg, theta[(b, int(ch[b]))], h, int(ch[b]))
            if K < D - 1:
                act[(y, K + 1)] = h
            else:
                losses[y], grad[(y, K)] = mse_loss(h, np.asarray(batches[y][1], dtype=np.float64))
        else:
            dy = grad.pop((y, K))
            grads = {}
            for b in reversed(blocks[K]):
                key = (b, int(ch[b]))
                dy, grads[key] = _block_bwd(cfg, theta[key], tapes.pop((y, b)), dy)
            if K > 0:
                grad[(y, K - 1)] = dy
            sgd_apply(theta, grads, cfg["lr"])
    return {k: pack(cfg, k[0], k[1], v) for k, v in theta.items()}, losses
