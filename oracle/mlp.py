"""MLP candidate (configs[0] "toy supernet ... MLP choice blocks (width 64)").

Block internals are not given by the paper (Table 5 P:L439-450 lists op types only); the
reading is SURVEY §8c A17: ``y = x + tanh(x W^T + b)``, W [d,d] row-major [out,in], b [d].
Packing order (SURVEY §8b get_params): W then b.
"""
import numpy as np


def layout(cfg):
    d = cfg["width"]
    return [("W", (d, d), "uniform", d), ("b", (d,), "uniform", d)]


def forward(p, x):
    """x: [B, d] float64.  Returns (y, tape)."""
    z = x @ p["W"].T + p["b"]
    h = np.tanh(z)
    return x + h, (x, h)


def backward(p, tape, dy):
    """Returns (dx, grads) — dx uses the pre-update weights (reading A4)."""
    x, h = tape
    dz = dy * (1.0 - h * h)
    dx = dy + dz @ p["W"]
    return dx, {"W": dz.T @ x, "b": dz.sum(axis=0)}
