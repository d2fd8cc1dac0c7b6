"""Seeded synthetic workload generators shared by the tests, the oracle harness and bench.py.

This module holds NO arithmetic of the method (no forward/backward, no scheduling, no
update rule).  It only produces inputs: workload configurations, subnet choice vectors,
input batches and the counter-based initial parameter values.  Both sides of every parity
test receive what this module generates:

* the CUDA path receives choice vectors and batches through the C ABI and generates its own
  initial parameters with its own C++ implementation of the same counter hash;
* the oracle (``oracle/``) receives the same choice vectors and batches, and the initial
  parameters from :func:`init_packed` below.

Workload recipe:
* choices: uniform per choice block (§3 "Preliminaries": "per choice block
  uniform sampling"), NumPy PCG64 ``default_rng(arch_seed)``, arch_seed = 0;
* batch y: inputs and targets N(0,1) float32 from ``default_rng([data_seed, y])``,
  data_seed = 1, so batch y does not depend on how many subnets are generated;
* parameters: U(-1/sqrt(fan_in), 1/sqrt(fan_in)) from a splitmix64 counter hash keyed by
  (init_seed, candidate uid = b*n + c, element index i); LayerNorm gamma = 1, beta = 0.
"""
from __future__ import annotations

import copy
import numpy as np

ARCH_SEED = 0
DATA_SEED = 1
INIT_SEED = 2

# ----------------------------------------------------------------------------------------
# Workload configurations (BASELINE.json "configs").  Plain dicts so the
# oracle and the binding each interpret them with their own code.
# ----------------------------------------------------------------------------------------
CONFIGS = {
    # configs[0]: "toy supernet: 4 layers x 4 MLP choice blocks (width 64), 2 stages,
    # 16 subnets, batch 8, fp32"
    "toy": dict(family="mlp", n_blocks=4, n_choices=4, batch=8, width=64, lr=0.05,
                compute_dtype="fp32", n_stages=2, n_subnets=16),
    # configs[2]: "Transformer supernet (24 layers, choices over FFN width/heads, seq 128,
    # batch 32) bf16".  n = 4 = {h 8,16} x {f 2048,4096}.
    "transformer": dict(family="transformer", n_blocks=24, n_choices=4, batch=32,
                        d_model=1024, seq_len=128,
                        choice_heads=[8, 8, 16, 16], choice_ffn=[2048, 4096, 2048, 4096],
                        lr=0.01, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # configs[3]: "large Transformer supernet (48 layers x 8 choices)".
    "large_transformer": dict(family="transformer", n_blocks=48, n_choices=8, batch=32,
                              d_model=2048, seq_len=128,
                              choice_heads=[16] * 4 + [32] * 4,
                              choice_ffn=[4096, 8192, 12288, 16384] * 2,
                              lr=0.01, compute_dtype="bf16", n_stages=8, n_subnets=64),
    # NLP.c3 analog (Table 1: 48 choice blocks x 24 layers per block) over Table 5's
    # NLP ops (reading A38): {8/16-head attention, Conv 3x1, Sep Conv 7x1, Light
    # Conv 5x1 with 8/16 weight-sharing heads} x FFN {1024, 2048, 3072}; d, seq and batch of
    # configs[2].
    "nlp_c3": dict(family="transformer", n_blocks=48, n_choices=24, batch=32, d_model=1024, seq_len=128,
                   choice_op=[op for op in (0, 1, 2, 3) for _ in range(6)],
                   choice_heads=[h for _ in range(4) for h in (8, 16) for _ in range(3)],
                   choice_ffn=[f for _ in range(8) for f in (1024, 2048, 3072)],
                   lr=0.01, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # The other Table 1 NLP spaces (48 choice blocks x 96 / 72 / 48 layers), executed
    # (round 2): each layer a distinct (Table 5 op, heads, FFN width) combination over the
    # NLP.c3 op set; NLP.c2 fits all-resident in HBM (~18e9 params x 6 B), c1 / c0 run with
    # context switching (bench --budget-x).
    "nlp_c2": dict(family="transformer", n_blocks=48, n_choices=48, batch=32, d_model=1024, seq_len=128,
                   choice_op=[op for op in (0, 1, 2, 3) for _ in range(12)],
                   choice_heads=[h for _ in range(4) for h in (8, 16) for _ in range(6)],
                   choice_ffn=[f for _ in range(8) for f in (512, 1024, 1536, 2048, 3072, 4096)],
                   lr=0.01, compute_dtype="bf16", n_stages=8, n_subnets=256),
    "nlp_c1": dict(family="transformer", n_blocks=48, n_choices=72, batch=32, d_model=1024, seq_len=128,
                   choice_op=[op for op in (0, 1, 2, 3) for _ in range(18)],
                   choice_heads=[h for _ in range(4) for h in (8, 16) for _ in range(9)],
                   choice_ffn=[f for _ in range(8) for f in (512, 768, 1024, 1536, 2048, 2560, 3072, 3584, 4096)],
                   lr=0.01, compute_dtype="bf16", n_stages=8, n_subnets=256),
    "nlp_c0": dict(family="transformer", n_blocks=48, n_choices=96, batch=32, d_model=1024, seq_len=128,
                   choice_op=[op for op in (0, 1, 2, 3) for _ in range(24)],
                   choice_heads=[h for _ in range(4) for h in (8, 16) for _ in range(12)],
                   choice_ffn=[f for _ in range(8) for f in (256, 512, 768, 1024, 1280, 1536, 2048, 2560,
                                                            3072, 3328, 3584, 4096)],
                   lr=0.01, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # small supernet with every NLP op (parity tests of A38): Conv 3x1, Sep Conv 7x1, Light
    # Conv 5x1 (H = 4), attention
    "tiny_nlp": dict(family="transformer", n_blocks=4, n_choices=4, batch=2, d_model=192, seq_len=128,
                     choice_op=[1, 2, 3, 0], choice_heads=[3, 2, 4, 3], choice_ffn=[320, 384, 192, 256],
                     lr=0.01, compute_dtype="bf16", n_stages=2, n_subnets=8),
    # Small transformer used by the parity tests: several GEMM tiles in every dimension
    # and ragged tails (d=192 is 1.5 x 128; f=320 is 2.5 x 128), seq 128 like the real one.
    "tiny_transformer": dict(family="transformer", n_blocks=4, n_choices=3, batch=2,
                             d_model=192, seq_len=128,
                             choice_heads=[3, 2, 3], choice_ffn=[320, 384, 192],
                             lr=0.01, compute_dtype="bf16", n_stages=2, n_subnets=8),
    # configs[1]: "SPOS-style CNN supernet (20 layers x 4 choices, synthetic 224x224 images,
    # batch 64)": repeats [4,4,8,4], C_out [64,160,320,640], choices {Shuffle 3/5/7, Xception}.
    # lr 0.001 (A29): at 0.01 the 100-step sequential trajectory on random labels is
    # chaotic (fp32 vs fp64 storage alone differ by 3e-2 after 100 steps).
    "spos": dict(family="spos", n_blocks=20, n_choices=4, batch=64, image_hw=224, num_classes=1000,
                 stage_repeats=[4, 4, 8, 4], stage_channels=[64, 160, 320, 640], stem_channels=16,
                 head_channels=1024, choice_kernel=[3, 5, 7, 3], choice_xception=[0, 0, 0, 1],
                 lr=0.001, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # CV.c3 analog (Table 1: 32 choice blocks x 12 layers per block) over Table 5's CV
    # op types: Shuffle/Xception (separable) x k 3/5/7 x dilation 1/2 (A36);
    # same stages and image size as configs[1].
    "cv_c3": dict(family="spos", n_blocks=32, n_choices=12, batch=64, image_hw=224, num_classes=1000,
                  stage_repeats=[8, 8, 8, 8], stage_channels=[64, 160, 320, 640], stem_channels=16,
                  head_channels=1024, choice_kernel=[3, 5, 7] * 4, choice_xception=[0] * 6 + [1] * 6,
                  choice_dilation=[1, 1, 1, 2, 2, 2] * 2,
                  lr=0.001, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # The other Table 1 CV spaces (32 choice blocks x 24 / 48 layers), executed
    # (round 2): CV.c3's 12 op types (Shuffle / Xception x k 3/5/7 x dilation 1/2), each
    # present 2 / 4 times as separately trained candidates.
    "cv_c2": dict(family="spos", n_blocks=32, n_choices=24, batch=64, image_hw=224, num_classes=1000,
                  stage_repeats=[8, 8, 8, 8], stage_channels=[64, 160, 320, 640], stem_channels=16,
                  head_channels=1024, choice_kernel=[3, 5, 7] * 8, choice_xception=([0] * 6 + [1] * 6) * 2,
                  choice_dilation=[1, 1, 1, 2, 2, 2] * 4,
                  lr=0.001, compute_dtype="bf16", n_stages=8, n_subnets=256),
    "cv_c1": dict(family="spos", n_blocks=32, n_choices=48, batch=64, image_hw=224, num_classes=1000,
                  stage_repeats=[8, 8, 8, 8], stage_channels=[64, 160, 320, 640], stem_channels=16,
                  head_channels=1024, choice_kernel=[3, 5, 7] * 16, choice_xception=([0] * 6 + [1] * 6) * 4,
                  choice_dilation=[1, 1, 1, 2, 2, 2] * 8,
                  lr=0.001, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # configs[1] with Table 5's dense "Conv 3x3" (reading A40) in place of Shuffle 3: the CV
    # op set {Conv 3x3, Sep Conv 5x5 (Shuffle 5), Shuffle 7, Xception} at full size
    "spos_dense": dict(family="spos", n_blocks=20, n_choices=4, batch=64, image_hw=224, num_classes=1000,
                       stage_repeats=[4, 4, 8, 4], stage_channels=[64, 160, 320, 640], stem_channels=16,
                       head_channels=1024, choice_kernel=[3, 5, 7, 3], choice_xception=[2, 0, 0, 1],
                       lr=0.001, compute_dtype="bf16", n_stages=8, n_subnets=256),
    # small SPOS supernet with Table 5's dense "Conv 3x3" candidates (choice_xception 2, reading
    # A40) beside Shuffle 5 and Xception 3 (parity tests)
    "tiny_spos_dense": dict(family="spos", n_blocks=5, n_choices=4, batch=4, image_hw=64, num_classes=10,
                            stage_repeats=[1, 2, 1, 1], stage_channels=[32, 64, 96, 128], stem_channels=16,
                            head_channels=64, choice_kernel=[3, 5, 3, 3], choice_xception=[2, 0, 1, 2],
                            lr=0.001, compute_dtype="bf16", n_stages=2, n_subnets=8),
    # small SPOS supernet with dilated candidates (parity tests of A36)
    "tiny_spos_dil": dict(family="spos", n_blocks=5, n_choices=4, batch=4, image_hw=64, num_classes=10,
                          stage_repeats=[1, 2, 1, 1], stage_channels=[32, 64, 96, 128], stem_channels=16,
                          head_channels=64, choice_kernel=[3, 7, 5, 3], choice_xception=[0, 0, 1, 1],
                          choice_dilation=[2, 2, 2, 1], lr=0.001, compute_dtype="bf16", n_stages=2,
                          n_subnets=8),
    # small SPOS supernet for parity tests: every channel count a multiple of 16
    "tiny_spos": dict(family="spos", n_blocks=5, n_choices=4, batch=4, image_hw=64, num_classes=10,
                      stage_repeats=[1, 2, 1, 1], stage_channels=[32, 64, 96, 128], stem_channels=16,
                      head_channels=64, choice_kernel=[3, 5, 7, 3], choice_xception=[0, 0, 0, 1],
                      lr=0.001, compute_dtype="bf16", n_stages=2, n_subnets=8),
}


def sweep_config(n_choices: int) -> dict:
    """configs[4]: search-space sweep; C3 with a uniform candidate shape (h=16, f=3072)."""
    return dict(family="transformer", n_blocks=24, n_choices=n_choices, batch=32,
                d_model=1024, seq_len=128, choice_heads=[16] * n_choices,
                choice_ffn=[3072] * n_choices, lr=0.01, compute_dtype="bf16",
                n_stages=8, n_subnets=256)


def get_config(name: str, **overrides) -> dict:
    cfg = copy.deepcopy(CONFIGS[name])
    cfg.update(overrides)
    cfg.setdefault("init_seed", INIT_SEED)
    return cfg


# ----------------------------------------------------------------------------------------
# Subnet choice vectors
# ----------------------------------------------------------------------------------------
def sample_choices(n_subnets: int, n_blocks: int, n_choices: int,
                   seed: int = ARCH_SEED) -> np.ndarray:
    """Uniform per-block sampling.  Row y is subnet SN_y's choice vector."""
    rng = np.random.default_rng(seed)
    return rng.integers(0, n_choices, size=(n_subnets, n_blocks), dtype=np.int64).astype(np.int32)


# ----------------------------------------------------------------------------------------
# Batches
# ----------------------------------------------------------------------------------------
def batch_shape(cfg: dict) -> tuple:
    if cfg["family"] == "mlp":
        return (cfg["batch"], cfg["width"])
    if cfg["family"] == "transformer":
        return (cfg["batch"], cfg["seq_len"], cfg["d_model"])
    if cfg["family"] == "spos":
        return (cfg["batch"], cfg["image_hw"], cfg["image_hw"], 3)
    raise ValueError(cfg["family"])


def make_batch(cfg: dict, y: int, seed: int = DATA_SEED):
    """Input and target for subnet y: N(0,1) float32, independent of N.
    SPOS: the target is an int32 label vector, uniform in [0, num_classes)."""
    rng = np.random.default_rng([seed, int(y)])
    shp = batch_shape(cfg)
    x = rng.standard_normal(shp, dtype=np.float32)
    if cfg["family"] == "spos":
        t = rng.integers(0, cfg["num_classes"], size=cfg["batch"], dtype=np.int64).astype(np.int32)
    else:
        t = rng.standard_normal(shp, dtype=np.float32)
    return x, t


# ----------------------------------------------------------------------------------------
# Counter-based initial parameters (SURVEY §8c reading A21)
# ----------------------------------------------------------------------------------------
_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLD = np.uint64(0x9E3779B97F4A7C15)


def _splitmix64(x: np.ndarray) -> np.ndarray:
    with np.errstate(over="ignore"):
        z = x + _GOLD
        z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        z = z ^ (z >> np.uint64(31))
    return z


def hash_uniform(seed: int, uid: int, start: int, count: int) -> np.ndarray:
    """u_i = (splitmix64(seed ^ (uid*GOLD + i)) >> 40) * 2^-24 for i in [start, start+count)."""
    i = np.arange(start, start + count, dtype=np.uint64)
    with np.errstate(over="ignore"):
        key = np.uint64(seed) ^ (np.uint64(uid) * _GOLD + i)
    z = _splitmix64(key)
    return (z >> np.uint64(40)).astype(np.float32) * np.float32(2.0 ** -24)


def init_packed(seed: int, uid: int, segments) -> np.ndarray:
    """Packed float32 parameter vector of one candidate.

    ``segments`` is a list of (size, kind, fan_in) in packing order, kind in
    {"uniform", "ones", "zeros"}.  Element i of the packed vector (counted over all
    segments) uses counter i, so the value does not depend on how segments are grouped.
    """
    total = sum(s for s, _, _ in segments)
    out = np.empty(total, dtype=np.float32)
    off = 0
    for size, kind, fan_in in segments:
        if kind == "uniform":
            bound = np.float32(1.0) / np.sqrt(np.float32(fan_in))
            u = hash_uniform(seed, uid, off, size)
            out[off:off + size] = bound * (np.float32(2.0) * u - np.float32(1.0))
        elif kind == "ones":
            out[off:off + size] = 1.0
        elif kind == "zeros":
            out[off:off + size] = 0.0
        else:
            raise ValueError(kind)
        off += size
    return out


def cost_table_uniform(n_blocks: int, n_choices: int, cf: int = 1, cb: int = 2):
    """The canonical unit cost table of SURVEY §8c A8 (cf=1, cb=2 per block)."""
    return (np.full((n_blocks, n_choices), cf, dtype=np.int32),
            np.full((n_blocks, n_choices), cb, dtype=np.int32))
