"""Host-side C ABI tests (no GPU): the library loads and exports every declared symbol; the
C++ planner, dependency table, partition, residency planner and initialiser agree
bit-exactly with the oracle (SURVEY §4 tier T1)."""
import json
import os
import re

import numpy as np
import pytest

import synth
from oracle import csp, residency, train

npipe = pytest.importorskip("paper_conf_asplos_zhaolcscwzlc22_b200")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "naspipe.h")).read()
    declared = set(re.findall(r"^(?:int|void|const char\s*\*)\s+(naspipe_[a-z_0-9]+)\s*\(", hdr, re.M))
    assert declared, "no declarations parsed"
    for name in sorted(declared):
        assert hasattr(npipe.lib, name), name
    assert declared == set(npipe.EXPORTED_SYMBOLS)
    assert npipe.naspipe_abi_version() == 4


@pytest.mark.parametrize("name", ["toy", "tiny_transformer", "transformer", "tiny_nlp", "nlp_c3"])
def test_init_params_match_shared_hash(name):
    """Packed sizes and counter-hash init equal the oracle's layout (nlp: every op, A38)."""
    cfg = synth.get_config(name)
    spec = npipe.Spec(cfg)
    n = cfg["n_choices"]
    pairs = [(0, 0), (1, n - 1), (cfg["n_blocks"] - 1, n // 2)]
    if name in ("tiny_nlp", "nlp_c3"):
        pairs += [(2, c) for c in range(n)]
    for (b, c) in pairs:
        got = npipe.naspipe_init_params(spec, b, c)
        segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in train.candidate_layout(cfg, b, c)]
        assert npipe.naspipe_param_count(spec, b, c) == sum(s for s, _, _ in segs)
        if name in ("transformer", "nlp_c3") and (b, c) not in ((0, 0), (2, 6), (2, 12), (2, 18)):
            continue  # one full-size candidate is enough (12.6 M floats)
        ref = synth.init_packed(cfg["init_seed"], b * n + c, segs)
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), (b, c)


@pytest.mark.parametrize("name", ["tiny_spos", "spos", "tiny_spos_dil", "cv_c3", "tiny_spos_dense"])
def test_spos_layout_and_init_match_oracle(name):
    """SPOS candidates: packed sizes and counter-hash values equal the oracle's layout
    (oracle/spos.py layout) for every candidate kind (stride 1/2, Shuffle k=3/5/7, Xception
    k=3/5/7, dilation 1/2)."""
    cfg = synth.get_config(name)
    spec = npipe.Spec(cfg)
    n, m = cfg["n_choices"], cfg["n_blocks"]
    for b in range(m):
        for c in range(n):
            segs = [(int(np.prod(s)), kind, fan) for _, s, kind, fan in train.candidate_layout(cfg, b, c)]
            assert npipe.naspipe_param_count(spec, b, c) == sum(s for s, _, _ in segs), (b, c)
            if name in ("spos", "cv_c3") and b not in (0, 1, m - 1):
                continue
            got = npipe.naspipe_init_params(spec, b, c)
            ref = synth.init_packed(cfg["init_seed"], b * n + c, segs)
            assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), (b, c)
    fz = train.frozen_theta(cfg)
    for part, key in enumerate(["stem", "head", "fc"]):
        ref = fz[key]["w"].ravel().astype(np.float32)
        got = npipe.naspipe_init_frozen(spec, part, ref.size)
        assert np.array_equal(got.view(np.uint32), ref.view(np.uint32)), key


@pytest.mark.parametrize("name,m,n", [("nlp_c0", 48, 96), ("nlp_c1", 48, 72), ("nlp_c2", 48, 48), ("nlp_c3", 48, 24),
                                      ("cv_c1", 32, 48), ("cv_c2", 32, 24), ("cv_c3", 32, 12)])
def test_table1_space_configs(name, m, n):
    """Table 1's spaces as executable configs: m blocks x n candidates, every
    NLP candidate a distinct (op, heads, FFN) combination over Table 5's NLP ops, every CV
    candidate one of CV.c3's 12 op types; the library accepts every candidate and its packed
    size equals the oracle's layout (candidates of block 0 and the last block)."""
    cfg = synth.get_config(name)
    assert (cfg["n_blocks"], cfg["n_choices"]) == (m, n)
    keys = sorted(k for k in cfg if k.startswith("choice_"))
    assert all(len(cfg[k]) == n for k in keys)
    kinds = set(zip(*[cfg[k] for k in keys]))
    assert len(kinds) == (n if cfg["family"] == "transformer" else 12)
    spec = npipe.Spec(cfg)
    for b in (0, m - 1):
        for c in range(n):
            segs = [int(np.prod(s)) for _, s, _, _ in train.candidate_layout(cfg, b, c)]
            assert npipe.naspipe_param_count(spec, b, c) == sum(segs), (b, c)


def test_nlp_op_spec_validation():
    cfg = synth.get_config("tiny_nlp")
    for bad in (dict(choice_op=[1, 2, 4, 0]), dict(choice_op=[1, 2, -1, 0]), dict(choice_heads=[3, 2, 5, 3])):
        with pytest.raises(npipe.NaspipeError):
            npipe.naspipe_default_costs(npipe.Spec(dict(cfg, **bad)))
    # Light Conv heads need not give a 16-multiple head dim (only attention does): H = 12, d/H = 16
    npipe.naspipe_default_costs(npipe.Spec(dict(cfg, choice_heads=[3, 2, 12, 3])))
    cf, cb = npipe.naspipe_default_costs(npipe.Spec(synth.get_config("nlp_c3")))
    assert (cf >= 1).all() and (cb > cf).all()


def test_spos_spec_validation():
    cfg = synth.get_config("tiny_spos")
    for bad in (dict(stage_repeats=[1, 2, 1, 2]), dict(stage_channels=[32, 64, 80, 128]),
                dict(choice_kernel=[3, 5, 4, 3]), dict(image_hw=48), dict(head_channels=60),
                dict(choice_xception=[0, 0, 3, 1]), dict(choice_dilation=[1, 3, 1, 1]),
                # the dense Conv 3x3 (xception 2, reading A40) takes k 3 and dilation 1 only
                dict(choice_xception=[0, 2, 0, 1]), dict(choice_xception=[2, 0, 0, 1], choice_dilation=[2, 1, 1, 1]),
                dict(choice_dilation=[1, 0, 1, 1])):
        with pytest.raises(npipe.NaspipeError):
            npipe.naspipe_default_costs(npipe.Spec(dict(cfg, **bad)))
    cf, cb = npipe.naspipe_default_costs(npipe.Spec(synth.get_config("spos")))
    assert (cf >= 1).all() and (cb > cf).all()
    assert (npipe.naspipe_partition(npipe.Spec(synth.get_config("spos")), 8) == np.sort(
        npipe.naspipe_partition(npipe.Spec(synth.get_config("spos")), 8))).all()


def _random_case(seed):
    rng = np.random.default_rng(seed)
    N = int(rng.integers(3, 40))
    m = int(rng.integers(1, 9))
    n = int(rng.integers(1, 6))
    D = int(rng.integers(1, m + 1))
    W = int(rng.integers(1, 4 * D + 3))
    lam = int(rng.integers(0, 3))
    policy = int(rng.integers(0, 2))
    cf = rng.integers(0, 5, size=(m, n)).astype(np.int32)
    cb = rng.integers(0, 7, size=(m, n)).astype(np.int32)
    ch = synth.sample_choices(N, m, n, seed)
    cfg = dict(family="mlp", n_blocks=m, n_choices=n, batch=2, width=8, lr=0.05, compute_dtype="fp32",
               window=W, link_latency=lam, bwd_policy=policy, cost_fwd=cf, cost_bwd=cb)
    return cfg, ch, D


@pytest.mark.parametrize("seed", range(40))
def test_planner_matches_oracle_bit_exact(seed):
    cfg, ch, D = _random_case(seed)
    spec = npipe.Spec(cfg)
    sob = npipe.naspipe_partition(spec, D)
    wts = csp.block_partition_cost(cfg["cost_fwd"], cfg["cost_bwd"])
    np.testing.assert_array_equal(sob, csp.balanced_partition(wts, D))
    plan = npipe.naspipe_plan(spec, D, ch)
    tf, tb = csp.task_costs(ch, sob, cfg["cost_fwd"], cfg["cost_bwd"], D)
    ref = csp.simulate_csp(ch, sob, D, cfg["window"], tf, tb, lam=cfg["link_latency"], policy=cfg["bwd_policy"])
    got = [tuple(int(v) for v in row) for row in plan.trace()]
    assert got == [tuple(r) for r in ref["trace"]]
    assert plan.makespan() == ref["makespan"]
    st, bu = plan.idle(D)
    assert list(st) == ref["stall"] and list(bu) == ref["bubble"]
    for y in range(len(ch)):
        for K in range(D):
            assert plan.deps(y, K) == sorted(csp.deps(ch, sob, y, K))


def test_worked_example_through_c_abi():
    ch = np.array([[0, 0], [1, 0], [0, 1], [1, 1]])
    cfg = dict(family="mlp", n_blocks=2, n_choices=2, batch=2, width=8, compute_dtype="fp32", window=4,
               cost_fwd=np.ones((2, 2)), cost_bwd=np.full((2, 2), 2), stage_of_block=[0, 1])
    plan = npipe.naspipe_plan(npipe.Spec(cfg), 2, ch)
    assert plan.makespan() == 15
    s0 = [("F" if k == 0 else "B") + f"{y}@{t}" for t, K, k, y in plan.trace() if K == 0]
    assert s0 == ["F0@0", "F1@1", "B0@4", "F2@6", "B1@7", "F3@9", "B2@10", "B3@13"]
    # residency worked example 2 needs unit candidate sizes: check ordering semantics via
    # the oracle on the library's own plan at D = 1 with bytes = 4 * params (all equal)
    plan1 = npipe.naspipe_plan(npipe.Spec(dict(cfg, stage_of_block=[0, 0])), 1, ch)
    P = 4 * npipe.naspipe_param_count(npipe.Spec(cfg), 0, 0)
    ev, wb = plan1.residency(0, 3 * P, 2)
    got = [("LOAD" if op == 0 else "EVICT") + f"({i},{u})" for _, i, op, u in ev]
    assert got == ["LOAD(0,0)", "LOAD(0,2)", "LOAD(1,1)", "EVICT(4,2)", "LOAD(4,3)"]
    assert wb == 1


@pytest.mark.parametrize("seed", range(15))
def test_residency_matches_oracle(seed):
    cfg, ch, D = _random_case(100 + seed)
    cfg = dict(cfg, family="transformer", d_model=16, seq_len=16, compute_dtype="bf16",
               choice_heads=[1] * cfg["n_choices"],
               choice_ffn=[16 * (1 + c % 3) for c in range(cfg["n_choices"])])
    spec = npipe.Spec(cfg)
    plan = npipe.naspipe_plan(spec, D, ch)
    sob = npipe.naspipe_partition(spec, D)
    tr = plan.trace()
    n, m = cfg["n_choices"], cfg["n_blocks"]
    nbytes = {b * n + c: 4 * npipe.naspipe_param_count(spec, b, c) for b in range(m) for c in range(n)}
    rng = np.random.default_rng(seed)
    for K in range(D):
        order = [(int(k), int(y)) for t, KK, k, y in tr if KK == K]
        blocks = [b for b in range(m) if sob[b] == K]
        uses = residency.stage_uses(order, ch, blocks, n)
        need = max(sum(nbytes[u] for u in us) for us in uses)
        budget = int(need * rng.uniform(1.0, 3.0))
        for depth in (1, 2, 3):
            for horizon in (None, 1, 3, 8):
                ref = residency.simulate_residency(uses, [k for k, _ in order], nbytes, budget, L=depth,
                                                   horizon=horizon)
                ev, wb = plan.residency(K, budget, depth, -1 if horizon is None else horizon)
                got = [("LOAD" if op == 0 else "EVICT", int(i), int(u)) for _, i, op, u in ev]
                assert got == ref["events"], (K, depth, horizon)
                assert wb == len(ref["writebacks"])


def test_budget_error_and_invalid_args():
    cfg = dict(family="mlp", n_blocks=2, n_choices=2, batch=2, width=8, compute_dtype="fp32")
    spec = npipe.Spec(cfg)
    plan = npipe.naspipe_plan(spec, 1, np.array([[0, 0], [1, 1]]))
    P = 4 * npipe.naspipe_param_count(spec, 0, 0)
    with pytest.raises(npipe.NaspipeError) as e:
        plan.residency(0, P, 2)            # one task needs 2 candidates
    assert e.value.code == -6
    with pytest.raises(npipe.NaspipeError) as e:
        npipe.naspipe_plan(spec, 1, np.array([[0, 2]]))   # choice out of range
    assert e.value.code == -1
    with pytest.raises(npipe.NaspipeError):
        npipe.naspipe_plan(spec, 3, np.array([[0, 0]]))   # more stages than blocks
    bad = npipe.Spec(dict(cfg, family="transformer", d_model=24, seq_len=8, compute_dtype="bf16",
                          choice_heads=[1, 1], choice_ffn=[16, 16]))   # d_model % 16 != 0
    with pytest.raises(npipe.NaspipeError) as e:
        npipe.naspipe_param_count(bad, 0, 0)
    assert e.value.code == -1


def test_default_costs_and_partition_of_real_configs():
    for name, D in [("transformer", 8), ("large_transformer", 8), ("toy", 2)]:
        cfg = synth.get_config(name)
        spec = npipe.Spec(cfg)
        cf, cb = npipe.naspipe_default_costs(spec)
        assert (cf >= 1).all() and (cb >= cf).all()
        sob = npipe.naspipe_partition(spec, D)
        assert sob[0] == 0 and sob[-1] == D - 1 and np.all(np.diff(sob) >= 0)
        if name == "toy":
            assert list(sob) == [0, 0, 1, 1]


@pytest.mark.parametrize("sync", ["inorder", "asp", "bsp", "serial"])
@pytest.mark.parametrize("seed", range(12))
def test_sync_policies_match_oracle_bit_exact(sync, seed):
    """the C++ planner's INORDER / ASP / BSP schedules equal the oracle's."""
    cfg, ch, D = _random_case(100 + seed)
    cfg = dict(cfg, sync=sync, bulk_size=int(np.random.default_rng(seed).integers(0, 6)))
    spec = npipe.Spec(cfg)
    sob = npipe.naspipe_partition(spec, D)
    plan = npipe.naspipe_plan(spec, D, ch)
    tf, tb = csp.task_costs(ch, sob, cfg["cost_fwd"], cfg["cost_bwd"], D)
    ref = csp.simulate_csp(ch, sob, D, cfg["window"], tf, tb, lam=cfg["link_latency"], policy=cfg["bwd_policy"],
                           sync=sync, bulk=cfg["bulk_size"])
    assert [tuple(int(v) for v in row) for row in plan.trace()] == [tuple(r) for r in ref["trace"]]
    assert plan.makespan() == ref["makespan"]
    st, bu = plan.idle(D)
    assert list(st) == ref["stall"] and list(bu) == ref["bubble"]


def test_bsp_needs_resident_candidates():
    """BSP executes with every candidate resident (its accumulators live beside the
    masters); with a context-switch budget create fails with EINVAL before touching CUDA."""
    cfg = dict(synth.get_config("toy"), sync="bsp", hbm_weight_budget_bytes=1 << 20)
    with pytest.raises(npipe.NaspipeError) as e:
        npipe.naspipe_create(npipe.Spec(cfg), 1)
    assert e.value.code == -1


def test_mirrored_plan_matches_oracle_bit_exact():
    """naspipe_plan_mirrored (C++) vs oracle.csp.simulate_csp_mirrored: partitions, every
    task start, makespan and idle ticks, on the worked example and random cases."""
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "mirror_worked_example.json")))
    base = synth.get_config("toy")
    cfg = dict(base, n_blocks=3, n_choices=2, cost_fwd=np.array(g["cost_f"]), cost_bwd=np.array(g["cost_b"]), window=4)
    for key, lw in (("lam_w_0", 0), ("lam_w_3", 3)):
        r = npipe.naspipe_plan_mirrored(npipe.Spec(cfg), 2, g["choices"], lw)
        assert r["stage_of_block"].tolist() == g["stage_of_block"]
        assert r["trace"].tolist() == g[key]["trace"] and r["makespan"] == g[key]["makespan"]
    rng = np.random.default_rng(5)
    for _ in range(40):
        m, n = int(rng.integers(2, 8)), int(rng.integers(1, 5))
        D, N = int(rng.integers(1, min(m, 4) + 1)), int(rng.integers(1, 16))
        W, lam, lw = int(rng.integers(1, 6)), int(rng.integers(0, 3)), int(rng.integers(0, 4))
        ch = rng.integers(0, n, (N, m))
        cf, cb = rng.integers(0, 5, (m, n)), rng.integers(0, 9, (m, n))
        spec = npipe.Spec(dict(base, n_blocks=m, n_choices=n, cost_fwd=cf, cost_bwd=cb, window=W, link_latency=lam))
        r = npipe.naspipe_plan_mirrored(spec, D, ch, lw)
        sob = csp.subnet_partitions(ch.tolist(), cf, cb, D)
        o = csp.simulate_csp_mirrored(ch.tolist(), sob, D, W, cf, cb, lam=lam, lam_w=lw)
        assert np.array_equal(r["stage_of_block"], sob)
        assert [tuple(t) for t in r["trace"].tolist()] == [tuple(t) for t in o["trace"]]
        assert r["makespan"] == o["makespan"]
        assert r["stall"].tolist() == list(o["stall"]) and r["bubble"].tolist() == list(o["bubble"])


def test_mirrored_plan_rejects_other_policies():
    cfg = synth.get_config("toy")
    ch = synth.sample_choices(3, cfg["n_blocks"], cfg["n_choices"])
    for over in (dict(sync="asp"), dict(bwd_policy=1)):
        with pytest.raises(npipe.NaspipeError):
            npipe.naspipe_plan_mirrored(npipe.Spec(cfg, **over), 2, ch)
    with pytest.raises(npipe.NaspipeError):
        npipe.naspipe_plan_mirrored(npipe.Spec(cfg), 2, ch, -1)
    with pytest.raises(npipe.NaspipeError):
        npipe.naspipe_plan_mirrored(npipe.Spec(cfg), 2, np.full_like(ch, cfg["n_choices"]))


def test_recompute_flag_validation():
    """NASPIPE_FLAG_RECOMPUTE: transformer family only, never with ASP (EINVAL)."""
    ok = synth.get_config("tiny_transformer")
    npipe.naspipe_partition(npipe.Spec(ok, flags=npipe.FLAG_RECOMPUTE), 2)
    for cfg in (synth.get_config("toy"), synth.get_config("tiny_spos"), synth.get_config("tiny_transformer", sync="asp")):
        with pytest.raises(npipe.NaspipeError) as e:
            npipe.naspipe_partition(npipe.Spec(cfg, flags=npipe.FLAG_RECOMPUTE), 2)
        assert e.value.code == -1


def test_sass_gemm_kernels_are_tcgen05():
    """Every GEMM instantiation in libnaspipe.so issues tcgen05.mma (SASS UTCHMMA), reads
    TMEM (LDTM), is fed by TMA (UTMALDG) and has no legacy HMMA (tools/sass_census.py;
    profiles/r2_sass_census.md) -- a regression to a non-tcgen05 GEMM fails here."""
    import shutil
    import sys as _s
    if not os.path.exists("/usr/local/cuda/bin/cuobjdump") or shutil.which("c++filt") is None:
        pytest.skip("cuobjdump / c++filt not available")
    _s.path.insert(0, os.path.join(ROOT, "tools"))
    import sass_census
    kernels, names = sass_census.census()
    gemms = [k for k in kernels if "gemm_tc_kernel" in names[k] or "gemm_pair_kernel" in names[k]]
    assert len(gemms) >= 20, len(gemms)
    for k in gemms:
        c = kernels[k]
        assert c["UTCHMMA"] > 0 and c["LDTM"] > 0 and c["UTMALDG"] > 0 and c["HMMA"] == 0, (names[k], c)
