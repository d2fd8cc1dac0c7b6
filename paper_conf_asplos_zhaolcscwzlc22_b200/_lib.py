"""ctypes marshalling for include/naspipe.h.  No computation happens here."""
import ctypes as C
import os

import numpy as np

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libnaspipe.so")
if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: build it with "
                      "`python -m paper_conf_asplos_zhaolcscwzlc22_b200.build` (no CPU fallback exists)")
lib = C.CDLL(LIB_PATH)

ABI_VERSION = 4
SYNC = {"csp": 0, "inorder": 1, "asp": 2, "bsp": 3, "serial": 4}  # naspipe_sync (include/naspipe.h)
FAMILY = {"mlp": 0, "transformer": 1, "spos": 2}
DTYPE = {"fp32": 0, "bf16": 1}
BATCH_HOST, BATCH_DEVICE, BATCH_SYNTHETIC = 0, 1, 2
FLAG_TRACE, FLAG_VERSION_CHECK, FLAG_NULL_KERNELS, FLAG_TIMING, FLAG_RECOMPUTE, FLAG_MIRROR = 1, 2, 4, 8, 16, 32
FLAG_TIMED = 64
STATS_FIELDS = ["tasks", "kernel_launches", "h2d_bytes", "d2h_bytes", "p2p_bytes", "makespan_ticks",
                "dominant_launches", "dominant_flops", "dominant_ms", "res_loads", "res_evicts",
                "writebacks", "version_checks", "gemm_flops", "gemm_launches", "all_bytes"]

_i32p = C.POINTER(C.c_int32)
_i64p = C.POINTER(C.c_int64)


class _SpecStruct(C.Structure):
    _fields_ = [("abi_version", C.c_int32), ("family", C.c_int32), ("n_blocks", C.c_int32),
                ("n_choices", C.c_int32), ("batch", C.c_int32), ("compute_dtype", C.c_int32),
                ("width", C.c_int32), ("d_model", C.c_int32), ("seq_len", C.c_int32),
                ("choice_heads", _i32p), ("choice_ffn", _i32p), ("lr", C.c_float),
                ("init_seed", C.c_uint64), ("stage_of_block", _i32p), ("cost_fwd", _i32p),
                ("cost_bwd", _i32p), ("window", C.c_int32), ("lookahead", C.c_int32),
                ("residency_horizon", C.c_int32),
                ("hbm_weight_budget_bytes", C.c_int64), ("bwd_policy", C.c_int32),
                ("link_latency", C.c_int32), ("flags", C.c_int32),
                ("image_hw", C.c_int32), ("num_classes", C.c_int32), ("stem_channels", C.c_int32),
                ("head_channels", C.c_int32), ("n_cnn_stages", C.c_int32), ("stage_repeats", _i32p),
                ("stage_channels", _i32p), ("choice_kernel", _i32p), ("choice_xception", _i32p),
                ("sync_policy", C.c_int32), ("bulk_size", C.c_int32), ("choice_dilation", _i32p), ("choice_op", _i32p)]


class _BatchStruct(C.Structure):
    _fields_ = [("input", C.c_void_p), ("target", C.c_void_p), ("where", C.c_int32),
                ("synth_seed", C.c_uint64)]


def _sig(name, res, args):
    f = getattr(lib, name)
    f.restype = res
    f.argtypes = args
    return f


_SP = C.POINTER(_SpecStruct)
_sig("naspipe_last_error", C.c_char_p, [])
_sig("naspipe_abi_version", C.c_int, [])
_sig("naspipe_create", C.c_int, [_SP, C.c_int32, C.POINTER(C.c_void_p)])
_sig("naspipe_create_rank", C.c_int, [_SP, C.c_int32, C.c_int32, C.c_int32, C.c_void_p, C.POINTER(C.c_void_p)])
_sig("naspipe_submit", C.c_int, [C.c_void_p, _i32p, C.POINTER(_BatchStruct), _i64p])
_sig("naspipe_drain", C.c_int, [C.c_void_p])
_sig("naspipe_get_params", C.c_int, [C.c_void_p, C.c_int32, C.c_int32, C.POINTER(C.c_float), C.c_size_t])
_sig("naspipe_set_params", C.c_int, [C.c_void_p, C.c_int32, C.c_int32, C.POINTER(C.c_float), C.c_size_t])
_sig("naspipe_get_losses", C.c_int, [C.c_void_p, C.POINTER(C.c_float), C.c_int64])
_sig("naspipe_get_trace", C.c_int, [C.c_void_p, _i64p, C.c_size_t, C.POINTER(C.c_size_t)])
_sig("naspipe_get_stats", C.c_int, [C.c_void_p, C.POINTER(C.c_double)])
_sig("naspipe_set_timing", C.c_int, [C.c_void_p, C.c_int])
_sig("naspipe_get_residency_trace", C.c_int, [C.c_void_p, _i64p, C.c_size_t, C.POINTER(C.c_size_t)])
_sig("naspipe_get_timed_stats", C.c_int, [C.c_void_p, C.POINTER(C.c_double)])
_sig("naspipe_destroy", None, [C.c_void_p])
_sig("naspipe_param_count", C.c_int, [_SP, C.c_int32, C.c_int32, C.POINTER(C.c_size_t)])
_sig("naspipe_default_costs", C.c_int, [_SP, _i32p, _i32p])
_sig("naspipe_partition", C.c_int, [_SP, C.c_int32, _i32p])
_sig("naspipe_plan_mirrored", C.c_int, [_SP, C.c_int32, _i32p, C.c_int64, C.c_int32, _i32p, _i64p, C.c_size_t,
                                        C.POINTER(C.c_size_t), _i64p, _i64p, _i64p])
_sig("naspipe_init_params", C.c_int, [_SP, C.c_int32, C.c_int32, C.POINTER(C.c_float), C.c_size_t])
_sig("naspipe_init_frozen", C.c_int, [_SP, C.c_int32, C.POINTER(C.c_float), C.c_size_t])
_sig("naspipe_plan_create", C.c_int, [_SP, C.c_int32, _i32p, C.c_int64, C.POINTER(C.c_void_p)])
_sig("naspipe_plan_trace", C.c_int, [C.c_void_p, _i64p, C.c_size_t, C.POINTER(C.c_size_t)])
_sig("naspipe_plan_makespan", C.c_int, [C.c_void_p, _i64p])
_sig("naspipe_plan_deps", C.c_int, [C.c_void_p, C.c_int64, C.c_int32, _i64p, C.c_size_t, C.POINTER(C.c_size_t)])
_sig("naspipe_plan_residency", C.c_int, [C.c_void_p, C.c_int32, C.c_int64, C.c_int32, C.c_int32, _i64p,
                                         C.c_size_t, C.POINTER(C.c_size_t), _i64p])
_sig("naspipe_plan_idle", C.c_int, [C.c_void_p, _i64p, _i64p])
_sig("naspipe_plan_comm_schedule", C.c_int, [C.c_void_p, C.c_int32, _i64p, C.c_size_t, C.POINTER(C.c_size_t)])
_sig("naspipe_plan_destroy", None, [C.c_void_p])
_sig("naspipe_nccl_unique_id", C.c_int, [C.c_void_p])
_sig("naspipe_set_pdl", C.c_int, [C.c_int])
_sig("naspipe_create_rank_peer", C.c_int, [_SP, C.c_int32, C.c_int32, C.c_int32, C.POINTER(C.c_void_p)])
_sig("naspipe_peer_export", C.c_int, [C.c_void_p, C.c_void_p, C.c_size_t, C.POINTER(C.c_size_t)])
_sig("naspipe_peer_connect", C.c_int, [C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p, C.c_size_t])

EXPORTED_SYMBOLS = [
    "naspipe_create", "naspipe_create_rank", "naspipe_submit", "naspipe_drain", "naspipe_get_params",
    "naspipe_set_params", "naspipe_get_losses", "naspipe_get_trace", "naspipe_get_stats", "naspipe_set_timing",
    "naspipe_get_residency_trace", "naspipe_destroy", "naspipe_param_count", "naspipe_default_costs",
    "naspipe_partition", "naspipe_init_params", "naspipe_init_frozen", "naspipe_plan_create", "naspipe_plan_trace",
    "naspipe_plan_makespan", "naspipe_plan_deps", "naspipe_plan_residency", "naspipe_plan_destroy",
    "naspipe_plan_comm_schedule", "naspipe_plan_idle", "naspipe_plan_mirrored",
    "naspipe_nccl_unique_id", "naspipe_last_error", "naspipe_abi_version",
    "naspipe_create_rank_peer", "naspipe_peer_export", "naspipe_peer_connect", "naspipe_set_pdl",
    "naspipe_get_timed_stats"]


class NaspipeError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"naspipe error {code}: {msg}")
        self.code = code


def _check(rc):
    if rc != 0:
        raise NaspipeError(rc, lib.naspipe_last_error().decode(errors="replace"))


def _i32(a):
    a = np.ascontiguousarray(a, dtype=np.int32)
    return a, a.ctypes.data_as(_i32p)


class Spec:
    """naspipe_supernet_spec built from a workload dict (synth.CONFIGS style)."""

    def __init__(self, cfg, **over):
        cfg = dict(cfg, **over)
        s = _SpecStruct()
        s.abi_version = ABI_VERSION
        s.family = FAMILY[cfg["family"]]
        s.n_blocks, s.n_choices, s.batch = cfg["n_blocks"], cfg["n_choices"], cfg["batch"]
        s.compute_dtype = DTYPE[cfg.get("compute_dtype", "fp32")]
        s.width = cfg.get("width", 0)
        s.d_model, s.seq_len = cfg.get("d_model", 0), cfg.get("seq_len", 0)
        self._keep = []
        for name in ("choice_heads", "choice_ffn", "stage_of_block", "cost_fwd", "cost_bwd", "stage_repeats",
                     "stage_channels", "choice_kernel", "choice_xception", "choice_dilation", "choice_op"):
            if cfg.get(name) is not None:
                arr, ptr = _i32(np.asarray(cfg[name]).ravel())
                self._keep.append(arr)
                setattr(s, name, ptr)
        s.lr = cfg.get("lr", 0.01)
        s.init_seed = cfg.get("init_seed", 2)
        s.window = cfg.get("window", 0)
        s.lookahead = cfg.get("lookahead", 0)
        s.residency_horizon = cfg.get("residency_horizon", 0)
        s.hbm_weight_budget_bytes = cfg.get("hbm_weight_budget_bytes", 0)
        s.bwd_policy = cfg.get("bwd_policy", 0)
        s.link_latency = cfg.get("link_latency", 0)
        s.flags = cfg.get("flags", 0)
        s.image_hw, s.num_classes = cfg.get("image_hw", 0), cfg.get("num_classes", 0)
        s.stem_channels, s.head_channels = cfg.get("stem_channels", 0), cfg.get("head_channels", 0)
        s.n_cnn_stages = len(cfg.get("stage_repeats", []))
        s.sync_policy = SYNC[cfg.get("sync", "csp")]
        s.bulk_size = cfg.get("bulk_size", 0)
        self.struct = s
        self.cfg = cfg

    @property
    def ptr(self):
        return C.byref(self.struct)


class Handle:
    def __init__(self, ptr, spec):
        self.ptr = ptr
        self.spec = spec
        self.keep = []   # host buffers borrowed until the next drain

    def __del__(self):
        if getattr(self, "ptr", None):
            lib.naspipe_destroy(self.ptr)
            self.ptr = None


def naspipe_abi_version():
    return lib.naspipe_abi_version()


def naspipe_create(spec: Spec, n_stages: int) -> Handle:
    h = C.c_void_p()
    _check(lib.naspipe_create(spec.ptr, n_stages, C.byref(h)))
    return Handle(h, spec)


def naspipe_create_rank(spec: Spec, n_stages: int, stage_rank: int, device: int, nccl_ids: bytes) -> Handle:
    h = C.c_void_p()
    buf = C.create_string_buffer(bytes(nccl_ids), max(1, len(nccl_ids)))
    _check(lib.naspipe_create_rank(spec.ptr, n_stages, stage_rank, device, buf, C.byref(h)))
    return Handle(h, spec)


def naspipe_create_rank_peer(spec: Spec, n_stages: int, stage_rank: int, device: int) -> Handle:
    h = C.c_void_p()
    _check(lib.naspipe_create_rank_peer(spec.ptr, n_stages, stage_rank, device, C.byref(h)))
    return Handle(h, spec)


def naspipe_peer_export(h: Handle) -> bytes:
    n = C.c_size_t()
    _check(lib.naspipe_peer_export(h.ptr, None, 0, C.byref(n)))
    buf = C.create_string_buffer(n.value)
    _check(lib.naspipe_peer_export(h.ptr, buf, n.value, C.byref(n)))
    return buf.raw


def naspipe_peer_connect(h: Handle, prev_blob, next_blob) -> None:
    pb = C.create_string_buffer(bytes(prev_blob), len(prev_blob)) if prev_blob else None
    nb = C.create_string_buffer(bytes(next_blob), len(next_blob)) if next_blob else None
    _check(lib.naspipe_peer_connect(h.ptr, pb, len(prev_blob) if prev_blob else 0, nb,
                                    len(next_blob) if next_blob else 0))


def naspipe_set_pdl(enabled: bool) -> None:
    _check(lib.naspipe_set_pdl(1 if enabled else 0))


def naspipe_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _check(lib.naspipe_nccl_unique_id(buf))
    return buf.raw


def _ptr_of(x, keep):
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):          # torch tensor (pinned host or device)
        keep.append(x)
        return x.data_ptr()
    x = np.asarray(x)
    a = np.ascontiguousarray(x, dtype=np.int32 if np.issubdtype(x.dtype, np.integer) else np.float32)
    keep.append(a)
    return a.ctypes.data


def naspipe_submit(h: Handle, choice, input=None, target=None, where=BATCH_HOST, synth_seed=0) -> int:
    ch, chp = _i32(np.asarray(choice).ravel())
    b = _BatchStruct()
    b.input = _ptr_of(input, h.keep)
    b.target = _ptr_of(target, h.keep)
    b.where = where
    b.synth_seed = synth_seed
    y = C.c_int64()
    _check(lib.naspipe_submit(h.ptr, chp, C.byref(b), C.byref(y)))
    return y.value


def naspipe_drain(h: Handle):
    _check(lib.naspipe_drain(h.ptr))
    h.keep.clear()


def naspipe_destroy(h: Handle):
    if h.ptr:
        lib.naspipe_destroy(h.ptr)
        h.ptr = None


def naspipe_param_count(spec: Spec, block: int, choice: int) -> int:
    n = C.c_size_t()
    _check(lib.naspipe_param_count(spec.ptr, block, choice, C.byref(n)))
    return n.value


def naspipe_get_params(h: Handle, block: int, choice: int) -> np.ndarray:
    n = naspipe_param_count(h.spec, block, choice)
    out = np.empty(n, dtype=np.float32)
    _check(lib.naspipe_get_params(h.ptr, block, choice, out.ctypes.data_as(C.POINTER(C.c_float)), n))
    return out


def naspipe_set_params(h: Handle, block: int, choice: int, src):
    a = np.ascontiguousarray(src, dtype=np.float32)
    _check(lib.naspipe_set_params(h.ptr, block, choice, a.ctypes.data_as(C.POINTER(C.c_float)), a.size))


def naspipe_get_losses(h: Handle, n: int) -> np.ndarray:
    out = np.empty(n, dtype=np.float32)
    _check(lib.naspipe_get_losses(h.ptr, out.ctypes.data_as(C.POINTER(C.c_float)), n))
    return out


def _get_rows(fn, *args, width=4):
    n = C.c_size_t()
    _check(fn(*args, None, 0, C.byref(n)))
    out = np.zeros((n.value, width), dtype=np.int64)
    if n.value:
        _check(fn(*args, out.ctypes.data_as(_i64p), n.value, C.byref(n)))
    return out


def naspipe_get_trace(h: Handle) -> np.ndarray:
    """(tick, stage, kind 0=F/1=B, seq id) per executed task, in issue order."""
    return _get_rows(lib.naspipe_get_trace, h.ptr)


def naspipe_get_residency_trace(h: Handle) -> np.ndarray:
    return _get_rows(lib.naspipe_get_residency_trace, h.ptr)


def naspipe_get_stats(h: Handle) -> dict:
    out = (C.c_double * 16)()
    _check(lib.naspipe_get_stats(h.ptr, out))
    return dict(zip(STATS_FIELDS, list(out)))


TIMED_FIELDS = ("tasks", "backwards", "predictions", "hits", "host_ms", "reserved")


def naspipe_get_timed_stats(h: Handle) -> dict:
    """Timing-driven executor (FLAG_TIMED) counters: tasks issued, backward starts, Alg.3
    predictions made at them, predictions that were the stage's next forward, host loop ms."""
    out = (C.c_double * 6)()
    _check(lib.naspipe_get_timed_stats(h.ptr, out))
    return dict(zip(TIMED_FIELDS, list(out)))


def naspipe_set_timing(h: Handle, on: bool) -> None:
    _check(lib.naspipe_set_timing(h.ptr, 1 if on else 0))


def naspipe_default_costs(spec: Spec):
    m, n = spec.struct.n_blocks, spec.struct.n_choices
    cf = np.zeros(m * n, dtype=np.int32)
    cb = np.zeros(m * n, dtype=np.int32)
    _check(lib.naspipe_default_costs(spec.ptr, cf.ctypes.data_as(_i32p), cb.ctypes.data_as(_i32p)))
    return cf.reshape(m, n), cb.reshape(m, n)


def naspipe_partition(spec: Spec, n_stages: int) -> np.ndarray:
    out = np.zeros(spec.struct.n_blocks, dtype=np.int32)
    _check(lib.naspipe_partition(spec.ptr, n_stages, out.ctypes.data_as(_i32p)))
    return out


def naspipe_plan_mirrored(spec: Spec, n_stages: int, choices, mirror_latency: int = 0) -> dict:
    """Per-subnet balanced partitions with layer mirroring (planning only; include/naspipe.h):
    dict(stage_of_block [N][m], trace [T][4] (tick, stage, kind, y), makespan, stall [D], bubble [D])."""
    ch, chp = _i32(choices)
    N = ch.shape[0] if ch.ndim == 2 else 0
    m = spec.struct.n_blocks
    sob = np.zeros((N, m), dtype=np.int32)
    cap = 2 * N * n_stages
    tr = np.zeros((max(cap, 1), 4), dtype=np.int64)
    nt, ms = C.c_size_t(0), C.c_int64(0)
    stall = np.zeros(n_stages, dtype=np.int64)
    bubble = np.zeros(n_stages, dtype=np.int64)
    _check(lib.naspipe_plan_mirrored(spec.ptr, n_stages, chp, N, int(mirror_latency),
                                     sob.ctypes.data_as(_i32p), tr.ctypes.data_as(_i64p), cap, C.byref(nt),
                                     C.byref(ms), stall.ctypes.data_as(_i64p), bubble.ctypes.data_as(_i64p)))
    return dict(stage_of_block=sob, trace=tr[: nt.value], makespan=ms.value, stall=stall, bubble=bubble)


def naspipe_init_params(spec: Spec, block: int, choice: int) -> np.ndarray:
    n = naspipe_param_count(spec, block, choice)
    out = np.empty(n, dtype=np.float32)
    _check(lib.naspipe_init_params(spec.ptr, block, choice, out.ctypes.data_as(C.POINTER(C.c_float)), n))
    return out


def naspipe_init_frozen(spec: Spec, part: int, n: int) -> np.ndarray:
    out = np.empty(n, dtype=np.float32)
    _check(lib.naspipe_init_frozen(spec.ptr, part, out.ctypes.data_as(C.POINTER(C.c_float)), n))
    return out


class Plan:
    """Host-only CSP plan (naspipe_plan_create): trace, makespan, deps, residency."""

    def __init__(self, spec: Spec, n_stages: int, choices):
        ch, chp = _i32(np.asarray(choices).reshape(-1, spec.struct.n_blocks))
        self.spec = spec
        self.n_subnets = ch.shape[0]
        self.ptr = C.c_void_p()
        _check(lib.naspipe_plan_create(spec.ptr, n_stages, chp, ch.shape[0], C.byref(self.ptr)))

    def __del__(self):
        if getattr(self, "ptr", None):
            lib.naspipe_plan_destroy(self.ptr)
            self.ptr = None

    def trace(self) -> np.ndarray:
        return _get_rows(lib.naspipe_plan_trace, self.ptr)

    def makespan(self) -> int:
        v = C.c_int64()
        _check(lib.naspipe_plan_makespan(self.ptr, C.byref(v)))
        return v.value

    def deps(self, y: int, stage: int):
        return [int(v) for v in _get_rows(lib.naspipe_plan_deps, self.ptr, y, stage, width=1).ravel()]

    def idle(self, n_stages: int):
        """(stall ticks [D], bubble ticks [D])."""
        st = np.zeros(n_stages, dtype=np.int64)
        bu = np.zeros(n_stages, dtype=np.int64)
        _check(lib.naspipe_plan_idle(self.ptr, st.ctypes.data_as(_i64p), bu.ctypes.data_as(_i64p)))
        return st, bu

    def comm_schedule(self, rank: int) -> np.ndarray:
        """(op, peer, subnet id) rows: the p2p operations rank `rank` issues, in order."""
        return _get_rows(lib.naspipe_plan_comm_schedule, self.ptr, rank, width=3)

    def residency(self, stage: int, budget_bytes: int, depth: int = 0, horizon: int = -1):
        """horizon: -1 unbounded, 0 the spec's, > 0 reading A26's H."""
        n = C.c_size_t()
        wb = C.c_int64()
        _check(lib.naspipe_plan_residency(self.ptr, stage, budget_bytes, depth, horizon, None, 0, C.byref(n),
                                          C.byref(wb)))
        out = np.zeros((n.value, 4), dtype=np.int64)
        if n.value:
            _check(lib.naspipe_plan_residency(self.ptr, stage, budget_bytes, depth, horizon, out.ctypes.data_as(_i64p),
                                              n.value, C.byref(n), C.byref(wb)))
        return out, wb.value


def naspipe_plan(spec: Spec, n_stages: int, choices) -> Plan:
    return Plan(spec, n_stages, choices)
