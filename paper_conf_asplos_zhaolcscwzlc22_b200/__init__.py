"""B200-native NASPipe hot path: Python binding of the C ABI (include/naspipe.h).

Argument marshalling only — every step of the path (planning, transfers, kernels) runs in
libnaspipe.so.  There is no CPU fallback: importing this package fails loudly if the
library has not been built (``python -m paper_conf_asplos_zhaolcscwzlc22_b200.build``).
"""
from ._lib import (  # noqa: F401
    LIB_PATH, NaspipeError, Spec, naspipe_abi_version, naspipe_create, naspipe_create_rank, naspipe_create_rank_peer,
    naspipe_peer_export, naspipe_peer_connect, naspipe_set_pdl,
    naspipe_default_costs, naspipe_destroy, naspipe_drain, naspipe_get_losses,
    naspipe_get_params, naspipe_get_residency_trace, naspipe_get_stats, naspipe_get_trace,
    naspipe_init_params, naspipe_init_frozen, naspipe_nccl_unique_id, naspipe_param_count, naspipe_partition,
    naspipe_plan, naspipe_plan_mirrored, naspipe_set_params, naspipe_set_timing, naspipe_submit, lib, BATCH_HOST, BATCH_DEVICE,
    BATCH_SYNTHETIC, FLAG_TRACE, FLAG_VERSION_CHECK, FLAG_NULL_KERNELS, FLAG_TIMING, FLAG_RECOMPUTE, FLAG_MIRROR,
    FLAG_TIMED, naspipe_get_timed_stats, TIMED_FIELDS, STATS_FIELDS, EXPORTED_SYMBOLS,
)
