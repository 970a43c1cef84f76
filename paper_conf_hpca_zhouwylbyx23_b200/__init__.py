"""MPress D2D stripe swap, B200-native (Zhou et al., HPCA'23).

The product is ``libmpress.so`` (C ABI in ``include/mpress.h``); this package is
its thin Python binding (``api``).  See DESIGN.md.
"""
from .api import (  # noqa: F401
    OK, ALIGN, DEFAULT_GRANULE, EXPORTED, LIB_PATH, OPT_MAX_CTAS, OPT_ORDER, OPT_PATH, OPT_VARIANT, ORDER_INTERLEAVE, ORDER_PLAN, VARIANT_AUTO, PATH_BULK, PATH_CE,
    PATH_DIRECT, STATE_IN, STATE_IN_PENDING, STATE_OUT, STATE_OUT_PENDING, Context, Handle,
    CHOICE_CPU_SWAP, CHOICE_D2D, CHOICE_RECOMPUTE, DEVICE_HOST, NOT_RECOMPUTABLE, MPressError,
    OPT_TRANSPORT, TRANSPORT_LEGACY_IPC, TRANSPORT_LOCAL, TRANSPORT_VMM_FD, OPT_LAST_PATH, OPT_PDL, OPT_PACE_MBPS, OPT_SPLIT, SPLIT_BLOCKED, SPLIT_STRIDED, SPLIT_DYNAMIC, SPLIT_AUTO, PATH_AUTO, OPT_AUTO_OUT, OPT_AUTO_IN, OPT_AUTO_OUT_SMALL, OPT_AUTO_IN_SMALL, AUTO_SMALL_BYTES,
    Executor, Plan, compaction_plan, lib, map_search, partition_sequential, pointers, plan, plan_from_units, plan_global, schedule_1f1b,
    share_fds,
    torch_exchange,
)
from .api import (ERR_ALIGN, ERR_ARG, ERR_CUDA, ERR_NO_SPACE, ERR_PEER, ERR_STATE,  # noqa: F401
                  ERR_SYS)
