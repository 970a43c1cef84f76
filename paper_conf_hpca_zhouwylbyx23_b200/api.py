"""Thin ctypes binding of libmpress (include/mpress.h).  Marshalling only.

Every step of the swap path -- planning, peer mapping, the copy kernels,
events -- runs inside libmpress.so; this module turns Python lists into C
arrays, torch tensors into device pointers (``data_ptr()``) and torch
streams / events into ``cudaStream_t`` / ``cudaEvent_t``.  There is no
fallback: if the library is missing the import fails loudly.
"""
import ctypes
import os
from ctypes import (CFUNCTYPE, POINTER, byref, c_char_p, c_int, c_int32, c_int64,
                    c_size_t, c_uint32, c_uint64, c_void_p)

_HERE = os.path.dirname(os.path.abspath(__file__))
# MPRESS_LIB overrides the library path (A/B runs of two builds, tools/ab.py)
LIB_PATH = os.environ.get("MPRESS_LIB") or os.path.join(_HERE, "libmpress.so")

OK = 0
ERR_ARG, ERR_NO_SPACE, ERR_ALIGN, ERR_STATE, ERR_PEER, ERR_CUDA, ERR_SYS = -1, -2, -3, -4, -5, -6, -7
ALIGN = 256
DEFAULT_GRANULE = 65536
OPT_PATH, OPT_MAX_CTAS, OPT_VARIANT, OPT_ORDER = 1, 2, 3, 4
ORDER_INTERLEAVE, ORDER_PLAN = 0, 1
DEVICE_HOST = -1   # mpress_init_local: a pinned host pool as a peer (NEXT-4)
OPT_TRANSPORT = 5  # read-only
OPT_LAST_PATH = 6  # read-only: path of the last swap call
OPT_PDL = 7
OPT_PACE_MBPS = 12
OPT_SPLIT = 13
SPLIT_BLOCKED, SPLIT_STRIDED, SPLIT_DYNAMIC, SPLIT_AUTO = 0, 1, 2, 3
OPT_AUTO_OUT, OPT_AUTO_IN = 8, 9   # read-only: AUTO's uncapped-grid path per direction (large launches)
OPT_AUTO_OUT_SMALL, OPT_AUTO_IN_SMALL = 10, 11   # ... for launches < AUTO_SMALL_BYTES
AUTO_SMALL_BYTES = 32 << 20
TRANSPORT_LOCAL, TRANSPORT_VMM_FD, TRANSPORT_LEGACY_IPC = 0, 1, 2
VARIANT_AUTO = -1
PATH_DIRECT, PATH_BULK, PATH_CE, PATH_AUTO = 0, 1, 2, 3
STATE_OUT_PENDING, STATE_OUT, STATE_IN_PENDING, STATE_IN = 1, 2, 3, 4

_ERR_NAMES = {ERR_ARG: "ERR_ARG", ERR_NO_SPACE: "ERR_NO_SPACE", ERR_ALIGN: "ERR_ALIGN",
              ERR_STATE: "ERR_STATE", ERR_PEER: "ERR_PEER", ERR_CUDA: "ERR_CUDA",
              ERR_SYS: "ERR_SYS"}

EXPORTED = [
    "mpress_plan", "mpress_plan_stripes", "mpress_plan_units", "mpress_plan_get_info",
    "mpress_plan_free", "mpress_partition_sequential", "mpress_plan_global",
    "mpress_plan_from_units", "mpress_schedule_1f1b", "mpress_map_search",
    "mpress_compaction_plan", "mpress_executor_create", "mpress_executor_ops",
    "mpress_executor_slot", "mpress_executor_restore_to", "mpress_executor_before",
    "mpress_executor_after", "mpress_executor_release", "mpress_executor_set_option",
    "mpress_executor_get_option", "mpress_executor_free", "mpress_init",
    "mpress_init_local",
    "mpress_finalize", "mpress_stash_free", "mpress_set_option", "mpress_get_option", "mpress_autotune",
    "mpress_swap_out", "mpress_swap_in", "mpress_wait", "mpress_query", "mpress_handle_state",
    "mpress_handle_is_graph",
    "mpress_handle_slices", "mpress_handle_free", "mpress_peer_read", "mpress_peer_ptr", "mpress_last_launches",
    "mpress_share_fds", "mpress_last_error", "mpress_version",
]


class MPressError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__("%s (%d): %s" % (_ERR_NAMES.get(code, "?"), code, msg))
        self.code = code


class Stripe(ctypes.Structure):
    _fields_ = [("tensor", c_uint32), ("peer", c_uint32), ("src_off", c_uint64),
                ("dst_off", c_uint64), ("len", c_uint64)]


class PlanInfo(ctypes.Structure):
    _fields_ = [("world", c_int32), ("source", c_int32), ("n_tensors", c_uint32),
                ("n_stripes", c_uint32), ("granule", c_uint64), ("virtual_bytes", c_uint64),
                ("units", c_uint64)]


class Params1F1B(ctypes.Structure):
    _fields_ = [("stages", c_uint32), ("stage", c_uint32), ("micro_batches", c_uint32),
                ("duplex", c_uint32), ("t_fwd_ns", c_uint64), ("t_bwd_ns", c_uint64),
                ("t_out_ns", c_uint64), ("t_in_ns", c_uint64), ("t_slack_ns", c_uint64)]


class Slot1F1B(ctypes.Structure):
    _fields_ = [(n, c_uint64) for n in ("fwd_start", "fwd_end", "bwd_start", "bwd_end", "live_ns",
                                        "out_start", "out_end", "in_start", "in_end")] + \
               [("in_trigger", c_uint32), ("hidden", c_uint32), ("exposed_ns", c_uint64)]


class Summary1F1B(ctypes.Structure):
    _fields_ = [("makespan_ns", c_uint64), ("makespan_noswap_ns", c_uint64),
                ("peak_resident", c_uint32), ("peak_resident_noswap", c_uint32),
                ("ops", c_uint32), ("pad", c_uint32)]


EXCHANGE_FN = CFUNCTYPE(c_int, c_void_p, c_void_p, c_size_t, c_void_p)


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError("libmpress.so not built at %s: run "
                          "`python -c 'import __graft_entry__ as g; g.build()'`" % LIB_PATH)
    lib = ctypes.CDLL(LIB_PATH)
    P = c_void_p
    sig = {
        "mpress_plan": (c_int, [c_int, c_int, P, P, c_uint32, P, c_uint64, POINTER(P)]),
        "mpress_plan_stripes": (c_int, [P, POINTER(POINTER(Stripe)), POINTER(c_uint32), POINTER(POINTER(c_uint64))]),
        "mpress_plan_units": (c_int, [P, POINTER(POINTER(c_uint64))]),
        "mpress_plan_get_info": (c_int, [P, POINTER(PlanInfo)]),
        "mpress_plan_free": (None, [P]),
        "mpress_partition_sequential": (c_int, [c_int, P, P, c_uint32, P, P, P, P, c_uint64, P]),
        "mpress_plan_global": (c_int, [c_int, c_uint32, P, P, P, P, P, P, P, c_uint64, P,
                                       POINTER(c_uint64), POINTER(c_uint64)]),
        "mpress_plan_from_units": (c_int, [c_int, c_int, P, c_uint32, P, c_uint64, POINTER(P)]),
        "mpress_schedule_1f1b": (c_int, [POINTER(Params1F1B), P, P]),
        "mpress_executor_create": (c_int, [P, P, POINTER(Params1F1B), P, P, POINTER(P)]),
        "mpress_executor_ops": (c_int, [P]),
        "mpress_executor_slot": (c_int, [P, c_uint32, POINTER(Slot1F1B)]),
        "mpress_executor_restore_to": (c_int, [P, c_uint32, P]),
        "mpress_executor_before": (c_int, [P, c_uint32, P, POINTER(c_uint32), POINTER(c_uint32)]),
        "mpress_executor_after": (c_int, [P, c_uint32, P, P]),
        "mpress_executor_release": (c_int, [P, c_uint32, P]),
        "mpress_executor_set_option": (c_int, [P, c_int, c_int64]),
        "mpress_executor_get_option": (c_int, [P, c_int, POINTER(c_int64)]),
        "mpress_executor_free": (c_int, [P]),
        "mpress_compaction_plan": (c_int, [c_uint32, P, c_uint64, P, P, POINTER(c_uint64),
                                           POINTER(c_uint64)]),
        "mpress_map_search": (c_int, [c_int, P, P, P, P, P, c_uint64, P, POINTER(c_uint64),
                                      POINTER(c_uint64), POINTER(c_uint64)]),
        "mpress_init": (c_int, [c_int, c_int, c_int, P, EXCHANGE_FN, P, POINTER(P)]),
        "mpress_init_local": (c_int, [c_int, c_int, P, P, POINTER(P)]),
        "mpress_finalize": (c_int, [P]),
        "mpress_stash_free": (c_int, [P, P]),
        "mpress_set_option": (c_int, [P, c_int, c_int64]),
        "mpress_get_option": (c_int, [P, c_int, POINTER(c_int64)]),
        "mpress_autotune": (c_int, [P, c_uint64, c_int, P, P]),
        "mpress_swap_out": (c_int, [P, P, P, P, P, POINTER(P)]),
        "mpress_swap_in": (c_int, [P, P, P, P]),
        "mpress_wait": (c_int, [P, P, P]),
        "mpress_query": (c_int, [P, P]),
        "mpress_handle_state": (c_int, [P]),
        "mpress_handle_is_graph": (c_int, [P]),
        "mpress_handle_slices": (c_int, [P, P]),
        "mpress_handle_free": (c_int, [P, P, c_int]),
        "mpress_peer_read": (c_int, [P, c_int, c_uint64, c_uint64, P]),
        "mpress_peer_ptr": (c_int, [P, c_int, c_uint64, POINTER(P)]),
        "mpress_last_launches": (c_int, [P]),
        "mpress_share_fds": (c_int, [c_int, c_int, c_int, P, EXCHANGE_FN, P, P]),
        "mpress_last_error": (c_char_p, []),
        "mpress_version": (c_int, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


lib = _load()


def _check(rc):
    if rc < 0:
        raise MPressError(rc, lib.mpress_last_error().decode(errors="replace"))
    return rc


def _u64(values):
    return (c_uint64 * len(values))(*[int(v) for v in values])


def _ptr(x):
    """Device pointer of a torch tensor, or an int address."""
    if hasattr(x, "data_ptr"):
        return int(x.data_ptr())
    return int(x)


def pointers(tensors):
    """A reusable C array of the tensors' device addresses (marshal once,
    pass to swap_out / swap_in many times; the tensors must stay alive).
    A uint64 array: the same bytes as `void* const*` on the 64-bit ABI, and
    ~3x cheaper to build from a list of tensors than c_void_p items."""
    try:
        return (c_uint64 * len(tensors))(*[t.data_ptr() for t in tensors])
    except AttributeError:   # int addresses mixed in
        return (c_uint64 * len(tensors))(*[_ptr(t) for t in tensors])


def _ptr_array(x):
    if isinstance(x, ctypes.Array):
        return x
    return pointers(x)


def _stream(s, device=None):
    if s is None:
        import torch
        return c_void_p(torch.cuda.current_stream(device).cuda_stream)
    if hasattr(s, "cuda_stream"):
        return c_void_p(s.cuda_stream)
    return c_void_p(int(s))


def _event(e):
    if e is None:
        return None
    if hasattr(e, "cuda_event"):
        return c_void_p(e.cuda_event)
    return c_void_p(int(e))


# ------------------------------------------------------------------------- plans

class Plan:
    """Owner of an mpress_plan_t (the metadata table of one batch)."""

    def __init__(self, world, source, spare, bw, sizes, granule=0):
        if len(spare) != world or len(bw) != world:
            raise MPressError(ERR_ARG, "spare/bw must have `world` entries")
        h = c_void_p()
        _check(lib.mpress_plan(world, source, _u64(spare), _u64(bw), len(sizes), _u64(sizes),
                               granule, byref(h)))
        self._h = h
        self.world = world
        self.sizes = [int(s) for s in sizes]

    def __del__(self):
        h = getattr(self, "_h", None)
        if h is not None and h.value and lib is not None:
            lib.mpress_plan_free(h)
            self._h = None

    @property
    def handle(self):
        return self._h

    @property
    def info(self):
        i = PlanInfo()
        _check(lib.mpress_plan_get_info(self._h, byref(i)))
        return i

    @property
    def stripes(self):
        p = POINTER(Stripe)()
        n = c_uint32()
        _check(lib.mpress_plan_stripes(self._h, byref(p), byref(n), None))
        return [(p[i].tensor, p[i].peer, p[i].src_off, p[i].dst_off, p[i].len) for i in range(n.value)]

    @property
    def peer_bytes(self):
        pb = POINTER(c_uint64)()
        _check(lib.mpress_plan_stripes(self._h, None, None, byref(pb)))
        return [pb[i] for i in range(self.world)]

    @property
    def units(self):
        u = POINTER(c_uint64)()
        _check(lib.mpress_plan_units(self._h, byref(u)))
        return [u[i] for i in range(self.world)]


def plan(world, source, spare, bw, sizes, granule=0):
    return Plan(world, source, spare, bw, sizes, granule)


def plan_from_units(world, source, units, sizes, granule=0):
    """The plan of a batch for a given per-peer unit split (mpress_plan_from_units)."""
    p = Plan.__new__(Plan)
    h = c_void_p()
    _check(lib.mpress_plan_from_units(world, source, _u64(units), len(sizes), _u64(sizes),
                                      granule, byref(h)))
    p._h = h
    p.world = world
    p.sizes = [int(s) for s in sizes]
    return p


def schedule_1f1b(stages, stage, micro_batches, t_fwd_ns, t_bwd_ns, t_out_ns, t_in_ns, duplex=True,
                  slack_ns=0):
    """NEXT-2 (mpress_schedule_1f1b): (slots as dicts, summary dict)."""
    p = Params1F1B(stages, stage, micro_batches, 1 if duplex else 0, t_fwd_ns, t_bwd_ns,
                   t_out_ns, t_in_ns, slack_ns)
    slots = (Slot1F1B * micro_batches)()
    summ = Summary1F1B()
    _check(lib.mpress_schedule_1f1b(byref(p), slots, byref(summ)))
    names = [f[0] for f in Slot1F1B._fields_]
    return ([{n: getattr(s, n) for n in names} for s in slots],
            {f[0]: getattr(summ, f[0]) for f in Summary1F1B._fields_ if f[0] != "pad"})


class TensorStat(ctypes.Structure):
    _fields_ = [("bytes", c_uint64), ("live_ns", c_uint64), ("recompute_ns", c_uint64),
                ("cpu_swap_ns", c_uint64), ("d2d_swap_ns", c_uint64)]


NOT_RECOMPUTABLE = (1 << 64) - 1
CHOICE_CPU_SWAP, CHOICE_RECOMPUTE, CHOICE_D2D = 1, 2, 3


def compaction_plan(stats, d2d_capacity):
    """NEXT-4 (mpress_compaction_plan).  stats: dicts with bytes, live_ns,
    recompute_ns, cpu_swap_ns, d2d_swap_ns.  Returns (choices, overheads,
    total, d2d_bytes)."""
    n = len(stats)
    arr = (TensorStat * max(1, n))(*[TensorStat(t["bytes"], t["live_ns"], t["recompute_ns"],
                                                t["cpu_swap_ns"], t["d2d_swap_ns"]) for t in stats])
    ch = (c_uint32 * max(1, n))()
    ov = (c_uint64 * max(1, n))()
    tot, used = c_uint64(), c_uint64()
    _check(lib.mpress_compaction_plan(n, arr, d2d_capacity, ch, ov, byref(tot), byref(used)))
    return list(ch)[:n], list(ov)[:n], tot.value, used.value


def map_search(demand, spare, link, egress=None, ingress=None, granule=0):
    """NEXT-3 (mpress_map_search): (stage_to_gpu, (num, den), mappings evaluated)."""
    n = len(demand)
    out = (c_int32 * n)()
    num, den, ev = c_uint64(), c_uint64(), c_uint64()
    _check(lib.mpress_map_search(n, _u64(demand), _u64(spare), _u64([w for row in link for w in row]),
                                 _u64(egress) if egress else None, _u64(ingress) if ingress else None,
                                 granule, out, byref(num), byref(den), byref(ev)))
    return list(out), (num.value, den.value), ev.value


def plan_global(world, requests, spare, bw_matrix, egress=None, ingress=None, granule=0):
    """NEXT-1 (mpress_plan_global).  requests: [(source, sizes)].
    Returns (units {source: [world]}, (num, den)) with T* = num / den."""
    srcs = (c_int32 * len(requests))(*[r[0] for r in requests])
    ns = (c_uint32 * len(requests))(*[len(r[1]) for r in requests])
    flat = _u64([s for r in requests for s in r[1]])
    out = (c_uint64 * (len(requests) * world))()
    num, den = c_uint64(), c_uint64()
    _check(lib.mpress_plan_global(world, len(requests), srcs, ns, flat, _u64(spare),
                                  _u64([b for row in bw_matrix for b in row]),
                                  _u64(egress) if egress else None, _u64(ingress) if ingress else None,
                                  granule, out, byref(num), byref(den)))
    units = {r[0]: [out[i * world + p] for p in range(world)] for i, r in enumerate(requests)}
    return units, (num.value, den.value)


def partition_sequential(world, spare, bw_matrix, requests, granule=0):
    """requests: [(source, sizes, copies)] -> partition[s][p] (bytes)."""
    srcs = (c_int32 * len(requests))(*[r[0] for r in requests])
    ns = (c_uint32 * len(requests))(*[len(r[1]) for r in requests])
    cp = (c_uint32 * len(requests))(*[r[2] for r in requests])
    flat = _u64([s for r in requests for s in r[1]] or [0])
    bwm = _u64([b for row in bw_matrix for b in row])
    out = (c_uint64 * (world * world))()
    _check(lib.mpress_partition_sequential(world, _u64(spare), bwm, len(requests), srcs, ns, flat,
                                           cp, granule, out))
    return [[out[s * world + p] for p in range(world)] for s in range(world)]


# ------------------------------------------------------------------- exchange

def torch_exchange(group=None):
    """An all-gather callback over a torch.distributed process group (gloo for
    CPU bytes; an NCCL default group gets a gloo side group)."""
    import torch.distributed as dist
    if group is None and dist.get_backend() != "gloo":
        group = dist.new_group(backend="gloo")
    world = dist.get_world_size(group)

    def cb(user, mine, ln, out):
        try:
            import torch
            t = torch.frombuffer(bytearray(ctypes.string_at(mine, ln)), dtype=torch.uint8)
            outs = [torch.empty(ln, dtype=torch.uint8) for _ in range(world)]
            dist.all_gather(outs, t, group=group)
            buf = b"".join(bytes(o.numpy().tobytes()) for o in outs)
            ctypes.memmove(out, buf, len(buf))
            return 0
        except Exception as e:  # pragma: no cover - reported through the C status
            print("mpress exchange failed:", e)
            return -1
    return EXCHANGE_FN(cb)


def share_fds(world, rank, my_fd, want, exchange_cb):
    w = (c_int32 * world)(*[1 if x else 0 for x in want])
    out = (c_int32 * world)()
    _check(lib.mpress_share_fds(world, rank, my_fd, w, exchange_cb, None, out))
    return list(out)


# --------------------------------------------------------------- context / swap

class Handle:
    """An mpress_handle_t (one swapped batch).  Released by free(), by the
    garbage collector (forced), or when its context is finalized.  A graph
    handle (swap-out captured into a CUDA graph) is owned by its graph's
    replays, so the context keeps it alive until free() is called explicitly
    -- dropping the Python object must not release slices a replay uses."""

    def __init__(self, ctx, h, plan):
        self._ctx = ctx
        self._h = h
        self.plan = plan  # keeps the Plan alive while the handle exists
        ctx._handles.add(self)
        self.graph = _check(lib.mpress_handle_is_graph(h)) == 1
        if self.graph:
            ctx._graph_handles.add(self)

    def __del__(self):
        try:
            if self._h is not None and self._h.value and self._ctx._h is not None:
                lib.mpress_handle_free(self._ctx._h, self._h, 1)
        except Exception:  # pragma: no cover - interpreter shutdown
            pass
        self._h = None

    @property
    def state(self):
        return _check(lib.mpress_handle_state(self._h))

    def slices(self):
        out = (c_uint64 * self._ctx.world)()
        _check(lib.mpress_handle_slices(self._h, out))
        return list(out)

    def free(self, force=False):
        if self._h is not None and self._h.value:
            _check(lib.mpress_handle_free(self._ctx._h, self._h, 1 if force else 0))
        self._h = None
        self._ctx._graph_handles.discard(self)


class Executor:
    """mpress_executor_t: the paper's swap executor for the exporter
    stage of a 1F1B pipeline (see include/mpress.h)."""

    def __init__(self, ctx, plan_, stages, stage, micro_batches, t_fwd_ns, t_bwd_ns, t_out_ns, t_in_ns,
                 out_stream, in_stream, duplex=True, slack_ns=0):
        p = Params1F1B(stages, stage, micro_batches, 1 if duplex else 0, t_fwd_ns, t_bwd_ns,
                       t_out_ns, t_in_ns, slack_ns)
        h = c_void_p()
        _check(lib.mpress_executor_create(ctx._h, plan_.handle, byref(p), _stream(out_stream),
                                          _stream(in_stream), byref(h)))
        self._h, self._ctx, self.plan = h, ctx, plan_
        self.ops = _check(lib.mpress_executor_ops(h))

    def slot(self, m):
        s = Slot1F1B()
        _check(lib.mpress_executor_slot(self._h, m, byref(s)))
        return {f[0]: getattr(s, f[0]) for f in Slot1F1B._fields_}

    def restore_to(self, m, dst):
        _check(lib.mpress_executor_restore_to(self._h, m, _ptr_array(dst)))

    def before(self, op, compute=None):
        """Returns ('F' | 'B', micro-batch) of op `op`."""
        k, m = c_uint32(), c_uint32()
        _check(lib.mpress_executor_before(self._h, op, _stream(compute), byref(k), byref(m)))
        return ("F" if k.value == 0 else "B"), m.value

    def after(self, op, compute=None, activations=None):
        _check(lib.mpress_executor_after(self._h, op, _stream(compute),
                                         None if activations is None else _ptr_array(activations)))

    def release(self, m, stream=None):
        """mpress_executor_release: `stream` waits until micro-batch m's
        swap-out has read its activations, so they may be freed on it."""
        _check(lib.mpress_executor_release(self._h, m, _stream(stream)))

    def set_option(self, key, value):
        """mpress_executor_set_option: this executor's own swap options
        (a copy of the context's taken at creation)."""
        _check(lib.mpress_executor_set_option(self._h, key, int(value)))

    def get_option(self, key):
        v = c_int64()
        _check(lib.mpress_executor_get_option(self._h, key, byref(v)))
        return v.value

    def free(self):
        if self._h is not None:
            _check(lib.mpress_executor_free(self._h))
            self._h = None


class Context:
    """An mpress_ctx_t: this source's view of the peers' stash pools."""

    def __init__(self, h, world, source, device, exchange_cb=None):
        import weakref
        self._h = h
        self.world = world
        self.source = source
        self.device = device
        self._exchange = exchange_cb  # keep the ctypes callback alive
        self._handles = weakref.WeakSet()
        self._graph_handles = set()   # strong refs: released only by Handle.free()

    def __del__(self):
        # A local context can be released here; a distributed one must be
        # finalized collectively by the caller (mpress_finalize is a barrier).
        try:
            if self._h is not None and self._exchange is None:
                self.finalize()
        except Exception:  # pragma: no cover - interpreter shutdown
            pass

    @classmethod
    def local(cls, world, source, devices, partition):
        """Single process; every devices[p] equal = 1-GPU loopback."""
        h = c_void_p()
        devs = (c_int * world)(*devices)
        flat = _u64([partition[s][p] for s in range(world) for p in range(world)])
        _check(lib.mpress_init_local(world, source, devs, flat, byref(h)))
        return cls(h, world, source, devices[source])

    @classmethod
    def distributed(cls, device, world, rank, partition, exchange_cb=None):
        """Collective over torch.distributed (one process per GPU)."""
        if exchange_cb is None:
            exchange_cb = torch_exchange()
        h = c_void_p()
        flat = _u64([partition[s][p] for s in range(world) for p in range(world)])
        _check(lib.mpress_init(device, world, rank, flat, exchange_cb, None, byref(h)))
        return cls(h, world, rank, device, exchange_cb)

    def finalize(self):
        if self._h is not None:
            for hd in list(self._handles):   # the library frees them with the context
                hd._h = None
            self._graph_handles.clear()
            h, self._h = self._h, None
            _check(lib.mpress_finalize(h))

    @property
    def graph_handles(self):
        """Graph handles not yet freed (kept alive for their graphs' replays)."""
        return list(self._graph_handles)

    def set_option(self, key, value):
        _check(lib.mpress_set_option(self._h, key, int(value)))

    def get_option(self, key):
        v = c_int64()
        _check(lib.mpress_get_option(self._h, key, byref(v)))
        return v.value

    def autotune(self, probe_bytes=1 << 30, trials=5, stream=None):
        """mpress_autotune: time the direct and bulk kernels on this
        context's links (back-to-back launches over a `probe_bytes` working
        set) and let MPRESS_PATH_AUTO keep the faster per direction and size
        class (collective for a distributed context).  Returns the chosen
        paths (out / in for launches >= AUTO_SMALL_BYTES, out_small /
        in_small below) and the median ms per launch of every probe."""
        ms = (ctypes.c_float * 8)()
        _check(lib.mpress_autotune(self._h, probe_bytes, trials, _stream(stream, self.device), ms))
        names = [c + "_" + k + "_" + d for c in ("small", "large") for k in ("direct", "bulk") for d in ("out", "in")]
        return {"out": self.get_option(OPT_AUTO_OUT), "in": self.get_option(OPT_AUTO_IN),
                "out_small": self.get_option(OPT_AUTO_OUT_SMALL), "in_small": self.get_option(OPT_AUTO_IN_SMALL),
                "ms": dict(zip(names, ms))}

    def stash_free(self):
        out = (c_uint64 * self.world)()
        _check(lib.mpress_stash_free(self._h, out))
        return list(out)

    def swap_out(self, plan_, tensors, stream=None, after=None):
        """tensors: a list of tensors / addresses, or a `pointers(...)` array
        built once and reused (saves the per-call marshalling)."""
        h = c_void_p()
        _check(lib.mpress_swap_out(self._h, plan_.handle, _ptr_array(tensors),
                                   _stream(stream, self.device), _event(after), byref(h)))
        return Handle(self, h, plan_)

    def swap_in(self, handle, dst, stream=None):
        _check(lib.mpress_swap_in(self._h, handle._h, _ptr_array(dst), _stream(stream, self.device)))

    def wait(self, handle, stream=None):
        _check(lib.mpress_wait(self._h, handle._h, _stream(stream, self.device)))

    def query(self, handle):
        return _check(lib.mpress_query(self._h, handle._h)) == 1

    def peer_ptr(self, peer, offset=0):
        """mpress_peer_ptr: device address (int) of byte `offset` of this
        source's partition on `peer` (debug / test)."""
        out = c_void_p()
        _check(lib.mpress_peer_ptr(self._h, peer, offset, byref(out)))
        return out.value or 0

    def peer_read(self, peer, offset, length):
        buf = ctypes.create_string_buffer(max(1, length))
        _check(lib.mpress_peer_read(self._h, peer, offset, length, buf))
        return buf.raw[:length]

    @property
    def last_launches(self):
        return lib.mpress_last_launches(self._h)
