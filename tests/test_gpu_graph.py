"""Swaps captured into CUDA graphs (include/mpress.h, "CUDA graph capture").

A pipeline step that swaps can be captured once and replayed as one graph
launch.  Each replay must move the bytes the captured tensors hold at replay
time, bit-exactly (stash vs the oracle byte model, restored tensors vs the
generator), the graph handle's slices must stay reserved while eager swaps of
the same context run, and the misuse cases must fail with ERR_STATE."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev

import _swaputil as U

pytestmark = pytest.mark.gpu

PATHS = [mp.PATH_DIRECT, mp.PATH_BULK, mp.PATH_CE]


def _setup(path, copies=2):
    # golden G1 shape (weights 1:2:1, binding caps, tails) plus a multi-chunk tensor
    sizes, world, source = [1000, 70000, 300, 3 << 20], 4, 0
    spare, bw, G = [0, 2 << 20, 4 << 20, 1 << 20], [0, 1, 2, 1], 4096
    o = oracle.plan(world, source, spare, bw, sizes, G)
    pl = mp.plan(world, source, spare, bw, sizes, G)
    assert pl.stripes == [tuple(s) for s in o["stripes"]]
    ctx = U.loopback_ctx(world, source, pl.units, G, copies=copies)
    ctx.set_option(mp.OPT_PATH, path)
    return sizes, o, pl, ctx


def _refill(ts, seed):
    for i, t in enumerate(ts):
        synth_dev.fill(t, seed, i)
    torch.cuda.synchronize()


@pytest.mark.parametrize("path", PATHS)
def test_graph_replays_move_current_bytes(path):
    sizes, o, pl, ctx = _setup(path)
    try:
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        dst = [torch.full((n,), 0x5A, dtype=torch.uint8, device="cuda") for n in sizes]
        full = ctx.stash_free()
        s = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            h = ctx.swap_out(pl, src)
            ctx.swap_in(h, dst)
            ctx.wait(h)
        torch.cuda.synchronize()
        assert all(bool((d == 0x5A).all()) for d in dst)      # capture runs nothing
        held = ctx.stash_free()
        assert all(held[p] == full[p] - pl.units[p] * o["G"] for p in range(4))
        for rep in range(3):
            seed = 500 + rep
            _refill(src, seed)
            g.replay()
            torch.cuda.synchronize()
            assert ctx.query(h)
            host = U.host_inputs(sizes, seed)
            U.check_stash(ctx, h, o, host)
            for i, (d, e) in enumerate(zip(dst, host)):
                assert np.array_equal(d.cpu().numpy(), e), "replay %d: tensor %d differs" % (rep, i)

        # An eager swap beside the graph handle takes other slices.
        _refill(src, 777)
        h2 = ctx.swap_out(pl, src)
        a, b = h.slices(), h2.slices()
        for p in range(1, 4):
            n = pl.units[p] * o["G"]
            assert a[p] + n <= b[p] or b[p] + n <= a[p]
        dst2 = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        ctx.swap_in(h2, dst2)
        ctx.wait(h2)
        g.replay()                       # the graph still works beside it
        torch.cuda.synchronize()
        h2.free()
        for i, d in enumerate(dst2):
            assert synth_dev.check(d, 777, i) == 0
        for i, d in enumerate(dst):
            assert synth_dev.check(d, 777, i) == 0
        del g
        h.free()
        torch.cuda.synchronize()
        assert ctx.stash_free() == full
    finally:
        ctx.finalize()


def test_graph_cross_stream_join():
    """Swap-out on the capture stream, swap-in on a forked side stream, the
    capture stream joined back through mpress_wait."""
    sizes, o, pl, ctx = _setup(mp.PATH_DIRECT)
    try:
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        out = torch.zeros(1, dtype=torch.int64, device="cuda")
        g = torch.cuda.CUDAGraph()
        cap = torch.cuda.Stream()
        with torch.cuda.graph(g, stream=cap):
            side = torch.cuda.Stream()
            h = ctx.swap_out(pl, src)
            side.wait_stream(torch.cuda.current_stream())
            ctx.swap_in(h, dst, stream=side)
            ctx.wait(h, torch.cuda.current_stream())            # join
            out.copy_(dst[3][:8].view(torch.int64)[:1])           # consumer after the join
        for rep in range(2):
            _refill(src, 900 + rep)
            g.replay()
            torch.cuda.synchronize()
            for i, d in enumerate(dst):
                assert synth_dev.check(d, 900 + rep, i) == 0
            assert int(out.item()) == int(src[3][:8].view(torch.int64)[0].item())
        del g
        h.free()
    finally:
        ctx.finalize()


@pytest.mark.filterwarnings("ignore:The CUDA Graph is empty")  # refused calls leave the capture empty
def test_graph_misuse():
    sizes, o, pl, ctx = _setup(mp.PATH_DIRECT, copies=3)
    try:
        src = U.make_inputs(sizes, 11)
        dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        s = torch.cuda.Stream()
        # swap-out captured, swap-in eager -> ERR_STATE; free needs force
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            h = ctx.swap_out(pl, src)
        with pytest.raises(mp.MPressError) as ei:
            ctx.swap_in(h, dst)
        assert ei.value.code == mp.ERR_STATE
        with pytest.raises(mp.MPressError) as ei:
            h.free()
        assert ei.value.code == mp.ERR_STATE
        h.free(force=True)
        del g
        # eager swap-out, swap-in under capture -> ERR_STATE
        he = ctx.swap_out(pl, src)
        g2 = torch.cuda.CUDAGraph()
        with pytest.raises(mp.MPressError) as ei:
            with torch.cuda.graph(g2, stream=s):
                ctx.swap_in(he, dst)
        assert ei.value.code == mp.ERR_STATE
        ctx.swap_in(he, dst)            # the eager handle is unaffected
        ctx.wait(he)
        torch.cuda.synchronize()
        for i, d in enumerate(dst):
            assert synth_dev.check(d, 11, i) == 0
        he.free()
        # a graph handle's swap-in may be captured only once
        g3 = torch.cuda.CUDAGraph()
        with pytest.raises(mp.MPressError) as ei:
            with torch.cuda.graph(g3, stream=s):
                h3 = ctx.swap_out(pl, src)
                ctx.swap_in(h3, dst)
                ctx.swap_in(h3, dst)
        assert ei.value.code == mp.ERR_STATE
        h3.free()
    finally:
        ctx.finalize()


def test_graph_handle_survives_python_gc():
    """Dropping the Python handle of a captured swap must not release the
    slices its graph replays into; Context.graph_handles gives it back."""
    import gc
    sizes, o, pl, ctx = _setup(mp.PATH_DIRECT)
    try:
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=torch.cuda.Stream()):
            h = ctx.swap_out(pl, src)
            ctx.swap_in(h, dst)
        assert h.graph
        held = ctx.stash_free()
        del h
        gc.collect()
        assert ctx.stash_free() == held                 # still reserved
        _refill(src, 321)
        g.replay()
        torch.cuda.synchronize()
        for i, d in enumerate(dst):
            assert synth_dev.check(d, 321, i) == 0
        (hg,) = ctx.graph_handles
        del g
        hg.free()
        assert ctx.graph_handles == []
        assert ctx.stash_free() != held
    finally:
        ctx.finalize()
