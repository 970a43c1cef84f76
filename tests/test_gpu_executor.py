"""The native swap executor on the GPU: op order, restore buffers and
misuse errors; the byte-exact replay runs in test_gpu_pipeline.py."""
import pytest
import torch

import paper_conf_hpca_zhouwylbyx23_b200 as mp
from oracle import pipeline as P
from synth import device as synth_dev

pytestmark = pytest.mark.gpu


def _setup(M):
    sizes = [4096, 10000, 333]
    world = 3
    spare, bw = [0, 1 << 24, 1 << 24], [0, 1, 1]
    pl = mp.plan(world, 0, spare, bw, sizes, 4096)
    part = [[0] * world for _ in range(world)]
    part[0] = [M * u * 4096 for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    return ctx, pl, sizes


def test_executor_steps_and_errors():
    M = 3
    ctx, pl, sizes = _setup(M)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    comp = torch.cuda.current_stream()
    try:
        ex = mp.Executor(ctx, pl, 2, 0, M, 10_000, 20_000, 5_000, 5_000, s_out, s_in)
        assert ex.ops == 2 * M
        # B(0) before anything was swapped out
        with pytest.raises(mp.MPressError) as ei:
            ex.before(2, comp)
        assert ei.value.code == mp.ERR_STATE
        # F without activations
        with pytest.raises(mp.MPressError) as ei:
            ex.after(0, comp, None)
        assert ei.value.code == mp.ERR_ARG
        src = [[torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        dst = [[torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        for step in range(3):                       # the executor serves many steps
            for m in range(M):
                for i, t in enumerate(src[m]):
                    synth_dev.fill(t, 50 * step + m, i)
                ex.restore_to(m, dst[m])
            ops = []
            for j in range(ex.ops):
                kind, m = ex.before(j, comp)
                ops.append((kind, m))
                ex.after(j, comp, src[m] if kind == "F" else None)
            # the executor runs the oracle's 1F1B op order (reading R24) ...
            assert ops == P.stage_ops(2, 0, M)
            torch.cuda.synchronize()
            for m in range(M):
                for i, t in enumerate(dst[m]):
                    assert synth_dev.check(t, 50 * step + m, i) == 0, (step, m, i)
        # ... and swaps at the oracle's points: every slot equals
        # oracle.pipeline.schedule for the same parameters
        slots, _ = P.schedule(2, 0, M, 10_000, 20_000, 5_000, 5_000)
        assert [ex.slot(m) for m in range(M)] == slots
        ex.free()
    finally:
        ctx.finalize()


def test_executor_missing_restore_buffers():
    M = 2
    ctx, pl, sizes = _setup(M)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    comp = torch.cuda.current_stream()
    try:
        ex = mp.Executor(ctx, pl, 1, 0, M, 10_000, 20_000, 5_000, 5_000, s_out, s_in)
        src = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        kind, m = ex.before(0, comp)
        assert (kind, m) == ("F", 0)
        with pytest.raises(mp.MPressError) as ei:   # F(0) triggers its own swap-in (S = 1)
            ex.after(0, comp, src)
        assert ei.value.code == mp.ERR_STATE
        torch.cuda.synchronize()
        ex.free()
    finally:
        ctx.finalize()


@pytest.mark.filterwarnings("ignore:The CUDA Graph is empty")  # the refused capture records nothing
def test_executor_refuses_graph_capture():
    """An executor step recycles stash slices between micro-batches, so it
    must refuse to run while one of its streams is being captured."""
    M = 2
    ctx, pl, sizes = _setup(M)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    try:
        ex = mp.Executor(ctx, pl, 2, 0, M, 10_000, 20_000, 5_000, 5_000, s_out, s_in)
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        g = torch.cuda.CUDAGraph()
        with pytest.raises(mp.MPressError) as ei:
            with torch.cuda.graph(g, stream=torch.cuda.Stream()):
                ex.after(0, torch.cuda.current_stream(), src)
        assert ei.value.code == mp.ERR_STATE
        ex.free()
    finally:
        ctx.finalize()


def test_executor_release_then_reuse():
    """freeing the activations right after F(m) is the point of the
    swap.  After mpress_executor_release(m, compute) the caching
    allocator may hand their memory to the next op on the compute stream; the
    swap-out stream is held back by a sleep so that, without the release, the
    overwrite would land before the swap-out read the bytes."""
    M = 3
    ctx, pl, sizes = _setup(M)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    comp = torch.cuda.current_stream()
    try:
        ex = mp.Executor(ctx, pl, 2, 0, M, 10_000, 20_000, 5_000, 5_000, s_out, s_in)
        dst = [[torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        for m in range(M):
            ex.restore_to(m, dst[m])
        for j in range(ex.ops):
            kind, m = ex.before(j, comp)
            if kind == "F":
                act = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
                for i, t in enumerate(act):
                    synth_dev.fill(t, 900 + m, i)
                with torch.cuda.stream(s_out):
                    torch.cuda._sleep(20_000_000)      # ~10 ms: the swap-out starts late
                ex.after(j, comp, act)
                ex.release(m, comp)
                ptrs = {t.data_ptr() for t in act}
                del act                                  # freed on the compute stream
                reuse = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
                for t in reuse:
                    t.fill_(0xA5)                        # the next op overwrites the memory
                assert ptrs & {t.data_ptr() for t in reuse}, "allocator did not reuse the block"
                del reuse
            else:
                ex.after(j, comp, None)
        with pytest.raises(mp.MPressError) as ei:        # every handle is gone after B(m)
            ex.release(0, comp)
        assert ei.value.code == mp.ERR_STATE
        torch.cuda.synchronize()
        for m in range(M):
            for i, t in enumerate(dst[m]):
                assert synth_dev.check(t, 900 + m, i) == 0, (m, i)
        ex.free()
    finally:
        ctx.finalize()


@pytest.mark.parametrize("path", [mp.PATH_CE, mp.PATH_BULK, mp.PATH_DIRECT], ids=["ce", "bulk", "direct"])
def test_executor_own_swap_options(path):
    """mpress_executor_set_option: the executor's swaps run on its own path
    (OPT_LAST_PATH after a step) while the context keeps its own (a plain
    swap afterwards runs the context's); options are copied at creation,
    validated like mpress_set_option, and non-swap options are refused."""
    M = 2
    ctx, pl, sizes = _setup(M)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    comp = torch.cuda.current_stream()
    try:
        ctx.set_option(mp.OPT_MAX_CTAS, 5)
        ex = mp.Executor(ctx, pl, 2, 0, M, 10_000, 20_000, 5_000, 5_000, s_out, s_in)
        assert ex.get_option(mp.OPT_MAX_CTAS) == 5            # copied from the context
        assert ex.get_option(mp.OPT_PATH) == mp.PATH_AUTO
        ex.set_option(mp.OPT_PATH, path)
        ex.set_option(mp.OPT_MAX_CTAS, 0)
        assert ctx.get_option(mp.OPT_PATH) == mp.PATH_AUTO    # the context is unchanged
        assert ctx.get_option(mp.OPT_MAX_CTAS) == 5
        with pytest.raises(mp.MPressError) as ei:
            ex.set_option(mp.OPT_TRANSPORT, 0)                 # not a swap option
        assert ei.value.code == mp.ERR_ARG
        with pytest.raises(mp.MPressError):
            ex.set_option(mp.OPT_VARIANT, 99)
        src = [[torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        dst = [[torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        for m in range(M):
            for i, t in enumerate(src[m]):
                synth_dev.fill(t, 70 + m, i)
            ex.restore_to(m, dst[m])
        for j in range(ex.ops):
            kind, m = ex.before(j, comp)
            ex.after(j, comp, src[m] if kind == "F" else None)
        torch.cuda.synchronize()
        assert ctx.get_option(mp.OPT_LAST_PATH) == path
        for m in range(M):
            for i, t in enumerate(dst[m]):
                assert synth_dev.check(t, 70 + m, i) == 0, (m, i)
        h = ctx.swap_out(pl, src[0])                            # a plain swap: the context's options
        torch.cuda.synchronize()
        assert ctx.get_option(mp.OPT_LAST_PATH) in (mp.PATH_DIRECT, mp.PATH_BULK)   # AUTO at 5 CTAs
        h.free(force=True)
        ex.free()
    finally:
        ctx.finalize()
