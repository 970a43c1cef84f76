"""Context options and the free-space query (the spare_bytes argument of the
next mpress_plan, R21)."""
import pytest
import torch

import paper_conf_hpca_zhouwylbyx23_b200 as mp

pytestmark = pytest.mark.gpu


def test_options_and_stash_free():
    world = 3
    sizes = [1 << 20]
    pl = mp.plan(world, 0, [0, 1 << 30, 1 << 30], [0, 1, 1], sizes)
    part = [[0, 4 << 20, 4 << 20], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        assert ctx.get_option(mp.OPT_PATH) == mp.PATH_AUTO
        assert ctx.get_option(mp.OPT_VARIANT) == mp.VARIANT_AUTO
        assert ctx.get_option(mp.OPT_ORDER) == mp.ORDER_INTERLEAVE
        ctx.set_option(mp.OPT_MAX_CTAS, 12)
        assert ctx.get_option(mp.OPT_MAX_CTAS) == 12
        for key, bad in ((mp.OPT_PATH, 7), (mp.OPT_VARIANT, 99), (mp.OPT_ORDER, 5), (mp.OPT_MAX_CTAS, -1), (42, 0)):
            with pytest.raises(mp.MPressError) as ei:
                ctx.set_option(key, bad)
            assert ei.value.code == mp.ERR_ARG
        ctx.set_option(mp.OPT_PATH, mp.PATH_BULK)
        assert ctx.get_option(mp.OPT_VARIANT) == mp.VARIANT_AUTO   # reset with the path
        with pytest.raises(mp.MPressError):
            ctx.set_option(mp.OPT_VARIANT, 7)                        # bulk has 7 shapes (0-6)
        assert ctx.stash_free() == [0, 4 << 20, 4 << 20]
        src = [torch.zeros(sizes[0], dtype=torch.uint8, device="cuda")]
        h = ctx.swap_out(pl, src)
        free = ctx.stash_free()
        assert free[1] == (4 << 20) - pl.units[1] * 65536 and free[2] == (4 << 20) - pl.units[2] * 65536
        ctx.swap_in(h, src)
        torch.cuda.synchronize()
        assert ctx.stash_free() == [0, 4 << 20, 4 << 20]
        h.free()
    finally:
        ctx.finalize()


def test_auto_path_resolution():
    """MPRESS_PATH_AUTO: bulk (TMA) at a full grid, direct when the grid is
    capped to <= one CTA per SM; variants cannot be forced under AUTO; every
    resolution round-trips bit-exactly."""
    from synth import device as synth_dev
    world = 3
    sizes = [(3 << 20) + 5, 4096]
    pl = mp.plan(world, 0, [0, 1 << 30, 1 << 30], [0, 1, 1], sizes)
    part = [[0] + [u * 65536 for u in pl.units[1:]], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        with pytest.raises(mp.MPressError) as ei:
            ctx.set_option(mp.OPT_VARIANT, 0)
        assert ei.value.code == mp.ERR_ARG
        assert ctx.get_option(mp.OPT_LAST_PATH) == -1
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        for i, t in enumerate(src):
            synth_dev.fill(t, 4, i)
        sms = torch.cuda.get_device_properties(0).multi_processor_count
        for cap, want in ((0, mp.PATH_BULK), (sms + 1, mp.PATH_BULK), (sms, mp.PATH_DIRECT), (16, mp.PATH_DIRECT)):
            ctx.set_option(mp.OPT_MAX_CTAS, cap)
            dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
            h = ctx.swap_out(pl, src)
            assert ctx.get_option(mp.OPT_LAST_PATH) == want, cap
            ctx.swap_in(h, dst)
            torch.cuda.synchronize()
            assert all(synth_dev.check(d, 4, i) == 0 for i, d in enumerate(dst)), cap
            h.free()
    finally:
        ctx.finalize()
