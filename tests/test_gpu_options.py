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
            ctx.set_option(mp.OPT_VARIANT, 10)                       # bulk has 10 shapes (0-9)
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
    """MPRESS_PATH_AUTO: at a full grid the size class's kernel (direct for a
    small launch before any autotune), direct when the grid is capped to <=
    one CTA per SM; variants cannot be forced under AUTO; every resolution
    round-trips bit-exactly."""
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
        # a ~3 MiB launch is in the small class: direct before any autotune
        assert sum(sizes) < mp.AUTO_SMALL_BYTES
        small = ctx.get_option(mp.OPT_AUTO_OUT_SMALL)
        assert small == ctx.get_option(mp.OPT_AUTO_IN_SMALL) == mp.PATH_DIRECT
        for cap, want in ((0, small), (sms + 1, small), (sms, mp.PATH_DIRECT), (16, mp.PATH_DIRECT)):
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


def test_pdl_modes():
    """MPRESS_OPT_PDL: 0 never, 1 (default) uncapped grids only, 2 always;
    chains of swap kernels on one stream stay ordered in every mode (each
    PDL-launched kernel waits for its predecessor grid before touching
    memory), capped and uncapped, and the data round-trips bit-exactly."""
    from synth import device as synth_dev
    world = 3
    sizes = [(5 << 20) + 48, 65536 * 3 + 7, 4096]
    pl = mp.plan(world, 0, [0, 1 << 30, 1 << 30], [0, 1, 1], sizes)
    chain = 4
    part = [[0] + [chain * u * 65536 for u in pl.units[1:]], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        assert ctx.get_option(mp.OPT_PDL) == 1
        for bad in (-1, 3):
            with pytest.raises(mp.MPressError) as ei:
                ctx.set_option(mp.OPT_PDL, bad)
            assert ei.value.code == mp.ERR_ARG
        srcs = [[torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(chain)]
        for k, src in enumerate(srcs):
            for i, t in enumerate(src):
                synth_dev.fill(t, 50 + k, i)
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        for mode in (0, 1, 2):
            ctx.set_option(mp.OPT_PDL, mode)
            assert ctx.get_option(mp.OPT_PDL) == mode
            for path, cap in ((mp.PATH_DIRECT, 0), (mp.PATH_DIRECT, 8), (mp.PATH_BULK, 0), (mp.PATH_BULK, 8)):
                ctx.set_option(mp.OPT_PATH, path)
                ctx.set_option(mp.OPT_MAX_CTAS, cap)
                dsts = [[torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(chain)]
                with torch.cuda.stream(s):
                    hs = [ctx.swap_out(pl, src, stream=s) for src in srcs]
                    for h, dst in zip(hs, dsts):
                        ctx.swap_in(h, dst, stream=s)
                    # a second generation through the same slices, back to back
                    hs2 = [ctx.swap_out(pl, dst, stream=s) for dst in dsts]
                    for h, dst in zip(hs2, dsts):
                        ctx.swap_in(h, dst, stream=s)
                s.synchronize()
                for k, dst in enumerate(dsts):
                    assert all(synth_dev.check(d, 50 + k, i) == 0 for i, d in enumerate(dst)), (mode, path, cap, k)
                for h in hs + hs2:
                    h.free()
    finally:
        ctx.finalize()


def test_autotune_local():
    """mpress_autotune on a loopback context: both kernels timed per
    direction and size class, each choice is one of them, later AUTO swaps
    with an uncapped grid run the chosen kernel for their direction and size
    class (capped ones stay direct), and everything round-trips bit-exactly.
    A live handle refuses the probe."""
    from synth import device as synth_dev
    world = 4
    small = [(7 << 20) + 3, 1 << 20, 33]          # < AUTO_SMALL_BYTES per launch
    large = [48 << 20, 5]                          # >= AUTO_SMALL_BYTES
    assert sum(small) < mp.AUTO_SMALL_BYTES <= sum(large)
    spare, bw = [0] + [1 << 30] * 3, [0, 1, 1, 1]
    pls = {"small": mp.plan(world, 0, spare, bw, small), "large": mp.plan(world, 0, spare, bw, large)}
    part = [[0] + [2 * u * 65536 for u in pls["large"].units[1:]]] + [[0] * world for _ in range(3)]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        assert ctx.get_option(mp.OPT_AUTO_OUT) == ctx.get_option(mp.OPT_AUTO_IN) == mp.PATH_BULK
        assert ctx.get_option(mp.OPT_AUTO_OUT_SMALL) == ctx.get_option(mp.OPT_AUTO_IN_SMALL) == mp.PATH_DIRECT
        for bad in ((0, 3), (1 << 20, 0), (1 << 20, 65)):
            with pytest.raises(mp.MPressError) as ei:
                ctx.autotune(probe_bytes=bad[0], trials=bad[1])
            assert ei.value.code == mp.ERR_ARG
        free0 = ctx.stash_free()
        res = ctx.autotune(probe_bytes=64 << 20, trials=3)
        assert ctx.stash_free() == free0   # the probe's slices went back
        for k in ("out", "in", "out_small", "in_small"):
            assert res[k] in (mp.PATH_DIRECT, mp.PATH_BULK), res
        assert len(res["ms"]) == 8 and all(v > 0 for v in res["ms"].values()), res
        for cls, sizes in (("small", small), ("large", large)):
            pl = pls[cls]
            src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
            for i, t in enumerate(src):
                synth_dev.fill(t, 61, i)
            torch.cuda.synchronize()
            suffix = "" if cls == "large" else "_small"
            for cap in (0, 16):
                ctx.set_option(mp.OPT_MAX_CTAS, cap)
                dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
                h = ctx.swap_out(pl, src)
                assert ctx.get_option(mp.OPT_LAST_PATH) == (res["out" + suffix] if cap == 0 else mp.PATH_DIRECT)
                if cap == 0:
                    with pytest.raises(mp.MPressError) as ei:
                        ctx.autotune()
                    assert ei.value.code == mp.ERR_STATE
                ctx.swap_in(h, dst)
                assert ctx.get_option(mp.OPT_LAST_PATH) == (res["in" + suffix] if cap == 0 else mp.PATH_DIRECT)
                torch.cuda.synchronize()
                assert all(synth_dev.check(d, 61, i) == 0 for i, d in enumerate(dst)), (cls, cap)
                h.free()
    finally:
        ctx.finalize()


@pytest.mark.parametrize("path,cap", [(mp.PATH_DIRECT, 32), (mp.PATH_DIRECT, 0), (mp.PATH_BULK, 0)])
def test_pace_limits_rate_and_keeps_bytes(path, cap):
    """MPRESS_OPT_PACE_MBPS: a paced swap moves at most the requested rate
    (it only has to fit the live interval), and its stash and restored
    bytes still equal the oracle's byte model."""
    import oracle
    from _swaputil import check_stash, host_inputs, make_inputs
    from synth import device as synth_dev
    world, G = 4, 65536
    sizes = [(64 << 20) + 48, 3 << 20, 1000]
    spare, bw = [0, 1 << 30, 1 << 30, 1 << 30], [0, 1, 2, 1]
    pl = mp.plan(world, 0, spare, bw, sizes, G)
    o = oracle.plan(world, 0, spare, bw, sizes, G)
    part = [[0] * world for _ in range(world)]
    part[0] = [u * G for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        ctx.set_option(mp.OPT_MAX_CTAS, cap)
        src = make_inputs(sizes, 31)
        dst = [torch.zeros_like(t) for t in src]
        nbytes = sum(sizes)
        s = torch.cuda.Stream()
        for pace in (0, 100_000):          # off, then 100 GB/s
            ctx.set_option(mp.OPT_PACE_MBPS, pace)
            assert ctx.get_option(mp.OPT_PACE_MBPS) == pace
            e = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            e[0].record(s)
            h = ctx.swap_out(pl, src, stream=s)
            e[1].record(s)
            torch.cuda.synchronize()
            check_stash(ctx, h, o, host_inputs(sizes, 31))
            e[2].record(s)
            ctx.swap_in(h, dst, stream=s)
            e[3].record(s)
            torch.cuda.synchronize()
            h.free()
            for i, t in enumerate(dst):
                assert synth_dev.check(t, 31, i) == 0
                t.zero_()
            if pace:
                for a, b in ((e[0], e[1]), (e[2], e[3])):
                    gbs = nbytes / a.elapsed_time(b) / 1e6
                    assert 60 < gbs <= 100 * 1.03, gbs
        with pytest.raises(mp.MPressError):
            ctx.set_option(mp.OPT_PACE_MBPS, -1)
    finally:
        ctx.finalize()


@pytest.mark.parametrize("split", [0, 1, 2, 3], ids=["blocked", "strided", "dynamic", "auto"])
@pytest.mark.parametrize("path,variant,cap", [(mp.PATH_DIRECT, 7, 5), (mp.PATH_DIRECT, 11, 128),
                                              (mp.PATH_DIRECT, 5, 0), (mp.PATH_BULK, 3, 0),
                                              (mp.PATH_BULK, 6, 7)])
def test_split_modes_are_oracle_exact(split, path, variant, cap):
    """MPRESS_OPT_SPLIT: every way of sharing a launch's interleaved chunks
    among CTAs write exactly the oracle's stash bytes and restore every
    tensor, with ragged stripes over three peers of unequal weight."""
    import oracle
    from _swaputil import check_stash, host_inputs, make_inputs
    from synth import device as synth_dev
    world, G = 4, 65536
    sizes = [(5 << 20) + 48, 777, 3 << 20, 70001]
    spare, bw = [0, 1 << 30, 1 << 30, 1 << 30], [0, 1, 3, 2]
    pl = mp.plan(world, 0, spare, bw, sizes, G)
    o = oracle.plan(world, 0, spare, bw, sizes, G)
    part = [[0] * world for _ in range(world)]
    part[0] = [u * G for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        ctx.set_option(mp.OPT_VARIANT, variant)
        ctx.set_option(mp.OPT_MAX_CTAS, cap)
        ctx.set_option(mp.OPT_SPLIT, split)
        assert ctx.get_option(mp.OPT_SPLIT) == split
        src = make_inputs(sizes, 41)
        h = ctx.swap_out(pl, src)
        torch.cuda.synchronize()
        check_stash(ctx, h, o, host_inputs(sizes, 41))
        dst = [torch.zeros_like(t) for t in src]
        ctx.swap_in(h, dst)
        torch.cuda.synchronize()
        h.free()
        assert all(synth_dev.check(t, 41, i) == 0 for i, t in enumerate(dst))
        with pytest.raises(mp.MPressError):
            ctx.set_option(mp.OPT_SPLIT, 4)
    finally:
        ctx.finalize()


def test_autotune_waits_for_inflight_swap_in():
    """a freed IN_PENDING handle leaves its slices fenced by the
    swap-in's event; mpress_autotune uses the stash as probe scratch and must
    not write those bytes before that swap-in has read them.  The swap-in's
    stream is held back by a sleep, the handle freed, autotune run on
    another stream: the restored tensors must still be the original bytes."""
    from synth import device as synth_dev
    world, G = 3, 65536
    sizes = [8 << 20, 3 << 20]
    spare, bw = [0, 1 << 30, 1 << 30], [0, 1, 1]
    pl = mp.plan(world, 0, spare, bw, sizes, G)
    part = [[0] + [u * G for u in pl.units[1:]], [0] * 3, [0] * 3]   # room for exactly one handle
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        for i, t in enumerate(src):
            synth_dev.fill(t, 61, i)
        dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        s_in, s_probe = torch.cuda.Stream(), torch.cuda.Stream()
        torch.cuda.synchronize()
        h = ctx.swap_out(pl, src, stream=s_in)
        with torch.cuda.stream(s_in):
            torch.cuda._sleep(50_000_000)             # ~25 ms: the swap-in starts late
        ctx.swap_in(h, dst, stream=s_in)
        h.free()                                      # IN_PENDING: slices released, fenced
        ctx.autotune(probe_bytes=sum(sizes), trials=1, stream=s_probe)
        torch.cuda.synchronize()
        assert all(synth_dev.check(t, 61, i) == 0 for i, t in enumerate(dst))
    finally:
        ctx.finalize()


def test_peer_ptr_errors_and_identity():
    """mpress_peer_ptr (the device address behind the element-wise stash
    check): the bytes at the pointer are the ones mpress_peer_read returns;
    unmapped peers and out-of-range offsets are refused."""
    import numpy as np
    from synth import device as synth_dev
    world = 3
    sizes = [1 << 20]
    pl = mp.plan(world, 0, [0, 1 << 30, 0], [0, 1, 0], sizes)
    part = [[0, 2 << 20, 0], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        src = [torch.empty(sizes[0], dtype=torch.uint8, device="cuda")]
        synth_dev.fill(src[0], 71, 0)
        h = ctx.swap_out(pl, src)
        torch.cuda.synchronize()
        off = h.slices()[1]
        p = ctx.peer_ptr(1, off)
        assert synth_dev.check_ptr(p, sizes[0], 71, 0) == 0
        assert np.array_equal(np.frombuffer(ctx.peer_read(1, off, 4096), dtype=np.uint8),
                              src[0][:4096].cpu().numpy())
        with pytest.raises(mp.MPressError) as ei:
            ctx.peer_ptr(2, 0)                     # no partition on peer 2
        assert ei.value.code == mp.ERR_PEER
        with pytest.raises(mp.MPressError) as ei:
            ctx.peer_ptr(1, (2 << 20) + 1)         # past the partition
        assert ei.value.code == mp.ERR_ARG
        with pytest.raises(mp.MPressError):
            ctx.peer_ptr(5, 0)
        ctx.swap_in(h, src)
        torch.cuda.synchronize()
        h.free()
    finally:
        ctx.finalize()


def test_dynamic_claims_counter_ring_wraps_and_streams():
    """MPRESS_SPLIT_DYNAMIC: 600 launches (more than the 256 claim-counter
    slots, so every slot is reset by its launch's last CTA and reused) on two
    streams at once, at 1 CTA (the claims' serial case) and 8 CTAs;
    every restored byte equals the generator -- a slot left non-zero, or
    shared by two concurrent launches, would skip or duplicate chunks."""
    from synth import device as synth_dev
    world = 3
    sizes = [(1 << 20) + 4096 * 3 + 48, 333333]
    spare, bw = [0, 1 << 30, 1 << 30], [0, 2, 1]
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] * world for _ in range(world)]
    part[0] = [8 * u * mp.DEFAULT_GRANULE for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        ctx.set_option(mp.OPT_PATH, mp.PATH_BULK)
        ctx.set_option(mp.OPT_SPLIT, mp.SPLIT_DYNAMIC)
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        for i, t in enumerate(src):
            synth_dev.fill(t, 61, i)
        torch.cuda.synchronize()
        streams = [torch.cuda.Stream(), torch.cuda.Stream()]
        for cap in (1, 8):
            ctx.set_option(mp.OPT_MAX_CTAS, cap)
            dsts = []     # all kept alive until the sync (used on side streams)
            for k in range(150):
                s = streams[k % 2]
                dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
                s.wait_stream(torch.cuda.current_stream())
                h = ctx.swap_out(pl, src, stream=s)
                ctx.swap_in(h, dst, stream=s)
                h.free()
                dsts.append(dst)
            torch.cuda.synchronize()
            for dst in dsts:
                assert all(synth_dev.check(t, 61, i) == 0 for i, t in enumerate(dst)), cap
    finally:
        ctx.finalize()
