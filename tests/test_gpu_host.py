"""NEXT-4 on the GPU: a pinned host pool as a swap peer (GPU-CPU swap tier,
P:105).  The same plan / kernels / events move bytes over PCIe;
striping mixes NVLink-class peers and the host in proportion to the link
weights.  Bytes must be bit-exact."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import workloads

import _swaputil as U

pytestmark = pytest.mark.gpu


def _roundtrip(world, devices, spare, bw, sizes, seed, path):
    o = oracle.plan(world, 0, spare, bw, sizes)
    pl = mp.plan(world, 0, spare, bw, sizes)
    assert pl.stripes == [tuple(s) for s in o["stripes"]]
    part = [[0] * world for _ in range(world)]
    part[0] = [u * o["G"] for u in pl.units]
    ctx = mp.Context.local(world, 0, devices, part)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        src = U.make_inputs(sizes, seed)
        host = U.host_inputs(sizes, seed)
        s = torch.cuda.Stream()
        h = ctx.swap_out(pl, src, stream=s)
        s.synchronize()
        U.check_stash(ctx, h, o, host)
        for t in src:
            t.fill_(0)
        dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        ctx.swap_in(h, dst, stream=s)
        s.synchronize()
        for d, e in zip(dst, host):
            assert np.array_equal(d.cpu().numpy(), e)
        h.free()
    finally:
        ctx.finalize()
    return o


@pytest.mark.parametrize("path", [mp.PATH_DIRECT, mp.PATH_BULK, mp.PATH_CE])
def test_host_only_tier(path):
    _roundtrip(2, [0, mp.DEVICE_HOST], [0, 1 << 30], [0, 1], workloads.cfg1_sizes(), 11, path)


@pytest.mark.parametrize("path", [mp.PATH_DIRECT, mp.PATH_CE])
def test_mixed_nvlink_and_host_striping(path):
    """Three NVLink-class peers (900) and the host (55, PCIe-class): the host
    gets ~55/2755 of the batch."""
    world = 5
    o = _roundtrip(world, [0, 0, 0, 0, mp.DEVICE_HOST], [0] + [1 << 30] * 4, [0, 900, 900, 900, 55],
                   [1000, 70000, 3 << 20, 17], 12, path)
    assert 0 < o["units"][4] < o["units"][1]


def test_autotune_skips_host_pools():
    """mpress_autotune probes only device peers (a host pool is PCIe, and AUTO
    sends any swap touching one to the direct kernel anyway): with a device
    peer and a host peer it times the device peer, leaves the host pool's
    free space untouched, and AUTO swaps still run direct and bit-exact."""
    from synth import device as synth_dev
    world = 3
    spare, bw = [0, 1 << 30, 1 << 30], [0, 900, 55]
    sizes = [3 << 20, 4097]
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] + [2 * u * 65536 for u in pl.units[1:]], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0, 0, mp.DEVICE_HOST], part)
    try:
        free0 = ctx.stash_free()
        res = ctx.autotune(probe_bytes=1 << 20, trials=1)
        assert all(v > 0 for v in res["ms"].values()), res
        assert ctx.stash_free() == free0
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        for i, t in enumerate(src):
            synth_dev.fill(t, 81, i)
        dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        torch.cuda.synchronize()
        h = ctx.swap_out(pl, src)
        assert ctx.get_option(mp.OPT_LAST_PATH) == mp.PATH_DIRECT
        ctx.swap_in(h, dst)
        torch.cuda.synchronize()
        assert all(synth_dev.check(d, 81, i) == 0 for i, d in enumerate(dst))
        h.free()
    finally:
        ctx.finalize()


def test_auto_picks_copy_engines_for_host_only_launches():
    """MPRESS_PATH_AUTO per launch (round 2): every stripe to a host pool ->
    the copy engines (faster than any SM kernel over PCIe); device peers only
    -> the SM kernels even though the context also has a host pool; mixed ->
    direct.  Bytes equal the oracle's byte model in all three."""
    world = 3
    part_bytes = 64 << 20
    part = [[0, part_bytes, part_bytes], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0, 0, mp.DEVICE_HOST], part)
    try:
        sizes = [5 << 20, 4097]
        for bw, want in (([0, 0, 1], mp.PATH_CE), ([0, 1, 0], None), ([0, 900, 55], mp.PATH_DIRECT)):
            spare = [0, part_bytes if bw[1] else 0, part_bytes if bw[2] else 0]
            o = oracle.plan(world, 0, spare, bw, sizes)
            pl = mp.plan(world, 0, spare, bw, sizes)
            src = U.make_inputs(sizes, 91)
            h = ctx.swap_out(pl, src)
            torch.cuda.synchronize()
            ran = ctx.get_option(mp.OPT_LAST_PATH)
            if want is None:
                assert ran in (mp.PATH_DIRECT, mp.PATH_BULK)
            else:
                assert ran == want, (bw, ran)
            U.check_stash(ctx, h, o, U.host_inputs(sizes, 91))
            dst = [torch.zeros_like(t) for t in src]
            ctx.swap_in(h, dst)
            torch.cuda.synchronize()
            h.free()
            for d, e in zip(dst, U.host_inputs(sizes, 91)):
                assert np.array_equal(d.cpu().numpy(), e)
    finally:
        ctx.finalize()


@pytest.mark.parametrize("path", [mp.PATH_AUTO, mp.PATH_DIRECT, mp.PATH_BULK, mp.PATH_CE])
def test_pinned_host_tensors_as_swap_buffers(path):
    """Zero-copy e2e (bench `e2e_zero_copy`): pinned host tensors handed to
    mpress_swap_out / mpress_swap_in directly (UVA) -- the kernels read the
    host memory over PCIe into the device peers' stash and write it back;
    the stash equals the oracle's byte model and the host round trip is the
    identity."""
    world, G = 3, 65536
    sizes = [(3 << 20) + 48, 70001, 16]
    spare, bw = [0, 1 << 30, 1 << 30], [0, 1, 2]
    o = oracle.plan(world, 0, spare, bw, sizes, G)
    pl = mp.plan(world, 0, spare, bw, sizes, G)
    part = [[0] + [u * G for u in pl.units[1:]], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        host = U.host_inputs(sizes, 77)
        hsrc = [torch.from_numpy(h.copy()).pin_memory() for h in host]
        hdst = [torch.zeros(n, dtype=torch.uint8).pin_memory() for n in sizes]
        s = torch.cuda.Stream()
        h = ctx.swap_out(pl, hsrc, stream=s)
        s.synchronize()
        U.check_stash(ctx, h, o, host)
        ctx.swap_in(h, hdst, stream=s)
        s.synchronize()
        h.free()
        for d, e in zip(hdst, host):
            assert np.array_equal(d.numpy(), e)
    finally:
        ctx.finalize()
