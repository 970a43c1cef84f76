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
