"""Every kernel shape (MPRESS_OPT_VARIANT) on a ragged multi-peer batch, with
32-byte aligned and with only 16-byte aligned tensors (the 32-byte-vector
shapes must fall back), bit-exact against the oracle byte model."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev
from synth import splitmix64_bytes

pytestmark = pytest.mark.gpu

SIZES = [1000, 70000, 300, (1 << 20) + 48, 17, 65536 * 3]


@pytest.mark.parametrize("path,variant", [(mp.PATH_DIRECT, v) for v in range(14)] +
                         [(mp.PATH_BULK, v) for v in range(10)] +
                         [(mp.PATH_CE, 0)])
@pytest.mark.parametrize("misalign", [0, 16])
def test_variant_roundtrip(path, variant, misalign):
    world, G = 4, 4096
    spare, bw = [0, 1 << 26, 1 << 26, 1 << 26], [0, 1, 2, 1]
    o = oracle.plan(world, 0, spare, bw, SIZES, G)
    pl = mp.plan(world, 0, spare, bw, SIZES, G)
    part = [[0] * world for _ in range(world)]
    part[0] = [u * G for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        ctx.set_option(mp.OPT_VARIANT, variant)
        ctx.set_option(mp.OPT_MAX_CTAS, 37)
        # tensors placed at +misalign inside larger buffers
        bufs = [torch.empty(n + 64, dtype=torch.uint8, device="cuda") for n in SIZES]
        src = [b[misalign:misalign + n] for b, n in zip(bufs, SIZES)]
        for i, t in enumerate(src):
            synth_dev.fill(t, 77, i)
        torch.cuda.synchronize()
        h = ctx.swap_out(pl, src)
        torch.cuda.synchronize()
        host = [splitmix64_bytes(77, i, 0, n) for i, n in enumerate(SIZES)]
        sl = h.slices()
        for p, (buf, defined) in oracle.swap_out(o, host).items():
            got = np.frombuffer(ctx.peer_read(p, sl[p], len(buf)), dtype=np.uint8)
            assert not np.any((got != buf) & defined), p
        obufs = [torch.zeros(n + 64, dtype=torch.uint8, device="cuda") for n in SIZES]
        dst = [b[misalign:misalign + n] for b, n in zip(obufs, SIZES)]
        torch.cuda.synchronize()
        ctx.swap_in(h, dst)
        torch.cuda.synchronize()
        for i, (d, e) in enumerate(zip(dst, host)):
            assert np.array_equal(d.cpu().numpy(), e), i
        # nothing outside the tensors was written
        for b, n in zip(obufs, SIZES):
            full = b.cpu().numpy()
            assert not full[:misalign].any() and not full[misalign + n:].any()
        h.free()
    finally:
        ctx.finalize()
