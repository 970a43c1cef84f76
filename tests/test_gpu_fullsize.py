"""Full-size parity at BASELINE.json's sizes, in the launch configurations
bench.py times (default grid; AUTO's default kernel and the direct kernel,
the two mpress_autotune chooses between): EVERY stash byte of every stripe
of the oracle's plan checked in place on the device (mpress_peer_ptr + the
generator's check kernel) against the oracle's byte model, sampled windows
also copied to the host and compared with the generator there, and the
round trip checked on the device against the generator for every byte.
(Out-of-bounds / stray-write checks of every kernel shape: test_gpu_bounds.py.)"""
import random

import numpy as np
import pytest
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev
from synth import splitmix64_bytes, workloads

pytestmark = pytest.mark.gpu


def _sampled_roundtrip(world, source, spare, bw, sizes, seed, samples=64, path=None, variant=-1, max_ctas=0):
    o = oracle.plan(world, source, spare, bw, sizes)
    pl = mp.plan(world, source, spare, bw, sizes)
    assert pl.stripes == [tuple(s) for s in o["stripes"]]
    assert pl.units == o["units"] and pl.peer_bytes == o["peer_bytes"]
    part = [[0] * world for _ in range(world)]
    part[source] = [u * o["G"] for u in pl.units]
    ctx = mp.Context.local(world, source, [0] * world, part)
    try:
        if path is not None:
            ctx.set_option(mp.OPT_PATH, path)
            if variant >= 0:
                ctx.set_option(mp.OPT_VARIANT, variant)
        ctx.set_option(mp.OPT_MAX_CTAS, max_ctas)
        src = []
        for i, n in enumerate(sizes):
            t = torch.empty(n, dtype=torch.uint8, device="cuda")
            synth_dev.fill(t, seed, i)
            src.append(t)
        # the fills run on the current stream; the swap stream does not wait
        # for it on its own (non-blocking streams)
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        h = ctx.swap_out(pl, src, stream=s)
        s.synchronize()
        sl = h.slices()
        # every stash byte of every stripe, on the device: the oracle's byte
        # model (stash[p][dst_off:+len] =
        # tensor[i][src_off:+len]) over the oracle's own stripes, with the
        # tensor bytes regenerated from (seed, i, src_off)
        bad, checked = 0, 0
        for (i, p, so, do, ln) in o["stripes"]:
            bad += synth_dev.check_ptr(ctx.peer_ptr(p, sl[p] + do), ln, seed, i, start=so)
            checked += ln
        assert bad == 0, "%d of %d stash bytes differ from the oracle's byte model" % (bad, checked)
        assert checked == sum(sizes)
        rng = random.Random(seed)
        picks = list(o["stripes"])
        rng.shuffle(picks)
        # first/last bytes of every stripe + random interior windows
        for (i, p, so, do, ln) in o["stripes"]:
            for x in (0, max(0, ln - 4096)):
                n = min(4096, ln - x)
                got = np.frombuffer(ctx.peer_read(p, sl[p] + do + x, n), dtype=np.uint8)
                assert np.array_equal(got, splitmix64_bytes(seed, i, so + x, n)), (i, p, x)
        for (i, p, so, do, ln) in picks[:samples]:
            x = rng.randrange(0, ln)
            n = min(1 << 16, ln - x)
            got = np.frombuffer(ctx.peer_read(p, sl[p] + do + x, n), dtype=np.uint8)
            assert np.array_equal(got, splitmix64_bytes(seed, i, so + x, n)), (i, p, x)
        del src
        torch.cuda.empty_cache()
        dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        ctx.swap_in(h, dst, stream=s)
        s.synchronize()
        for i, d in enumerate(dst):
            assert synth_dev.check(d, seed, i) == 0, i
        h.free()
    finally:
        ctx.finalize()
    return o


@pytest.mark.parametrize("path", [None, mp.PATH_DIRECT], ids=["auto", "direct"])
def test_config3_gpt_adam_states_full_size(path):
    """BJ:9: 100 fp32 Adam m/v tensors (12.21 GB) -> peers 5,6,7 with 8/8/2 GiB
    spare: the cap binds on peer 7 (water-fill)."""
    c = workloads.CONFIGS[3]
    spare = workloads.spare_vector(8, 0, c["peers"], spare_by_peer=c["spare_by_peer"])
    bw = workloads.bw_vector(8, 0, c["peers"])
    o = _sampled_roundtrip(8, 0, spare, bw, workloads.cfg3_sizes(), seed=3000, path=path)
    assert o["units"][7] * o["G"] == 2 << 30


@pytest.mark.parametrize("path", [None, mp.PATH_DIRECT], ids=["auto", "direct"])
def test_config4_largest_size_seven_peers(path):
    """BJ:10: one 4 GiB uint8 tensor striped over 7 peers."""
    peers = list(range(1, 8))
    spare = workloads.spare_vector(8, 0, peers, spare=8 << 30)
    bw = workloads.bw_vector(8, 0, peers)
    _sampled_roundtrip(8, 0, spare, bw, [4 << 30], seed=4000, path=path)


@pytest.mark.parametrize("path", [None, mp.PATH_DIRECT], ids=["auto", "direct"])
def test_config2_x8_single_batch_full_size(path):
    """BJ:8: the 8 in-flight micro-batches (376 tensors, 7.03 GiB) as one plan
    over 3 peers."""
    peers = [1, 2, 3]
    spare = workloads.spare_vector(4, 0, peers, spare=24 << 30)
    bw = workloads.bw_vector(4, 0, peers)
    _sampled_roundtrip(4, 0, spare, bw, workloads.cfg2_sizes(8), seed=2000, path=path)


@pytest.mark.parametrize("path", [None, mp.PATH_DIRECT], ids=["auto", "direct"])
def test_stripe_longer_than_4gib(path):
    """One 6 GiB + 17 B tensor to one peer: a single stripe longer than 2^32
    bytes (64-bit lengths and offsets through the tables and the kernels'
    chunk arithmetic), with a ragged tail."""
    spare = [0, 8 << 30]
    _sampled_roundtrip(2, 0, spare, [0, 1], [(6 << 30) + 17], seed=4100, path=path)


@pytest.mark.parametrize("path,variant,cap", [(mp.PATH_BULK, 7, 148), (mp.PATH_AUTO, -1, 64)],
                         ids=["gemm_leg_bulk7x148", "auto_capped64"])
def test_config2_micro_batch_gemm_leg_settings(path, variant, cap):
    """BJ:8 / BJ:11: one full Bert stage-0 micro-batch (47 tensors, 900 MiB)
    over 3 peers in the launch configurations the bench's GEMM legs time
    (the one-warp TMA shape on every SM, with the AUTO split's dynamic
    claims; AUTO capped at 64 CTAs = direct shape 9): every stash byte
    against the oracle's byte model, every restored byte."""
    peers = [1, 2, 3]
    spare = workloads.spare_vector(4, 0, peers, spare=4 << 30)
    bw = workloads.bw_vector(4, 0, peers)
    _sampled_roundtrip(4, 0, spare, bw, workloads.cfg2_sizes(1), seed=2100 + cap, path=path, variant=variant,
                       max_ctas=cap)
