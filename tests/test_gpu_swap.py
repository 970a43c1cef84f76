"""GPU parity of the swap path (through the C ABI) against the oracle.

Loopback mode (mpress_init_local with every peer on cuda:0): the peers' stash
pools are disjoint cuMem allocations of the same B200, mapped exactly as a
peer's pool would be, so planner, mapping, kernels and scheduler all run.
Bytes must match bit-exactly (R18): stash content vs the oracle byte model,
restored tensors vs the generator."""
import random

import numpy as np
import pytest
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev
from synth import splitmix64_bytes, workloads

import _swaputil as U

pytestmark = pytest.mark.gpu

PATHS = [mp.PATH_DIRECT, mp.PATH_BULK, mp.PATH_CE]


def test_synth_device_matches_host():
    for tid, (start, n) in enumerate([(0, 1), (3, 29), (8, 4096), (13, 100003)]):
        t = torch.empty(n, dtype=torch.uint8, device="cuda")
        synth_dev.fill(t, 99, tid, start)
        assert np.array_equal(t.cpu().numpy(), splitmix64_bytes(99, tid, start, n))
        assert synth_dev.check(t, 99, tid, start) == 0


@pytest.mark.parametrize("path", PATHS)
def test_config1_roundtrip(path):
    c = workloads.CONFIGS[1]
    spare = workloads.spare_vector(2, 0, c["peers"], spare=c["spare"])
    U.run_roundtrip(workloads.cfg1_sizes(), 2, 0, spare, [0, 1], seed=1000, path=path)


@pytest.mark.parametrize("path", PATHS)
def test_golden_g1_tails_and_padding(path):
    # 3 peers with weights 1:2:1, caps binding, 8- and 12-byte tails
    U.run_roundtrip([1000, 70000, 300], 4, 0, [0, 16384, 65536, 8192], [0, 1, 2, 1],
                    G=4096, seed=7, path=path)


@pytest.mark.parametrize("path", PATHS)
def test_random_ragged_instances(path):
    rng = random.Random(31 + path)
    for t in range(12):
        world = rng.randint(2, 8)
        source = rng.randrange(world)
        G = 256 * rng.choice([1, 4, 64, 256])
        sizes = [rng.choice([1, 7, 16, 31, 255, 256, 4097, rng.randint(1, 3 << 20)])
                 for _ in range(rng.randint(1, 20))]
        V = oracle.virtual_layout(sizes)[1]
        K = (V + G - 1) // G
        bw = [0 if p == source else rng.choice([0, 1, 2, 3]) for p in range(world)]
        if sum(bw) == 0:
            bw[(source + 1) % world] = 1
        spare = [(K + 2) * G if bw[p] else 0 for p in range(world)]
        U.run_roundtrip(sizes, world, source, spare, bw, G=G, seed=100 + t, path=path,
                        max_ctas=rng.choice([0, 1, 3, 16]))


@pytest.mark.parametrize("path", [mp.PATH_DIRECT, mp.PATH_BULK])
def test_more_stripes_than_one_launch(path):
    # 2500 tensors -> > 1024 descriptors -> several launches of one swap
    rng = random.Random(5)
    sizes = [rng.randint(1, 3000) for _ in range(2500)]
    o = U.run_roundtrip(sizes, 3, 0, [0, 1 << 26, 1 << 26], [0, 1, 1], G=4096, seed=5, path=path)
    assert len(o["stripes"]) > 1024


def test_one_byte_and_exact_granule():
    U.run_roundtrip([1], 2, 1, [1 << 20, 0], [1, 0], G=256, seed=3)
    U.run_roundtrip([65536, 65536], 3, 0, [0, 65536, 65536], [0, 1, 1], seed=4)


def test_alignment_and_state_errors():
    pl = mp.plan(2, 0, [0, 1 << 20], [0, 1], [4096])
    ctx = U.loopback_ctx(2, 0, pl.units, 65536)
    try:
        buf = torch.zeros(8192, dtype=torch.uint8, device="cuda")
        with pytest.raises(mp.MPressError) as ei:
            ctx.swap_out(pl, [buf.data_ptr() + 1])
        assert ei.value.code == mp.ERR_ALIGN
        h = ctx.swap_out(pl, [buf])
        with pytest.raises(mp.MPressError) as ei:
            h.free()
        assert ei.value.code == mp.ERR_STATE
        # partition holds exactly one handle
        with pytest.raises(mp.MPressError) as ei:
            ctx.swap_out(pl, [buf])
        assert ei.value.code == mp.ERR_NO_SPACE
        ctx.swap_in(h, [buf])
        with pytest.raises(mp.MPressError) as ei:
            ctx.swap_in(h, [buf])
        assert ei.value.code == mp.ERR_STATE
        torch.cuda.synchronize()
        assert ctx.query(h)
        h.free()
        # plan for another source is refused
        other = mp.plan(2, 1, [1 << 20, 0], [1, 0], [4096])
        with pytest.raises(mp.MPressError) as ei:
            ctx.swap_out(other, [buf])
        assert ei.value.code == mp.ERR_PEER
    finally:
        ctx.finalize()


def test_slice_reuse_is_fenced_across_streams():
    """swap-out A, swap-in A on stream 1, then swap-out B into the same slice
    on stream 2: B's kernel must wait for A's swap-in (fence event)."""
    sizes = [8 << 20]
    pl = mp.plan(2, 0, [0, 1 << 30], [0, 1], sizes)
    ctx = U.loopback_ctx(2, 0, pl.units, 65536)
    try:
        a = U.make_inputs(sizes, 11)
        b = U.make_inputs(sizes, 12)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        for _ in range(5):
            ha = ctx.swap_out(pl, a, stream=s1)
            dst = [torch.empty(sizes[0], dtype=torch.uint8, device="cuda")]
            ctx.swap_in(ha, dst, stream=s1)
            hb = ctx.swap_out(pl, b, stream=s2)   # reuses A's slice
            assert hb.slices() == ha.slices()
            torch.cuda.synchronize()
            assert synth_dev.check(dst[0], 11, 0) == 0
            dst2 = [torch.empty(sizes[0], dtype=torch.uint8, device="cuda")]
            ctx.swap_in(hb, dst2, stream=s2)
            torch.cuda.synchronize()
            assert synth_dev.check(dst2[0], 12, 0) == 0
            ha.free()
            hb.free()
    finally:
        ctx.finalize()


def test_multiple_handles_in_flight_config2():
    """8 micro-batches of Bert stage-0 activations in flight at once (1F1B), 3 peers."""
    sizes = workloads.cfg2_sizes(1)
    world, peers = 4, [1, 2, 3]
    spare = workloads.spare_vector(world, 0, peers, spare=24 << 30)
    bw = workloads.bw_vector(world, 0, peers)
    o = oracle.plan(world, 0, spare, bw, sizes)
    pl = mp.plan(world, 0, spare, bw, sizes)
    ctx = U.loopback_ctx(world, 0, pl.units, o["G"], copies=8)
    try:
        s = torch.cuda.Stream()
        srcs, hs = [], []
        for m in range(8):
            src = U.make_inputs(sizes, 2000 + m)
            srcs.append(src)
            hs.append(ctx.swap_out(pl, src, stream=s))
        slices = [tuple(h.slices()) for h in hs]
        assert len(set(slices)) == 8
        # sampled stash windows vs the oracle plan + generator
        torch.cuda.synchronize()
        rng = random.Random(0)
        for m in (0, 7):
            sl = hs[m].slices()
            for (i, p, so, do, ln) in rng.sample(o["stripes"], 10):
                x = rng.randrange(0, ln)
                n = min(4096, ln - x)
                got = np.frombuffer(ctx.peer_read(p, sl[p] + do + x, n), dtype=np.uint8)
                assert np.array_equal(got, splitmix64_bytes(2000 + m, i, so + x, n))
        del srcs
        for m in reversed(range(8)):
            dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
            ctx.swap_in(hs[m], dst, stream=s)
            s.synchronize()
            for i, d in enumerate(dst):
                assert synth_dev.check(d, 2000 + m, i) == 0
            hs[m].free()
    finally:
        ctx.finalize()


@pytest.mark.parametrize("path", [mp.PATH_DIRECT, mp.PATH_BULK])
def test_large_tables_device_resident_ring_wraps(path):
    """Launches of more than 128 descriptors read a device-resident table
    (pinned staging slot -> device slot on the swap stream).  300 swap pairs
    of a 150-tensor plan (600 launches) are enqueued without a host sync, so
    the 256-slot ring wraps and slots are reused behind their kernels; every
    restored tensor is bit-exact.  The same plan captured into a CUDA graph
    (tables as kernel parameters there) round-trips too."""
    import numpy as np
    from synth import device as synth_dev
    world = 3
    rng = np.random.default_rng(5)
    sizes = [int(x) for x in rng.integers(1, 200_000, size=150)]
    pl = mp.plan(world, 0, [0, 1 << 30, 1 << 30], [0, 1, 2], sizes)
    assert len(pl.stripes) > 128
    part = [[0] + [4 * u * 65536 for u in pl.units[1:]], [0] * 3, [0] * 3]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        for i, t in enumerate(src):
            synth_dev.fill(t, 70, i)
        dst = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        ps, pd = mp.pointers(src), mp.pointers(dst)
        for _ in range(300):
            h = ctx.swap_out(pl, ps, stream=s)
            ctx.swap_in(h, pd, stream=s)
            h.free()
        s.synchronize()
        assert all(synth_dev.check(d, 70, i) == 0 for i, d in enumerate(dst))
        # graph capture: parameter tables (the ring is not used under capture)
        dst2 = [torch.zeros(n, dtype=torch.uint8, device="cuda") for n in sizes]
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            gh = ctx.swap_out(pl, src)
            ctx.swap_in(gh, dst2)
        g.replay()
        torch.cuda.synchronize()
        assert all(synth_dev.check(d, 70, i) == 0 for i, d in enumerate(dst2))
        gh.free()
        del g
    finally:
        ctx.finalize()
