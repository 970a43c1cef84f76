"""Bounds checks of every swap kernel shape with guard patterns of our own
(compute-sanitizer is closed on this GPU pool, so out-of-bounds and stray
writes are caught here by construction instead).

Every tensor, destination and stash partition sits inside a larger buffer
whose every other byte holds a seeded guard pattern (the generator's bytes of
a tensor id no swap uses).  After swap-out and after swap-in:

* the bytes inside each stripe equal the oracle's byte model (SURVEY §8(c)
  step 8: stash[p][dst_off:+len] = tensor[i][src_off:+len]; every restored
  tensor equals the original);
* EVERY byte outside them -- the gaps between tensors (placed 16-byte but
  not always 32-byte aligned, so both vector widths and the host alignment
  fall-back run), the stash partition around and between the stripes
  (including the padding R6 says is never copied), and the slack at the end
  of each partition -- still holds the guard pattern;
* the source buffers are unchanged by swap-out and the stash by swap-in
  (the kernels only load from the side they read).

Shapes: every MPRESS_OPT_VARIANT of the direct (14) and bulk (9) kernels,
each at grids of 1 and 3 CTAs (many pieces per CTA: the bulk ring wraps,
per-lane cursors finish at different times) and at its default grid, all
three CTA splits (blocked, strided, dynamic claims); the copy engines; AUTO; a > 128-descriptor launch (device-resident
tables); a pinned host-pool peer (NEXT-4)."""
import random

import pytest
import torch

import oracle
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev

pytestmark = pytest.mark.gpu

GUARD_SEED = 0x6A7D
SIZES = [1 << 20, 300007, 40, 3 * 4096 + 5, 17, 65536, 1]


def _layout(sizes, rng):
    """Offsets of `sizes` inside one buffer, 16-byte aligned, about half of
    them not 32-byte aligned, with guard gaps of 16 B .. ~5 KiB between."""
    offs, cur = [], 4096 + 16 * rng.randrange(0, 64)
    for n in sizes:
        cur = (cur + 15) // 16 * 16
        if cur % 32 == 0 and rng.random() < 0.5:
            cur += 16
        offs.append(cur)
        cur += n + 16 * rng.randrange(1, 320)
    return offs, cur + 4096


def _gaps(regions, total):
    """Complement of the (start, length) regions inside [0, total)."""
    out, cur = [], 0
    for a, n in sorted(regions):
        if a > cur:
            out.append((cur, a - cur))
        cur = max(cur, a + n)
    if total > cur:
        out.append((cur, total - cur))
    return out


def _guard_bad(base, regions, total, guard_id):
    return sum(synth_dev.check_ptr(base + a, n, GUARD_SEED, guard_id, start=a)
               for a, n in _gaps(regions, total))


class _Guarded:
    """Tensors of `sizes` carved out of one guard-filled buffer."""

    def __init__(self, sizes, rng, guard_id, seed=None):
        self.offs, self.total = _layout(sizes, rng)
        self.buf = torch.empty(self.total, dtype=torch.uint8, device="cuda")
        self.guard_id = guard_id
        synth_dev.fill(self.buf, GUARD_SEED, guard_id)
        self.tensors = [self.buf[o:o + n] for o, n in zip(self.offs, sizes)]
        if seed is not None:
            for i, t in enumerate(self.tensors):
                synth_dev.fill(t, seed, i)

    def guard_bad(self):
        regions = [(o, t.numel()) for o, t in zip(self.offs, self.tensors)]
        return _guard_bad(self.buf.data_ptr(), regions, self.total, self.guard_id)


def _check_stash(ctx, o, part_bytes, sl, seed):
    """(bytes of stripes differing from the oracle's byte model, guard bytes
    overwritten anywhere else in the partitions)."""
    bad_model = 0
    regions = {p: [] for p in part_bytes}
    for (i, p, so, do, ln) in o["stripes"]:
        bad_model += synth_dev.check_ptr(ctx.peer_ptr(p, sl[p] + do), ln, seed, i, start=so)
        regions[p].append((sl[p] + do, ln))
    bad_guard = sum(_guard_bad(ctx.peer_ptr(p, 0), regions[p], n, 1000 + p) for p, n in part_bytes.items())
    return bad_model, bad_guard


def _guarded_roundtrip(sizes, path, variant=-1, caps=(0,), split=0, host_peer=False, seed=11):
    world, peers = 4, [1, 2, 3]
    spare = [0, 1 << 30, 1 << 30, 1 << 30]
    bw = [0, 1, 2, 3]
    o = oracle.plan(world, 0, spare, bw, sizes)
    pl = mp.plan(world, 0, spare, bw, sizes)
    assert pl.stripes == [tuple(s) for s in o["stripes"]]
    G = o["G"]
    # each partition: the plan's units plus 64 KiB + 4 KiB of guard slack
    part_bytes = {p: pl.units[p] * G + G + 4096 for p in peers if pl.units[p]}
    part = [[0] * world for _ in range(world)]
    for p, n in part_bytes.items():
        part[0][p] = n
    devices = [0, 0, 0, mp.DEVICE_HOST if host_peer else 0]
    ctx = mp.Context.local(world, 0, devices, part)
    rng = random.Random(seed)
    try:
        ctx.set_option(mp.OPT_PATH, path)
        if variant >= 0:
            ctx.set_option(mp.OPT_VARIANT, variant)
        ctx.set_option(mp.OPT_SPLIT, split)
        for cap in caps:
            ctx.set_option(mp.OPT_MAX_CTAS, cap)
            src = _Guarded(sizes, rng, 900, seed=seed)
            dst = _Guarded(sizes, rng, 901)
            for p, n in part_bytes.items():
                synth_dev.fill_ptr(ctx.peer_ptr(p, 0), n, GUARD_SEED, 1000 + p)
            torch.cuda.synchronize()
            s = torch.cuda.Stream()
            h = ctx.swap_out(pl, src.tensors, stream=s)
            s.synchronize()
            sl = h.slices()
            what = (path, variant, cap, split)
            assert _check_stash(ctx, o, part_bytes, sl, seed) == (0, 0), what
            assert src.guard_bad() == 0, what
            assert sum(synth_dev.check(t, seed, i) for i, t in enumerate(src.tensors)) == 0, what
            ctx.swap_in(h, dst.tensors, stream=s)
            s.synchronize()
            assert sum(synth_dev.check(t, seed, i) for i, t in enumerate(dst.tensors)) == 0, what
            assert dst.guard_bad() == 0, what
            assert _check_stash(ctx, o, part_bytes, sl, seed) == (0, 0), what
            h.free()
    finally:
        ctx.finalize()


@pytest.mark.parametrize("variant", range(14))
def test_guard_direct_every_shape(variant):
    _guarded_roundtrip(SIZES, mp.PATH_DIRECT, variant, caps=(1, 3, 0), seed=100 + variant)


@pytest.mark.parametrize("variant", range(10))
def test_guard_bulk_every_shape(variant):
    _guarded_roundtrip(SIZES, mp.PATH_BULK, variant, caps=(1, 3, 0), seed=200 + variant)


@pytest.mark.parametrize("split", [1, 2], ids=["strided", "dynamic"])
@pytest.mark.parametrize("path", [mp.PATH_DIRECT, mp.PATH_BULK], ids=["direct", "bulk"])
def test_guard_other_splits(path, split):
    _guarded_roundtrip(SIZES, path, caps=(1, 2, 0), split=split, seed=300 + 10 * split + path)


@pytest.mark.parametrize("variant", list(range(14)))
def test_guard_dynamic_split_direct_every_shape(variant):
    _guarded_roundtrip(SIZES, mp.PATH_DIRECT, variant, caps=(3, 0), split=2, seed=700 + variant)


@pytest.mark.parametrize("variant", list(range(10)))
def test_guard_dynamic_split_bulk_every_shape(variant):
    _guarded_roundtrip(SIZES, mp.PATH_BULK, variant, caps=(3, 0), split=2, seed=800 + variant)


@pytest.mark.parametrize("path", [mp.PATH_AUTO, mp.PATH_CE], ids=["auto", "ce"])
def test_guard_auto_and_copy_engines(path):
    _guarded_roundtrip(SIZES, path, caps=(0, 5), seed=400 + path)


@pytest.mark.parametrize("path", [mp.PATH_DIRECT, mp.PATH_BULK], ids=["direct", "bulk"])
def test_guard_device_resident_tables(path):
    """> 128 descriptors in one launch: the kernel reads its table from the
    device-resident ring instead of the parameter block."""
    sizes = [1 + (i * 7919) % 5000 for i in range(140)]
    _guarded_roundtrip(sizes, path, caps=(0, 3), seed=500 + path)


@pytest.mark.parametrize("path", [mp.PATH_AUTO, mp.PATH_DIRECT, mp.PATH_BULK], ids=["auto", "direct", "bulk"])
def test_guard_host_pool_peer(path):
    """NEXT-4: peer 3 is a pinned host pool (its guard pattern written and
    checked through its device mapping)."""
    _guarded_roundtrip(SIZES, path, caps=(0,), host_peer=True, seed=600 + path)


def test_guard_detects_a_stray_write():
    """Negative control: 64 bytes written just past the last stripe of a
    slice (and 64 into a source gap) are reported by the same checks."""
    sizes = [300007, 40]
    world, spare, bw = 2, [0, 1 << 30], [0, 1]
    o = oracle.plan(world, 0, spare, bw, sizes)
    pl = mp.plan(world, 0, spare, bw, sizes)
    part_bytes = {1: pl.units[1] * o["G"] + o["G"]}
    ctx = mp.Context.local(world, 0, [0, 0], [[0, part_bytes[1]], [0, 0]])
    try:
        src = _Guarded(sizes, random.Random(7), 900, seed=7)
        synth_dev.fill_ptr(ctx.peer_ptr(1, 0), part_bytes[1], GUARD_SEED, 1001)
        torch.cuda.synchronize()
        h = ctx.swap_out(pl, src.tensors)
        torch.cuda.synchronize()
        sl = h.slices()
        assert _check_stash(ctx, o, part_bytes, sl, 7) == (0, 0)
        end = max(do + ln for (_, _, _, do, ln) in o["stripes"])
        synth_dev.fill_ptr(ctx.peer_ptr(1, sl[1] + end), 64, 12345, 1)
        synth_dev.fill(src.buf, 12345, 2, nbytes=64)        # the first 64 B of the source buffer: a gap
        torch.cuda.synchronize()
        assert _check_stash(ctx, o, part_bytes, sl, 7)[1] >= 56
        assert src.guard_bad() >= 56
        h.free(force=True)
    finally:
        ctx.finalize()
