"""Scheduler fuzz on the GPU: random interleavings of swap-outs, swap-ins,
waits, queries and frees across two streams, with a partition that only
holds a few handles at once (slices are reused under fences, R21/R22) and a
mix of kernel paths.  Every restored tensor must equal the generator."""
import os
import random

import pytest
import torch

import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import device as synth_dev

pytestmark = pytest.mark.gpu


# MPRESS_FUZZ_EXTRA=N adds N more seeds (a soak run; the default suite runs 3)
SEEDS = [1, 2, 3] + list(range(1000, 1000 + int(os.environ.get("MPRESS_FUZZ_EXTRA", "0"))))


@pytest.mark.parametrize("seed", SEEDS)
def test_random_interleavings(seed):
    rng = random.Random(seed)
    world = 4
    # every third seed: 140 small tensors, so launches exceed 128 descriptors
    # and read device-resident tables (the staging/device ring) mid-interleaving
    if seed % 3 == 0:
        sizes = [rng.randint(1, 64 << 10) for _ in range(140)]
    else:
        sizes = [rng.randint(1, 3 << 20) for _ in range(5)]
    spare = [0, 1 << 30, 1 << 30, 1 << 30]
    bw = [0, 1, 2, 1]
    pl = mp.plan(world, 0, spare, bw, sizes, 4096)
    part = [[0] * world for _ in range(world)]
    part[0] = [3 * u * 4096 for u in pl.units]          # room for 3 handles
    ctx = mp.Context.local(world, 0, [0] * world, part)
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    live = []        # (handle, seed, dst or None, stream)
    next_seed = 100 * seed
    checked = 0
    try:
        for step in range(120):
            op = rng.random()
            if op < 0.45:
                if step % 17 == 0:
                    ctx.set_option(mp.OPT_PATH, rng.choice([mp.PATH_DIRECT, mp.PATH_BULK, mp.PATH_CE,
                                                            mp.PATH_AUTO]))
                    ctx.set_option(mp.OPT_MAX_CTAS, rng.choice([0, 1, 7, 64]))
                    ctx.set_option(mp.OPT_PDL, rng.choice([0, 1, 2]))
                    ctx.set_option(mp.OPT_SPLIT, rng.choice([mp.SPLIT_BLOCKED, mp.SPLIT_STRIDED, mp.SPLIT_DYNAMIC, mp.SPLIT_AUTO]))
                    ctx.set_option(mp.OPT_PACE_MBPS, rng.choice([0, 0, 200_000, 2_000_000]))
                src = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
                for i, t in enumerate(src):
                    synth_dev.fill(t, next_seed, i)
                s = rng.choice(streams)
                ev = torch.cuda.Event()
                ev.record()                      # the fills ran on the current stream
                try:
                    h = ctx.swap_out(pl, src, stream=s, after=ev)
                except mp.MPressError as e:
                    assert e.code == mp.ERR_NO_SPACE  # partition full: 3 handles out
                    continue
                # the sources may be dropped once the swap-out is done
                ctx.wait(h, torch.cuda.current_stream())
                del src
                live.append([h, next_seed, None, s])
                next_seed += 1
            elif op < 0.8 and live:
                item = rng.choice([x for x in live if x[2] is None] or [None])
                if item is None:
                    continue
                dst = [torch.full((n,), 0x33, dtype=torch.uint8, device="cuda") for n in sizes]
                s = rng.choice(streams)
                s.wait_stream(torch.cuda.current_stream())   # dst's fill ran there
                ctx.swap_in(item[0], dst, stream=s)
                item[2], item[3] = dst, s
            elif live:
                item = rng.choice(live)
                if item[2] is None:
                    if rng.random() < 0.5:
                        assert ctx.query(item[0]) in (True, False)
                    continue
                ctx.wait(item[0], torch.cuda.current_stream())
                torch.cuda.current_stream().synchronize()
                for i, d in enumerate(item[2]):
                    assert synth_dev.check(d, item[1], i) == 0, (step, item[1], i)
                checked += 1
                item[0].free()
                live.remove(item)
        torch.cuda.synchronize()
        for h, sd, dst, s in live:
            if dst is None:
                dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
                ctx.swap_in(h, dst, stream=s)
            torch.cuda.synchronize()
            for i, d in enumerate(dst):
                assert synth_dev.check(d, sd, i) == 0
            checked += 1
            h.free()
    finally:
        ctx.finalize()
    assert checked >= 10
