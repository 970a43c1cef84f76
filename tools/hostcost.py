#!/usr/bin/env python
"""Host-side cost of one swap pair (swap_out + swap_in + handle free) for a
small batch: through the Python binding, and through raw ctypes calls with
prebuilt argument arrays (the C ABI's own cost).  The GPU is kept busy by a
long kernel first so host time, not GPU time, is measured."""
import ctypes
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_hpca_zhouwylbyx23_b200 as mp  # noqa: E402
from paper_conf_hpca_zhouwylbyx23_b200 import api  # noqa: E402
from synth import device as synth_dev  # noqa: E402


def main():
    n_tensors = int(sys.argv[1]) if len(sys.argv) > 1 else 4
    pdl = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    sizes = [4096] * n_tensors
    world = 4
    spare = [0, 1 << 30, 1 << 30, 1 << 30]
    bw = [0, 1, 1, 1]
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] * world for _ in range(world)]
    part[0] = [64 * u * mp.DEFAULT_GRANULE for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    ctx.set_option(mp.OPT_PDL, pdl)
    src = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
    dst = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
    s = torch.cuda.Stream()
    base = torch.zeros(1, dtype=torch.int64, device="cuda")
    res = {}
    # stays below the stream's queue depth (the host would block); large
    # descriptor tables (28 KB of kernel parameters) fill the launch queue sooner
    R = int(sys.argv[3]) if len(sys.argv) > 3 else 150
    for mode in ("python", "ctypes"):
        synth_dev.stamp(base, s)
        synth_dev.gate(base, 2_000_000_000, s)     # ~2 s of GPU work queued first
        ptr_s = (ctypes.c_void_p * n_tensors)(*[t.data_ptr() for t in src])
        ptr_d = (ctypes.c_void_p * n_tensors)(*[t.data_ptr() for t in dst])
        st = ctypes.c_void_p(s.cuda_stream)
        h = ctypes.c_void_p()
        t0 = time.perf_counter()
        for _ in range(R):
            if mode == "python":
                hh = ctx.swap_out(pl, src, stream=s)
                ctx.swap_in(hh, dst, stream=s)
                hh.free()
            else:
                api.lib.mpress_swap_out(ctx._h, pl.handle, ptr_s, st, None, ctypes.byref(h))
                api.lib.mpress_swap_in(ctx._h, h, ptr_d, st)
                api.lib.mpress_handle_free(ctx._h, h, 0)
        res[mode + "_us_per_pair"] = (time.perf_counter() - t0) / R * 1e6
        torch.cuda.synchronize()
    res["n_tensors"] = n_tensors
    res["stripes"] = len(pl.stripes)
    res["pdl"] = pdl
    print(json.dumps(res))
    ctx.finalize()


if __name__ == "__main__":
    main()
