#!/usr/bin/env python
"""Tuning sweeps on one B200 (loopback peers): swap GB/s per path x grid cap x
size, and the slowdown of a concurrent bf16 GEMM (the second half of the
BASELINE metric).  Prints one JSON object per row.  Not the bench: bench.py
keeps the driver's contract; this explains it.

  python tools/sweep.py paths        # cfg2 micro-batch, every path x cap
  python tools/sweep.py sizes        # cfg4 sizes 4 KiB .. 4 GiB, 1/3/7 peers
  python tools/sweep.py gemm         # GEMM slowdown vs swap path x cap
  python tools/sweep.py power        # GEMM slowdown vs SM clock and board power
  python tools/sweep.py windows      # GEMM slowdown in the power-capped regime (bench gemm_windows protocol)
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_hpca_zhouwylbyx23_b200 as mp  # noqa: E402
from synth import device as synth_dev  # noqa: E402
from synth import workloads  # noqa: E402

PATHS = {"direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK, "ce": mp.PATH_CE, "auto": mp.PATH_AUTO}


def setup(sizes, peers_n, copies=1):
    world = peers_n + 1
    peers = list(range(1, world))
    spare = workloads.spare_vector(world, 0, peers, spare=64 << 30)
    bw = workloads.bw_vector(world, 0, peers)
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] * world for _ in range(world)]
    part[0] = [copies * u * mp.DEFAULT_GRANULE for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    ctx.set_option(mp.OPT_PDL, int(os.environ.get("SWEEP_PDL", "1")))
    ctx.set_option(mp.OPT_SPLIT, int(os.environ.get("SWEEP_SPLIT", "3")))
    src = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
    for i, t in enumerate(src):
        synth_dev.fill(t, 77, i)
    dst = [torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes]
    return ctx, pl, src, dst


def time_swaps(ctx, pl, src, dst, reps, stream):
    outs, ins = [], []
    for r in range(reps + 2):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(stream)
        h = ctx.swap_out(pl, src, stream=stream)
        e[1].record(stream)
        ctx.swap_in(h, dst, stream=stream)
        e[2].record(stream)
        h.free()
        if r >= 2:
            outs.append(e)
    torch.cuda.synchronize()
    to = [a.elapsed_time(b) for a, b, c in outs]
    ti = [b.elapsed_time(c) for a, b, c in outs]
    return statistics.median(to), statistics.median(ti)


def paths():
    sizes = workloads.cfg2_sizes(1)
    nbytes = sum(sizes)
    ctx, pl, src, dst = setup(sizes, 3)
    s = torch.cuda.Stream()
    nvar = {"direct": 14, "bulk": 9, "ce": 1, "auto": 0}  # plus -1 = auto
    only = os.environ.get("SWEEP_PATHS")        # e.g. "direct"
    var_sel = os.environ.get("SWEEP_VARIANTS")  # e.g. "0,5,6,8"
    cap_sel = os.environ.get("SWEEP_CAPS")      # e.g. "0,148,296"
    for name, path in PATHS.items():
        if only and name not in only.split(","):
            continue
        caps = [0] if name == "ce" else [0, 8, 16, 32, 64, 148, 296, 444, 592]
        if cap_sel and name != "ce":
            caps = [int(x) for x in cap_sel.split(",")]
        variants = ([-1] if name != "ce" else []) + list(range(nvar[name]))
        if var_sel and name != "ce":
            variants = [int(x) for x in var_sel.split(",")]
        for var in variants:
            for cap in caps:
                ctx.set_option(mp.OPT_PATH, path)
                if name != "ce":
                    ctx.set_option(mp.OPT_VARIANT, var)
                ctx.set_option(mp.OPT_MAX_CTAS, cap)
                for order in (mp.ORDER_INTERLEAVE, mp.ORDER_PLAN):
                    ctx.set_option(mp.OPT_ORDER, order)
                    to, ti = time_swaps(ctx, pl, src, dst, 10, s)
                    print(json.dumps({"sweep": "paths", "path": name, "variant": var, "max_ctas": cap,
                                      "order": order, "out_gbs": nbytes / to / 1e6,
                                      "in_gbs": nbytes / ti / 1e6,
                                      "hbm_gbs_out": 2 * nbytes / to / 1e6}), flush=True)
    ctx.finalize()


def sizes_sweep():
    s = torch.cuda.Stream()
    for peers_n in (1, 3, 7):
        for size in workloads.cfg4_sizes():
            ctx, pl, src, dst = setup([size], peers_n, copies=2)
            for name in os.environ.get("SWEEP_SIZE_PATHS", "direct,bulk,ce").split(","):
                ctx.set_option(mp.OPT_PATH, PATHS[name])
                reps = 20 if size < (256 << 20) else 5
                to, ti = time_swaps(ctx, pl, src, dst, reps, s)
                # back to back: R swap pairs enqueued while the GPU is busy, so
                # host enqueue time hides behind the previous pair
                R = 50 if size < (64 << 20) else 4
                torch.cuda.synchronize()
                warm = ctx.swap_out(pl, src, stream=s)   # keeps the GPU busy first
                ctx.swap_in(warm, dst, stream=s)
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(s)
                for _ in range(R):
                    h = ctx.swap_out(pl, src, stream=s)
                    ctx.swap_in(h, dst, stream=s)
                    h.free()
                e1.record(s)
                torch.cuda.synchronize()
                warm.free()
                pair_us = e0.elapsed_time(e1) * 1e3 / R
                # the pair captured once into a CUDA graph, one replay timed
                g = torch.cuda.CUDAGraph()
                with torch.cuda.graph(g, stream=s):
                    gh = ctx.swap_out(pl, src)
                    ctx.swap_in(gh, dst)
                ts = []
                with torch.cuda.stream(s):
                    for r in range(12):
                        e0.record()
                        g.replay()
                        e1.record()
                        torch.cuda.synchronize()
                        if r >= 2:
                            ts.append(e0.elapsed_time(e1) * 1e3)
                del g
                gh.free()
                graph_us = statistics.median(ts)
                print(json.dumps({"sweep": "sizes", "peers": peers_n, "bytes": size, "path": name,
                                  "out_gbs": size / to / 1e6, "in_gbs": size / ti / 1e6,
                                  "out_us": to * 1e3, "in_us": ti * 1e3,
                                  "b2b_pair_us": pair_us,
                                  "b2b_gbs": 2 * size / pair_us / 1e3,
                                  "graph_pair_us": graph_us}), flush=True)
            ctx.finalize()
            del src, dst
            torch.cuda.empty_cache()


def host():
    """NEXT-4: the pinned host pool as the only peer (GPU-CPU swap over PCIe)."""
    s = torch.cuda.Stream()
    for size in (64 << 20, 256 << 20, 1 << 30):
        sizes = [size]
        pl = mp.plan(2, 0, [0, 4 << 30], [0, 1], sizes)
        part = [[0, pl.units[1] * mp.DEFAULT_GRANULE], [0, 0]]
        ctx = mp.Context.local(2, 0, [0, mp.DEVICE_HOST], part)
        src = [torch.empty(size, dtype=torch.uint8, device="cuda")]
        synth_dev.fill(src[0], 5, 0)
        dst = [torch.empty(size, dtype=torch.uint8, device="cuda")]
        torch.cuda.synchronize()
        combos = [("direct", -1, 0), ("direct", -1, 32), ("bulk", -1, 0), ("ce", 0, 0)]
        if os.environ.get("HOST_COMBOS"):      # e.g. "bulk:7:148;direct:9:148"
            combos = [(f[0], int(f[1]), int(f[2])) for f in
                      (x.split(":") for x in os.environ["HOST_COMBOS"].split(";"))]
        for name, var, cap in combos:
            ctx.set_option(mp.OPT_PATH, PATHS[name])
            if name != "ce":
                ctx.set_option(mp.OPT_VARIANT, var)
            ctx.set_option(mp.OPT_MAX_CTAS, cap)
            to, ti = time_swaps(ctx, pl, src, dst, 4, s)
            print(json.dumps({"sweep": "host", "bytes": size, "path": name, "variant": var, "max_ctas": cap,
                              "out_gbs": size / to / 1e6, "in_gbs": size / ti / 1e6}), flush=True)
        ctx.finalize()


def gemm():
    """GEMM slowdown with the bench's protocol: for every (path, variant, cap)
    an alone round and a with-swap round of 24 GEMMs alternate, and only GEMMs
    that ran entirely inside the swap window count."""
    sizes = workloads.cfg2_sizes(1)
    nbytes = sum(sizes)
    ctx, pl, src, dst = setup(sizes, 3)
    shapes = {"8192^3": (8192, 8192, 8192), "gpt_fc1": (4096, 5120, 20480)}
    comp = torch.cuda.current_stream()
    swap = torch.cuda.Stream()
    G = 24
    for sname, (M, K, N) in shapes.items():
        a = torch.randn(M, K, dtype=torch.bfloat16, device="cuda")
        b = torch.randn(K, N, dtype=torch.bfloat16, device="cuda")
        c = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")

        def gemms():
            evs = []
            for _ in range(G):
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(comp)
                torch.matmul(a, b, out=c)
                e1.record(comp)
                evs.append((e0, e1))
            return evs

        gemms()
        torch.cuda.synchronize()
        if os.environ.get("GEMM_COMBOS"):  # e.g. "direct:4:64,96,128;ce:0:0"
            combos = []
            for part in os.environ["GEMM_COMBOS"].split(";"):
                f = part.split(":")     # path:variant:caps[:pace MB/s]
                pace = int(f[3]) if len(f) > 3 else 0
                combos += [(f[0], int(f[1]), int(cap), pace) for cap in f[2].split(",")]
        else:
            combos = [("direct", v, cap, 0) for v in (0, 1, 4) for cap in (16, 32, 64, 96, 148)]
            combos += [("bulk", 0, cap, 0) for cap in (8, 16, 32)] + [("ce", 0, 0, 0)]
        rounds = int(os.environ.get("GEMM_ROUNDS", "2"))
        for name, var, cap, pace in combos:
            ctx.set_option(mp.OPT_PATH, PATHS[name])
            if name != "ce":
                ctx.set_option(mp.OPT_VARIANT, var)
            ctx.set_option(mp.OPT_MAX_CTAS, cap)
            ctx.set_option(mp.OPT_PACE_MBPS, pace)
            to, ti = time_swaps(ctx, pl, src, dst, 3, swap)
            alone, during, gbs, ratios = [], [], [], []
            for _ in range(rounds):
                evs = gemms()
                torch.cuda.synchronize()
                alone += [x.elapsed_time(y) for x, y in evs[4:]]
                n_swap = int(2.0 * G * statistics.median(alone) / (to + ti)) + 2
                s0 = torch.cuda.Event(enable_timing=True)
                s1 = torch.cuda.Event(enable_timing=True)
                s0.record(swap)
                for _ in range(n_swap):
                    h = ctx.swap_out(pl, src, stream=swap)
                    ctx.swap_in(h, dst, stream=swap)
                    h.free()
                s1.record(swap)
                evs = gemms()
                torch.cuda.synchronize()
                win = s0.elapsed_time(s1)
                d_r = [x.elapsed_time(y) for x, y in evs[4:]
                       if s0.elapsed_time(x) >= 0 and s0.elapsed_time(y) <= win]
                during += d_r
                if d_r:
                    ratios.append(statistics.median(d_r) / statistics.median(alone[-(G - 4):]) - 1)
                gbs.append(2 * n_swap * nbytes / win / 1e6)
            am = statistics.median(alone)
            dm = statistics.median(during) if during else float("nan")
            print(json.dumps({"sweep": "gemm", "shape": sname, "path": name, "variant": var,
                              "max_ctas": cap, "pace_mbps": pace, "alone_ms": am, "gemm_ms": dm,
                              "slowdown": dm / am - 1,
                              "slowdown_paired_median": statistics.median(ratios) if ratios else None,
                              "rounds": len(ratios),
                              "counted": len(during), "swap_alone_gbs": 2 * nbytes / (to + ti) / 1e6,
                              "swap_gbs_under_gemm": statistics.median(gbs)}), flush=True)
    ctx.finalize()


def power():
    """Where the concurrent GEMM's slowdown comes from: for each swap setting,
    SECONDS of back-to-back bf16 8192^3 GEMMs with the swap looping beside
    them for the whole window, NVML sampling the SM clock and board power
    every 20 ms; alone windows alternate with the swap windows.  If the GEMM
    loses time in proportion to the SM clock drop, the interference is the
    power cap (moving bytes costs watts), not SMs taken by the swap."""
    import threading
    import time

    import pynvml
    pynvml.nvmlInit()
    nv = pynvml.nvmlDeviceGetHandleByIndex(torch.cuda.current_device())
    seconds = float(os.environ.get("POWER_SECONDS", "3"))
    sizes = workloads.cfg2_sizes(1)
    nbytes = sum(sizes)
    ctx, pl, src, dst = setup(sizes, 3)
    comp = torch.cuda.current_stream()
    swap = torch.cuda.Stream()
    M = 8192
    a = torch.randn(M, M, dtype=torch.bfloat16, device="cuda")
    b = torch.randn(M, M, dtype=torch.bfloat16, device="cuda")
    c = torch.empty(M, M, dtype=torch.bfloat16, device="cuda")

    def sample(stop, out):
        while not stop.is_set():
            out.append((pynvml.nvmlDeviceGetClockInfo(nv, pynvml.NVML_CLOCK_SM),
                        pynvml.nvmlDeviceGetPowerUsage(nv) / 1000.0))
            time.sleep(0.02)

    def window(setting):
        if setting:
            name, var, cap, pace = setting
            ctx.set_option(mp.OPT_PATH, PATHS[name])
            if name != "ce":
                ctx.set_option(mp.OPT_VARIANT, var)
            ctx.set_option(mp.OPT_MAX_CTAS, cap)
            ctx.set_option(mp.OPT_PACE_MBPS, pace)
        per_pair = 0.0
        if setting:   # one pair alone sizes the swap batch that covers 20 GEMMs
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(swap)
            h = ctx.swap_out(pl, src, stream=swap)
            ctx.swap_in(h, dst, stream=swap)
            e1.record(swap)
            h.free()
            torch.cuda.synchronize()
            per_pair = e0.elapsed_time(e1)
        torch.cuda.synchronize()
        stop, smp = threading.Event(), []
        th = threading.Thread(target=sample, args=(stop, smp))
        th.start()
        t0 = time.time()
        n_gemm = n_swap = 0
        gms = sms = 0.0
        while time.time() - t0 < seconds:
            g0 = torch.cuda.Event(enable_timing=True)
            g1 = torch.cuda.Event(enable_timing=True)
            s0 = torch.cuda.Event(enable_timing=True)
            s1 = torch.cuda.Event(enable_timing=True)
            k = 0
            if setting:   # under contention a pair is slower: 1.1x alone-time cover is enough
                k = max(1, int(1.1 * 20 * 0.75 / per_pair) + 1)
                s0.record(swap)
                for _ in range(k):
                    h = ctx.swap_out(pl, src, stream=swap)
                    ctx.swap_in(h, dst, stream=swap)
                    h.free()
                s1.record(swap)
            g0.record(comp)
            for _ in range(20):
                torch.matmul(a, b, out=c)
            g1.record(comp)
            torch.cuda.synchronize()
            n_gemm += 20
            n_swap += k
            gms += g0.elapsed_time(g1)
            if setting:
                sms += s0.elapsed_time(s1)
        stop.set()
        th.join()
        keep = smp[len(smp) // 5:] or smp   # drop the ramp
        row = {"sweep": "power", "setting": "alone" if not setting else "%s var=%d cap=%d pace=%d" % setting,
               "gemm_tflops": 2 * M ** 3 * n_gemm / (gms / 1e3) / 1e12,
               "sm_mhz_median": statistics.median(x for x, _ in keep),
               "power_w_median": statistics.median(w for _, w in keep), "samples": len(keep)}
        if setting:
            row["swap_gbs"] = 2 * n_swap * nbytes / sms / 1e6
            row["swap_busy_over_gemm_busy"] = sms / gms
        print(json.dumps(row), flush=True)
        return row

    window(None)   # warm to the sustained power state
    settings = [("direct", 7, 32, 0), ("direct", 7, 64, 0), ("direct", 9, 64, 0), ("direct", 7, 148, 0),
                ("ce", 0, 0, 0)]
    if os.environ.get("POWER_SETTINGS"):   # e.g. "direct:7:16,32,64;bulk:5:148;direct:9:148:847059;ce:0:0"
        settings = []
        for part in os.environ["POWER_SETTINGS"].split(";"):
            f = part.split(":")
            pace = int(f[3]) if len(f) > 3 else 0
            settings += [(f[0], int(f[1]), int(c), pace) for c in f[2].split(",")]
    for st in settings:
        al = window(None)
        wi = window(st)
        print(json.dumps({"sweep": "power_pair", "setting": wi["setting"],
                          "slowdown": al["gemm_tflops"] / wi["gemm_tflops"] - 1,
                          "sm_clock_ratio": wi["sm_mhz_median"] / al["sm_mhz_median"],
                          "swap_gbs": wi["swap_gbs"]}), flush=True)
    ctx.finalize()


def windows():
    """GEMM slowdown in the power-capped regime (bench.py gemm_windows'
    protocol): per round an alone window of W back-to-back bf16 8192^3 GEMMs,
    then at once a with-swap window of W more beside the looping swap, one
    synchronise per round; per setting `rounds` rounds after a settle.
    WINDOW_COMBOS="direct:9:148:847059;ce:0:0:0" (path:variant:cap:pace)."""
    import random
    sizes = workloads.cfg2_sizes(1)
    nbytes = sum(sizes)
    ctx, pl, src, dst = setup(sizes, 3)
    comp = torch.cuda.current_stream()
    swap = torch.cuda.Stream()
    M = 8192
    W = int(os.environ.get("WINDOW", "200"))
    rounds = int(os.environ.get("WINDOW_ROUNDS", "10"))
    a = torch.randn(M, M, dtype=torch.bfloat16, device="cuda")
    b = torch.randn(M, M, dtype=torch.bfloat16, device="cuda")
    c = torch.empty(M, M, dtype=torch.bfloat16, device="cuda")
    combos = [x.split(":") for x in os.environ.get(
        "WINDOW_COMBOS", "direct:9:148:847059;direct:9:148:600000;direct:7:64:0;ce:0:0:0").split(";")]
    t0 = __import__("time").time()
    while __import__("time").time() - t0 < 3.0:          # settle into the power-capped regime
        for _ in range(W):
            torch.matmul(a, b, out=c)
        torch.cuda.synchronize()
    for name, var, cap, pace in combos:
        ctx.set_option(mp.OPT_PATH, PATHS[name])
        if name != "ce":
            ctx.set_option(mp.OPT_VARIANT, int(var))
        ctx.set_option(mp.OPT_MAX_CTAS, int(cap))
        ctx.set_option(mp.OPT_PACE_MBPS, int(pace))
        to, ti = time_swaps(ctx, pl, src, dst, 3, swap)
        ratios, alone, gbs = [], [], []
        for _ in range(rounds):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(6)]
            ev[0].record(comp)
            for _ in range(W):
                torch.matmul(a, b, out=c)
            ev[1].record(comp)
            gemm_ms = statistics.median(alone) if alone else 0.8
            n_swap = int(1.5 * W * gemm_ms / (to + ti)) + 2
            swap.wait_event(ev[1])
            ev[2].record(swap)
            # a few swaps, then the GEMM window, then the rest: the host must
            # not be still enqueueing swaps (the copy engines take ~3 us of host
            # time per stripe) when the GEMM window should start
            for k in range(n_swap):
                if k == 3:
                    comp.wait_event(ev[2])
                    ev[4].record(comp)
                    for _ in range(W):
                        torch.matmul(a, b, out=c)
                    ev[5].record(comp)
                h = ctx.swap_out(pl, src, stream=swap)
                ctx.swap_in(h, dst, stream=swap)
                h.free()
            ev[3].record(swap)
            torch.cuda.synchronize()
            am = ev[0].elapsed_time(ev[1]) / W
            alone.append(am)
            if ev[5].elapsed_time(ev[3]) >= 0:
                ratios.append(ev[4].elapsed_time(ev[5]) / W / am - 1)
                gbs.append(2 * n_swap * nbytes / ev[2].elapsed_time(ev[3]) / 1e6)
        rng = random.Random(0)
        meds = sorted(statistics.median(rng.choices(ratios, k=len(ratios))) for _ in range(2000)) if ratios else []
        print(json.dumps({"sweep": "windows", "path": name, "variant": int(var), "max_ctas": int(cap),
                          "pace_mbps": int(pace), "window": W, "rounds": len(ratios),
                          "alone_tflops": 2 * M ** 3 / (statistics.median(alone) / 1e3) / 1e12,
                          "slowdown": statistics.median(ratios) if ratios else None,
                          "ci95": [meds[49], meds[1949]] if meds else None,
                          "swap_gbs_during": statistics.median(gbs) if gbs else None,
                          "swap_alone_gbs": 2 * nbytes / (to + ti) / 1e6}), flush=True)
    ctx.finalize()


if __name__ == "__main__":
    what = sys.argv[1] if len(sys.argv) > 1 else "paths"
    {"paths": paths, "sizes": sizes_sweep, "gemm": gemm, "host": host, "power": power, "windows": windows}[what]()
