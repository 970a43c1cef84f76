#!/usr/bin/env python
"""NEXT-2 on the GPU: replay the exporter stage of a 1F1B pipeline with D2D
swaps hidden behind its compute.

One stage (the exporter, stage e of S) runs on this GPU:
  * F(m) / B(m) = bf16 GEMMs sized like the stage's forward / backward
    (B = 2 x F); the other stages are absent, so every op is gated on
    the device (%globaltimer) to its start in the no-swap 1F1B timeline --
    the bubbles the other stages impose;
  * swap-out of micro-batch m's activations (a Bert stage-0 micro-batch:
    47 tensors, 900 MiB) is enqueued on the swap-out stream after F(m)
    (mpress_swap_out with `after` = F(m)'s event); its swap-in on the swap-in
    stream after the trigger op mpress_schedule_1f1b picked; B(m) waits on
    the swap-in (mpress_wait);
  * the same step is timed without swaps, and every restored tensor is
    checked against the generator.
Loopback peers (1 GPU): the swap's bytes also load the GEMMs' HBM.
Prints one JSON object per configuration.
  python tools/replay_1f1b.py [--stages 8 4 2] [--micro-batches 8] [--scale 1]
"""
import argparse
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


def gemm_op(n, a, b, c):
    def run():
        for _ in range(n):
            torch.matmul(a, b, out=c)
    return run


def timed(fn, stream, reps=5):
    ts = []
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        with torch.cuda.stream(stream):
            fn()
        e1.record(stream)
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts[1:]) * 1e6  # ns


def replay(S, e, M, scale, n_fwd_gemms, max_ctas, seed=7000, slack=0.5, pace_frac=0.0, path="auto:-1"):
    """pace_frac > 0: pace every swap launch (MPRESS_OPT_PACE_MBPS) to take
    pace_frac of the 1F1B period t_f + t_b, and give the scheduler those
    paced swap times.  In the steady state the swap-out stream and the
    swap-in stream each move one micro-batch per period, so the period -- not
    one micro-batch's live interval -- bounds how slow a swap may be
    (round-2 finding: pacing to 0.7 of the shortest live interval made the
    serialised swap-ins miss their backwards)."""
    sizes = [max(16, b // scale) for b in workloads.cfg2_sizes(1)]
    world, peers = 4, [1, 2, 3]
    spare = workloads.spare_vector(world, 0, peers, spare=64 << 30)
    bw = workloads.bw_vector(world, 0, peers)
    pl = mp.plan(world, 0, spare, bw, sizes)
    part = [[0] * world for _ in range(world)]
    part[0] = [M * u * mp.DEFAULT_GRANULE for u in pl.units]
    ctx = mp.Context.local(world, 0, [0] * world, part)
    ctx.set_option(mp.OPT_MAX_CTAS, max_ctas)
    pname, pvar = path.split(":")
    ctx.set_option(mp.OPT_PATH, {"auto": mp.PATH_AUTO, "direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK,
                                 "ce": mp.PATH_CE}[pname])
    if pname in ("direct", "bulk"):
        ctx.set_option(mp.OPT_VARIANT, int(pvar))
    comp = torch.cuda.current_stream()
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    try:
        src = [[torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        dst = [[torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes] for _ in range(M)]
        for m in range(M):
            for i, t in enumerate(src[m]):
                synth_dev.fill(t, seed + m, i)
        T, h = 4096, 1024      # Bert-large stage: 8 x 512 tokens, hidden 1024
        a = torch.randn(T, h, dtype=torch.bfloat16, device="cuda")
        w = torch.randn(h, 4 * h, dtype=torch.bfloat16, device="cuda")
        c = torch.empty(T, 4 * h, dtype=torch.bfloat16, device="cuda")
        fwd = gemm_op(n_fwd_gemms, a, w, c)
        bwd = gemm_op(2 * n_fwd_gemms, a, w, c)
        t_f = int(timed(fwd, comp))
        t_b = int(timed(bwd, comp))

        # swap times of one micro-batch, alone
        outs, ins = [], []
        for _ in range(4):
            e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            e0.record(s_out)
            hh = ctx.swap_out(pl, src[0], stream=s_out)
            e1.record(s_out)
            ctx.swap_in(hh, dst[0], stream=s_out)
            e2.record(s_out)
            torch.cuda.synchronize()
            hh.free()
            outs.append(e0.elapsed_time(e1))
            ins.append(e1.elapsed_time(e2))
        t_out = int(statistics.median(outs[1:]) * 1e6)
        t_in = int(statistics.median(ins[1:]) * 1e6)
        pace_mbps = 0
        if pace_frac > 0:
            # bytes per ns = GB/s; x1000 = MB/s; never slower than 1 GB/s
            pace_mbps = max(1000, int(sum(sizes) / (pace_frac * (t_f + t_b)) * 1000))
            ctx.set_option(mp.OPT_PACE_MBPS, pace_mbps)
            t_paced = int(sum(sizes) / (pace_mbps / 1000))          # ns per paced launch
            t_out, t_in = max(t_out, t_paced), max(t_in, t_paced)

        # swap-ins keep `slack` x t_in of lead: the swap slows down beside the
        # GEMMs (shared HBM in loopback), so the alone-measured t_in is optimistic
        sched, summ = mp.schedule_1f1b(S, e, M, t_f, t_b, t_out, t_in, slack_ns=int(slack * t_in))
        base_sched, _ = mp.schedule_1f1b(S, e, M, t_f, t_b, 0, 0)   # the no-swap timeline
        ops = []
        W = min(S - 1 - e, M)
        ops += [("F", m) for m in range(W)]
        for i in range(M):
            if W + i < M:
                ops.append(("F", W + i))
            ops.append(("B", i))
        start_of = {("F", m): base_sched[m]["fwd_start"] for m in range(M)}
        start_of.update({("B", m): base_sched[m]["bwd_start"] for m in range(M)})
        base = torch.zeros(1, dtype=torch.int64, device="cuda")

        # the native executor issues the swaps: swap-out after F(m),
        # swap-in after its scheduled trigger op, B(m) waits for it
        ex = mp.Executor(ctx, pl, S, e, M, t_f, t_b, t_out, t_in, s_out, s_in,
                         slack_ns=int(slack * t_in))
        assert ex.ops == len(ops)
        src_ptr = [mp.pointers(src[m]) for m in range(M)]
        for m in range(M):
            ex.restore_to(m, dst[m])

        def step(with_swap):
            ev = []
            synth_dev.stamp(base, comp)
            t0 = torch.cuda.Event(enable_timing=True)
            t0.record(comp)
            for j, (kind, m) in enumerate(ops):
                synth_dev.gate(base, start_of[(kind, m)], comp)
                if with_swap:
                    assert ex.before(j, comp) == (kind, m)
                b4 = torch.cuda.Event(enable_timing=True)
                b4.record(comp)
                (fwd if kind == "F" else bwd)()
                x = torch.cuda.Event(enable_timing=True)
                x.record(comp)
                ev.append((b4, x))
                if with_swap:
                    ex.after(j, comp, src_ptr[m] if kind == "F" else None)
            t1 = torch.cuda.Event(enable_timing=True)
            t1.record(comp)
            torch.cuda.synchronize()
            compute = sum(a.elapsed_time(b) for a, b in ev) * 1e6
            return t0.elapsed_time(t1) * 1e6, compute

        step(False)
        step(True)
        runs = [step(False) for _ in range(3)]
        no = statistics.median(r[0] for r in runs)
        comp_no = statistics.median(r[1] for r in runs)
        for m in range(M):
            for t in dst[m]:
                t.zero_()
        runs = [step(True) for _ in range(3)]
        yes = statistics.median(r[0] for r in runs)
        comp_yes = statistics.median(r[1] for r in runs)
        bad = sum(synth_dev.check(t, seed + m, i) for m in range(M) for i, t in enumerate(dst[m]))
        ex.free()
        mb = sum(sizes)
        return {
            "stages": S, "stage": e, "micro_batches": M, "micro_batch_bytes": mb,
            "swap_max_ctas": max_ctas, "swap_path": path, "swap_in_slack": slack, "pace_frac": pace_frac,
            "pace_mbps": pace_mbps,
            "t_fwd_ms": t_f / 1e6, "t_bwd_ms": t_b / 1e6, "t_out_ms": t_out / 1e6, "t_in_ms": t_in / 1e6,
            "schedule_params_ns": {"t_fwd": t_f, "t_bwd": t_b, "t_out": t_out, "t_in": t_in,
                                   "slack": int(slack * t_in)},
            "schedule_slots": sched, "schedule_summary": summ,
            "swap_gbs_alone": 2 * mb / ((t_out + t_in) / 1e9) / 1e9,
            "live_interval_ms": [s["live_ns"] / 1e6 for s in sched],
            "predicted_hidden": sum(s["hidden"] for s in sched),
            "predicted_makespan_ms": summ["makespan_ns"] / 1e6,
            "predicted_makespan_noswap_ms": summ["makespan_noswap_ns"] / 1e6,
            "peak_resident_sets": summ["peak_resident"], "peak_resident_sets_noswap": summ["peak_resident_noswap"],
            "memory_saved_gib": (summ["peak_resident_noswap"] - summ["peak_resident"]) * mb / 2**30,
            "measured_stage_ms_noswap": no / 1e6, "measured_stage_ms_swap": yes / 1e6,
            "measured_overhead": yes / no - 1,
            "compute_ms_noswap": comp_no / 1e6, "compute_ms_swap": comp_yes / 1e6,
            "compute_slowdown": comp_yes / comp_no - 1,
            "restored_bytes_wrong": int(bad),
        }
    finally:
        ctx.finalize()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--stages", type=int, nargs="+", default=[8, 4, 2])
    ap.add_argument("--micro-batches", type=int, default=8)
    ap.add_argument("--scale", type=int, default=1, help="divide the 900 MiB micro-batch by this")
    ap.add_argument("--fwd-gemms", type=int, default=10)
    ap.add_argument("--max-ctas", type=int, default=64)
    ap.add_argument("--slack", type=float, default=0.5, help="swap-in lead, in units of t_in")
    ap.add_argument("--path", nargs="+", default=["auto:-1"],
                    help="swap path:variant settings to replay, e.g. auto:-1 bulk:7 ce:0")
    ap.add_argument("--pace-frac", type=float, nargs="+", default=[0.0],
                    help="0 = unpaced; f > 0 = pace each swap launch to take f x the 1F1B period t_f + t_b")
    args = ap.parse_args()
    for S in args.stages:
        for path in args.path:
            for f in args.pace_frac:
                r = replay(S, 0, args.micro_batches, args.scale, args.fwd_gemms, args.max_ctas,
                           slack=args.slack, pace_frac=f, path=path)
                print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
