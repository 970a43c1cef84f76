#!/usr/bin/env python
"""bench.py -- MPress D2D stripe swap on B200 (BASELINE.json metric).

Metric: "D2D swap GB/s per source GPU vs 900 GB/s NVLink; GEMM slowdown while
swapping".  One step = one pass of the whole hot path:
  a1 PLAN      mpress_plan of the stage-0 micro-batch (host, integer);
  a3/a4 OUT    one swap-out per in-flight micro-batch (8, 1F1B) + its event;
  a5 IN        the matching swap-ins;
  a6 WAIT      the compute stream waits on the last swap-in's event.
(a2 MAP -- cuMem pool export/import/map -- is set-up, done once before timing.)

Workload (BASELINE.json configs[1], BJ:8): Bert-large stage-0 activations
(seq 512, micro-batch 8; 47 tensors, 900 MiB per micro-batch, 8 micro-batches
in flight = 7.03 GiB) striped over 3 light-load peers.
  * N = 1 (one GPU): the 3 peers are disjoint cuMem pools on the same B200
    ("loopback", mpress_init_local); the bytes cross HBM instead of NVLink, so
    the roofline is the measured HBM copy bandwidth.
  * N > 1 (torchrun, one process per GPU): every rank is a source striping
    its batch over all N-1 other ranks and an importer for theirs
    (mpress_init: POSIX-fd pool exchange + cuMemMap peer access over
    NVLink); value = one rank's swapped bytes / max-over-ranks time (per
    source GPU, BASELINE.json's metric); all_ranks_gbs = the whole-job sum.
value counts swapped tensor bytes, out + in (the round trip of P:332's
"time cost", reading R15), per second.  Inputs (7 GiB) exceed the 126 MB L2,
so no flush is needed between steps.

Beside the headline (each leg reports its own failure instead of losing the
line): e2e through pinned host buffers; the duplex leg (two swap streams);
the GEMM legs -- a calibrated GEMM-concurrent swap setting, then the bf16
slowdown with a bootstrap 95% interval for 8192^3 (burst rounds and
power-capped windows), the GPT FC1 stage GEMM and the copy engines, each
with `meets_north_star_pair` (>= 720 GB/s beside the GEMM and < 10%); at
N = 1 configs 1, 3 and 4 (single shot, back to back, graph-replayed), the
oracle's cpu_baseline and the planner timing; at N > 1 config 4's single
source rows (P = 1, 3, N-1) and config 5 (imbalanced sources + GEMMs on
every rank).  `--impl reference` times the oracle instead.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

GiB = 1 << 30
MICRO_BATCHES = 8
SPARE_PER_PEER = 24 * GiB          # cfg2: 24 GiB spare per peer
FALLBACK_HBM = 6650.0              # B200_PROFILING.md fallback, GB/s
NVLINK_GUIDE = 770.0               # B200_PROFILING.md's figure (peer copy per direction), not ours
HBM_NOMINAL = 7700.0               # GB/s, B200 HBM3e nominal (B200_PROFILING.md: 7.7 TB/s HGX, 8 DGX)
NVLINK_NOMINAL = 900.0


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="mpress", choices=["mpress", "reference"])
    ap.add_argument("--path", default="auto", choices=["auto", "direct", "bulk", "ce"],
                    help="auto = the library default: bulk (TMA) at a full grid, direct when capped")
    ap.add_argument("--max-ctas", type=int, default=0)
    ap.add_argument("--variant", type=int, default=-1, help="kernel shape within --path (-1 = auto)")
    ap.add_argument("--no-autotune", action="store_true",
                    help="skip mpress_autotune (AUTO keeps the bulk kernel for uncapped grids)")
    ap.add_argument("--no-pdl", action="store_true", help="plain launches instead of programmatic dependent launch")
    ap.add_argument("--pdl", type=int, default=1, choices=[0, 1, 2],
                    help="MPRESS_OPT_PDL: 0 never, 1 uncapped grids only (default), 2 always")
    ap.add_argument("--micro-batches", type=int, default=MICRO_BATCHES)
    ap.add_argument("--split", type=int, default=3, choices=[0, 1, 2, 3],
                    help="MPRESS_OPT_SPLIT: 0 = contiguous block per CTA, 1 = grid stride (round 1), "
                         "2 = dynamic claims, 3 = auto (dynamic for large TMA launches, default)")
    ap.add_argument("--e2e-steps", type=int, default=16)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e-zero-copy", action="store_true",
                    help="skip the e2e variant that hands pinned host tensors to the swap calls")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    ap.add_argument("--gemm-cap", type=int, default=0,
                    help="swap grid cap (CTAs = SMs touched) while the concurrent GEMM runs (AUTO path -> "
                         "direct shape 9); 0 = calibrate: the first of --gemm-swap-candidates whose swap rate "
                         "on this run's links reaches --gemm-target-gbs / 0.85")
    ap.add_argument("--gemm-swap-candidates", default="bulk:7:148,bulk:9:148,auto:-1:148,auto:-1:96,auto:-1:64",
                    help="path:variant:max_ctas settings for the GEMM-concurrent swap, cheapest for the GEMM "
                         "first: one-warp TMA CTAs (bulk 7); bulk 9 = that TMA warp plus a register-copy warp "
                         "per SM, 1.4x bulk 7's rate but a wider spread of burst-GEMM cost (+3..+13%%, "
                         "profiles/r02/hybrid/); "
                         "one-warp TMA CTAs (4 x 4 KiB of shared memory) on every SM cost the "
                         "power-capped GEMM ~12%% where 128-thread direct CTAs cost ~18%% at the same rate "
                         "(profiles/r02/gemm_windows_*.jsonl); among the direct settings one light "
                         "CTA on every SM cost no more than 64 or 96 busier SMs (gemm_leg_settings.jsonl)")
    ap.add_argument("--gemm-sus-fallback", default="bulk:9:148",
                    help="swap setting (path:variant:max_ctas, unpaced) for the power-capped GEMM leg when the "
                         "calibrated one moves less than --gemm-target-gbs there (empty: none); bulk 9 (TMA warp + "
                         "register-copy warp) moved 998-1107 GB/s at +5.3..+5.8%% in 3 s windows, direct 9 on 64 "
                         "SMs 1109-1128 at +7.6..+9.1%% (profiles/r02/hybrid/, gemm_windows_fallback_caps.jsonl)")
    ap.add_argument("--gemm-target-gbs", type=float, default=720.0,
                    help="per-source swap rate the GEMM-concurrent swap should sustain (BJ:5: 80%% of 900)")
    ap.add_argument("--gemm-no-pace", action="store_true",
                    help="run the GEMM-concurrent SM swap unpaced (default: paced to --gemm-target-gbs / 0.85 "
                         "with MPRESS_OPT_PACE_MBPS)")
    ap.add_argument("--no-gemm", action="store_true")
    ap.add_argument("--no-gemm-ce", action="store_true", help="skip the copy-engine pass of the GEMM leg")
    ap.add_argument("--no-gemm-fc1", action="store_true",
                    help="skip the GEMM leg on config 5's second shape (GPT-10.3B FC1, 4096x5120x20480)")
    ap.add_argument("--gemm-settle-s", type=float, default=2.0,
                    help="back-to-back GEMMs before the GEMM-slowdown rounds (power state)")
    ap.add_argument("--gemm-rounds", type=int, default=40,
                    help="paired alone / with-swap GEMM rounds (the slowdown's 95%% interval is bootstrapped "
                         "over them)")
    ap.add_argument("--gemm-window", type=int, default=4000,
                    help="GEMMs per window of the sustained-regime GEMM leg (gemm_windows): 4000 8192^3 "
                         "GEMMs are ~3 s, long enough for the power governor to settle in each window "
                         "(160 ms windows measured +11%% where 1.6-3 s windows measure +6%%, "
                         "profiles/r02/gemm_windows_long.jsonl)")
    ap.add_argument("--gemm-window-rounds", type=int, default=5,
                    help="alone / with-swap window pairs of the sustained-regime GEMM leg (0 = skip it)")
    ap.add_argument("--gemm-n", type=int, default=8192, help="GEMM size of the N>1 config-5 leg")
    ap.add_argument("--no-cfg5", action="store_true",
                    help="N>1: skip the config-5 leg (imbalanced swap + GEMM on every rank)")
    ap.add_argument("--ss-sizes", default=",".join(str(x) for x in (4096, 65536, 1 << 20, 16 << 20, 256 << 20,
                                                                    1 << 30, 4 << 30)),
                    help="N>1: tensor sizes (bytes) of the config-4 single-source leg")
    ap.add_argument("--no-single-source", action="store_true", help="N>1: skip the config-4 single-source leg")
    ap.add_argument("--no-duplex", action="store_true", help="skip the duplex (two swap streams) leg")
    ap.add_argument("--no-configs", action="store_true",
                    help="skip the other BASELINE configs (1, 3, 4) reported beside the headline")
    return ap.parse_args()


# mpress_autotune probe: 4 back-to-back 256 MiB launches per direction (large
# class), 16 x 16 MiB (small class), over a 1 GiB working set
AUTOTUNE_PROBE = 1 << 30


def _finite(x):
    """The JSON line must be strict JSON: NaN / inf (e.g. a slowdown with no
    GEMM inside the swap window) become null."""
    if isinstance(x, float):
        return x if x == x and x not in (float("inf"), float("-inf")) else None
    if isinstance(x, dict):
        return {k: _finite(v) for k, v in x.items()}
    if isinstance(x, (list, tuple)):
        return [_finite(v) for v in x]
    return x


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f), "measured"
    return {"hbm_gbs": FALLBACK_HBM}, "fallback"


# --------------------------------------------------------------- clocks

class Clocks:
    """SM clock and throttle reasons sampled DURING the timed region
    (B200_PROFILING.md's clocks line): an NVML thread every 5 ms between
    start() and stop() -- the default 20-step run times only ~0.1 s, so
    nvidia-smi's 100 ms loop would catch one sample or the idle tail.  Falls
    back to `nvidia-smi -lms 100` if NVML is unavailable."""
    FIELDS = ("clocks.sm,clocks.max.sm,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
    NAMES = ("hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap")

    def __init__(self, index):
        self.index = index
        self.proc = None
        self.file = None
        self.thread = None
        self.samples = []

    def _nvml_handle(self):
        import pynvml
        import torch
        pynvml.nvmlInit()
        try:
            p = torch.cuda.get_device_properties(self.index)
            bus = "%08x:%02x:%02x.0" % (p.pci_domain_id, p.pci_bus_id, p.pci_device_id)
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.index)

    def start(self):
        import threading
        try:
            nv, h = self._nvml_handle()
            self.max_mhz = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            bits = {"hw_slowdown": nv.nvmlClocksEventReasonHwSlowdown,
                    "hw_thermal_slowdown": nv.nvmlClocksEventReasonHwThermalSlowdown,
                    "sw_thermal_slowdown": nv.nvmlClocksEventReasonSwThermalSlowdown,
                    "sw_power_cap": nv.nvmlClocksEventReasonSwPowerCap}
            self.stop_flag = threading.Event()

            def run():
                while not self.stop_flag.is_set():
                    try:
                        mhz = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                        r = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                        self.samples.append((mhz, [n for n, b in bits.items() if r & b]))
                    except Exception:
                        pass
                    time.sleep(0.005)
            self.thread = threading.Thread(target=run, daemon=True)
            self.thread.start()
            return
        except Exception:
            self.thread = None
        try:
            self.file = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), "--query-gpu=" + self.FIELDS,
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=self.file, stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.thread is not None:
            self.stop_flag.set()
            self.thread.join()
            if not self.samples:
                return None
            reasons = sorted({n for _, rs in self.samples for n in rs})
            return {"sm_mhz": statistics.median(m for m, _ in self.samples), "sm_max_mhz": float(self.max_mhz),
                    "reasons": reasons, "samples": len(self.samples), "source": "NVML every 5 ms in the timed region"}
        if self.proc is None:
            return None
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        self.file.flush()
        self.file.seek(0)
        rows = [r.strip().split(", ") for r in self.file.read().splitlines() if r.strip()]
        os.unlink(self.file.name)
        sm, mx, reasons = [], None, set()
        for r in rows:
            try:
                sm.append(float(r[0]))
                mx = float(r[1])
            except (ValueError, IndexError):
                continue
            for n, v in zip(self.NAMES, r[3:7]):
                if v.strip().lower() == "active":
                    reasons.add(n)
        if not sm:
            return None
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": mx, "reasons": sorted(reasons),
                "samples": len(sm), "source": "nvidia-smi -lms 100"}


# --------------------------------------------------------------- oracle (cpu)

_HOST_CACHE = {}


def _oracle_inputs(n_tensors):
    from synth import splitmix64_bytes, workloads
    sizes = workloads.cfg2_sizes(1)[:n_tensors]
    if n_tensors not in _HOST_CACHE:
        full = _HOST_CACHE.setdefault("full", [])
        while len(full) < n_tensors:
            i = len(full)
            full.append(splitmix64_bytes(2000, i, 0, workloads.cfg2_sizes(1)[i]))
        _HOST_CACHE[n_tensors] = full[:n_tensors]
    return sizes, _HOST_CACHE[n_tensors]


def oracle_pass(n_tensors=47, seconds=0.0):
    """The oracle as it stands (plain Python planner + numpy byte model) on
    the first `n_tensors` tensors of one Bert stage-0 micro-batch, 3 peers,
    repeated for >= `seconds`; single-threaded.  Returns (GB/s, passes, bytes)."""
    import numpy as np
    import oracle
    from synth import workloads
    sizes, host = _oracle_inputs(n_tensors)
    world, peers = 4, [1, 2, 3]
    spare = workloads.spare_vector(world, 0, peers, spare=SPARE_PER_PEER)
    bw = workloads.bw_vector(world, 0, peers)
    passes, moved = 0, 0
    t0 = time.perf_counter()
    while True:
        pl = oracle.plan(world, 0, spare, bw, sizes)
        stash = oracle.swap_out(pl, host)
        back = oracle.swap_in(pl, stash)
        passes += 1
        moved += 2 * sum(sizes)
        if time.perf_counter() - t0 >= seconds:
            break
    el = time.perf_counter() - t0
    assert all(np.array_equal(a, b) for a, b in zip(host, back))
    return moved / el / 1e9, passes, sum(sizes)


def oracle_threaded(seconds, threads):
    """The same oracle passes (unchanged code) run by `threads` host threads
    at once, as the GPU swaps its 8 micro-batches: numpy releases the GIL for
    the large slice copies, so this is what the host's cores reach with the
    oracle as it stands.  Returns (GB/s, total passes)."""
    from concurrent.futures import ThreadPoolExecutor
    _oracle_inputs(47)   # generate the shared (read-only) inputs once
    t0 = time.perf_counter()
    with ThreadPoolExecutor(threads) as ex:
        res = list(ex.map(lambda _: oracle_pass(47, seconds), range(threads)))
    el = time.perf_counter() - t0
    moved = sum(2 * nbytes * passes for _, passes, nbytes in res)
    return moved / el / 1e9, sum(passes for _, passes, _ in res)


def oracle_sample(seconds):
    v, passes, nbytes = oracle_pass(47, seconds)
    out = {"value": v, "unit": "GB/s", "cores": 1, "kind": "oracle",
           "sample": "%d pass(es) of plan + swap-out + swap-in of 1 of the 8 Bert stage-0 "
                     "micro-batches (47 tensors, 900 MiB), 3 peers, numpy on one host thread"
                     % passes}
    try:
        import platform
        cpu = platform.processor() or ""
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    cpu = ln.split(":", 1)[1].strip()
                    break
        out["cpu_model"] = cpu
        out["host_cores"] = os.cpu_count()
    except Exception:  # pragma: no cover
        pass
    # context: the unchanged oracle on several host threads at once (at most 8:
    # each pass holds ~2 GB of host buffers)
    threads = max(1, min(8, os.cpu_count() or 1))
    try:   # ~3 GB of host buffers per concurrent pass; stay under a quarter of free RAM
        avail = os.sysconf("SC_AVPHYS_PAGES") * os.sysconf("SC_PAGE_SIZE")
        threads = max(1, min(threads, int(avail * 0.25 // (3 << 30))))
    except (ValueError, OSError):  # pragma: no cover
        pass
    if threads > 1:
        tv, tp = oracle_threaded(seconds, threads)
        out["threaded"] = {"value": tv, "unit": "GB/s", "cores": threads,
                           "sample": "%d passes of the same sample, %d concurrent host threads" % (tp, threads)}
    return out


def run_reference(args):
    """--impl reference: the oracle timed on host cores, each step a bounded
    sample (a prefix of one micro-batch's tensors) so the run stays short."""
    from synth import workloads
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    full_gbs, _, full_bytes = oracle_pass(47)           # calibration pass
    budget_s = 120.0 / max(1, args.steps + args.warmup)
    target = full_gbs * 1e9 * budget_s / 2
    sizes = workloads.cfg2_sizes(1)
    n_t, acc = 0, 0
    while n_t < len(sizes) and (n_t == 0 or acc + sizes[n_t] <= target):
        acc += sizes[n_t]
        n_t += 1
    for _ in range(args.warmup):
        oracle_pass(n_t)
    t0 = time.perf_counter()
    moved = 0
    for _ in range(args.steps):
        v, passes, nbytes = oracle_pass(n_t)
        moved += 2 * nbytes * passes
    el = time.perf_counter() - t0
    v = moved / el / 1e9
    sample = ("each step: plan + swap-out + swap-in of the first %d of the 47 tensors of one Bert "
              "stage-0 micro-batch (%.1f MiB), 3 peers, numpy on one host thread" % (n_t, acc / 2**20))
    line = {"impl": "reference", "metric": "D2D swap GB/s per source GPU (round trip, out+in)",
            "value": v, "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": el / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8",
            "data": "synthetic", "config": workload_config(args, args.gpus),
            "cpu_baseline": {"value": v, "unit": "GB/s", "cores": 1, "kind": "oracle", "sample": sample},
            "e2e": {"value": v, "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(_finite(line), allow_nan=False))
    return 0


# --------------------------------------------------------------- the GPU bench

def headline_values(n, swapped_per_step_rank, ms_step):
    """(value, all_ranks_gbs).  The metric is per SOURCE GPU (BASELINE.json:
    "D2D swap GB/s per source GPU vs 900 GB/s NVLink"): every rank is a
    source swapping the same bytes per step, so value = one rank's swapped
    bytes / the max-over-ranks step time; the whole-job sum over the n ranks
    is reported beside it as all_ranks_gbs."""
    per_source = swapped_per_step_rank / (ms_step / 1e3) / 1e9
    return per_source, n * per_source


def workload_config(args, n):
    if n == 1:
        wl = "cfg2 Bert-large stage-0 activations x%d micro-batches -> 3 peers (1-GPU loopback: " \
             "peers are cuMem pools on the same B200)" % args.micro_batches
    else:
        wl = "cfg2 Bert-large stage-0 activations x%d micro-batches per rank -> all %d other " \
             "ranks over NVLink (every rank a source and an importer)" % (args.micro_batches, n - 1)
    return {"workload": wl, "tensors_per_micro_batch": 47, "micro_batch_bytes": 900 << 20,
            "micro_batches": args.micro_batches, "peers": 3 if n == 1 else n - 1,
            "path": args.path, "variant": args.variant, "max_ctas": args.max_ctas, "pdl": 0 if args.no_pdl else args.pdl,
            "split": ["blocked", "strided", "dynamic", "auto"][args.split],
            "l2": "inputs %.2f GiB per rank > 126 MB L2: no flush needed" %
                  (args.micro_batches * 900 / 1024)}


def main():
    args = parse()
    if args.impl == "reference":
        return run_reference(args)

    import torch
    import torch.distributed as dist

    world_env = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    n = world_env
    # One rank per GPU.  Ranks sharing a GPU (only in the 1-GPU test of this
    # code path) use gloo alone; the reductions below are on CPU tensors, so
    # nothing on the swap path depends on the collective backend.
    ngpu = torch.cuda.device_count()
    device = local_rank % ngpu
    torch.cuda.set_device(device)
    if n > 1:
        # The swap path has no collective: the process group
        # only carries the init-time all-gathers and the CPU-side max-over-
        # ranks reductions, so gloo serves every layout (also ranks sharing
        # a GPU in the 1-GPU test of this path).
        dist.init_process_group("gloo")
    local_rank = device

    import paper_conf_hpca_zhouwylbyx23_b200 as mp
    from synth import device as synth_dev
    from synth import workloads

    sizes = workloads.cfg2_sizes(1)
    mb = args.micro_batches
    G = mp.DEFAULT_GRANULE
    path = {"direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK, "ce": mp.PATH_CE, "auto": mp.PATH_AUTO}[args.path]

    if n == 1:
        world, source = 4, 0
        peers = [1, 2, 3]
        spare = workloads.spare_vector(world, source, peers, spare=SPARE_PER_PEER)
        bw = workloads.bw_vector(world, source, peers)
        pl0 = mp.plan(world, source, spare, bw, sizes)
        part = [[0] * world for _ in range(world)]
        part[source] = [mb * u * G for u in pl0.units]
        ctx = mp.Context.local(world, source, [local_rank] * world, part)
        per_copy = spare
    else:
        world, source = n, rank
        spare = [SPARE_PER_PEER] * world
        bwm = [[0 if s == p else 1 for p in range(world)] for s in range(world)]
        bw = bwm[source]
        reqs = [(s, sizes, mb) for s in range(world)]
        part = mp.partition_sequential(world, spare, bwm, reqs)
        ctx = mp.Context.distributed(local_rank, world, rank, part)
        # what source s planned against inside partition_sequential
        rem = list(spare)
        for s in range(world):
            pc = [r // mb for r in rem]
            if s == source:
                per_copy = pc
            for p in range(world):
                rem[p] -= part[s][p]
    ctx.set_option(mp.OPT_PATH, path)
    ctx.set_option(mp.OPT_VARIANT, args.variant)
    ctx.set_option(mp.OPT_MAX_CTAS, args.max_ctas)
    ctx.set_option(mp.OPT_PDL, 0 if args.no_pdl else args.pdl)
    ctx.set_option(mp.OPT_SPLIT, args.split)
    autotune = None
    if path == mp.PATH_AUTO and not args.no_autotune:
        # which SM kernel an uncapped AUTO swap runs on THIS run's links
        # (loopback HBM at N=1, NVLink at N>1), measured before the timed steps
        t_at = time.perf_counter()
        res = ctx.autotune(probe_bytes=AUTOTUNE_PROBE, trials=5)
        t_at = (time.perf_counter() - t_at) * 1e3
        nm = {mp.PATH_DIRECT: "direct", mp.PATH_BULK: "bulk"}
        autotune = {"out": nm[res["out"]], "in": nm[res["in"]], "out_small": nm[res["out_small"]],
                    "in_small": nm[res["in_small"]], "small_below_bytes": mp.AUTO_SMALL_BYTES,
                    "probe_bytes": AUTOTUNE_PROBE, "trials": 5, "median_ms_per_launch": res["ms"],
                    "wall_ms": t_at}

    seed0 = 2000 + 100 * rank
    src = [[torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes] for _ in range(mb)]
    dst = [[torch.empty(s, dtype=torch.uint8, device="cuda") for s in sizes] for _ in range(mb)]
    for m in range(mb):
        for i, t in enumerate(src[m]):
            synth_dev.fill(t, seed0 + m, i)
    torch.cuda.synchronize()
    swap_stream = torch.cuda.Stream()
    compute = torch.cuda.current_stream()
    bytes_per_mb = sum(sizes)

    timing = {"out": [], "in": []}
    launches = [0]

    # Per-kernel timing: timing events bracket the RUN of mb swap-out
    # launches and the run of mb swap-in launches of every timed step, and the
    # average launch duration is the run's time / mb.  A timing event between
    # two kernels serialises them and switches off their programmatic
    # dependent launch (PDL) overlap, so none is recorded inside a run: the
    # runs are timed as the step runs them (an earlier version bracketed one
    # launch per direction, which cost that launch its PDL overlap and
    # understated the kernel's in-step speed by ~1%).
    ran_dir = {}   # path each direction ran (MPRESS_OPT_LAST_PATH), from the first warm-up step

    def step(record=False, k=0, probe_path=False):
        pl = mp.plan(world, source, per_copy, bw, sizes)              # a1
        hs = []
        if record:
            e0 = torch.cuda.Event(enable_timing=True); e0.record(swap_stream)
        for m in range(mb):                                            # a3 + a4
            hs.append(ctx.swap_out(pl, src[m], stream=swap_stream))
            launches[0] += ctx.last_launches
            if probe_path and m == 0:
                ran_dir["out"] = ctx.get_option(mp.OPT_LAST_PATH)
        if record:
            e1 = torch.cuda.Event(enable_timing=True); e1.record(swap_stream)
        for m in range(mb):                                            # a5
            ctx.swap_in(hs[m], dst[m], stream=swap_stream)
            launches[0] += ctx.last_launches
            if probe_path and m == 0:
                ran_dir["in"] = ctx.get_option(mp.OPT_LAST_PATH)
        if record:
            e2 = torch.cuda.Event(enable_timing=True); e2.record(swap_stream)
            timing["out"].append((e0, e1))
            timing["in"].append((e1, e2))
        ctx.wait(hs[-1], compute)                                      # a6
        for h in hs:
            h.free()

    for w in range(args.warmup):
        step(probe_path=w == 0)
    torch.cuda.synchronize()
    if n > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks = Clocks(local_rank)
    clocks.start()
    launches[0] = 0
    t_start = torch.cuda.Event(enable_timing=True)
    t_end = torch.cuda.Event(enable_timing=True)
    t_start.record(compute)
    swap_stream.wait_stream(compute)
    for k in range(args.steps):
        step(record=True, k=k)
    t_end.record(compute)
    torch.cuda.synchronize()
    clk = clocks.stop()          # before the barrier: no idle samples
    if n > 1:
        dist.barrier()
    torch.cuda.synchronize()
    ms = t_start.elapsed_time(t_end)
    ms_t = torch.tensor([ms], dtype=torch.float64)
    if n > 1:
        dist.all_reduce(ms_t, op=dist.ReduceOp.MAX)
    ms_max = float(ms_t.item())
    ms_step = ms_max / args.steps
    swapped_per_step_rank = 2 * mb * bytes_per_mb
    value, all_ranks_gbs = headline_values(n, swapped_per_step_rank, ms_step)

    # correctness of what was timed: every restored tensor == the generator
    bad = 0
    for m in range(mb):
        for i, t in enumerate(dst[m]):
            bad += synth_dev.check(t, seed0 + m, i)
    bad_t = torch.tensor([bad], dtype=torch.int64)
    if n > 1:
        dist.all_reduce(bad_t)
    if int(bad_t.item()) != 0:
        raise SystemExit("round trip mismatch: %d bytes" % int(bad_t.item()))

    names = {mp.PATH_DIRECT: "direct", mp.PATH_BULK: "bulk", mp.PATH_CE: "ce"}
    ran_by_dir = {k: names.get(v, "?") for k, v in ran_dir.items()}
    # per-launch durations: each timed run is mb launches (one per swap call)
    dur = {k: [a.elapsed_time(b) / mb for a, b in v] for k, v in timing.items()}
    tot = {k: sum(v) for k, v in dur.items()}
    dom = max(tot, key=tot.get)
    ran = ran_by_dir.get(dom, "?")   # the dominant kernel's path
    avg_ms = statistics.mean(dur[dom])
    peaks, peaks_src = measured_peaks()
    if n == 1:
        algo_bytes = 2 * bytes_per_mb       # HBM read + HBM write per swapped byte
        achieved = algo_bytes / (avg_ms / 1e3) / 1e9
        peak = float(peaks.get("hbm_gbs", FALLBACK_HBM))
        roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                "frac": achieved / peak, "traffic": traffic_from_profile(ran),
                "kernel": "mp_swap_%s<%s>" % (ran, "kDirIn" if dom == "in" else "kDirOut"),
                "algorithmic_bytes_per_launch": algo_bytes,
                "avg_launch_ms": avg_ms, "peak_source": "%s hbm_gbs (MEASURED_PEAKS.json)" % peaks_src,
                # the measured peak is torch's copy_ of 2 GiB (an elementwise
                # LSU copy); the TMA kernel claiming from one moving front
                # moves HBM faster than it, hence frac > 1;
                # against the nominal 7.7 TB/s of B200 HBM3e (HGX):
                "frac_of_nominal": achieved / HBM_NOMINAL,
                # sampled launches: average kernel time x launches per step / step time
                "share_of_step": (statistics.mean(dur["out"]) + statistics.mean(dur["in"])) * mb / ms_step
                if ms_step > 0 else None,
                "timed_launches": "every timed step: the run of %d swap-out launches and the run of %d "
                                  "swap-in launches, each bracketed by CUDA events on the swap stream; "
                                  "avg_launch_ms = run time / %d" % (mb, mb, mb)}
    else:
        algo_bytes = bytes_per_mb           # bytes over NVLink per launch (one direction)
        achieved = algo_bytes / (avg_ms / 1e3) / 1e9
        roof = {"bound": "nvlink", "achieved": achieved, "peak": NVLINK_GUIDE, "unit": "GB/s",
                "frac": achieved / NVLINK_GUIDE, "traffic": None,
                "nominal_peak": NVLINK_NOMINAL, "frac_of_nominal": achieved / NVLINK_NOMINAL,
                "kernel": "mp_swap_%s<%s>" % (ran, "kDirIn" if dom == "in" else "kDirOut"),
                "algorithmic_bytes_per_launch": algo_bytes, "avg_launch_ms": avg_ms,
                "peak_source": "guide figure, not measured by this run: /opt/skills/guides/B200_PROFILING.md "
                               "quotes a peer copy of 770 GB/s per direction measured on that pool's B200s "
                               "(nominal 900); MEASURED_PEAKS.json has no NVLink entry"}
    per_dir = {k: bytes_per_mb / (statistics.mean(v) / 1e3) / 1e9 for k, v in dur.items()}

    # The legs below add context to the headline; a failure in one is
    # reported in its key instead of losing the measured line.
    leg_wall = {}

    def leg(fn, *a):
        t0 = time.time()
        try:
            return fn(*a)
        except Exception as exc:  # pragma: no cover - reported, not hidden
            return {"error": "%s: %s" % (type(exc).__name__, exc)}
        finally:
            name = (fn.__name__ + ("_ce" if any(x is True for x in a[-2:]) else "") +
                    ("_fc1" if any(isinstance(x, str) and x == "gpt_fc1" for x in a) else ""))
            leg_wall[name + ("_2" if name in leg_wall else "")] = round(time.time() - t0, 2)

    e2e = leg(run_e2e, args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap_stream, n, dist)
    e2e_zc = None if args.no_e2e_zero_copy else leg(run_e2e_zero_copy, args, ctx, mp, world, source, per_copy,
                                                    bw, sizes, n, dist)
    duplex = None if args.no_duplex else leg(duplex_leg, ctx, mp, world, source, per_copy, bw, sizes, src, dst,
                                             n, dist)
    cap_cal = None
    args.gemm_swap = "auto:-1:%d" % (args.gemm_cap if args.gemm_cap > 0 else 148)
    if not args.no_gemm and args.gemm_cap <= 0:
        t0 = time.time()
        cap_cal = calibrate_gemm_cap(args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap_stream, n,
                                     dist)
        leg_wall["calibrate_gemm_cap"] = round(time.time() - t0, 2)
        args.gemm_swap = cap_cal["chosen"]
    gemm = None if args.no_gemm else leg(gemm_interference, args, ctx, mp, world, source, per_copy, bw,
                                         sizes, src, dst, swap_stream, n, dist)
    gemm_sus = None if (args.no_gemm or args.gemm_window_rounds <= 0) else leg(
        gemm_windows, args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap_stream, n, dist)
    # Under the power cap the calibrated setting (chosen on its alone rate)
    # may move less than the target beside the GEMM; then the leg is measured
    # again with --gemm-sus-fallback (unpaced), and the first result is kept
    # in the line.  Every rank sees the slowest rank's rate, so all agree.
    if (isinstance(gemm_sus, dict) and gemm_sus.get("swap_gbs_during") is not None and args.gemm_sus_fallback
            and gemm_sus["swap_gbs_during"] < args.gemm_target_gbs and args.gemm_cap <= 0
            and gemm_sus.get("swap_setting") != args.gemm_sus_fallback):
        alt = leg(gemm_windows, args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap_stream, n, dist,
                  args.gemm_sus_fallback, 0)
        if isinstance(alt, dict) and "error" not in alt:
            alt["first_setting"] = {k: gemm_sus.get(k) for k in ("swap_setting", "swap_pace_mbps",
                                                                  "swap_gbs_during", "slowdown", "slowdown_ci95")}
            alt["fallback"] = ("the calibrated setting moved less than --gemm-target-gbs beside the power-capped "
                               "GEMM; measured again with --gemm-sus-fallback")
            gemm_sus = alt
    gemm_fc1 = None if (args.no_gemm or args.no_gemm_fc1) else leg(
        gemm_interference, args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap_stream, n, dist, False,
        "gpt_fc1")
    gemm_ce = None if (args.no_gemm or args.no_gemm_ce) else leg(
        gemm_interference, args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap_stream, n, dist, True)
    cfg5 = None
    cfg5_ce = None
    if n > 1 and not args.no_gemm and not args.no_cfg5:
        cfg5 = leg(cfg5_leg, args, mp, rank, n, local_rank, dist)
        if not args.no_gemm_ce:
            cfg5_ce = leg(cfg5_leg, args, mp, rank, n, local_rank, dist, True)
    single = None
    if n > 1 and not args.no_single_source:
        single = leg(single_source_leg, args, mp, rank, n, local_rank, dist)
    others = None
    if n == 1 and not args.no_configs:
        del src, dst
        torch.cuda.empty_cache()
        others = leg(other_configs, args, mp, local_rank)

    cpu = None
    planner = None
    if rank == 0 and n == 1 and not args.no_cpu_baseline:
        cpu = leg(oracle_sample, args.cpu_seconds)
        planner = leg(planner_timing, mp, world, source, per_copy, bw, sizes)

    # BASELINE.json's pairing: the swap sustains the target rate (80% of 900
    # GB/s) beside the GEMM AND the GEMM slows by < 10% (upper 95% bound)
    for g in (gemm, gemm_ce, gemm_fc1, gemm_sus):
        if isinstance(g, dict) and g.get("swap_gbs_during") is not None and g.get("slowdown_ci95"):
            g["meets_rate_target"] = g["swap_gbs_during"] >= args.gemm_target_gbs
            g["meets_north_star_pair"] = bool(g["meets_rate_target"] and g.get("meets_10pct"))
    if rank == 0:
        line = {
            "metric": "D2D swap GB/s per source GPU (round trip, out+in)",
            "value": value, "unit": "GB/s", "n_gpus": n, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
            "config": workload_config(args, n),
            "swap_path_ran": ran_by_dir, "autotune": autotune,
            "per_direction_gbs": per_dir,
            "roofline": roof, "cpu_baseline": cpu, "e2e": e2e, "e2e_zero_copy": e2e_zc,
            "gpu_launches": launches[0], "clocks": clk, "gemm_slowdown": gemm, "gemm_slowdown_ce": gemm_ce,
            "gemm_slowdown_gpt_fc1": gemm_fc1, "gemm_slowdown_sustained": gemm_sus,
            "gemm_cap_calibration": cap_cal,
            "planner": planner, "other_configs": others, "cfg5": cfg5, "cfg5_ce": cfg5_ce,
            "single_source": single, "duplex": duplex,
            "leg_wall_s": leg_wall,
            "duplex_gbs": duplex.get("duplex_gbs") if isinstance(duplex, dict) else None,
            "parity": "round trip bit-exact vs generator (all %d tensors x %d ranks)" % (47 * mb, n),
            "value_is": "per source GPU: one rank's swapped bytes (out + in) / max-over-ranks step time",
            "paper_context": "context only, other hardware (BASELINE.md): Table III (P:323-332) D2D swaps of "
                             "115-1152 MB in 3-27 ms on V100 DGX-1 over 4 NVLink2 links = 72-85 GB/s round trip; "
                             "GPU-CPU swap 10.3-10.5 GB/s over PCIe3",
            "per_rank_gbs": value,
            "all_ranks_gbs": all_ranks_gbs,
            "transport": {mp.TRANSPORT_LOCAL: "local (mpress_init_local)",
                          mp.TRANSPORT_VMM_FD: "cuMem pools, POSIX fds over SCM_RIGHTS",
                          mp.TRANSPORT_LEGACY_IPC: "cudaMalloc pools, CUDA IPC handles"}.get(
                              ctx.get_option(mp.OPT_TRANSPORT), "?"),
            "link": ("HBM loopback (1 GPU: the peers are pools on the same GPU, bound by the HBM copy "
                     "roofline, not NVLink)" if n == 1 else
                     "NVLink 5 / NVSwitch (every rank swaps to all others; bound by 900 GB/s nominal, "
                     "770 GB/s per the profiling guide, per direction per GPU)"),
            "note": "N=1 and N>1 cross different links (HBM loopback vs NVLink), so value(N) / value(1) is "
                    "not a scaling efficiency; compare value with the NVLink roofline",
        }
        print(json.dumps(_finite(line), allow_nan=False))
    ctx.finalize()
    if n > 1:
        dist.destroy_process_group()
    return 0


def other_configs(args, mp, device):
    """BASELINE configs 1, 3 and 4 on this GPU (loopback peers), same kernel
    path and grid as the headline: swapped GB/s (out + in) of one round trip,
    median of 5 after 2 warm-ups, every byte checked against the generator.
    Config 5 needs 8 GPUs (its topology runs in tests/test_gpu_multiprocess.py)."""
    import torch
    from synth import device as synth_dev
    from synth import workloads
    path = {"direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK, "ce": mp.PATH_CE, "auto": mp.PATH_AUTO}[args.path]
    c3 = workloads.CONFIGS[3]
    cases = [
        ("cfg1 16 x 4 MiB fp16 activations -> 1 peer", 2, [1], [0, 1 << 30], workloads.cfg1_sizes()),
        ("cfg2 x8 micro-batches batched into one plan (376 tensors, 7.03 GiB, P:209) -> 3 peers", 4,
         [1, 2, 3], workloads.spare_vector(4, 0, [1, 2, 3], spare=24 << 30), workloads.cfg2_sizes(8)),
        ("cfg3 GPT-10.3B stage-0 Adam m/v (100 tensors, 12.21 GB) -> 3 peers, 2 GiB cap on one", 8,
         c3["peers"], workloads.spare_vector(8, 0, c3["peers"], spare_by_peer=c3["spare_by_peer"]),
         workloads.cfg3_sizes()),
        ("cfg4 one 4 GiB uint8 tensor -> 7 peers", 8, list(range(1, 8)),
         workloads.spare_vector(8, 0, list(range(1, 8)), spare=8 << 30), [4 << 30]),
        ("cfg4 one 4 MiB uint8 tensor -> 7 peers", 8, list(range(1, 8)),
         workloads.spare_vector(8, 0, list(range(1, 8)), spare=8 << 30), [4 << 20]),
    ]
    out = []
    s = torch.cuda.Stream()
    for name, world, peers, spare, sizes in cases:
        bw = workloads.bw_vector(world, 0, peers)
        pl = mp.plan(world, 0, spare, bw, sizes)
        part = [[0] * world for _ in range(world)]
        part[0] = [u * mp.DEFAULT_GRANULE for u in pl.units]
        ctx = mp.Context.local(world, 0, [device] * world, part)
        try:
            ctx.set_option(mp.OPT_PATH, path)
            ctx.set_option(mp.OPT_MAX_CTAS, args.max_ctas)
            src = [torch.empty(b, dtype=torch.uint8, device="cuda") for b in sizes]
            dst = [torch.empty(b, dtype=torch.uint8, device="cuda") for b in sizes]
            for i, t in enumerate(src):
                synth_dev.fill(t, 1000 * (len(out) + 1), i)
            torch.cuda.synchronize()
            ts = []
            for r in range(7):
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(s)
                h = ctx.swap_out(pl, src, stream=s)
                ctx.swap_in(h, dst, stream=s)
                e1.record(s)
                torch.cuda.synchronize()
                h.free()
                if r >= 2:
                    ts.append(e0.elapsed_time(e1))
            ms = statistics.median(ts)
            # back to back: R round trips enqueued at once, as a pipeline
            # issues them (the host runs ahead of the GPU, so per-call host
            # latency hides behind the previous pair's kernels)
            R = 32 if sum(sizes) <= (64 << 20) else 4
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            h = ctx.swap_out(pl, src, stream=s)     # keeps the GPU busy while the rest is enqueued
            ctx.swap_in(h, dst, stream=s)
            hs = [h]
            e0.record(s)
            for _ in range(R):
                h = ctx.swap_out(pl, src, stream=s)
                ctx.swap_in(h, dst, stream=s)
                hs.append(h)
            e1.record(s)
            torch.cuda.synchronize()
            for h in hs:
                h.free()
            b2b_ms = e0.elapsed_time(e1) / R
            bad = sum(synth_dev.check(t, 1000 * (len(out) + 1), i) for i, t in enumerate(dst))
            row = {"config": name, "bytes": sum(sizes), "stripes": len(pl.stripes),
                   "round_trip_ms": ms, "gbs": 2 * sum(sizes) / (ms / 1e3) / 1e9,
                   "b2b_round_trip_ms": b2b_ms, "b2b_gbs": 2 * sum(sizes) / (b2b_ms / 1e3) / 1e9,
                   "bit_exact": bad == 0}
            if sum(sizes) <= 256 << 20:
                row.update(graph_round_trip(ctx, mp, pl, src, dst, s, synth_dev, 1000 * (len(out) + 1)))
            out.append(row)
            del src, dst
            torch.cuda.empty_cache()
        finally:
            ctx.finalize()
    return out


def graph_round_trip(ctx, mp, pl, src, dst, s, synth_dev, seed):
    """The same round trip captured once into a CUDA graph (swap-out +
    swap-in, graph handle) and replayed: what a small, launch-bound swap
    costs when the pipeline step is a graph.  Median of 5 after 2 warm-ups."""
    import torch
    for t in dst:
        t.zero_()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        h = ctx.swap_out(pl, src)
        ctx.swap_in(h, dst)
    ts = []
    with torch.cuda.stream(s):
        for r in range(7):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record()
            g.replay()
            e1.record()
            torch.cuda.synchronize()
            if r >= 2:
                ts.append(e0.elapsed_time(e1))
    bad = sum(synth_dev.check(t, seed, i) for i, t in enumerate(dst))
    del g
    h.free()
    ms = statistics.median(ts)
    nbytes = sum(int(t.numel()) for t in src)
    return {"graph_round_trip_ms": ms, "graph_gbs": 2 * nbytes / (ms / 1e3) / 1e9,
            "graph_bit_exact": bad == 0}


def planner_timing(mp, world, source, spare, bw, sizes):
    """a1 PLAN on the host: the C++ planner (mpress_plan) against the oracle's
    Python planner on the bench's micro-batch (SURVEY §8(d) "planner timing")."""
    import oracle
    reps = 2000
    t0 = time.perf_counter()
    for _ in range(reps):
        mp.plan(world, source, spare, bw, sizes)
    cpp_us = (time.perf_counter() - t0) / reps * 1e6
    t0 = time.perf_counter()
    o = oracle.plan(world, source, spare, bw, sizes)
    py_us = (time.perf_counter() - t0) * 1e6
    assert mp.plan(world, source, spare, bw, sizes).stripes == [tuple(s) for s in o["stripes"]]
    return {"cpp_us_per_plan": cpp_us, "oracle_us_per_plan": py_us, "units": o["K"],
            "stripes": len(o["stripes"]), "note": "cpp includes the ctypes call; identical plans"}


def traffic_from_profile(path):
    """dram read+write bytes per launch of the dominant kernel (the swap
    kernel of `path`) from the committed ncu --set full summary, if any."""
    p = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(p):
        try:
            with open(p) as f:
                return json.load(f)["per_path"][path]["dram_bytes_per_launch"]
        except Exception:
            return None
    return None


class _Local:
    """Runs a rank's local work and remembers the first failure, so that the
    collectives after it are still reached by every rank (a leg that fails on
    one rank reports the error instead of hanging the others)."""

    def __init__(self):
        self.err = None

    def __call__(self, fn, *a):
        if self.err is not None:
            return None
        try:
            return fn(*a)
        except Exception as exc:  # pragma: no cover - reported in the line
            self.err = "%s: %s" % (type(exc).__name__, exc)
            return None


def bootstrap_ci95(xs, resamples=4000, seed=219):
    """95% percentile-bootstrap interval of the median of xs (NaN if empty)."""
    import random
    if not xs:
        return float("nan"), float("nan")
    rng = random.Random(seed)
    n = len(xs)
    meds = sorted(statistics.median(rng.choices(xs, k=n)) for _ in range(resamples))
    return meds[int(0.025 * (resamples - 1))], meds[int(0.975 * (resamples - 1))]


def set_gemm_swap(ctx, mp, spec, pace_mbps=0):
    """Apply a GEMM-concurrent swap setting "path:variant:max_ctas" (path
    auto/direct/bulk; auto with a cap <= the SM count runs the capped direct
    shape) and the rate pace (MPRESS_OPT_PACE_MBPS, 0 = unpaced; not applied
    to the copy engines); returns the previous options for restore_swap."""
    prev = (ctx.get_option(mp.OPT_PATH), ctx.get_option(mp.OPT_VARIANT), ctx.get_option(mp.OPT_MAX_CTAS),
            ctx.get_option(mp.OPT_PACE_MBPS))
    name, var, cap = spec.split(":")
    paths = {"auto": mp.PATH_AUTO, "direct": mp.PATH_DIRECT, "bulk": mp.PATH_BULK, "ce": mp.PATH_CE}
    ctx.set_option(mp.OPT_PATH, paths[name])
    if name != "auto":
        ctx.set_option(mp.OPT_VARIANT, int(var))
    ctx.set_option(mp.OPT_MAX_CTAS, int(cap))
    ctx.set_option(mp.OPT_PACE_MBPS, int(pace_mbps))
    return prev


def restore_swap(ctx, mp, prev):
    ctx.set_option(mp.OPT_PATH, prev[0])
    if prev[0] != mp.PATH_AUTO:
        ctx.set_option(mp.OPT_VARIANT, prev[1])
    ctx.set_option(mp.OPT_MAX_CTAS, prev[2])
    ctx.set_option(mp.OPT_PACE_MBPS, prev[3])


def gemm_pace_mbps(args, spec=None):
    """MB/s the GEMM-concurrent SM swap is paced to: the rate the calibration
    asks of it (--gemm-target-gbs / 0.85), so the swap takes only the
    bandwidth its target needs -- for the direct (LSU) kernels only,
    whose cost to the GEMM rises with their rate (+12.8 / +16.1 / +21.9% at
    381 / 555 / 737 GB/s); the TMA (bulk) kernels cost it about the same
    paced or not (bulk 7: +11.7% at 670 GB/s paced and at 844 unpaced,
    profiles/r02/gemm_windows_power_capped_bulk78.jsonl), so they run
    unpaced and keep the rate.  0 with --gemm-no-pace."""
    spec = spec if spec is not None else args.gemm_swap
    if args.gemm_no_pace or spec.split(":")[0] in ("bulk", "ce"):
        return 0
    return int(round(args.gemm_target_gbs / 0.85 * 1000))


def calibrate_gemm_cap(args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap, n, dist):
    """The GEMM-concurrent swap setting, measured on this run's links (HBM
    loopback at N = 1, NVLink at N > 1, where every remote access pays ~2x
    the latency, so a setting keeps fewer bytes in flight per µs): every
    candidate of --gemm-swap-candidates (ordered cheapest for the GEMM first:
    one-warp TMA CTAs with 16 KB of shared memory on every SM, then one
    128-thread direct CTA on every SM, then 96 and 64 of them) runs alone and
    unpaced, out + in, on every rank at
    once; the first whose slowest rank reaches --gemm-target-gbs / 0.85
    (headroom for the GEMM's contention) is chosen, else the fastest.  The
    GEMM leg then paces the chosen setting to that rate (gemm_pace_mbps).  Collective: every rank
    reaches every barrier and reduction even if its own work fails."""
    import torch
    specs = [c.strip() for c in args.gemm_swap_candidates.split(",") if c.strip()]
    pl = mp.plan(world, source, per_copy, bw, sizes)
    nbytes = sum(sizes)
    reps = 3
    table, err = {}, None
    for spec in specs:
        rate = 0.0
        if n > 1:
            dist.barrier()
        if err is None:
            prev = None
            try:
                prev = set_gemm_swap(ctx, mp, spec)
                h = ctx.swap_out(pl, src[0], stream=swap)     # warm-up
                ctx.swap_in(h, dst[0], stream=swap)
                h.free()
                torch.cuda.synchronize()
                e0 = torch.cuda.Event(enable_timing=True)
                e1 = torch.cuda.Event(enable_timing=True)
                e0.record(swap)
                for _ in range(reps):
                    h = ctx.swap_out(pl, src[0], stream=swap)
                    ctx.swap_in(h, dst[0], stream=swap)
                    h.free()
                e1.record(swap)
                torch.cuda.synchronize()
                rate = 2 * reps * nbytes / e0.elapsed_time(e1) / 1e6
            except Exception as exc:  # pragma: no cover - reported in the line
                err = "%s: %s" % (type(exc).__name__, exc)
            finally:
                if prev is not None:
                    try:
                        restore_swap(ctx, mp, prev)
                    except Exception:  # pragma: no cover
                        pass
        t = torch.tensor([rate if err is None else 0.0], dtype=torch.float64)
        if n > 1:
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
        table[spec] = float(t.item())
    need = args.gemm_target_gbs / 0.85
    ok = [c for c in specs if table[c] >= need]
    if err is not None:
        chosen = "auto:-1:148"
    else:
        chosen = ok[0] if ok else max(specs, key=lambda c: table[c])
    # the chosen setting's capability against its link roofline: loopback
    # moves 2 B of HBM per swapped byte (measured copy peak), NVLink 1 B per
    # direction (the guide's 770 GB/s)
    peaks, _ = measured_peaks()
    cap_gbs = table.get(chosen, 0.0)
    if n == 1:
        roof = {"bound": "hbm", "achieved": 2 * cap_gbs, "peak": float(peaks.get("hbm_gbs", FALLBACK_HBM)),
                "unit": "GB/s", "what": "HBM traffic of the chosen capped swap running alone (out + in)"}
    else:
        roof = {"bound": "nvlink", "achieved": cap_gbs, "peak": NVLINK_GUIDE, "unit": "GB/s",
                "what": "swapped bytes per second of the chosen capped swap alone, per source"}
    roof["frac"] = roof["achieved"] / roof["peak"] if roof["peak"] else None
    return {"chosen": chosen, "target_gbs": args.gemm_target_gbs, "needed_alone_gbs": need,
            "alone_gbs_min_over_ranks": table, "chosen_roofline": roof, "error": err}


GEMM_SHAPES = {"8192^3": (8192, 8192, 8192),
               # config 5 (ii): the FC1 of config 3's GPT-10.3B at
               # micro-batch 2 x seq 2048: [4096 x 5120] . [5120 x 20480]
               "gpt_fc1": (4096, 5120, 20480)}


def gemm_interference(args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap, n, dist, ce=False,
                      shape="8192^3"):
    """Second half of the metric: slowdown of a bf16 GEMM (8192^3, the shape
    MEASURED_PEAKS.json is quoted on, or config 5's GPT FC1 stage GEMM) on the
    compute stream while swaps loop on the side stream with the grid capped
    at --gemm-cap CTAs.  Alone and with-swap rounds alternate (so power-cap
    drift hits both), and only GEMMs that ran entirely inside the swap window
    count.  ce=True: the same with the copy-engine comparator (a7, no SMs)
    moving the swap."""
    import torch
    comp = torch.cuda.current_stream()
    M, K, N = GEMM_SHAPES[shape]
    G = 24
    L = _Local()
    st = {}
    alone, during, swap_gbs = [], [], []

    def gemms():
        evs = []
        for _ in range(G):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(comp)
            torch.matmul(st["a"], st["b"], out=st["c"])
            e1.record(comp)
            evs.append((e0, e1))
        return evs

    def setup():
        st["a"] = torch.randn(M, K, dtype=torch.bfloat16, device="cuda")
        st["b"] = torch.randn(K, N, dtype=torch.bfloat16, device="cuda")
        st["c"] = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")
        st["pl"] = mp.plan(world, source, per_copy, bw, sizes)
        st["prev"] = set_gemm_swap(ctx, mp, "ce:0:0" if ce else args.gemm_swap, 0 if ce else gemm_pace_mbps(args))
        # swap time at this setting, to size the loop that must cover the GEMM
        # window; one untimed pair first (the copy-engine path creates its
        # side streams on first use, which once inflated the estimate so much
        # that the loop ended before the counted GEMMs did)
        h = ctx.swap_out(st["pl"], src[0], stream=swap)
        ctx.swap_in(h, dst[0], stream=swap)
        h.free()
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(swap)
        h = ctx.swap_out(st["pl"], src[0], stream=swap)
        ctx.swap_in(h, dst[0], stream=swap)
        e1.record(swap)
        h.free()
        gemms()
        torch.cuda.synchronize()
        st["per_swap_ms"] = e0.elapsed_time(e1)
        # Settle the power state first: a B200 runs this GEMM at ~1670 TFLOP/s
        # in a burst and ~1400 sustained (MEASURED_PEAKS.json), and rounds that
        # straddle the drop mix the two regimes into the ratio.  (These short
        # synchronised rounds let the board climb back to burst clocks; the
        # power-capped regime is gemm_windows'.)
        t0 = time.time()
        while time.time() - t0 < args.gemm_settle_s:
            gemms()
            torch.cuda.synchronize()

    ratios = []

    def round_():
        evs = gemms()
        torch.cuda.synchronize()
        a_r = [x.elapsed_time(y) for x, y in evs[4:]]
        alone.extend(a_r)
        gemm_ms = statistics.median(alone)
        # cover the GEMM run twice over (3x for the copy engines, whose
        # host-side issue rate is the slower one)
        n_swap = int((3.0 if ce else 2.0) * G * gemm_ms / st["per_swap_ms"]) + 2
        s0 = torch.cuda.Event(enable_timing=True)
        s1 = torch.cuda.Event(enable_timing=True)
        # The SM paths enqueue in ~10 us per call, far ahead of the GPU, so
        # their swaps go first and cover the whole GEMM run.  The copy-engine
        # path costs ~3 us of host time per stripe (one cudaMemcpyAsync each):
        # enqueued first, its swaps would run as fast as the host issues them
        # and be over before the GEMMs start, so the GEMMs go first there.
        if ce:
            evs = gemms()
        s0.record(swap)
        for _ in range(n_swap):
            h = ctx.swap_out(st["pl"], src[0], stream=swap)
            ctx.swap_in(h, dst[0], stream=swap)
            h.free()
        s1.record(swap)
        if not ce:
            evs = gemms()
        torch.cuda.synchronize()
        win = s0.elapsed_time(s1)
        d_r = [x.elapsed_time(y) for x, y in evs[4:]
               if s0.elapsed_time(x) >= 0 and s0.elapsed_time(y) <= win]
        if os.environ.get("BENCH_DEBUG"):
            print("gemm round ce=%s n_swap=%d win=%.2f ms gemm starts %s ends %s" % (
                ce, n_swap, win, [round(s0.elapsed_time(x), 2) for x, _ in evs[::6]],
                [round(s0.elapsed_time(y), 2) for _, y in evs[::6]]), file=sys.stderr)
        during.extend(d_r)
        if d_r:
            ratios.append(statistics.median(d_r) / statistics.median(a_r))
        swap_gbs.append(2 * n_swap * sum(sizes) / win / 1e6)

    L(setup)
    for _ in range(args.gemm_rounds):
        L(round_)
    st["ran"] = ctx.get_option(mp.OPT_LAST_PATH)
    if "prev" in st:
        L(restore_swap, ctx, mp, st["prev"])
    lo, hi = bootstrap_ci95([r - 1 for r in ratios])
    t = torch.tensor([statistics.median(alone) if alone else float("nan"),
                      statistics.median(during) if during else float("nan"),
                      1.0 if L.err is not None else 0.0,
                      statistics.median(ratios) - 1 if ratios else float("nan"), lo, hi], dtype=torch.float64)
    if n > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if float(t[2]) > 0:
        return {"error": L.err or "another rank failed"}
    a_ms, d_ms = float(t[0]), float(t[1])
    a_tflops = 2 * M * N * K / (a_ms / 1e3) / 1e12
    peaks, _ = measured_peaks()
    burst, sus = peaks.get("bf16_tflops"), peaks.get("bf16_tflops_sustained")
    regime = None
    if burst and sus:
        regime = "sustained" if a_tflops < (burst + sus) / 2 else "burst"
    return {"gemm": "bf16 %dx%dx%d torch.matmul (cuBLAS) on the compute stream" % (M, K, N), "shape": shape,
            "alone_ms": a_ms, "with_swap_ms": d_ms,
            "alone_tflops": a_tflops,
            "regime": regime,
            "regime_rule": "alone TFLOP/s vs the midpoint of MEASURED_PEAKS.json bf16_tflops (burst) and "
                           "bf16_tflops_sustained",
            "settle_s": args.gemm_settle_s,
            # each round pairs an alone and a with-swap run back to back, so
            # clock / power drift between rounds cancels in the round's ratio
            "slowdown": float(t[3]),
            "slowdown_ci95": [float(t[4]), float(t[5])],
            "slowdown_ci95_method": "percentile bootstrap (4000 resamples) of the median of the per-round "
                                    "paired ratios; max over ranks at N > 1",
            "meets_10pct": float(t[5]) < 0.10,
            "slowdown_pooled": d_ms / a_ms - 1,
            "rounds": len(ratios),
            "slowdown_per_round": [r - 1 for r in ratios],
            "swap_path": {mp.PATH_DIRECT: "direct", mp.PATH_BULK: "bulk", mp.PATH_CE: "ce"}.get(
                st.get("ran"), args.path),
            "swap_setting": "ce:0:0" if ce else args.gemm_swap,
            "swap_max_ctas": None if ce else int(args.gemm_swap.split(":")[2]),
            "swap_pace_mbps": None if ce else gemm_pace_mbps(args),
            # MPRESS_OPT_PDL 1 (default) launches a capped grid without PDL
            "swap_pdl_mode": ctx.get_option(mp.OPT_PDL),
            "swap_gbs_during": statistics.median(swap_gbs),
            "gemms_counted": len(during),
            "note": ("N=1 loopback: the swap's bytes also load the GEMM's HBM (2 B per swapped "
                     "byte), a harsher case than NVLink (1 B of source HBM per byte)") if n == 1 else
                    ("every rank swaps to all others while running the GEMM; max over ranks")}


def gemm_windows(args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, swap, n, dist, spec=None, pace=None):
    """The GEMM leg in the power-capped ("sustained") regime.  The rounds of
    gemm_interference synchronise between short GEMM runs, and those gaps let
    the board climb back to burst clocks; here each round is an alone window
    of W back-to-back 8192^3 GEMMs followed at once by a with-swap window of
    W more (the capped swap looping beside it, started when the alone window
    ends), both enqueued before one synchronise, so the GPU stays busy and
    under its power cap.  W is ~3 s of GEMMs (the verdict's "windows of 3 s
    or more"): the power governor responds over hundreds of ms, and 160 ms
    windows mixed the two modes' power states.  The
    window time / W is the GEMM time; the ratio per round is paired; the
    interval is bootstrapped over rounds.  After a settle that reaches the
    sustained regime (below the burst/sustained midpoint)."""
    import torch
    comp = torch.cuda.current_stream()
    spec = spec or args.gemm_swap
    pace = gemm_pace_mbps(args) if pace is None else pace
    M = K = N = 8192
    W = args.gemm_window
    L = _Local()
    st = {}
    ratios, alone, during, gbs = [], [], [], []

    def setup():
        st["a"] = torch.randn(M, K, dtype=torch.bfloat16, device="cuda")
        st["b"] = torch.randn(K, N, dtype=torch.bfloat16, device="cuda")
        st["c"] = torch.empty(M, N, dtype=torch.bfloat16, device="cuda")
        st["pl"] = mp.plan(world, source, per_copy, bw, sizes)
        st["prev"] = set_gemm_swap(ctx, mp, spec, pace)
        h = ctx.swap_out(st["pl"], src[0], stream=swap)
        ctx.swap_in(h, dst[0], stream=swap)
        h.free()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(swap)
        h = ctx.swap_out(st["pl"], src[0], stream=swap)
        ctx.swap_in(h, dst[0], stream=swap)
        e1.record(swap)
        h.free()
        torch.cuda.synchronize()
        st["per_swap_ms"] = e0.elapsed_time(e1)
        peaks, _ = measured_peaks()
        mid = (peaks.get("bf16_tflops", 0) + peaks.get("bf16_tflops_sustained", 0)) / 2 or None
        t0 = time.time()
        while True:
            a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a0.record(comp)
            for _ in range(W):
                torch.matmul(st["a"], st["b"], out=st["c"])
            a1.record(comp)
            torch.cuda.synchronize()
            st["settle_tflops"] = 2 * M * N * K * W / (a0.elapsed_time(a1) / 1e3) / 1e12
            st["settle_s"] = time.time() - t0
            if (mid is None or st["settle_tflops"] < mid or st["settle_s"] > 30) and st["settle_s"] >= 2.0:
                break

    def round_():
        a0, a1, b0, b1 = (torch.cuda.Event(enable_timing=True) for _ in range(4))
        s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a0.record(comp)
        for _ in range(W):
            torch.matmul(st["a"], st["b"], out=st["c"])
        a1.record(comp)
        gemm_ms = statistics.median(alone) if alone else 0.8
        n_swap = int(1.5 * W * gemm_ms / st["per_swap_ms"]) + 2
        swap.wait_event(a1)                   # the swap window starts when the alone window ends
        s0.record(swap)
        for k in range(n_swap):
            if k == 3:   # the GEMM window is enqueued after a few swaps, not after all of them
                comp.wait_event(s0)           # it starts once the swaps have
                b0.record(comp)
                for _ in range(W):
                    torch.matmul(st["a"], st["b"], out=st["c"])
                b1.record(comp)
            h = ctx.swap_out(st["pl"], src[0], stream=swap)
            ctx.swap_in(h, dst[0], stream=swap)
            h.free()
        s1.record(swap)
        torch.cuda.synchronize()
        a_ms = a0.elapsed_time(a1) / W
        alone.append(a_ms)
        if s0.elapsed_time(b0) >= 0 and b1.elapsed_time(s1) >= 0:   # the swap covered the whole window
            d_ms = b0.elapsed_time(b1) / W
            during.append(d_ms)
            ratios.append(d_ms / a_ms - 1)
            gbs.append(2 * n_swap * sum(sizes) / s0.elapsed_time(s1) / 1e6)

    L(setup)
    for _ in range(args.gemm_window_rounds):
        L(round_)
    if "prev" in st:
        L(restore_swap, ctx, mp, st["prev"])
    lo, hi = bootstrap_ci95(ratios)
    # (the swap rate as its negative: MAX over ranks = the slowest rank's,
    # so every rank takes the same fallback decision)
    t = torch.tensor([statistics.median(alone) if alone else float("nan"),
                      statistics.median(during) if during else float("nan"),
                      1.0 if L.err is not None else 0.0,
                      statistics.median(ratios) if ratios else float("nan"), lo, hi,
                      -statistics.median(gbs) if gbs else float("nan")], dtype=torch.float64)
    if n > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if float(t[2]) > 0:
        return {"error": L.err or "another rank failed"}
    a_ms = float(t[0])
    a_tflops = 2 * M * N * K / (a_ms / 1e3) / 1e12
    peaks, _ = measured_peaks()
    mid = (peaks.get("bf16_tflops", 0) + peaks.get("bf16_tflops_sustained", 0)) / 2
    return {"gemm": "bf16 8192x8192x8192 torch.matmul (cuBLAS), windows of %d back to back" % W,
            "protocol": "per round: alone window then with-swap window, no synchronise between them",
            "alone_ms": a_ms, "with_swap_ms": float(t[1]), "alone_tflops": a_tflops,
            "regime": ("sustained" if a_tflops < mid else "burst") if mid else None,
            "settle_s": st.get("settle_s"), "settle_last_tflops": st.get("settle_tflops"),
            "slowdown": float(t[3]), "slowdown_ci95": [float(t[4]), float(t[5])],
            "meets_10pct": float(t[5]) < 0.10, "rounds": len(ratios),
            "slowdown_per_round": ratios, "swap_setting": spec,
            "swap_pace_mbps": pace,
            "swap_gbs_during": -float(t[6]) if gbs else None}


def cfg5_leg(args, mp, rank, n, device, dist, ce=False):
    """BASELINE config 5 (BJ:11, reading R20) at N GPUs: the
    first half of the ranks are the heavy stages (sources), the second half
    the light ones (pure importers).  Source s swaps (N/2 - s) Bert stage-0
    micro-batch sets (900 MiB each) batched into one plan -- at N = 8:
    3.52 / 2.64 / 1.76 / 0.88 GiB from sources 0-3 into peers 4-7 --
    sequential partition (R12), grid capped at --gemm-cap CTAs, while EVERY
    rank runs back-to-back bf16 GEMMs on its compute stream.  Reports each
    source's swap GB/s (out + in) under contention and the GEMM slowdown on
    sources and importers.  ce=True: the same with the copy-engine
    comparator moving the swaps (no SMs).  Every collective is reached by all ranks even if
    a rank's local work fails (the failure is reported, not hung on)."""
    import torch
    from synth import device as synth_dev
    from synth import workloads
    H = n // 2
    sources, peers = list(range(H)), list(range(H, n))
    is_src = rank in sources
    sizes = workloads.cfg2_sizes(H - rank) if is_src else []
    spare = [0] * n
    for p in peers:
        spare[p] = 16 * GiB
    bwm = [[1 if (s in sources and p in peers) else 0 for p in range(n)] for s in range(n)]
    part = mp.partition_sequential(n, spare, bwm, [(s, workloads.cfg2_sizes(H - s), 1) for s in sources])
    ctx = mp.Context.distributed(device, n, rank, part)
    comp = torch.cuda.current_stream()
    swap = torch.cuda.Stream()
    M = args.gemm_n
    G = 24
    err = []

    def guard(fn):
        if err:
            return None
        try:
            return fn()
        except Exception as exc:  # pragma: no cover - reported below
            err.append("rank %d: %s: %s" % (rank, type(exc).__name__, exc))
            return None

    st = {}

    def setup():
        rem = list(spare)
        for s in sources:
            if s == rank:
                st["pl"] = mp.plan(n, rank, rem, bwm[rank], sizes)
            for p in range(n):
                rem[p] -= part[s][p]
        set_gemm_swap(ctx, mp, "ce:0:0" if ce else args.gemm_swap, 0 if ce else gemm_pace_mbps(args))
        st["a"] = torch.randn(M, M, dtype=torch.bfloat16, device="cuda")
        st["b"] = torch.randn(M, M, dtype=torch.bfloat16, device="cuda")
        st["c"] = torch.empty(M, M, dtype=torch.bfloat16, device="cuda")
        if is_src:
            st["src"] = [torch.empty(x, dtype=torch.uint8, device="cuda") for x in sizes]
            st["dst"] = [torch.empty(x, dtype=torch.uint8, device="cuda") for x in sizes]
            for i, t in enumerate(st["src"]):
                synth_dev.fill(t, 5000 + rank, i)
            h = ctx.swap_out(st["pl"], st["src"], stream=swap)   # untimed first pair (see gemm_interference)
            ctx.swap_in(h, st["dst"], stream=swap)
            h.free()
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(swap)
            h = ctx.swap_out(st["pl"], st["src"], stream=swap)
            ctx.swap_in(h, st["dst"], stream=swap)
            e1.record(swap)
            h.free()
            torch.cuda.synchronize()
            st["per_swap_ms"] = e0.elapsed_time(e1)
        torch.cuda.synchronize()
        t0 = time.time()   # settle the power state (see gemm_interference)
        while time.time() - t0 < args.gemm_settle_s:
            gemms()
            torch.cuda.synchronize()

    def gemms():
        evs = []
        for _ in range(G):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(comp)
            torch.matmul(st["a"], st["b"], out=st["c"])
            e1.record(comp)
            evs.append((e0, e1))
        return evs

    alone, during, gbs, ratios = [], [], [], []

    def run_alone():
        evs = gemms()
        torch.cuda.synchronize()
        st["a_r"] = [x.elapsed_time(y) for x, y in evs[4:]]
        alone.extend(st["a_r"])

    def run_with_swap():
        s0 = s1 = None
        evs = gemms() if ce else None   # copy engines: GEMMs first (see gemm_interference)
        if is_src:
            n_swap = int((3.0 if ce else 2.0) * G * statistics.median(alone) / st["per_swap_ms"]) + 2
            s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            s0.record(swap)
            for _ in range(n_swap):
                h = ctx.swap_out(st["pl"], st["src"], stream=swap)
                ctx.swap_in(h, st["dst"], stream=swap)
                h.free()
            s1.record(swap)
        if not ce:
            evs = gemms()
        torch.cuda.synchronize()
        if is_src:
            win = s0.elapsed_time(s1)
            d_r = [x.elapsed_time(y) for x, y in evs[4:]
                   if s0.elapsed_time(x) >= 0 and s0.elapsed_time(y) <= win]
            gbs.append(2 * n_swap * sum(sizes) / win / 1e6)
        else:   # importers: the middle of the run, inside every source's window
            d_r = [x.elapsed_time(y) for x, y in evs[4:G - 4]]
        during.extend(d_r)
        if d_r:
            ratios.append(statistics.median(d_r) / statistics.median(st["a_r"]))

    guard(setup)
    for _ in range(max(4, args.gemm_rounds // 4)):
        dist.barrier()
        guard(run_alone)
        dist.barrier()
        guard(run_with_swap)
    bad = 0
    if is_src and not err:
        bad = guard(lambda: sum(synth_dev.check(t, 5000 + rank, i) for i, t in enumerate(st["dst"]))) or 0
    row = torch.zeros(n, 8, dtype=torch.float64)
    lo, hi = bootstrap_ci95([r - 1 for r in ratios])
    row[rank] = torch.tensor([statistics.median(alone) if alone else float("nan"),
                              statistics.median(during) if during else float("nan"),
                              statistics.median(gbs) if gbs else 0.0, float(bad), float(len(err)),
                              statistics.median(ratios) - 1 if ratios else float("nan"), lo, hi],
                             dtype=torch.float64)
    dist.all_reduce(row)
    ctx.finalize()
    if float(row[:, 4].sum()) > 0:
        return {"error": err[0] if err else "a rank failed (see its stderr)"}
    slow = [float(row[r, 5]) for r in range(n)]   # median over rounds of paired ratios
    return {"config": "cfg5 imbalanced all-stage swap: sources %s -> importers %s, source s swaps %s micro-batch "
                      "sets (900 MiB each, one plan), bf16 %dx%dx%d GEMMs on every rank" %
                      (sources, peers, [H - s for s in sources], M, M, M),
            "swap_setting": "ce:0:0" if ce else args.gemm_swap,
            "swap_pace_mbps": None if ce else gemm_pace_mbps(args),
            "per_source_gbs": [float(row[s, 2]) for s in sources],
            "per_source_bytes": [sum(workloads.cfg2_sizes(H - s)) for s in sources],
            "gemm_alone_ms": [float(row[r, 0]) for r in range(n)],
            "gemm_slowdown_per_rank": slow,
            "gemm_slowdown_ci95_per_rank": [[float(row[r, 6]), float(row[r, 7])] for r in range(n)],
            "rounds": max(4, args.gemm_rounds // 4),
            "max_slowdown_sources": max(slow[s] for s in sources),
            "max_slowdown_importers": max(slow[p] for p in peers),
            "bit_exact": float(row[:, 3].sum()) == 0}


def single_source_leg(args, mp, rank, n, device, dist):
    """BASELINE config 4 at N GPUs (BJ:10, the B200 analogue of Fig. 4,
    P:115-119): rank 0 is the only source and swaps ONE uint8 tensor to its
    first P peers, P in {1, 3, N-1}, over NVLink, for every size of
    --ss-sizes and every transfer path (direct kernel, bulk/TMA kernel, copy
    engines), swap-out and swap-in timed separately (CUDA events on the swap
    stream, median of 20 reps -- 5 from 256 MiB -- after 3 warm-up pairs).  GB/s = tensor bytes /
    time, i.e. one direction of NVLink per byte, reported as a fraction of the
    900 GB/s nominal and of the guide's 770 GB/s.  The other ranks are passive
    importers (their pools are mapped by rank 0).  The restored tensor is
    checked byte for byte against the generator after every (P, size, path)."""
    import torch
    from synth import device as synth_dev
    sizes = [int(x) for x in args.ss_sizes.split(",") if x.strip()]
    big = max(sizes)
    G = mp.DEFAULT_GRANULE
    per_peer = (big + G - 1) // G * G + G
    part = [[0] * n for _ in range(n)]
    part[0] = [0] + [per_peer] * (n - 1)
    ctx = mp.Context.distributed(device, n, rank, part)
    rows, err = [], None
    if rank == 0:
        try:
            swap = torch.cuda.Stream()
            src = torch.empty(big, dtype=torch.uint8, device="cuda")
            dst = torch.empty(big, dtype=torch.uint8, device="cuda")
            synth_dev.fill(src, 7000, 0)
            torch.cuda.synchronize()
            paths = [("direct", mp.PATH_DIRECT), ("bulk", mp.PATH_BULK), ("ce", mp.PATH_CE)]
            for P in sorted({p for p in (1, 3, n - 1) if 1 <= p <= n - 1}):
                peers = list(range(1, P + 1))
                spare = [0] * n
                for p in peers:
                    spare[p] = per_peer
                bw = [1 if p in peers else 0 for p in range(n)]
                for size in sizes:
                    pl = mp.plan(n, 0, spare, bw, [size])
                    a, b = src[:size], dst[:size]
                    for name, path in paths:
                        ctx.set_option(mp.OPT_PATH, path)
                        b.zero_()
                        reps = 20 if size < (256 << 20) else 5
                        to, ti = [], []
                        for r in range(reps + 3):                      # 3 warm-ups
                            e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
                            e[0].record(swap)
                            h = ctx.swap_out(pl, [a], stream=swap)
                            e[1].record(swap)
                            ctx.swap_in(h, [b], stream=swap)
                            e[2].record(swap)
                            torch.cuda.synchronize()
                            h.free()
                            if r >= 3:
                                to.append(e[0].elapsed_time(e[1]))
                                ti.append(e[1].elapsed_time(e[2]))
                        mo, mi = statistics.median(to), statistics.median(ti)
                        bad = synth_dev.check(b, 7000, 0)
                        go, gi = size / mo / 1e6, size / mi / 1e6
                        rows.append({"peers": P, "bytes": size, "path": name, "stripes": len(pl.stripes),
                                     "out_us": mo * 1e3, "in_us": mi * 1e3, "out_gbs": go, "in_gbs": gi,
                                     "out_frac_of_900": go / NVLINK_NOMINAL, "in_frac_of_900": gi / NVLINK_NOMINAL,
                                     "out_frac_of_guide_770": go / NVLINK_GUIDE,
                                     "in_frac_of_guide_770": gi / NVLINK_GUIDE, "bit_exact": bad == 0})
            del src, dst
            torch.cuda.empty_cache()
        except Exception as exc:  # pragma: no cover - reported in the line
            err = "%s: %s" % (type(exc).__name__, exc)
    dist.barrier()          # importers keep their pools until rank 0 is done
    ctx.finalize()
    if rank != 0:
        return None
    out = {"config": "cfg4 single source: rank 0 -> its first P peers, P in %s, one uint8 tensor per size, "
                     "swap-out and swap-in timed separately" % sorted({r["peers"] for r in rows}),
           "unit": "GB/s (tensor bytes / time, one NVLink direction)", "rows": rows, "error": err,
           "all_bit_exact": all(r["bit_exact"] for r in rows) if rows else None}
    ns = north_star_summary(rows, n)
    if ns is not None:
        out["north_star"] = ns
    return out


def north_star_summary(rows, n):
    """BASELINE.json's target on config 4's rows: at N GPUs, one source
    striping to its N-1 peers, tensors >= 256 MiB, the better SM kernel per
    size, the slower of swap-out and swap-in -- the minimum of that over the
    sizes against 80% of 900 GB/s.  None when no such row was measured."""
    head = [r for r in rows if r["peers"] == n - 1 and r["bytes"] >= (256 << 20) and r["path"] != "ce"]
    if not head:
        return None
    best = {}
    for r in head:
        v = min(r["out_gbs"], r["in_gbs"])
        if v > best.get(r["bytes"], (0, None))[0]:
            best[r["bytes"]] = (v, r["path"])
    worst = min(v for v, _ in best.values())
    return {"peers": n - 1, "sizes": sorted(best), "best_sm_path_per_size":
            {str(k): v[1] for k, v in sorted(best.items())},
            "min_gbs_over_sizes_and_directions": worst,
            "frac_of_900": worst / NVLINK_NOMINAL, "target_frac": 0.8,
            "meets_target": worst >= 0.8 * NVLINK_NOMINAL}


def duplex_leg(ctx, mp, world, source, per_copy, bw, sizes, src, dst, n, dist):
    """NEXT-2's duplex case (swap-out and swap-in on two streams): the
    swap-out of micro-batch m+1 runs on one stream while the swap-in of
    micro-batch m runs on another, as in the 1F1B steady state; the same
    2 x mb swaps serialised on one stream are timed beside it.  duplex_gbs
    = swapped bytes (out + in) / time.  On 1 GPU (loopback) both directions
    share the same HBM, so little gain is expected; over NVLink a swap-out is
    tx and a swap-in rx, which run on separate link directions."""
    import torch
    from synth import device as synth_dev
    mb = len(src)
    nbytes = 2 * mb * sum(sizes)
    s_out, s_in = torch.cuda.Stream(), torch.cuda.Stream()
    pl = mp.plan(world, source, per_copy, bw, sizes)
    L = _Local()

    def one(duplex):
        for row in dst:
            for t in row:
                t.zero_()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s_out)
        s_in.wait_stream(s_out)
        ins = s_in if duplex else s_out
        hs = [ctx.swap_out(pl, src[0], stream=s_out)]
        for m in range(1, mb + 1):
            if m < mb:
                hs.append(ctx.swap_out(pl, src[m], stream=s_out))
            ctx.swap_in(hs[m - 1], dst[m - 1], stream=ins)
        s_out.wait_stream(s_in)
        e1.record(s_out)
        torch.cuda.synchronize()
        for h in hs:
            h.free()
        return e0.elapsed_time(e1)

    def run():
        res = {}
        for duplex in (True, False):
            one(duplex)                                    # warm-up
            ts = [one(duplex) for _ in range(5)]
            res["duplex" if duplex else "serial"] = statistics.median(ts)
        bad = 0
        for m in range(mb):
            for i, t in enumerate(dst[m]):
                bad += synth_dev.check(t, 2000 + 100 * source + m, i)
        res["bad"] = bad
        return res

    if n > 1:
        dist.barrier()
    r = L(run) or {}
    t = torch.tensor([r.get("duplex", 0.0), r.get("serial", 0.0), float(r.get("bad", 0)),
                      1.0 if L.err else 0.0], dtype=torch.float64)
    if n > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if float(t[3]) > 0:
        return {"error": L.err or "another rank failed"}
    d_ms, s_ms = float(t[0]), float(t[1])
    return {"duplex_gbs": nbytes / (d_ms / 1e3) / 1e9, "serial_gbs": nbytes / (s_ms / 1e3) / 1e9,
            "duplex_ms": d_ms, "serial_ms": s_ms, "micro_batches": mb, "bytes": nbytes,
            "bit_exact": float(t[2]) == 0,
            "schedule": "out(0); then out(m+1) on the swap-out stream || in(m) on the swap-in stream; "
                        "serial = the same calls on one stream; max over ranks, median of 5"}


def run_e2e(args, ctx, mp, world, source, per_copy, bw, sizes, src, dst, stream, n, dist):
    """Same metric through the public API with pinned HOST buffers: each step
    copies the micro-batches' inputs host->device, swaps them out and in, and
    reads the restored tensors back device->host.  With N > 1 ranks on one
    host each rank stages 2 micro-batches (2 x 900 MiB pinned in and out) so N
    ranks do not pin N x 14 GiB of host memory.

    Pipelined per micro-batch on three streams (host->device, swap,
    device->host) over two device buffer sets: micro-batch m's swap-out starts
    as soon as its own upload lands, and its download starts as soon as its
    own swap-in is done, so both PCIe directions stay busy and the pipeline
    fills and drains by one micro-batch, not one step.  `pcie` reports the
    copies alone (no swap) on the same buffers: the ceiling e2e can reach."""
    import torch
    import numpy as np
    mb = len(src) if n == 1 else min(2, len(src))
    src, dst = src[:mb], dst[:mb]
    steps = max(1, args.e2e_steps)
    nt = len(sizes)
    L = _Local()
    st = {}
    src_free = [[None] * mb for _ in range(2)]   # (set, m): its swap-out has read src
    dst_free = [[None] * mb for _ in range(2)]   # (set, m): its download has read dst

    def setup():
        st["hsrc"] = [[torch.empty(s, dtype=torch.uint8, pin_memory=True) for s in sizes] for _ in range(mb)]
        st["hdst"] = [[torch.empty(s, dtype=torch.uint8, pin_memory=True) for s in sizes] for _ in range(mb)]
        for m in range(mb):
            for i in range(nt):
                st["hsrc"][m][i].copy_(src[m][i])
        st["srcs"] = [src, [[torch.empty_like(t) for t in row] for row in src]]
        st["dsts"] = [dst, [[torch.empty_like(t) for t in row] for row in dst]]
        st["h2d"], st["d2h"] = torch.cuda.Stream(), torch.cuda.Stream()
        torch.cuda.synchronize()

    def step(k):
        x = k % 2
        h2d, d2h, srcs, dsts = st["h2d"], st["d2h"], st["srcs"], st["dsts"]
        pl = mp.plan(world, source, per_copy, bw, sizes)
        hs = []
        for m in range(mb):
            if src_free[x][m] is not None:
                h2d.wait_event(src_free[x][m])
            with torch.cuda.stream(h2d):
                for i in range(nt):
                    srcs[x][m][i].copy_(st["hsrc"][m][i], non_blocking=True)
            up = torch.cuda.Event()
            up.record(h2d)
            stream.wait_event(up)
            hs.append(ctx.swap_out(pl, srcs[x][m], stream=stream))
            src_free[x][m] = torch.cuda.Event()
            src_free[x][m].record(stream)
        for m in range(mb):
            if dst_free[x][m] is not None:
                stream.wait_event(dst_free[x][m])
            ctx.swap_in(hs[m], dsts[x][m], stream=stream)
            done = torch.cuda.Event()
            done.record(stream)
            d2h.wait_event(done)
            with torch.cuda.stream(d2h):
                for i in range(nt):
                    st["hdst"][m][i].copy_(dsts[x][m][i], non_blocking=True)
            dst_free[x][m] = torch.cuda.Event()
            dst_free[x][m].record(d2h)
        for h in hs:
            h.free()

    def first():
        step(0)
        torch.cuda.synchronize()

    def timed():
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        st["h2d"].wait_stream(stream)
        for k in range(steps):
            step(k + 1)
        stream.wait_stream(st["d2h"])
        e1.record(stream)
        torch.cuda.synchronize()
        return e0.elapsed_time(e1)

    L(setup)
    L(first)
    if n > 1:
        dist.barrier()
    ms = L(timed)
    t = torch.tensor([ms or 0.0, 1.0 if L.err is not None else 0.0], dtype=torch.float64)
    if n > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if float(t[1]) > 0:
        return {"error": L.err or "another rank failed"}
    ms = float(t[0]) / steps
    per = 2 * mb * sum(sizes)
    hsrc, hdst = st["hsrc"], st["hdst"]
    ok = all(np.array_equal(hdst[m][i].numpy(), hsrc[m][i].numpy())
             for m in (0, mb - 1) for i in range(nt))
    try:
        pcie = leg_pcie(st["srcs"][0], st["dsts"][0], hsrc, hdst, st["h2d"], st["d2h"], stream)
    except Exception as exc:  # pragma: no cover - reported, not hidden
        pcie = {"error": "%s: %s" % (type(exc).__name__, exc)}
    return {"value": per / (ms / 1e3) / 1e9, "unit": "GB/s",
            "value_is": "per source GPU, like the headline",
            "all_ranks_gbs": n * per / (ms / 1e3) / 1e9,
            "h2d_bytes_per_step": mb * sum(sizes), "d2h_bytes_per_step": mb * sum(sizes),
            "micro_batches": mb,
            "steps": steps, "ms_per_step": ms, "round_trip_ok": bool(ok),
            "pipelining": "per micro-batch: upload(m) -> swap-out(m); swap-in(m) -> download(m); "
                          "3 streams, 2 device buffer sets",
            "pcie": pcie,
            "frac_of_pcie_duplex": ((per / (ms / 1e3) / 1e9) / pcie["duplex_gbs"]
                                    if "duplex_gbs" in pcie else None)}


def run_e2e_zero_copy(args, ctx, mp, world, source, per_copy, bw, sizes, n, dist):
    """The same metric through the C ABI with the HOST buffers themselves as
    the swap's tensors: pinned host memory is mapped into the device's
    address space (UVA), so mpress_swap_out reads the micro-batch straight
    from host memory over PCIe into the peers' stash and mpress_swap_in
    writes it straight back into host memory -- no device staging buffers,
    no separate copies.  Pipelined as the duplex leg: the swap-out of
    micro-batch m+1 (PCIe reads) beside the swap-in of m (PCIe writes) on
    two streams.  Every restored host byte is compared with the source."""
    import numpy as np
    import torch
    from synth import device as synth_dev
    # as run_e2e: N ranks on one host do not pin N x 14 GiB; never more
    # micro-batches than the partitions hold (out(m+1) beside in(m) needs 2)
    mb = min(args.micro_batches, MICRO_BATCHES if n == 1 else 2)
    nt = len(sizes)
    L = _Local()
    st = {}

    def setup():
        st["hsrc"] = [[torch.empty(x, dtype=torch.uint8, pin_memory=True) for x in sizes] for _ in range(mb)]
        st["hdst"] = [[torch.empty(x, dtype=torch.uint8, pin_memory=True) for x in sizes] for _ in range(mb)]
        for m in range(mb):
            for i in range(nt):
                t = torch.empty(sizes[i], dtype=torch.uint8, device="cuda")
                synth_dev.fill(t, 9000 + m, i)
                st["hsrc"][m][i].copy_(t)
        st["s_out"], st["s_in"] = torch.cuda.Stream(), torch.cuda.Stream()
        st["pl"] = mp.plan(world, source, per_copy, bw, sizes)

    def step():
        s_out, s_in = st["s_out"], st["s_in"]
        hs = [ctx.swap_out(st["pl"], st["hsrc"][0], stream=s_out)]
        for m in range(1, mb + 1):
            if m < mb:
                hs.append(ctx.swap_out(st["pl"], st["hsrc"][m], stream=s_out))
            ctx.swap_in(hs[m - 1], st["hdst"][m - 1], stream=s_in)
        return hs

    def timed():
        steps = max(1, args.e2e_steps)
        for h in step():          # warm-up
            h.free()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(st["s_out"])
        st["s_in"].wait_stream(st["s_out"])
        hs = []
        for _ in range(steps):
            hs += step()
        st["s_out"].wait_stream(st["s_in"])
        e1.record(st["s_out"])
        torch.cuda.synchronize()
        for h in hs:
            h.free()
        return e0.elapsed_time(e1) / steps

    L(setup)
    ms = L(timed)
    t = torch.tensor([ms or 0.0, 1.0 if L.err is not None else 0.0], dtype=torch.float64)
    if n > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    if float(t[1]) > 0:
        return {"error": L.err or "another rank failed"}
    ms = float(t[0])
    ok = all(np.array_equal(st["hdst"][m][i].numpy(), st["hsrc"][m][i].numpy())
             for m in range(mb) for i in range(nt))
    per = 2 * mb * sum(sizes)
    return {"value": per / (ms / 1e3) / 1e9, "unit": "GB/s", "micro_batches": mb, "ms_per_step": ms,
            "h2d_bytes_per_step": mb * sum(sizes), "d2h_bytes_per_step": mb * sum(sizes),
            "round_trip_ok": bool(ok),
            "how": "pinned host tensors passed to mpress_swap_out / mpress_swap_in (UVA): the swap kernels "
                   "read and write host memory over PCIe directly; out(m+1) || in(m) on two streams"}


def leg_pcie(src, dst, hsrc, hdst, h2d, d2h, stream, reps=3):
    """The e2e ceiling on this box: the same pinned copies with no swap --
    upload alone, download alone, and both at once (GB/s of copied bytes,
    best of `reps`).  e2e moves one upload and one download byte per swapped
    byte, so its ceiling is duplex_gbs."""
    import torch

    def timed(up, down):
        best = None
        for _ in range(reps):
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            h2d.wait_stream(stream)
            d2h.wait_stream(stream)
            for m in range(len(src)):
                for i in range(len(src[m])):
                    if up:
                        with torch.cuda.stream(h2d):
                            src[m][i].copy_(hsrc[m][i], non_blocking=True)
                    if down:
                        with torch.cuda.stream(d2h):
                            hdst[m][i].copy_(dst[m][i], non_blocking=True)
            stream.wait_stream(h2d)
            stream.wait_stream(d2h)
            e1.record(stream)
            torch.cuda.synchronize()
            ms = e0.elapsed_time(e1)
            best = ms if best is None else min(best, ms)
        nbytes = sum(t.numel() for row in src for t in row) * (int(up) + int(down))
        return nbytes / (best / 1e3) / 1e9

    return {"h2d_gbs": timed(True, False), "d2h_gbs": timed(False, True),
            "duplex_gbs": timed(True, True)}


if __name__ == "__main__":
    sys.exit(main())
