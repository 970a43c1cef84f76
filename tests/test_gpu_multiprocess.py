"""The cross-process peer-mapping path on one GPU: two processes (both on
cuda:0, as torchrun would place ranks on GPUs 0 and 1), each exporting a cuMem
stash pool as a POSIX fd, receiving the other's over SCM_RIGHTS, mapping it
and swapping into it.  This is the code path of an N-GPU run; only the
physical link differs (HBM instead of NVLink)."""
import os
import socket
import tempfile

import pytest
import torch.multiprocessing as tmp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, outdir, path, transport="fd"):
    import numpy as np
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    if transport == "legacy":
        os.environ["MPRESS_IPC"] = "legacy"   # CUDA IPC handles via the all-gather
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import paper_conf_hpca_zhouwylbyx23_b200 as mp
    from synth import device as synth_dev
    from synth import splitmix64_bytes

    sizes = [1000 + 37 * rank, 3 << 20, 5, 70001]
    spare = [256 << 20] * world
    bwm = [[0 if s == p else 1 for p in range(world)] for s in range(world)]
    reqs = [(s, sizes, 2) for s in range(world)]   # every rank is a source
    part = mp.partition_sequential(world, spare, bwm, reqs, 4096)
    ctx = mp.Context.distributed(0, world, rank, part)
    err = ""
    try:
        ctx.set_option(mp.OPT_PATH, path)
        want = mp.TRANSPORT_LEGACY_IPC if transport == "legacy" else mp.TRANSPORT_VMM_FD
        assert ctx.get_option(mp.OPT_TRANSPORT) == want
        if path == mp.PATH_AUTO:   # collective probe on the real (here: loopback) peers
            res = ctx.autotune(probe_bytes=8 << 20, trials=2)
            assert res["out"] in (mp.PATH_DIRECT, mp.PATH_BULK) and res["in"] in (mp.PATH_DIRECT, mp.PATH_BULK)
            assert all(v > 0 for v in res["ms"].values()), res
        per_copy = [r // 2 for r in spare]
        pl = mp.plan(world, rank, per_copy, bwm[rank], sizes, 4096)
        o = oracle.plan(world, rank, per_copy, bwm[rank], sizes, 4096)
        assert pl.stripes == [tuple(s) for s in o["stripes"]]
        seed = 500 + rank
        src = []
        for i, n in enumerate(sizes):
            t = torch.empty(n, dtype=torch.uint8, device="cuda")
            synth_dev.fill(t, seed, i)
            src.append(t)
        torch.cuda.synchronize()
        h = ctx.swap_out(pl, src)
        torch.cuda.synchronize()
        host = [splitmix64_bytes(seed, i, 0, n) for i, n in enumerate(sizes)]
        model = oracle.swap_out(o, host)
        sl = h.slices()
        for p, (buf, defined) in model.items():
            got = np.frombuffer(ctx.peer_read(p, sl[p], len(buf)), dtype=np.uint8)
            assert not np.any((got != buf) & defined), "stash bytes differ on peer %d" % p
        dist.barrier()   # both ranks wrote into each other's pools
        for t in src:
            t.fill_(0)
        dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
        ctx.swap_in(h, dst)
        torch.cuda.synchronize()
        for i, d in enumerate(dst):
            assert synth_dev.check(d, seed, i) == 0, "tensor %d not restored" % i
        h.free()
    except Exception as e:  # report through the file so the parent sees it
        err = repr(e)
    finally:
        ctx.finalize()
    with open(os.path.join(outdir, "r%d.txt" % rank), "w") as f:
        f.write(err or "ok")
    dist.destroy_process_group()


@pytest.mark.parametrize("path,transport", [(0, "fd"), (1, "fd"), (0, "legacy"), (3, "fd")])
def test_two_processes_one_gpu(path, transport):
    with tempfile.TemporaryDirectory() as d:
        tmp.spawn(_worker, args=(2, _free_port(), d, path, transport), nprocs=2, join=True)
        for r in range(2):
            assert open(os.path.join(d, "r%d.txt" % r)).read() == "ok"


def _cfg5_worker(rank, world, port, outdir):
    """Config 5 topology (Table IV): sources 0-3 swap (4-s) scaled
    Bert micro-batch sets into importers 4-7 concurrently; sequential partition
    (R12) computed identically on every rank."""
    import numpy as np
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import paper_conf_hpca_zhouwylbyx23_b200 as mp
    from synth import device as synth_dev
    from synth import splitmix64_bytes, workloads

    def sizes_of(s):  # 1/64-scale Bert sets, ragged tails
        return [max(1, b // 64 + 7 * s) for b in workloads.cfg5_source_sizes(s)]

    sources, peers = [0, 1, 2, 3], [4, 5, 6, 7]
    spare = [0] * 4 + [400 << 20] * 4
    bwm = [[1 if (s in sources and p in peers) else 0 for p in range(world)] for s in range(world)]
    reqs = [(s, sizes_of(s), 1) for s in sources]
    part = mp.partition_sequential(world, spare, bwm, reqs)
    opart, oplans = oracle.sequential_partition(world, spare, bwm, reqs)
    err = "" if part == opart else "partition differs from the oracle"
    ctx = mp.Context.distributed(0, world, rank, part)
    try:
        # collective: the importers (no peers of their own) only join the barriers
        res = ctx.autotune(probe_bytes=4 << 20, trials=1)
        if rank in peers:
            assert all(v == 0 for v in res["ms"].values()), res
            assert res["out"] == res["in"] == mp.PATH_BULK
            assert res["out_small"] == res["in_small"] == mp.PATH_DIRECT
        else:
            assert all(v > 0 for v in res["ms"].values()), res
        if rank in sources and not err:
            sizes = sizes_of(rank)
            rem = list(spare)
            for s in sources:   # the spare each source planned against
                if s == rank:
                    break
                rem = [r - part[s][p] for p, r in enumerate(rem)]
            pl = mp.plan(world, rank, rem, bwm[rank], sizes)
            o = oplans[rank]
            assert pl.stripes == [tuple(x) for x in o["stripes"]]
            src = []
            for i, n in enumerate(sizes):
                t = torch.empty(n, dtype=torch.uint8, device="cuda")
                synth_dev.fill(t, 5000 + rank, i)
                src.append(t)
            torch.cuda.synchronize()
            h = ctx.swap_out(pl, src)
            torch.cuda.synchronize()
            host = [splitmix64_bytes(5000 + rank, i, 0, n) for i, n in enumerate(sizes)]
            sl = h.slices()
            for p, (buf, defined) in oracle.swap_out(o, host).items():
                got = np.frombuffer(ctx.peer_read(p, sl[p], len(buf)), dtype=np.uint8)
                assert not np.any((got != buf) & defined), "stash differs on peer %d" % p
            dst = [torch.empty(n, dtype=torch.uint8, device="cuda") for n in sizes]
            ctx.swap_in(h, dst)
            torch.cuda.synchronize()
            for i, d in enumerate(dst):
                assert synth_dev.check(d, 5000 + rank, i) == 0
            h.free()
        dist.barrier()
    except Exception as e:
        err = repr(e)
    finally:
        ctx.finalize()
    with open(os.path.join(outdir, "r%d.txt" % rank), "w") as f:
        f.write(err or "ok")
    dist.destroy_process_group()


def test_config5_eight_processes_one_gpu():
    with tempfile.TemporaryDirectory() as d:
        tmp.spawn(_cfg5_worker, args=(8, _free_port(), d), nprocs=8, join=True)
        for r in range(8):
            assert open(os.path.join(d, "r%d.txt" % r)).read() == "ok", r


def test_bench_torchrun_two_ranks_one_gpu():
    """bench.py's N>1 path (every rank a source and an importer, mpress_init
    over the process group) under torchrun, both ranks on the one GPU."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=%d" % _free_port(), "bench.py", "--gpus", "2",
           "--steps", "3", "--warmup", "1", "--micro-batches", "2", "--e2e-steps", "1", "--no-gemm",
           "--ss-sizes", "4096,1048576,67108864"]
    r = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["value"] > 0 and line["roofline"]["bound"] == "nvlink"
    assert "bit-exact" in line["parity"]
    # value is per source GPU; the whole-job sum is its own key
    assert line["value"] == line["per_rank_gbs"] and abs(line["all_ranks_gbs"] - 2 * line["value"]) < 1e-6
    # config 4 single source: P = 1 peer at N = 2, three sizes x three paths, out and in
    ss = line["single_source"]
    assert ss["error"] is None and ss["all_bit_exact"], ss
    assert {(r["peers"], r["bytes"], r["path"]) for r in ss["rows"]} == \
        {(1, b, p) for b in (4096, 1048576, 67108864) for p in ("direct", "bulk", "ce")}
    assert all(r["out_gbs"] > 0 and r["in_gbs"] > 0 for r in ss["rows"])
    d = line["duplex"]
    assert d["bit_exact"] and line["duplex_gbs"] == d["duplex_gbs"] > 0


def test_bench_cfg5_leg_two_ranks_one_gpu():
    """bench.py's config-5 leg (sources = first half of the ranks, importers =
    second half, GEMMs on every rank) under torchrun, both ranks on one GPU:
    every collective is reached, bytes come back bit-exact, the line carries
    per-source GB/s and per-rank GEMM slowdowns."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", "--master-port=%d" % _free_port(), "bench.py", "--gpus", "2",
           "--steps", "2", "--warmup", "1", "--micro-batches", "1", "--e2e-steps", "1", "--gemm-n", "2048",
           "--gemm-window", "200", "--gemm-window-rounds", "2"]
    r = subprocess.run(cmd, cwd=root, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([l for l in r.stdout.splitlines() if l.startswith("{")][-1])
    c5 = line["cfg5"]
    assert "error" not in c5, c5
    assert c5["bit_exact"] and len(c5["per_source_gbs"]) == 1 and c5["per_source_gbs"][0] > 0
    assert len(c5["gemm_slowdown_per_rank"]) == 2
    assert "error" not in line["gemm_slowdown"], line["gemm_slowdown"]
