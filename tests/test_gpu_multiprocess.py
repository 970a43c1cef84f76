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


def _worker(rank, world, port, outdir, path):
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


@pytest.mark.parametrize("path", [0, 1])
def test_two_processes_one_gpu(path):
    with tempfile.TemporaryDirectory() as d:
        tmp.spawn(_worker, args=(2, _free_port(), d, path), nprocs=2, join=True)
        for r in range(2):
            assert open(os.path.join(d, "r%d.txt" % r)).read() == "ok"
