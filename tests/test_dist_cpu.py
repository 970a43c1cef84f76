"""Multi-process host logic on CPU (gloo, world size 2 and 3): the fd-passing
rendezvous mpress_init uses for cuMem pool handles (SCM_RIGHTS over Unix
sockets, csrc/fdpass.cpp), driven through the torch process-group exchange
callback, and the rank-independence of plans/partitions (§8(b) multi-source:
every rank computes the same table with no communication)."""
import os
import socket
import tempfile

import pytest
import torch.multiprocessing as tmp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, want_matrix, outdir):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_hpca_zhouwylbyx23_b200 as mp
    from synth import workloads

    fd = os.memfd_create("mpress-test-%d" % rank)
    os.write(fd, ("payload-of-rank-%d" % rank).encode())
    cb = mp.torch_exchange()
    fds = mp.share_fds(world, rank, fd, want_matrix[rank], cb)
    got = {}
    for p, f in enumerate(fds):
        if f >= 0:
            os.lseek(f, 0, os.SEEK_SET)
            got[p] = os.read(f, 64).decode()
            os.close(f)
    os.close(fd)

    # every rank computes the same partition table (no communication)
    c = workloads.CONFIGS[5]
    spare = workloads.spare_vector(8, 0, c["peers"], spare=c["spare"])
    bwm = [workloads.bw_vector(8, s, c["peers"]) for s in range(8)]
    reqs = [(s, workloads.cfg5_source_sizes(s), 2) for s in c["sources"]]
    part = mp.partition_sequential(8, spare, bwm, reqs)
    with open(os.path.join(outdir, "r%d.txt" % rank), "w") as f:
        f.write(repr((got, part)))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,want", [
    (2, [[0, 1], [1, 0]]),
    (3, [[0, 1, 1], [0, 0, 0], [1, 1, 0]]),
])
def test_share_fds_gloo(world, want):
    with tempfile.TemporaryDirectory() as d:
        for attempt in range(2):
            try:
                tmp.spawn(_worker, args=(world, _free_port(), want, d), nprocs=world, join=True)
                break
            except Exception as exc:  # the probed port can be taken before gloo's store binds it
                msg = str(exc).lower()
                if attempt or not any(k in msg for k in ("address", "port", "store", "connect")):
                    raise
        results = [eval(open(os.path.join(d, "r%d.txt" % r)).read()) for r in range(world)]
    for r, (got, part) in enumerate(results):
        expect = {p: "payload-of-rank-%d" % p for p in range(world) if want[r][p] and p != r}
        assert got == expect
        assert part == results[0][1]


def _slow_rank1_worker(rank, world, port, outdir):
    """Rank 1 enters the listen barrier (exchange #2) 3 s late, so a foreign
    process can reach rank 0's socket first."""
    import ctypes
    import time
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import paper_conf_hpca_zhouwylbyx23_b200 as mp

    inner = mp.torch_exchange()
    calls = [0]

    def slow(user, mine, ln, out):
        calls[0] += 1
        if rank == 1 and calls[0] == 2:
            time.sleep(3.0)
        return inner(user, mine, ln, out)
    from paper_conf_hpca_zhouwylbyx23_b200.api import EXCHANGE_FN
    cb = EXCHANGE_FN(slow)
    fd = os.memfd_create("mpress-peercred-%d" % rank)
    os.write(fd, ("payload-of-rank-%d" % rank).encode())
    fds = mp.share_fds(world, rank, fd, [[0, 0], [1, 0]][rank], cb)
    got = None
    if fds[0] >= 0:
        os.lseek(fds[0], 0, os.SEEK_SET)
        got = os.read(fds[0], 64).decode()
    with open(os.path.join(outdir, "r%d.txt" % rank), "w") as f:
        f.write(repr(got))
    dist.barrier()
    dist.destroy_process_group()


def test_share_fds_refuses_foreign_peer():
    """the abstract socket name is visible in /proc/net/unix, so a
    process that is not one of the job's ranks can connect.  It must get no
    descriptor (SO_PEERCRED check), its connection must not use up the
    served rank's slot, and rank 1 must still receive rank 0's fd."""
    import array
    import time
    with tempfile.TemporaryDirectory() as d:
        before = set(open("/proc/net/unix").read().split())
        ctx = tmp.spawn(_slow_rank1_worker, args=(2, _free_port(), d), nprocs=2, join=False)
        name, t0 = None, time.time()
        while name is None and time.time() - t0 < 60:
            for tok in open("/proc/net/unix").read().split():
                if tok.startswith("@mpress.") and tok.endswith(".0") and tok not in before:
                    name = tok
            time.sleep(0.01)
        assert name is not None, "rank 0 never listened"
        s = socket.socket(socket.AF_UNIX, socket.SOCK_STREAM)
        s.settimeout(30)
        s.connect("\0" + name[1:])
        fds = array.array("i")
        msg, anc, _, _ = s.recvmsg(16, socket.CMSG_LEN(fds.itemsize))
        s.close()
        assert msg == b"" and anc == [], "a foreign process received the pool descriptor"
        while not ctx.join():
            pass
        assert eval(open(os.path.join(d, "r1.txt")).read()) == "payload-of-rank-0"
