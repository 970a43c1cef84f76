"""CPU tests of the C ABI: the library loads without a GPU, exports every
symbol include/mpress.h declares, and its planner (a different algorithm:
water-fill + exact fix-up, csrc/plan.cpp) reproduces the oracle's plans
bit-exactly.  No compute call touches a GPU here."""
import os
import random
import re
import subprocess

import pytest

import oracle
from oracle import PlanError
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import workloads

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GOLDEN = os.path.join(ROOT, "tests", "golden")


def _declared():
    src = open(os.path.join(ROOT, "include", "mpress.h")).read()
    return sorted(set(re.findall(r"MPRESS_API\s+[\w\s\*]*?\b(mpress_\w+)\s*\(", src)))


def test_exports_every_declared_symbol():
    declared = _declared()
    assert len(declared) >= 20
    out = subprocess.run(["nm", "-D", "--defined-only", mp.LIB_PATH], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\sT\s(mpress_\w+)", out))
    assert set(declared) == exported
    assert set(declared) == set(mp.EXPORTED)
    for name in declared:
        assert hasattr(mp.lib, name)


def test_version_and_error_text():
    assert mp.lib.mpress_version() == 1
    with pytest.raises(mp.MPressError) as ei:
        mp.plan(2, 0, [0, 1 << 30], [0, 1], [100], granule=100)
    assert ei.value.code == mp.ERR_ARG
    assert "256" in str(ei.value)


def _compare(world, source, spare, bw, sizes, G):
    try:
        o = oracle.plan(world, source, spare, bw, sizes, G)
    except PlanError as e:
        with pytest.raises(mp.MPressError) as ei:
            mp.plan(world, source, spare, bw, sizes, G)
        assert ei.value.code == e.code
        return False
    c = mp.plan(world, source, spare, bw, sizes, G)
    assert c.units == o["units"]
    assert c.peer_bytes == o["peer_bytes"]
    assert c.stripes == [tuple(s) for s in o["stripes"]]
    info = c.info
    assert (info.virtual_bytes, info.units, info.granule) == (o["V"], o["K"], o["G"])
    assert info.n_stripes == len(o["stripes"]) and info.n_tensors == len(sizes)
    return True


@pytest.mark.parametrize("fname", sorted(f for f in os.listdir(GOLDEN) if f.startswith("g") and f.endswith(".json")))
def test_golden_parity(fname):
    import json
    g = json.load(open(os.path.join(GOLDEN, fname)))
    if "expect" in g:
        assert _compare(g["world"], g["source"], g["spare"], g["bw"], g["sizes"], g["granule"])
    else:
        assert _compare(g["world"], g["source"], g["feasible_spare"], g["bw"], g["sizes"], g["granule"])
        assert not _compare(g["world"], g["source"], g["infeasible_spare"], g["bw"], g["sizes"], g["granule"])


def test_random_plan_parity():
    """10 000 random instances (weights 0..900 and huge, caps binding or not)."""
    rng = random.Random(2023)
    feasible = 0
    for t in range(10000):
        world = rng.randint(1, 8)
        source = rng.randrange(world)
        G = 256 * rng.choice([1, 2, 3, 16, 256])
        kind = t % 4
        if kind == 0:    # small weights, many ties
            bw = [rng.choice([0, 1, 2, 3]) for _ in range(world)]
        elif kind == 1:  # NVLink-ish GB/s weights
            bw = [rng.choice([0, 25, 50, 100, 900]) for _ in range(world)]
        elif kind == 2:  # arbitrary
            bw = [rng.randint(0, 1000) for _ in range(world)]
        else:            # huge weights (128-bit cross products)
            bw = [rng.choice([0, (1 << 63) + rng.randint(0, 1 << 40), rng.randint(1, 1 << 62)]) for _ in range(world)]
        n = rng.randint(1, 12)
        sizes = [rng.choice([1, 15, 16, 17, 255, 256, 257, rng.randint(1, 40 * G)]) for _ in range(n)]
        V = oracle.virtual_layout(sizes)[1]
        K = (V + G - 1) // G
        spare = [rng.randint(0, 2 * K // max(1, world - 1) + 2) * G + rng.randint(0, G - 1) for _ in range(world)]
        feasible += _compare(world, source, spare, bw, sizes, G)
    assert feasible > 4000


def test_large_unit_counts_parity():
    """Water-fill starting point far from trivial: K ~ 1e5..1e6 units."""
    rng = random.Random(7)
    for _ in range(20):
        world = 8
        bw = [0] + [rng.randint(1, 1 << 20) for _ in range(7)]
        sizes = [rng.randint(1, 1 << 30) for _ in range(rng.randint(1, 5))]
        V = oracle.virtual_layout(sizes)[1]
        K = (V + 65535) // 65536
        spare = [0] + [rng.randint(K // 8, K) * 65536 for _ in range(7)]
        _compare(world, 0, spare, bw, sizes, 0)


@pytest.mark.parametrize("cfg", [1, 2, 3, 5])
def test_config_plans_parity(cfg):
    c = workloads.CONFIGS[cfg]
    if cfg == 1:
        sizes = workloads.cfg1_sizes()
    elif cfg == 2:
        sizes = workloads.cfg2_sizes(8)
    elif cfg == 3:
        sizes = workloads.cfg3_sizes()
    else:
        sizes = workloads.cfg5_source_sizes(0)
    if cfg == 3:
        spare = workloads.spare_vector(c["world"], 0, c["peers"], spare_by_peer=c["spare_by_peer"])
    else:
        spare = workloads.spare_vector(c["world"], 0, c["peers"], spare=c["spare"])
    bw = workloads.bw_vector(c["world"], 0, c["peers"])
    assert _compare(c["world"], 0, spare, bw, sizes, 0)


def test_config4_sweep_parity():
    for world, P in workloads.CONFIGS[4]["sweeps"]:
        peers = list(range(1, P + 1))
        spare = workloads.spare_vector(world, 0, peers, spare=workloads.CONFIGS[4]["spare"])
        bw = workloads.bw_vector(world, 0, peers)
        for s in workloads.cfg4_sizes():
            assert _compare(world, 0, spare, bw, [s], 0)


def test_partition_parity():
    rng = random.Random(12)
    for t in range(300):
        world = rng.randint(2, 8)
        spare = [rng.randint(0, 64) * 4096 for _ in range(world)]
        bwm = [[0 if s == p else rng.choice([0, 1, 2, 25, 50]) for p in range(world)] for s in range(world)]
        srcs = rng.sample(range(world), rng.randint(1, world))
        reqs = [(s, [rng.randint(1, 20000) for _ in range(rng.randint(1, 4))], rng.randint(1, 3)) for s in srcs]
        try:
            op, _ = oracle.sequential_partition(world, spare, bwm, reqs, 4096)
        except PlanError as e:
            with pytest.raises(mp.MPressError) as ei:
                mp.partition_sequential(world, spare, bwm, reqs, 4096)
            assert ei.value.code == e.code
            continue
        cp = mp.partition_sequential(world, spare, bwm, reqs, 4096)
        assert cp == op


def test_partition_config5_parity():
    c = workloads.CONFIGS[5]
    world = 8
    spare = workloads.spare_vector(world, 0, c["peers"], spare=c["spare"])
    bwm = [workloads.bw_vector(world, s, c["peers"]) for s in range(world)]
    reqs = [(s, workloads.cfg5_source_sizes(s), 1) for s in c["sources"]]
    op, _ = oracle.sequential_partition(world, spare, bwm, reqs)
    assert mp.partition_sequential(world, spare, bwm, reqs) == op


def test_init_argument_errors_without_gpu():
    """Partition validation happens before any CUDA call (R21: a source never
    stashes on itself; partitions are 256-byte multiples)."""
    import ctypes
    P = ctypes.c_void_p
    h = P()
    devs = (ctypes.c_int * 2)(0, 0)
    bad_self = (ctypes.c_uint64 * 4)(256, 0, 0, 0)
    assert mp.lib.mpress_init_local(2, 0, devs, bad_self, ctypes.byref(h)) == mp.ERR_ARG
    assert "itself" in mp.lib.mpress_last_error().decode()
    bad_align = (ctypes.c_uint64 * 4)(0, 100, 0, 0)
    assert mp.lib.mpress_init_local(2, 0, devs, bad_align, ctypes.byref(h)) == mp.ERR_ARG
    assert mp.lib.mpress_init_local(2, 2, devs, bad_align, ctypes.byref(h)) == mp.ERR_ARG
    assert mp.lib.mpress_finalize(None) == 0
    assert mp.lib.mpress_autotune(None, 1 << 20, 3, None, None) == mp.ERR_ARG
    v = ctypes.c_int64()
    assert mp.lib.mpress_get_option(None, mp.OPT_AUTO_OUT, ctypes.byref(v)) == mp.ERR_ARG
    with pytest.raises(mp.MPressError) as ei:
        mp.plan(3, 0, [0, 1], [0, 1, 1], [10])
    assert ei.value.code == mp.ERR_ARG


def test_plan_overflow_and_zero_size_rejected():
    with pytest.raises(mp.MPressError) as ei:
        mp.plan(2, 0, [0, 1 << 40], [0, 1], [1 << 63, 1 << 63])
    assert ei.value.code == mp.ERR_ARG
    with pytest.raises(mp.MPressError) as ei:
        mp.plan(2, 0, [0, 1 << 40], [0, 1], [5, 0])
    assert ei.value.code == mp.ERR_ARG


def test_header_constants_match_the_binding():
    """Every integer constant include/mpress.h defines (options, paths,
    orders, transports, states, errors, choices) has a twin with the same
    value in the package namespace (MPRESS_X -> mp.X), so a constant added to
    the ABI cannot be missing from the binding the bench and tests use."""
    src = open(os.path.join(ROOT, "include", "mpress.h")).read()
    defs = dict(re.findall(r"#define\s+MPRESS_(\w+)\s+\(?(-?\d+)u?\)?", src))
    skip = {"VERSION"}
    checked = 0
    for name, val in defs.items():
        if name in skip:
            continue
        assert hasattr(mp, name), "mp.%s missing (MPRESS_%s in mpress.h)" % (name, name)
        assert getattr(mp, name) == int(val), name
        checked += 1
    assert checked >= 30
