"""NEXT-1: joint plan of several exporters (Fig. 6, score P:213,
reading R23).  CPU only.

Pins of the oracle: the candidate-scan oracle equals exhaustive enumeration
on tiny inputs; with one exporter and no ports the joint optimum reduces to
the single-source planner's makespan (itself pinned by brute force and the
paper's worked ratio, tests/test_oracle.py).  Parity of the library: the
optimal time T* is unique and must match exactly; the assignment is one of
many optima (R19), so it is checked for validity and for reaching T*."""
import random
from fractions import Fraction

import pytest

import oracle
from oracle import PlanError, ERR_NO_SPACE
import paper_conf_hpca_zhouwylbyx23_b200 as mp
from synth import workloads


def _random_case(rng, max_world=5, max_units=5, ports=False):
    world = rng.randint(2, max_world)
    n_src = rng.randint(1, min(3, world))
    sources = rng.sample(range(world), n_src)
    G = 256
    spare = [rng.randint(0, max_units) * G + rng.randint(0, 255) for _ in range(world)]
    bw = [[0 if s == p else rng.choice([0, 1, 2, 3, 5]) for p in range(world)] for s in range(world)]
    reqs = [(s, [rng.randint(1, max_units * G) for _ in range(rng.randint(1, 2))]) for s in sources]
    eg = [rng.choice([0, 2, 3, 7]) for _ in range(world)] if ports else None
    ig = [rng.choice([0, 2, 3, 7]) for _ in range(world)] if ports else None
    return world, sources, reqs, spare, bw, eg, ig, G


def _demands(reqs, G):
    return [oracle.global_plan.demand_units(sz, G) for _, sz in reqs]


@pytest.mark.parametrize("ports", [False, True])
def test_scan_oracle_equals_brute_force(ports):
    rng = random.Random(156 + ports)
    checked = 0
    for _ in range(400):
        world, sources, reqs, spare, bw, eg, ig, G = _random_case(rng, ports=ports)
        K = _demands(reqs, G)
        if sum(K) > 7:
            continue
        try:
            b = oracle.brute_force_global(world, sources, K, spare, bw, eg, ig, G)
        except PlanError as e:
            assert e.code == ERR_NO_SPACE
            with pytest.raises(PlanError):
                oracle.scan_global(world, sources, K, spare, bw, eg, ig, G)
            continue
        T, x = oracle.scan_global(world, sources, K, spare, bw, eg, ig, G)
        assert T == b
        assert oracle.assignment_time(x, sources, world, bw, eg, ig) <= T
        checked += 1
    assert checked > 100


def test_single_exporter_reduces_to_the_planner():
    """One exporter, no ports: T* = min max k_p/B_p = the planner's makespan (R1)."""
    rng = random.Random(213)
    for _ in range(200):
        world = rng.randint(2, 6)
        s = rng.randrange(world)
        G = 256
        spare = [rng.randint(0, 12) * G for _ in range(world)]
        bw = [[0 if a == p else rng.choice([0, 1, 2, 25, 50]) for p in range(world)] for a in range(world)]
        sizes = [rng.randint(1, 10 * G)]
        try:
            pl = oracle.plan(world, s, spare, bw[s], sizes, G)
        except PlanError:
            continue
        T, _ = oracle.scan_global(world, [s], [pl["K"]], spare, bw, None, None, G)
        assert T == oracle.makespan(pl["units"], [b if b else 1 for b in bw[s]])


def _check_library(world, reqs, spare, bw, eg, ig, G):
    sources = [s for s, _ in reqs]
    K = _demands(reqs, G)
    try:
        T, _ = oracle.scan_global(world, sources, K, spare, bw, eg, ig, G)
    except PlanError as e:
        with pytest.raises(mp.MPressError) as ei:
            mp.plan_global(world, reqs, spare, bw, eg, ig, G)
        assert ei.value.code == e.code
        return False
    units, (num, den) = mp.plan_global(world, reqs, spare, bw, eg, ig, G)
    assert Fraction(num, den) == T
    x = [units[s] for s in sources]
    caps = [sp // G for sp in spare]
    for si, s in enumerate(sources):
        assert sum(x[si]) == K[si]
        for p in range(world):
            if x[si][p]:
                assert p != s and bw[s][p] > 0
    for p in range(world):
        assert sum(x[si][p] for si in range(len(sources))) <= caps[p]
    assert oracle.assignment_time(x, sources, world, bw, eg, ig) == T
    # every row is a valid plan, identical to the oracle's layout of that split
    for (s, sizes), row in zip(reqs, x):
        c = mp.plan_from_units(world, s, row, sizes, G)
        o = oracle.plan_from_units(world, s, row, sizes, G)
        assert c.stripes == [tuple(t) for t in o["stripes"]]
        assert c.peer_bytes == o["peer_bytes"]
    return True


@pytest.mark.parametrize("ports", [False, True])
def test_library_matches_oracle(ports):
    rng = random.Random(204 + ports)
    ok = 0
    for _ in range(300):
        world, sources, reqs, spare, bw, eg, ig, G = _random_case(rng, max_world=6, max_units=12,
                                                                  ports=ports)
        ok += _check_library(world, reqs, spare, bw, eg, ig, G)
    assert ok > 100


def test_dgx1_ratio_two_exporters():
    """P:153 weights (GPU0->GPU3 twice GPU0->GPU1) with two exporters sharing
    GPU3: the joint optimum is checked against the oracle."""
    world, G = 4, 4096
    bw = [[0, 25, 0, 50], [0, 0, 25, 50], [0] * 4, [0] * 4]
    spare = [0, 0, 64 * G, 48 * G]
    reqs = [(0, [30 * G]), (1, [30 * G])]
    assert _check_library(world, reqs, spare, bw, None, None, G)


def test_config5_nvswitch_ports():
    """Config 5 (BJ:11, Table IV): sources 0-3 -> importers 4-7 on
    NVSwitch (equal links, 900 GB/s ports).  The joint optimum is bounded
    below by source 0's egress (its 3.5 GiB at one port) and the sequential
    plans (R12) already reach it; the joint planner must not do worse."""
    c = workloads.CONFIGS[5]
    world, G = 8, 1 << 20   # 1 MiB units keep the scan oracle fast
    spare = workloads.spare_vector(world, 0, c["peers"], spare=c["spare"])
    bw = [workloads.bw_vector(world, s, c["peers"], weight=900) for s in range(world)]
    reqs = [(s, workloads.cfg5_source_sizes(s)) for s in c["sources"]]
    eg = [900] * world
    ig = [900] * world
    units, (num, den) = mp.plan_global(world, reqs, spare, bw, eg, ig, G)
    K0 = oracle.global_plan.demand_units(reqs[0][1], G)
    assert Fraction(num, den) == Fraction(K0, 900)   # egress-bound at source 0
    # the sequential partition's time under the same model
    part, plans = oracle.sequential_partition(world, spare, bw, [(s, sz, 1) for s, sz in reqs], G)
    x = [plans[s]["units"] for s, _ in reqs]
    seq = oracle.assignment_time(x, [s for s, _ in reqs], world, bw, eg, ig)
    assert Fraction(num, den) <= seq


def test_capacity_bound_joint_beats_sequential():
    """When an importer's spare binds, planning sources one after the other
    (R12) can strand a later source on slow links; the joint plan cannot be
    worse and here is strictly better."""
    world, G = 4, 4096
    bw = [[0, 0, 4, 4], [0, 0, 4, 1], [0] * 4, [0] * 4]
    spare = [0, 0, 8 * G, 8 * G]
    reqs = [(0, [8 * G]), (1, [8 * G])]
    units, (num, den) = mp.plan_global(world, reqs, spare, bw, None, None, G)
    _, plans = oracle.sequential_partition(world, spare, bw, [(s, sz, 1) for s, sz in reqs], G)
    seq = oracle.assignment_time([plans[0]["units"], plans[1]["units"]], [0, 1], world, bw, None, None)
    # sequential strands source 1 on its slow link (T = 4); jointly, source 0
    # keeps 1 unit on GPU2 and 7 on GPU3, source 1 takes 7 on GPU2 and 1 on
    # GPU3: T = max(7/4, 1/1) = 7/4 (hand-checked: a = 1 minimises
    # max(a, (8-a)/4) over the split a + b = 8 the capacities force)
    assert seq == 4 and Fraction(num, den) == Fraction(7, 4)
    assert _check_library(world, reqs, spare, bw, None, None, G)


def test_errors():
    with pytest.raises(mp.MPressError) as ei:
        mp.plan_global(3, [(0, [4096]), (0, [4096])], [0, 1 << 20, 1 << 20], [[0, 1, 1]] * 3, granule=4096)
    assert ei.value.code == mp.ERR_ARG
    with pytest.raises(mp.MPressError) as ei:
        mp.plan_global(2, [(0, [1 << 20])], [0, 4096], [[0, 1], [1, 0]], granule=4096)
    assert ei.value.code == mp.ERR_NO_SPACE
    with pytest.raises(mp.MPressError) as ei:
        mp.plan_from_units(3, 0, [1, 0, 0], [4096], 4096)
    assert ei.value.code == mp.ERR_ARG
    with pytest.raises(mp.MPressError) as ei:
        mp.plan_from_units(3, 0, [0, 2, 0], [4096], 4096)
    assert ei.value.code == mp.ERR_ARG
