"""Pins of the oracle against what the paper and the mathematics fix.

None of these checks re-types the oracle's own loop: they use golden plans
derived by hand from the paper's passages (tests/golden/*.json), exhaustive
search of the P:213 objective, a continuous water-fill bound for P:209
proportionality, invariants of Fig. 6 line 3 (capacity), a per-byte
virtual-address definition of the stash content, and the round-trip identity
(P:378).  Runs on CPU only.
"""
import glob
import json
import os
import random
from fractions import Fraction

import numpy as np
import pytest

import oracle
from oracle import PlanError, ERR_ARG, ERR_NO_SPACE
from synth import splitmix64_bytes, workloads

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- golden plans

@pytest.mark.parametrize("fname", ["g1_weights_caps_padding.json", "g2_dgx1_ratio.json",
                                   "g3_config1.json", "g4_symmetric.json"])
def test_golden_plan(fname):
    g = _golden(fname)
    pl = oracle.plan(g["world"], g["source"], g["spare"], g["bw"], g["sizes"], g["granule"])
    e = g["expect"]
    assert pl["offsets"] == e["offsets"]
    assert pl["V"] == e["V"] and pl["K"] == e["K"]
    assert pl["units"] == e["units"]
    assert pl["peer_bytes"] == e["peer_bytes"]
    assert [list(s) for s in pl["stripes"]] == e["stripes"]
    assert oracle.makespan(pl["units"], [b if b else 1 for b in g["bw"]]) == Fraction(*e["makespan"])


def test_golden_no_space_boundary():
    g = _golden("g5_no_space_boundary.json")
    pl = oracle.plan(g["world"], g["source"], g["feasible_spare"], g["bw"], g["sizes"], g["granule"])
    assert pl["units"] == g["expect_feasible_units"]
    with pytest.raises(PlanError) as ei:
        oracle.plan(g["world"], g["source"], g["infeasible_spare"], g["bw"], g["sizes"], g["granule"])
    assert ei.value.code == ERR_NO_SPACE


def test_argument_errors():
    with pytest.raises(PlanError) as ei:
        oracle.plan(2, 0, [0, 1 << 30], [0, 1], [100], granule=100)
    assert ei.value.code == ERR_ARG
    with pytest.raises(PlanError) as ei:
        oracle.plan(2, 2, [0, 1 << 30], [0, 1], [100])
    assert ei.value.code == ERR_ARG
    with pytest.raises(PlanError) as ei:
        oracle.plan(2, 0, [0, 1 << 30], [0, 1], [])
    assert ei.value.code == ERR_ARG


def test_source_and_zero_weight_excluded():
    # R10: the source's own entry is ignored and weight 0 means "not a neighbour"
    pl = oracle.plan(4, 1, [1 << 30] * 4, [5, 9, 0, 5], [1 << 20], granule=4096)
    assert pl["units"][1] == 0 and pl["units"][2] == 0
    assert pl["units"][0] + pl["units"][3] == 256


# ---------------------------------------------------------------- random instance helpers

def _random_instance(rng, max_world=8, max_units=60, max_cap=30, weights=None):
    world = rng.randint(2, max_world)
    source = rng.randrange(world)
    G = 256 * rng.choice([1, 2, 4, 16])
    spare = [rng.randint(0, max_cap) * G + rng.randint(0, G - 1) for _ in range(world)]
    wpool = weights or list(range(0, 901))
    bw = [rng.choice(wpool) for _ in range(world)]
    n = rng.randint(1, 6)
    total = rng.randint(1, max_units) * G
    sizes = []
    for _ in range(n):
        sizes.append(max(1, rng.randint(1, max(1, total // n))))
    return world, source, spare, bw, sizes, G


def _cands(world, source, spare, bw, G):
    return [p for p in range(world) if p != source and bw[p] > 0 and spare[p] // G > 0]


def _water_fill(K, caps, bw):
    """Continuous x_p = min(cap_p, lam*B_p) with sum x_p = K (exact Fractions)."""
    lo, hi = Fraction(0), Fraction(max(c for c in caps) , min(bw)) + 1
    pts = sorted({Fraction(c, b) for c, b in zip(caps, bw)} | {Fraction(0)})
    # find the segment in which the piecewise-linear total reaches K
    def total(lam):
        return sum(min(Fraction(c), lam * b) for c, b in zip(caps, bw))
    prev = Fraction(0)
    for t in pts + [hi]:
        if total(t) >= K:
            # linear on [prev, t]
            free = sum(b for c, b in zip(caps, bw) if Fraction(c, b) > prev)
            base = total(prev)
            lam = prev + (K - base) / free
            return [min(Fraction(c), lam * b) for c, b in zip(caps, bw)]
        prev = t
    raise AssertionError("infeasible water fill")


def _check_invariants(pl, world, source, spare, bw, sizes, G):
    units, pb, st = pl["units"], pl["peer_bytes"], pl["stripes"]
    K = pl["K"]
    assert sum(units) == K
    for p in range(world):
        # Fig. 6 line 3: never exceed the peer's spare memory
        assert pb[p] <= units[p] * G <= spare[p]
        if p == source or bw[p] == 0:
            assert units[p] == 0
    # stripes cover every tensor exactly once (sum of sub-block sizes = tensor size)
    cover = [[] for _ in sizes]
    for (i, p, so, do, ln) in st:
        assert ln > 0
        cover[i].append((so, so + ln))
        assert do + ln <= pb[p]
        assert so % 256 == 0 and do % 256 == 0
    for i, s in enumerate(sizes):
        iv = sorted(cover[i])
        assert iv[0][0] == 0 and iv[-1][1] == s
        for a, b in zip(iv, iv[1:]):
            assert a[1] == b[0]
    # stash ranges of one peer never overlap
    for p in range(world):
        iv = sorted((do, do + ln) for (i, q, so, do, ln) in st if q == p)
        for a, b in zip(iv, iv[1:]):
            assert a[1] <= b[0]


# ---------------------------------------------------------------- P:213 optimality (brute force)

def test_brute_force_optimal_makespan():
    rng = random.Random(213)
    checked = 0
    for _ in range(3000):
        world = rng.randint(2, 5)
        source = rng.randrange(world)
        G = 256
        spare = [rng.randint(0, 10) * G for _ in range(world)]
        bw = [rng.choice([0, 1, 2, 3, 5, 25, 50]) for _ in range(world)]
        sizes = [rng.randint(1, 6 * G) for _ in range(rng.randint(1, 3))]
        cands = _cands(world, source, spare, bw, G)
        K = (oracle.virtual_layout(sizes)[1] + G - 1) // G
        if K > 14 or len(cands) > 4:
            continue
        best = oracle.brute_force_makespan(K, [spare[p] // G for p in cands], [bw[p] for p in cands])
        try:
            pl = oracle.plan(world, source, spare, bw, sizes, G)
        except PlanError as e:
            assert e.code == ERR_NO_SPACE
            assert best is None           # infeasibility agrees with exhaustive search
            continue
        assert best is not None
        assert oracle.makespan(pl["units"], [b if b else 1 for b in bw]) == best
        _check_invariants(pl, world, source, spare, bw, sizes, G)
        checked += 1
    assert checked > 1000


# ---------------------------------------------------------------- P:209 proportionality

def test_bandwidth_proportional_bound():
    """x_p - 1 < k_p <= x_p + P - 1, x = continuous capped water-fill (P:209 + P:160)."""
    rng = random.Random(209)
    for _ in range(1500):
        world, source, spare, bw, sizes, G = _random_instance(rng)
        cands = _cands(world, source, spare, bw, G)
        try:
            pl = oracle.plan(world, source, spare, bw, sizes, G)
        except PlanError as e:
            assert e.code == ERR_NO_SPACE
            assert sum(spare[p] // G for p in cands) < (oracle.virtual_layout(sizes)[1] + G - 1) // G
            continue
        _check_invariants(pl, world, source, spare, bw, sizes, G)
        x = _water_fill(pl["K"], [spare[p] // G for p in cands], [bw[p] for p in cands])
        P = len(cands)
        for xp, p in zip(x, cands):
            k = pl["units"][p]
            assert xp - 1 < k <= xp + P - 1


def test_symmetric_equal_subblocks():
    """P:151 on equal links and ample spare: k_p in {floor(K/P), ceil(K/P)}, extras to low indices."""
    rng = random.Random(151)
    for _ in range(300):
        P = rng.randint(1, 7)
        world = P + 1
        K = rng.randint(1, 200)
        G = 4096
        pl = oracle.plan(world, 0, [0] + [1 << 40] * P, [0] + [3] * P, [K * G], G)
        q, r = divmod(K, P)
        assert pl["units"] == [0] + [q + 1] * r + [q] * (P - r)


# ---------------------------------------------------------------- byte model

def _virtual_address_expectation(pl, tensors, p):
    """Per-byte definition: stash byte x of peer p holds virtual address a = O_p + x,
    i.e. byte a - off_i of the tensor i with off_i <= a < off_i + S_i (None = padding)."""
    O = sum(pl["units"][q] for q in range(p)) * pl["G"]
    exp = []
    for x in range(pl["peer_bytes"][p]):
        a = O + x
        v = None
        for i, off in enumerate(pl["offsets"]):
            if off <= a < off + pl["sizes"][i]:
                v = int(tensors[i][a - off])
        exp.append(v)
    return exp


def test_byte_model_matches_virtual_addresses_g1():
    g = _golden("g1_weights_caps_padding.json")
    pl = oracle.plan(g["world"], g["source"], g["spare"], g["bw"], g["sizes"], g["granule"])
    tensors = [splitmix64_bytes(7, i, 0, s) for i, s in enumerate(g["sizes"])]
    stash = oracle.swap_out(pl, tensors)
    for p, (buf, defined) in stash.items():
        exp = _virtual_address_expectation(pl, tensors, p)
        for x, v in enumerate(exp):
            assert defined[x] == (v is not None)
            if v is not None:
                assert buf[x] == v


def test_round_trip_identity_random():
    """swap-out followed by swap-in is the identity, for random bits (R18)."""
    rng = random.Random(378)
    for t in range(200):
        world, source, spare, bw, sizes, G = _random_instance(rng)
        try:
            pl = oracle.plan(world, source, spare, bw, sizes, G)
        except PlanError:
            continue
        tensors = [splitmix64_bytes(t, i, 0, s) for i, s in enumerate(sizes)]
        stash = oracle.swap_out(pl, tensors)
        back = oracle.swap_in(pl, stash)
        for a, b in zip(tensors, back):
            assert np.array_equal(a, b)


# ---------------------------------------------------------------- generator pin

def test_splitmix64_known_value():
    # splitmix64 with state 0: first output 0xE220A8397B1DCDAF (Steele et al. reference)
    b = splitmix64_bytes(0, 0, 0, 8)
    assert int.from_bytes(bytes(b), "little") == 0xE220A8397B1DCDAF
    # second output of the reference stream = finaliser(2*gamma) = word index ... not
    # directly comparable; check windowing consistency instead
    full = splitmix64_bytes(5, 3, 0, 100)
    assert np.array_equal(full[13:77], splitmix64_bytes(5, 3, 13, 64))


# ---------------------------------------------------------------- workloads + partition

def test_workload_sizes():
    assert sum(workloads.cfg1_sizes()) == 64 << 20
    s2 = workloads.cfg2_sizes()
    assert len(s2) == 47 and sum(s2) == 900 << 20
    # per layer = 34*s*b*h + 5*a*s^2*b bytes (ref [39])
    s, b, h, a = 512, 8, 1024, 16
    assert sum(s2[2:17]) == 34 * s * b * h + 5 * a * s * s * b
    s3 = workloads.cfg3_sizes()
    assert len(s3) == 100 and min(s3) == 20 * 1024 and abs(sum(s3) / 1e9 - 12.21) < 0.01


def test_config3_capacity_binds():
    c = workloads.CONFIGS[3]
    spare = workloads.spare_vector(8, 0, c["peers"], spare_by_peer=c["spare_by_peer"])
    bw = workloads.bw_vector(8, 0, c["peers"])
    pl = oracle.plan(8, 0, spare, bw, workloads.cfg3_sizes())
    G = pl["G"]
    assert pl["units"][7] * G == 2 << 30            # peer 7 capped at its 2 GiB
    assert abs(pl["units"][5] - pl["units"][6]) <= 1  # the rest split equally


def test_sequential_partition_config5():
    c = workloads.CONFIGS[5]
    world = 8
    spare = workloads.spare_vector(world, 0, c["peers"], spare=c["spare"])
    bw_rows = [workloads.bw_vector(world, s, c["peers"]) for s in range(world)]
    reqs = [(s, workloads.cfg5_source_sizes(s), 1) for s in c["sources"]]
    part, plans = oracle.sequential_partition(world, spare, bw_rows, reqs)
    for p in range(world):
        assert sum(part[s][p] for s in range(world)) <= spare[p]
    for s in c["sources"]:
        assert sum(part[s]) >= sum(workloads.cfg5_source_sizes(s))
        # equal weights and ample spare: each source spreads over all 4 peers
        u = [plans[s]["units"][p] for p in c["peers"]]
        assert max(u) - min(u) <= 1
