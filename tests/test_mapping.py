"""NEXT-3: device-stage mapping search (Fig. 6 lines 10-26, P:172-213,
reading R25).  CPU only.  Pins: a hand-derived 3-GPU chain, the symmetric
case (on symmetric links every mapping scores the same, so the
paper skips the search), and the inner score = the NEXT-1 optimum (pinned in
test_global_plan.py).  The library must pick the same mapping as the oracle
(both take the lexicographically first optimum) with the same T*."""
import json
import os
import random
import time
from fractions import Fraction
from itertools import permutations

import pytest

from oracle import mapping as OM
from oracle import global_plan as OG
import paper_conf_hpca_zhouwylbyx23_b200 as mp

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def test_chain_by_hand():
    """GPU0 -2- GPU1 -1- GPU2 (no GPU0-GPU2 link).  Stage 0 must swap 6 units
    into stages 1 and 2 (12 units of spare each).  On GPU1 it reaches both
    peers and splits 4:2 -> T = 6/3 = 2; on GPU0 only GPU1 (T = 6/2 = 3); on
    GPU2 only GPU1 (T = 6/1 = 6).  First optimal mapping in lexicographic
    order: stage 0 -> GPU1, stage 1 -> GPU0, stage 2 -> GPU2."""
    G = 4096
    link = [[0, 2, 0], [2, 0, 1], [0, 1, 0]]
    demand, spare = [6 * G, 0, 0], [0, 12 * G, 12 * G]
    T, m, ev = OM.mapping_search(3, demand, spare, link, G=G)
    assert (T, m, ev) == (Fraction(2), [1, 0, 2], 6)
    got, (num, den), ev2 = mp.map_search(demand, spare, link, granule=G)
    assert got == [1, 0, 2] and Fraction(num, den) == 2 and ev2 == 6


def test_symmetric_links_every_mapping_ties():
    """with symmetric links the mapping does not matter."""
    G = 4096
    n = 4
    link = [[0 if i == j else 3 for j in range(n)] for i in range(n)]
    demand, spare = [5 * G, 3 * G, 0, 0], [0, 0, 6 * G, 6 * G]
    scores = set()
    for perm in permutations(range(n)):
        srcs = [perm[s] for s in range(n) if demand[s]]
        K = [OG.demand_units([demand[s]], G) for s in range(n) if demand[s]]
        sp = [0] * n
        for s in range(n):
            if not demand[s]:
                sp[perm[s]] = spare[s]
        scores.add(OG.scan_global(n, srcs, K, sp, link, None, None, G)[0])
    assert len(scores) == 1
    got, (num, den), _ = mp.map_search(demand, spare, link, granule=G)
    assert Fraction(num, den) in scores and got == [0, 1, 2, 3]


def test_library_matches_oracle_random():
    rng = random.Random(172)
    for _ in range(25):
        n = rng.randint(2, 5)
        G = 4096
        link = [[0] * n for _ in range(n)]
        for i in range(n):
            for j in range(i + 1, n):
                link[i][j] = link[j][i] = rng.choice([0, 1, 2])
        demand = [rng.choice([0, 0, rng.randint(1, 4) * G]) for _ in range(n)]
        if not any(demand):
            demand[0] = 2 * G
        spare = [0 if d else rng.randint(0, 5) * G for d in demand]
        try:
            T, m, ev = OM.mapping_search(n, demand, spare, link, G=G)
        except Exception as e:
            with pytest.raises(mp.MPressError) as ei:
                mp.map_search(demand, spare, link, granule=G)
            assert ei.value.code == mp.ERR_NO_SPACE, e
            continue
        got, (num, den), ev2 = mp.map_search(demand, spare, link, granule=G)
        assert (got, Fraction(num, den), ev2) == (m, T, ev)


def test_dgx1v_eight_gpus_search_time():
    """the search takes at most 47 s single-threaded for the extreme
    case.  8 stages on a DGX-1V-like topology (tests/golden/m1), stages 0-3
    overflowing into 4-7 (Table IV P:347-350 pattern)."""
    L = json.load(open(os.path.join(GOLDEN, "m1_dgx1v_links.json")))["links"]
    GiB = 1 << 30
    demand = [20 * GiB, 14 * GiB, 9 * GiB, 4 * GiB, 0, 0, 0, 0]
    spare = [0, 0, 0, 0, 12 * GiB, 12 * GiB, 12 * GiB, 12 * GiB]
    t0 = time.perf_counter()
    got, (num, den), ev = mp.map_search(demand, spare, L, granule=256 << 20)
    dt = time.perf_counter() - t0
    assert ev == 40320 and dt < 47
    # the identity mapping (stages 0-3 on GPUs 0-3) gives each overflowed GPU
    # a single NVLink into GPUs 4-7, whose 12 GiB cannot hold stage 0's 20 GiB:
    # without the search the D2D swap fails outright
    G = 256 << 20
    K = [OG.demand_units([d], G) for d in demand[:4]]
    srcs = [0, 1, 2, 3]
    with pytest.raises(mp.MPressError) as ei:
        mp.plan_global(8, [(s, [demand[s]]) for s in srcs], spare, L, granule=G)
    assert ei.value.code == mp.ERR_NO_SPACE
    # and the chosen mapping reaches its score
    sp = [0] * 8
    for s in range(8):
        if not demand[s]:
            sp[got[s]] = spare[s]
    _, (n2, d2) = mp.plan_global(8, [(got[s], [demand[s]]) for s in range(4)], sp, L, granule=G)
    assert Fraction(n2, d2) == Fraction(num, den)
    assert K  # units used by the identity check above
