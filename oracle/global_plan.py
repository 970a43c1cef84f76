"""ORACLE (test infrastructure only) -- NEXT-1: joint plan of several exporters.

Fig. 6: from each importer's view, enumerate "all possible ways
to distribute mem of spare_amount to candidates" (lines 2-8), combine the
single-GPU plans into global plans ("permutation", line 20) and keep the one
with the best score, "the reciprocal of the maximal time cost of D2D swap"
(garbled as "ratio of revenue to cost" in line 22; reading R1).

Model (reading R23).  Every source s swaps its batch of K_s units
(G-byte units, the batch layout of plan.py) at the same time.  x[s][p] units
of s go to importer p.  The time of the assignment is

    T(x) = max(  max_{s,p: x>0} x[s][p] / B[s][p]      per-link (DGX-1)
               , max_s  sum_p x[s][p] / E[s]           source egress port (NVSwitch)
               , max_p  sum_s x[s][p] / I[p] )         importer ingress port (NVSwitch)

with E / I = 0 meaning "no port limit", subject to sum_p x[s][p] = K_s,
sum_s x[s][p] <= cap_p = spare_p // G, x[s][p] = 0 when B[s][p] = 0 or p = s.

Two independent oracles:
  brute_force_global -- enumerates every integer x (tiny inputs), the plain
                        reading of Fig. 6;
  scan_global        -- walks the finite candidate set of T values (every
                        k/w for an integer k and a weight w of the model) in
                        increasing order and returns the first T at which a
                        plain Edmonds-Karp max-flow routes all units.  It is
                        pinned to brute_force_global on tiny inputs.
The optimal T* is unique; the optimal x is not (R19), so tests compare T* and
check the library's x for validity and T(x) = T*.
"""
from fractions import Fraction
from itertools import product

from .plan import PlanError, ERR_ARG, ERR_NO_SPACE, virtual_layout


def demand_units(sizes, G):
    return (virtual_layout(sizes)[1] + G - 1) // G


def assignment_time(x, sources, world, bw, egress, ingress):
    """T(x) as an exact Fraction (0 for an empty assignment)."""
    t = Fraction(0)
    for si, s in enumerate(sources):
        for p in range(world):
            if x[si][p] > 0:
                t = max(t, Fraction(x[si][p], bw[s][p]))
        if egress and egress[s] > 0:
            t = max(t, Fraction(sum(x[si]), egress[s]))
    if ingress:
        for p in range(world):
            if ingress[p] > 0:
                t = max(t, Fraction(sum(x[si][p] for si in range(len(sources))), ingress[p]))
    return t


def _check(world, sources, K, spare, bw, G):
    if G % 256 or G <= 0:
        raise PlanError(ERR_ARG, "granule must be a positive multiple of 256")
    if len(set(sources)) != len(sources) or any(not 0 <= s < world for s in sources):
        raise PlanError(ERR_ARG, "bad source list")
    caps = [spare[p] // G for p in range(world)]
    return caps


def brute_force_global(world, sources, demands, spare, bw, egress=None, ingress=None, G=4096):
    """min T over all integer assignments (tiny inputs), or raises NO_SPACE."""
    caps = _check(world, sources, demands, spare, bw, G)
    S = len(sources)
    # per source: all ways to split K_s over its candidate importers
    options = []
    for si, s in enumerate(sources):
        cand = [p for p in range(world) if p != s and bw[s][p] > 0 and caps[p] > 0]
        splits = []
        for ks in product(*[range(min(caps[p], demands[si]) + 1) for p in cand]):
            if sum(ks) == demands[si]:
                row = [0] * world
                for p, k in zip(cand, ks):
                    row[p] = k
                splits.append(row)
        options.append(splits)
    best = None
    for combo in product(*options):
        if any(sum(combo[si][p] for si in range(S)) > caps[p] for p in range(world)):
            continue
        t = assignment_time(combo, sources, world, bw, egress, ingress)
        if best is None or t < best:
            best = t
    if best is None:
        raise PlanError(ERR_NO_SPACE, "no feasible assignment")
    return best


def _max_flow(n, cap, s, t):
    """Edmonds-Karp on a dense capacity matrix (copied); returns (flow, cap_left)."""
    cap = [row[:] for row in cap]
    flow = 0
    while True:
        prev = [-1] * n
        prev[s] = s
        queue = [s]
        for u in queue:
            for v in range(n):
                if prev[v] < 0 and cap[u][v] > 0:
                    prev[v] = u
                    queue.append(v)
        if prev[t] < 0:
            return flow, cap
        # bottleneck
        b, v = None, t
        while v != s:
            u = prev[v]
            b = cap[u][v] if b is None else min(b, cap[u][v])
            v = u
        v = t
        while v != s:
            u = prev[v]
            cap[u][v] -= b
            cap[v][u] += b
            v = u
        flow += b


def feasible(T, world, sources, demands, caps, bw, egress, ingress):
    """Can every unit be routed with time <= T?  Returns x or None."""
    S = len(sources)
    n = 2 + S + world
    src, snk = 0, 1
    cap = [[0] * n for _ in range(n)]
    for si, s in enumerate(sources):
        if egress and egress[s] > 0 and Fraction(demands[si]) > T * egress[s]:
            return None
        cap[src][2 + si] = demands[si]
        for p in range(world):
            if p != s and bw[s][p] > 0:
                cap[2 + si][2 + S + p] = int(T * bw[s][p])  # floor
    for p in range(world):
        c = caps[p]
        if ingress and ingress[p] > 0:
            c = min(c, int(T * ingress[p]))
        cap[2 + S + p][snk] = c
    flow, left = _max_flow(n, cap, src, snk)
    if flow != sum(demands):
        return None
    return [[cap[2 + si][2 + S + p] - left[2 + si][2 + S + p] for p in range(world)] for si in range(S)]


def scan_global(world, sources, demands, spare, bw, egress=None, ingress=None, G=4096):
    """(T*, x): the first feasible T in the sorted candidate set."""
    caps = _check(world, sources, demands, spare, bw, G)
    total = sum(demands)
    weights = set()
    for s in sources:
        for p in range(world):
            if p != s and bw[s][p] > 0:
                weights.add(bw[s][p])
        if egress and egress[s] > 0:
            weights.add(egress[s])
    if ingress:
        weights |= {w for w in ingress if w > 0}
    cands = sorted({Fraction(k, w) for w in weights for k in range(0, total + 1)})
    for T in cands:
        x = feasible(T, world, sources, demands, caps, bw, egress, ingress)
        if x is not None:
            return T, x
    raise PlanError(ERR_NO_SPACE, "no feasible assignment")
