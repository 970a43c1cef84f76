"""ORACLE (test infrastructure only) -- exhaustive minimum makespan.

P:213: "we compute the score as the reciprocal of the maximal time cost of D2D
swap for a fixed assignment."  With k_p units on a link of weight B_p the time
on that link is k_p / B_p (R1), so the best score is

    1 / min over { k : sum k_p = K, 0 <= k_p <= cap_p, k_p = 0 if B_p = 0 }
              of max_p k_p / B_p

which this module finds by enumerating every k (tiny inputs only).  It is the
independent pin of the greedy planner's optimality; it knows nothing about
tie-breaking, layout or stripes.
"""
from fractions import Fraction
from itertools import product


def makespan(units, bw):
    """max_p k_p / B_p over peers that got units (exact Fraction)."""
    m = Fraction(0)
    for k, b in zip(units, bw):
        if k > 0:
            m = max(m, Fraction(k, b))
    return m


def brute_force_makespan(K, caps, bw):
    """Minimum makespan over all feasible unit vectors, or None if infeasible.

    caps[p] and bw[p] per candidate peer (bw > 0).  Enumerates the full grid.
    """
    best = None
    ranges = [range(c + 1) for c in caps]
    for k in product(*ranges):
        if sum(k) != K:
            continue
        m = makespan(k, bw)
        if best is None or m < best:
            best = m
    return best
