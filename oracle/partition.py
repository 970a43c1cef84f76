"""ORACLE (test infrastructure only) -- multi-source stash reservation (R12, R21).

Fig. 6 lines 2-8 distribute each importer's spare amount among the
overflowed exporters.  The paper's "all possible ways ... permutation" search is
garbled and out of the hot path; the reading used here (R12) is the
deterministic sequential one: plan the sources in ascending index, each against
the spare memory the earlier sources left, and reserve ``copies * k_p * G``
bytes of peer p for source s (``copies`` = how many handles of that plan may be
in flight at once, e.g. 8 micro-batches under 1F1B).  A source with
``copies`` in flight plans against floor(remaining_p / copies) per peer.
"""
from .plan import plan as _plan


def sequential_partition(world, spare, bw_rows, requests, granule=0):
    """requests: list of (source, sizes, copies), any order.

    Returns (partition, plans): partition[s][p] = bytes of peer p's pool owned
    by source s; plans[s] = the oracle plan of source s.
    """
    remaining = list(spare)
    partition = [[0] * world for _ in range(world)]
    plans = {}
    for source, sizes, copies in sorted(requests, key=lambda r: r[0]):
        # each of the `copies` in-flight handles gets an equal share
        per_copy = [r // copies for r in remaining]
        pl = _plan(world, source, per_copy, bw_rows[source], sizes, granule)
        for p in range(world):
            r = copies * pl["units"][p] * pl["G"]
            remaining[p] -= r
            partition[source][p] += r
        plans[source] = pl
    return partition, plans
