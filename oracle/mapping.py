"""ORACLE (test infrastructure only) -- NEXT-3: device-stage mapping search.

Fig. 6 lines 10-26 and P:211-213: enumerate every mapping of
pipeline stages to GPUs ("all_map", line 13); for each, let every GPU with
spare memory distribute it to the overflowed GPUs among its NVLink
neighbours (assign_mem, lines 2-8), combine the per-GPU plans and score the
combination by "the reciprocal of the maximal time cost of D2D swap";
keep the best mapping.  On symmetric NVLink the search is skipped.

Reading R25: the inner "distribute + combine + score" is the
NEXT-1 joint optimum T*(mapping) (global_plan.py, reading R23), with each
overflowed stage's demand as one batch of `demand[s]` bytes; mappings are
enumerated in lexicographic order of (gpu of stage 0, gpu of stage 1, ...)
and the first one with the smallest T* wins.  A mapping whose spare cannot
hold the demand is skipped; if none fits -> NO_SPACE.
"""
from itertools import permutations

from .global_plan import scan_global, demand_units
from .plan import PlanError, ERR_NO_SPACE


def mapping_search(n, demand, spare, link, egress=None, ingress=None, G=1 << 20):
    """Returns (best T* as a Fraction, stage_to_gpu list, mappings evaluated)."""
    best, best_map, evaluated = None, None, 0
    for perm in permutations(range(n)):
        evaluated += 1
        sources = [perm[s] for s in range(n) if demand[s] > 0]
        if not sources:
            continue
        K = [demand_units([demand[s]], G) for s in range(n) if demand[s] > 0]
        sp = [0] * n
        for s in range(n):
            sp[perm[s]] = spare[s] if demand[s] == 0 else 0
        try:
            T, _ = scan_global(n, sources, K, sp, link, egress, ingress, G)
        except PlanError:
            continue
        if best is None or T < best:
            best, best_map = T, list(perm)
    if best is None:
        raise PlanError(ERR_NO_SPACE, "no mapping fits the demand")
    return best, best_map, evaluated
