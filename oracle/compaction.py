"""ORACLE (test infrastructure only) -- NEXT-4: the memory-compaction
decision rule (§III-D) between GPU-CPU swap, recomputation and
D2D swap, on per-tensor cost statistics (Table III).

Paper passages
  P:219  swaps "can run in parallel with the forward and backward
         computation"; when the live interval exceeds the swap time, "no extra
         time delay is introduced";
  fn.2  GPU-CPU swap overhead = swap cost - live interval;
  P:97-103     recomputation re-runs the forward: its cost is extra time;
  P:224-232    initial assignment: GPU-CPU swap for long-lived tensors,
         recomputation for activations whose extra latency is smaller than the
         GPU-CPU swap's, GPU-CPU swap for the rest; then, step by step, the
         tensors whose optimizations "introduce the most extra overhead" move to
         D2D swap "whenever possible, e.g., when there is spare GPU memory",
         accepting a change only if it performs better;
  P:358-364    Table III's reasoning: ties go to the option that spends no
         spare GPU memory (t1: GPU-CPU over D2D; t3: recomputation over D2D).

Reading R26: overhead(swap) = max(0, cost - live); overhead
(recompute) = its cost; initial = the lower of GPU-CPU swap and recomputation
(ties -> GPU-CPU swap, which uses neither GPU memory nor compute); then tensors
in order of current overhead (largest first, ties -> lower index) switch to
D2D if its overhead is strictly lower and the tensor fits in the remaining
spare bytes.
"""

CPU, RECOMPUTE, D2D = 1, 2, 3
NOT_RECOMPUTABLE = (1 << 64) - 1


def overhead(cost, live):
    return cost - live if cost > live else 0


def compaction_plan(stats, d2d_capacity):
    """stats: list of dicts with bytes, live_ns, recompute_ns, cpu_swap_ns,
    d2d_swap_ns.  Returns (choices, overheads, total, d2d_bytes)."""
    choice, ovh = [], []
    for t in stats:
        c = overhead(t["cpu_swap_ns"], t["live_ns"])
        r = t["recompute_ns"]
        if r != NOT_RECOMPUTABLE and r < c:
            choice.append(RECOMPUTE)
            ovh.append(r)
        else:
            choice.append(CPU)
            ovh.append(c)
    order = sorted(range(len(stats)), key=lambda i: (-ovh[i], i))
    left = d2d_capacity
    used = 0
    for i in order:
        t = stats[i]
        d = overhead(t["d2d_swap_ns"], t["live_ns"])
        if d < ovh[i] and t["bytes"] <= left:
            choice[i], ovh[i] = D2D, d
            left -= t["bytes"]
            used += t["bytes"]
    return choice, ovh, sum(ovh), used


def brute_force_total(stats, d2d_capacity):
    """Minimum total overhead over every assignment (tiny inputs)."""
    from itertools import product
    best = None
    for combo in product((CPU, RECOMPUTE, D2D), repeat=len(stats)):
        cap = d2d_capacity
        tot = 0
        ok = True
        for t, c in zip(stats, combo):
            if c == CPU:
                tot += overhead(t["cpu_swap_ns"], t["live_ns"])
            elif c == RECOMPUTE:
                if t["recompute_ns"] == NOT_RECOMPUTABLE:
                    ok = False
                    break
                tot += t["recompute_ns"]
            else:
                cap -= t["bytes"]
                tot += overhead(t["d2d_swap_ns"], t["live_ns"])
        if ok and cap >= 0 and (best is None or tot < best):
            best = tot
    return best
