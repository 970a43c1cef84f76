"""ORACLE (test infrastructure only) -- NEXT-2: 1F1B swap schedule with the
live-interval check.

Paper passages
  P:62-77, P:87-89 (Fig. 1)  inter-operator parallel training: the mini-batch
        is split into M micro-batches pipelined over S stages; early stages
        keep more micro-batches' activations alive (PipeDream 1F1B, DAPPLE).
  P:145, P:236  swap-out / swap-in operators run by the executor on two extra
        CUDA streams, one for swap-out and one for swap-in, next to compute.
  P:219 + fn.1  a swap costs nothing when the tensor's live interval
        ("the difference between the timestamps of its backward and forward
        passes") exceeds the swap time; fn.2: extra time = swap cost -
        live interval.
  P:281  computation-balanced partitioning: every stage has the same
        per-micro-batch forward / backward time.

Model (reading R24), all times integers (ns):
  * stage k runs W_k = min(S-1-k, M) warm-up forwards, then alternates
    F(W_k+i), B(i), then the remaining backwards (1F1B);
  * every resource (a stage, a swap stream) runs its ops in a fixed order;
    an op starts at max(end of the resource's previous op, end of each of its
    dependencies) and lasts t_f / t_b / t_out / t_in;
  * dependencies: F(m)@k needs F(m)@k-1; B(m)@k needs B(m)@k+1 (last stage:
    its own F(m)); at the exporter stage e, B(m)@e also needs swap-in(m);
    swap-out(m) needs F(m)@e; swap-in(m) needs swap-out(m) and its trigger op;
  * trigger op j(m) = the last op of stage e (in stage order, from F(m) up to
    before B(m)) whose no-swap end <= B_start_noswap(m) - t_in - slack: the swap-in
    is issued as late as the no-swap timeline allows it to still be hidden;
  * swap-op order = the executor's enqueue order: after op j of stage e,
    first the swap-out of the micro-batch j produced (if j is a forward), then
    the swap-ins triggered by j (ascending m).  duplex: swap-outs and swap-ins
    on two streams; otherwise both on one stream in that order;
  * resident activation sets at stage e: [F_start(m), B_end(m)) without
    swapping, [F_start(m), out_end(m)) and [in_start(m), B_end(m)) with; at
    one instant, releases happen before acquisitions.
This is list scheduling with fixed per-resource orders, so every start time is
determined; the simulation below just evaluates the definition.
"""


def stage_ops(S, k, M):
    """1F1B op order of stage k: list of ('F'|'B', m)."""
    W = min(S - 1 - k, M)
    ops = [("F", m) for m in range(W)]
    for i in range(M):
        if W + i < M:
            ops.append(("F", W + i))
        ops.append(("B", i))
    return ops


def _run(queues, deps, dur):
    """queues: {resource: [op, ...]}; deps(op) -> [ops]; dur(op) -> ns.
    Returns (start, end) dicts over all ops."""
    start, end = {}, {}
    pos = {r: 0 for r in queues}
    free = {r: 0 for r in queues}
    remaining = sum(len(q) for q in queues.values())
    while remaining:
        progressed = False
        for r, q in queues.items():
            while pos[r] < len(q):
                op = q[pos[r]]
                ds = deps(op)
                if any(d not in end for d in ds):
                    break
                t = max([free[r]] + [end[d] for d in ds])
                start[op], end[op] = t, t + dur(op)
                free[r] = end[op]
                pos[r] += 1
                remaining -= 1
                progressed = True
        if not progressed:
            raise RuntimeError("cyclic dependencies")
    return start, end


def _compute_queues(S, M):
    return {("stage", k): [(k,) + op for op in stage_ops(S, k, M)] for k in range(S)}


def _base_deps(S, op):
    k, kind, m = op
    if kind == "F":
        return [(k - 1, "F", m)] if k > 0 else []
    return [(k + 1, "B", m)] if k < S - 1 else [(k, "F", m)]


def timeline_noswap(S, M, tf, tb):
    return _run(_compute_queues(S, M), lambda op: _base_deps(S, op),
                lambda op: tf if op[1] == "F" else tb)


def schedule(S, e, M, tf, tb, t_out, t_in, duplex=True, slack=0):
    """(slots, summary) for exporter stage e; slots[m] has the fields of
    mpress_1f1b_slot, summary those of mpress_1f1b_summary (include/mpress.h)."""
    assert 0 <= e < S and M >= 1
    s0, e0 = timeline_noswap(S, M, tf, tb)
    ops = stage_ops(S, e, M)
    idx = {op: j for j, op in enumerate(ops)}
    trig = []
    for m in range(M):
        target = s0[(e, "B", m)] - t_in - slack
        j = idx[("F", m)]
        for jj in range(idx[("F", m)], idx[("B", m)]):
            if e0[(e,) + ops[jj]] <= target:
                j = jj
        trig.append(j)
    order = []
    for j, (kind, m) in enumerate(ops):
        if kind == "F":
            order.append(("out", m))
        order += [("in", mm) for mm in range(M) if trig[mm] == j]
    queues = _compute_queues(S, M)
    if duplex:
        queues["out"] = [op for op in order if op[0] == "out"]
        queues["in"] = [op for op in order if op[0] == "in"]
    else:
        queues["swap"] = order

    def deps(op):
        if op[0] == "out":
            return [(e, "F", op[1])]
        if op[0] == "in":
            return [("out", op[1]), (e,) + ops[trig[op[1]]]]
        d = _base_deps(S, op)
        if op[0] == e and op[1] == "B":
            d = d + [("in", op[2])]
        return d

    def dur(op):
        return {"out": t_out, "in": t_in, "F": tf, "B": tb}[op[0] if op[0] in ("out", "in") else op[1]]

    s1, e1 = _run(queues, deps, dur)
    slots = []
    for m in range(M):
        b = (e, "B", m)
        jb = idx[("B", m)]
        ready = max([e1[(e,) + ops[jb - 1]]] + [e1[d] for d in _base_deps(S, b)])
        slots.append(dict(
            fwd_start=s1[(e, "F", m)], fwd_end=e1[(e, "F", m)], bwd_start=s1[b], bwd_end=e1[b],
            live_ns=s0[b] - e0[(e, "F", m)],
            out_start=s1[("out", m)], out_end=e1[("out", m)],
            in_start=s1[("in", m)], in_end=e1[("in", m)],
            in_trigger=trig[m], hidden=1 if e1[("in", m)] <= ready else 0,
            exposed_ns=s1[b] - s0[b]))
    compute = [op for op in e1 if isinstance(op[0], int)]
    summary = dict(
        makespan_ns=max(e1[op] for op in compute), makespan_noswap_ns=max(e0.values()),
        peak_resident=_peak([(s1[(e, "F", m)], e1[("out", m)]) for m in range(M)] +
                            [(s1[("in", m)], e1[(e, "B", m)]) for m in range(M)]),
        peak_resident_noswap=_peak([(s0[(e, "F", m)], e0[(e, "B", m)]) for m in range(M)]),
        ops=len(ops))
    return slots, summary


def _peak(intervals):
    """Max number of overlapping [a, b) intervals (releases before acquisitions)."""
    ev = []
    for a, b in intervals:
        if b > a:
            ev.append((a, 1))
            ev.append((b, -1))
    ev.sort()
    cur = best = 0
    for _, d in ev:
        cur += d
        best = max(best, cur)
    return best
