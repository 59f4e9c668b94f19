"""Discrete-event simulator of 1F1B pipeline scheduling (test-only pin).

Independent of the oracle: it executes the schedule of PipeDream-Flush / Megatron
1F1B (ref [28], [29]) event by event and reports the makespan
and the peak number of in-flight microbatches (forward done, backward not yet)
per stage. Stage i (0-based) runs min(p-i-1, N) warm-up forwards, then
alternates one forward and one backward, then drains the remaining backwards.
F(i,m) waits for F(i-1,m); B(i,m) waits for B(i+1,m) and F(i,m).
"""


def simulate(f, b, N, sync=None):
    """f[i], b[i]: forward/backward time of one microbatch on stage i.
    sync[i]: time of stage i's end-of-iteration gradient sync (after its last backward).
    Returns (makespan, peak_inflight[i])."""
    p = len(f)
    sync = sync or [0] * p
    order = []
    for i in range(p):
        w = min(p - i - 1, N)
        seq = [("F", m) for m in range(w)]
        nf, nb = w, 0
        while nb < N:
            if nf < N:
                seq.append(("F", nf))
                nf += 1
            seq.append(("B", nb))
            nb += 1
        order.append(seq)
    done = {}
    pos = [0] * p
    t_free = [0] * p
    inflight = [0] * p
    peak = [0] * p
    progress = True
    while progress:
        progress = False
        for i in range(p):
            while pos[i] < len(order[i]):
                kind, m = order[i][pos[i]]
                if kind == "F":
                    dep = [done.get(("F", i - 1, m))] if i > 0 else []
                else:
                    dep = [done.get(("F", i, m))]
                    if i < p - 1:
                        dep.append(done.get(("B", i + 1, m)))
                if any(d is None for d in dep):
                    break
                start = max([t_free[i]] + dep)
                end = start + (f[i] if kind == "F" else b[i])
                done[(kind, i, m)] = end
                t_free[i] = end
                if kind == "F":
                    inflight[i] += 1
                    peak[i] = max(peak[i], inflight[i])
                else:
                    inflight[i] -= 1
                pos[i] += 1
                progress = True
    assert all(pos[i] == len(order[i]) for i in range(p)), "deadlock"
    makespan = max(t_free[i] + sync[i] for i in range(p))
    return makespan, peak
