"""Memory timeline of one pipeline stage under 1F1B with recomputation (test-only pin).

Independent of the oracle: it replays the stage's 1F1B order (the one of sim1f1b:
min(p-i-1, N) warm-up forwards, then one forward / one backward, then the remaining
backwards) op by op and tracks the bytes allocated at every instant:
  - weights, gradients and optimizer state: W, always resident;
  - forward of op j: its transient `peak` while it runs; afterwards its stash stays until
    its backward: `act` bytes, or only `keep` bytes if the op is recomputed (activation
    checkpointing: the rest is discarded and rebuilt in backward);
  - backward of op j (ops in reverse order): a recomputed op first rebuilds the
    discarded `act - keep` bytes (its forward is re-run), then runs with its
    transient `peak`; afterwards its stash (and the rebuilt part) is freed.
Returns the largest total. Eq. 1 with the stage max term of P:L234 is an upper
bound of this timeline; it is reached when the op with the largest transient is the
stage's last op (the first backward, when all in-flight microbatches are stashed).
"""


def stage_memory_peak(ops, W, p, i, N):
    """ops: list of (act, keep, peak, rc) in op order; W: resident bytes; stage i of p."""
    w = min(p - i - 1, N)
    seq = [("F", m) for m in range(w)]
    nf, nb = w, 0
    while nb < N:
        if nf < N:
            seq.append(("F", nf))
            nf += 1
        seq.append(("B", nb))
        nb += 1
    stash = 0
    best = W
    for kind, _ in seq:
        if kind == "F":
            for act, keep, peak, rc in ops:
                best = max(best, W + stash + peak)
                stash += keep if rc else act
        else:
            for act, keep, peak, rc in reversed(ops):
                rebuilt = (act - keep) if rc else 0
                best = max(best, W + stash + rebuilt + peak)
                stash -= keep if rc else act
    assert stash == 0
    return best
