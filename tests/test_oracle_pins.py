"""Pins for the CPU oracle (no GPU): each test checks the oracle against something
the paper or mathematics fixes, not against a retyped copy of its formulas.

P:Lnn = PAPER.md line; R# = reading in DESIGN.md §3.
"""
import itertools
import json
import os

import numpy as np
import pytest

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P
from tests.sim1f1b import simulate

NF = 10
FC, FM, BC, BM, ACT, KEEP, PEAK, RESH, P2PF, P2PB = range(NF)


def mkprof(recs, op_type, n_tp=1, n_b=8, n_dp=1, G=1, C=1 << 40, Bg=8, wmem=None, dps=None):
    """recs: dict type -> fn(tpl, b) -> list of NF values."""
    T = len(recs)
    rec = np.zeros((T, n_tp, n_b, NF), np.int64)
    for t in range(T):
        for tpl in range(n_tp):
            for b in range(n_b):
                rec[t, tpl, b] = recs[t](tpl, b)
    wm = np.zeros((T, n_tp, 2), np.int64) if wmem is None else np.asarray(wmem, np.int64)
    dp = np.zeros((T, n_tp, n_dp), np.int64) if dps is None else np.asarray(dps, np.int64)
    return P.from_tables("hand", op_type, rec, wm, dp, G, C, Bg)


def cand(stage_sizes, tpdp=None, rc=None):
    """Row of codes for consecutive stages of the given sizes."""
    out = []
    j = 0
    for i, n in enumerate(stage_sizes):
        tpl, dpl = (tpdp[i] if tpdp else (0, 0))
        for k in range(n):
            r = rc[j] if rc else 0
            out.append(ai.code(1 if k == 0 else 0, tpl, dpl, r))
            j += 1
    return out


def ev(prof, rows, hdrs, full=True):
    return oracle.evaluate(prof, np.array(rows, np.uint8), np.array(hdrs, np.uint64), full=full)


# --------------------------------------------------------------------------
# Eq. 2 (R1) and Eq. 1 (R2) against a discrete-event 1F1B simulation
# --------------------------------------------------------------------------
@pytest.mark.parametrize("p", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("mbs_log2", [0, 1, 2, 3])
def test_uniform_pipeline_matches_1f1b_simulation(p, mbs_log2):
    """Uniform stages: Eq. 2 (reading R1) gives the 1F1B makespan (N+p-1)(f+b)
    and Eq. 1 gives min(p-i, N) in-flight activations on stage i."""
    k = 3  # ops per stage
    f_op, b_op = 7, 13
    prof = mkprof({0: lambda tpl, b: [f_op, 0, b_op, 0, 1, 0, 0, 0, 0, 0]}, [0] * (p * k), G=p, Bg=8)
    N = 8 >> mbs_log2
    out = ev(prof, [cand([k] * p)], [ai.header(mbs_log2, p)])
    assert out["info"][0] & oracle.INFO_INVALID == 0
    mk, peak = simulate([f_op * k] * p, [b_op * k] * p, N)
    assert int(out["iter"][0]) == mk == (N + p - 1) * (f_op + b_op) * k
    for i in range(p):
        assert int(out["stage_mem"][0, i]) == k * peak[i] == k * min(p - i, N)


def test_inflight_rule_on_nonuniform_stages():
    """The in-flight count min(p-i, N) of Eq. 1 (R2) is structural: it holds for any
    stage times in the 1F1B simulation, so Mem_i/A_i must equal the simulated peak."""
    rng = np.random.default_rng(5)
    for _ in range(20):
        p = int(rng.integers(1, 7))
        sizes = [int(x) for x in rng.integers(1, 5, size=p)]
        L = sum(sizes)
        prof = mkprof({0: lambda tpl, b: [3, 0, 5, 0, 1, 0, 0, 0, 0, 0]}, [0] * L, G=p, Bg=16)
        mbs_log2 = int(rng.integers(0, 5))
        N = 16 >> mbs_log2
        out = ev(prof, [cand(sizes)], [ai.header(mbs_log2, p)])
        f = [float(rng.uniform(1, 9)) for _ in range(p)]
        b = [float(rng.uniform(1, 9)) for _ in range(p)]
        _, peak = simulate(f, b, N)
        for i in range(p):
            assert int(out["stage_mem"][0, i]) == sizes[i] * peak[i]


def test_p1_is_gradient_accumulation():
    """p = 1: T = N*S + D (N microbatches back to back, then the DP sync)."""
    prof = mkprof({0: lambda tpl, b: [11 * (b + 1), 2, 23 * (b + 1), 3, 0, 0, 0, 0, 0, 0]},
                  [0] * 5, n_b=2, n_dp=2, G=2, Bg=16, dps=[[[0, 1000]]])
    # one stage, dp = 2, mbs = 4 -> per-GPU batch 2 (b index 1), N = 4
    out = ev(prof, [cand([5], tpdp=[(0, 1)])], [ai.header(2, 1)])
    mk, _ = simulate([5 * (22 + 2)], [5 * (46 + 3)], 4, sync=[5 * 1000])
    assert int(out["iter"][0]) == mk


def test_dp_sync_on_first_stage_matches_simulation():
    """R6: the DP gradient sync is added once to its own stage. Stage 0 finishes last
    in 1F1B, so a sync on stage 0 adds exactly to the simulated makespan."""
    p, k = 3, 2
    prof = mkprof({0: lambda tpl, b: [5, 0, 9, 0, 0, 0, 0, 0, 0, 0],
                   1: lambda tpl, b: [5, 0, 9, 0, 0, 0, 0, 0, 0, 0]},
                  [1, 1] + [0] * 4, n_dp=2, G=p, Bg=8,
                  dps=[[[0, 0]], [[40, 40]]])
    # op type 1 carries a DP sync only when dp > 1 ... stage 0 runs dp=1 -> use dps[1][0][0]
    prof.dps[1, 0, 0] = 40
    out = ev(prof, [cand([k] * p)], [ai.header(1, p)])
    N = 4
    mk, _ = simulate([5 * k] * p, [9 * k] * p, N, sync=[80, 0, 0])
    assert int(out["iter"][0]) == mk


def test_dp_sync_on_any_stage_with_free_backward_matches_simulation():
    """R6 on every stage: with a zero-time backward the 1F1B backward cascade is instant,
    every stage ends its last backward at the same time, and the iteration ends with the
    slowest stage's own DP sync: makespan = (N+p-1)F + max_i D_i. Eq. 2 gives the same only
    if D_i is added to stage i's own T_i (not summed over stages, not added to others)."""
    rng = np.random.default_rng(11)
    for _ in range(30):
        p = int(rng.integers(2, 6))
        k = int(rng.integers(1, 4))
        d = [int(x) for x in rng.integers(0, 400, size=p)]
        recs = {i: (lambda tpl, bb: [5, 0, 0, 0, 0, 0, 0, 0, 0, 0]) for i in range(p)}
        types = [i for i in range(p) for _ in range(k)]
        dps = [[[d[i]]] for i in range(p)]
        prof = mkprof(recs, types, G=p, Bg=8, dps=dps)
        mbs_log2 = int(rng.integers(0, 4))
        N = 8 >> mbs_log2
        out = ev(prof, [cand([k] * p)], [ai.header(mbs_log2, p)])
        assert out["info"][0] & oracle.INFO_INVALID == 0
        mk, _ = simulate([5 * k] * p, [0] * p, N, sync=[k * x for x in d])
        assert int(out["iter"][0]) == mk == (N + p - 1) * 5 * k + k * max(d)
        # per stage: T_i = the makespan when only stage i synchronises (attribution of D_i)
        for i in range(p):
            mk_i, _ = simulate([5 * k] * p, [0] * p, N, sync=[k * d[i] if s == i else 0 for s in range(p)])
            assert int(out["stage_T"][0, i]) == mk_i


# --------------------------------------------------------------------------
# recomputation (R3, R7)
# --------------------------------------------------------------------------
def test_recompute_adds_forward_and_never_adds_memory():
    """inc-rc on op j (Table 1 row 9: Comp up, Mem down): stage i's per-microbatch
    time grows by F_j, so T_i grows by N*F_j and every other T_k by F_j (Eq. 2);
    Mem_i does not grow (R3)."""
    prof = P.toy_b()
    codes, hdr = ai.search_shaped(prof, 11, 0, 400, group_size=16, invalid_permille=0)
    base = oracle.evaluate(prof, codes, hdr, full=True)
    rng = np.random.default_rng(3)
    checked = 0
    for c in range(len(hdr)):
        if base["info"][c] & oracle.INFO_INVALID:
            continue
        j = int(rng.integers(0, prof.n_ops))
        if codes[c, j] & 0x10:
            continue
        row = codes[c].copy()
        row[j] |= 0x10
        new = oracle.evaluate(prof, row[None, :], hdr[c:c + 1], full=True)
        p = (int(hdr[c]) >> 8) & 0xFF
        i = int(np.sum(codes[c, :j + 1] & 1)) - 1
        mbs_log2 = int(hdr[c]) & 0xFF
        N = prof.global_batch >> mbs_log2
        tpl = (int(codes[c, j]) >> 1) & 7
        dpl = (int(codes[c, j]) >> 5) & 7
        r = prof.rec[prof.op_type[j], tpl, mbs_log2 - dpl]
        F = int(r[FC] + r[FM])
        for k in range(p):
            d = int(new["stage_T"][0, k]) - int(base["stage_T"][c, k])
            assert d == (N * F if k == i else F)
        assert int(new["stage_mem"][0, i]) <= int(base["stage_mem"][c, i])
        assert int(new["iter"][0]) >= int(base["iter"][c])
        checked += 1
    assert checked > 100


# --------------------------------------------------------------------------
# zero-cost operator invariance (north_star)
# --------------------------------------------------------------------------
def test_zero_cost_op_move_changes_nothing():
    rng = np.random.default_rng(9)
    recs = {0: lambda tpl, b: [0] * NF}
    for t in range(1, 4):
        vals = [int(x) for x in rng.integers(1, 1000, size=NF)]
        vals[KEEP] = vals[ACT] // 2
        vals[P2PF] = vals[P2PB] = 0
        recs[t] = (lambda v: (lambda tpl, b: v))(vals)
    op_type = [1, 2, 0, 3, 1, 0, 2, 3]
    wm = np.zeros((4, 1, 2), np.int64)
    wm[1:] = rng.integers(0, 100, size=(3, 1, 2))
    dps = np.zeros((4, 1, 1), np.int64)
    prof = mkprof(recs, op_type, G=2, Bg=8, wmem=wm, dps=dps, C=1 << 40)
    # boundary before op 2 (zero op in stage 1) vs after it (zero op in stage 0)
    a = ev(prof, [cand([2, 6])], [ai.header(1, 2)])
    b = ev(prof, [cand([3, 5])], [ai.header(1, 2)])
    for key in ["iter", "max_mem", "info", "stage_T", "stage_mem", "stage_comp", "stage_comm"]:
        assert np.array_equal(a[key], b[key]), key


# --------------------------------------------------------------------------
# Heuristic-1 on the Fig. 3 scenario, worked by hand: tests/golden/fig3_scenario.json
# --------------------------------------------------------------------------
GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def _golden(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def fig3_profile():
    g = _golden("fig3_scenario.json")
    tab = {tuple(int(x) for x in k.split(",")): v for k, v in g["records"].items()}
    pr = g["profile"]
    return mkprof({0: lambda tpl, b: tab[(tpl, b)]}, [0] * pr["n_ops"], n_tp=pr["n_tp"], n_b=pr["n_b"],
                  n_dp=pr["n_dp"], G=pr["n_devices"], C=pr["mem_capacity"], Bg=pr["global_batch"])


def test_fig3_scenario():
    g = _golden("fig3_scenario.json")
    prof = fig3_profile()
    cs = g["candidates"]
    rows = [cand(c["stage_sizes"], tpdp=[tuple(t) for t in c["tpdp"]]) for c in cs]
    out = ev(prof, rows, [ai.header(c["mbs_log2"], c["p"]) for c in cs])
    info = out["info"]
    for i, c in enumerate(cs):
        e = g["expected"][c["name"]]
        assert bool(info[i] & oracle.INFO_OOM) == e["oom"], c["name"]
        if "bottleneck" in e:
            assert info[i] & 0xFF == e["bottleneck"], c["name"]
        if "stage_mem" in e:
            assert list(out["stage_mem"][i, :len(e["stage_mem"])]) == e["stage_mem"]
        if "max_mem" in e:
            assert out["max_mem"][i] == e["max_mem"]
        if "iter" in e:
            assert out["iter"][i] == e["iter"], c["name"]
    assert out["iter"][2] < out["iter"][1]  # the migration is faster
    # "better": feasible beats infeasible, then faster
    assert oracle.select(out) == tuple(g["expected"]["select"])


def test_bottleneck_ties_take_lowest_stage():
    prof = mkprof({0: lambda tpl, b: [5, 0, 5, 0, 1, 1, 0, 0, 0, 0]}, [0] * 6, G=3, Bg=1, C=1 << 40)
    out = ev(prof, [cand([2, 2, 2])], [ai.header(0, 3)])   # N = 1: equal T, equal Mem
    assert out["info"][0] & 0xFF == 0
    prof.mem_capacity = 0                                   # all stages OOM, equal Mem
    out = ev(prof, [cand([2, 2, 2])], [ai.header(0, 3)])
    assert out["info"][0] & oracle.INFO_OOM and out["info"][0] & 0xFF == 0


# --------------------------------------------------------------------------
# record lookup: which (type, tp, per-GPU batch) entry is read (R8)
# --------------------------------------------------------------------------
def test_lookup_fingerprint():
    """Single-op model, one stage: T = N*F + D with only fwd_comp set to a fingerprint
    of (type, tpl, b) and dps to a fingerprint of (type, tpl, dpl): a transposed index
    or a wrong per-GPU batch (mbs/dp) shows up as a different number."""
    n_tp = n_dp = 4
    n_b = 4

    def fp(t, tpl, b):
        return 1 + b + 10 * tpl + 100 * t

    recs = {t: (lambda t: (lambda tpl, b: [fp(t, tpl, b), 0, 0, 0, 0, 0, 0, 0, 0, 0]))(t) for t in range(2)}
    dps = np.zeros((2, n_tp, n_dp), np.int64)
    for t, tpl, dpl in itertools.product(range(2), range(n_tp), range(n_dp)):
        dps[t, tpl, dpl] = 1000 * (1 + dpl + 10 * tpl + 100 * t)
    for t in range(2):
        for G in [1, 2, 4, 8]:
            kG = G.bit_length() - 1
            prof = mkprof(recs, [t], n_tp=n_tp, n_b=n_b, n_dp=n_dp, G=G, Bg=64, dps=dps)
            rows, hdrs, exp = [], [], []
            for tpl in range(kG + 1):
                dpl = kG - tpl
                for mbs_log2 in range(dpl, dpl + n_b):
                    rows.append([ai.code(1, tpl, dpl, 0)])
                    hdrs.append(ai.header(mbs_log2, 1))
                    N = 64 >> mbs_log2
                    exp.append(N * fp(t, tpl, mbs_log2 - dpl) + dps[t, tpl, dpl])
            out = ev(prof, rows, hdrs)
            assert [int(x) for x in out["iter"]] == exp


def test_memory_terms_special_cases():
    """One stage, N = 1: Mem = sum W + sum A + max_j peak (P:L229 + P:L234, R4)."""
    vals = [(10, 3, 7, 5), (20, 20, 40, 1), (30, 0, 11, 9)]  # (act, keep, peak, W)
    recs = {t: (lambda v: (lambda tpl, b: [1, 0, 1, 0, v[0], v[1], v[2], 0, 0, 0]))(v)
            for t, v in enumerate(vals)}
    wm = np.array([[[v[3], 0]] for v in vals], np.int64)
    prof = mkprof(recs, [0, 1, 2], G=1, Bg=1, wmem=wm)
    out = ev(prof, [cand([3])], [ai.header(0, 1)])
    assert out["max_mem"][0] == (5 + 1 + 9) + (10 + 20 + 30) + 40
    # recompute op 0: keeps 3 instead of 10, re-materialises 7 transiently (R3)
    out = ev(prof, [cand([3], rc=[1, 0, 0])], [ai.header(0, 1)])
    assert out["max_mem"][0] == 15 + (3 + 20 + 30) + max(7 + 7, 40, 11)


# --------------------------------------------------------------------------
# R5 (inter-stage sends) against the 1F1B simulation: a send occupies its sender
# after the compute and the receiver waits for its end, i.e. the simulation runs with
# F'_i = F_i + [i < p-1] c_fwd and B'_i = B_i + [i > 0] c_bwd. The edge stage that sends
# nothing in one direction gets the same amount of extra compute instead, so the pipeline
# is uniform and Eq. 2 (R1) is exact -- but only if the oracle charges p2p_fwd of each
# non-last stage's LAST op and p2p_bwd of each non-first stage's FIRST op, per microbatch.
# The other ops carry different p2p values that must not be charged.
# --------------------------------------------------------------------------
@pytest.mark.parametrize("p", [2, 3, 4, 5])
@pytest.mark.parametrize("mbs_log2", [0, 1, 3])
def test_p2p_forward_sends_match_1f1b_simulation(p, mbs_log2):
    k, f, b, c = 3, 7, 13, 5
    recs = {0: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, 0, 1000, 0],     # inner op: p2p_fwd never charged
            1: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, 0, c, 0],        # last op of stages 0..p-2
            2: lambda tpl, bb: [f + c, 0, b, 0, 0, 0, 0, 0, 3000, 0]}  # last op of the last stage
    types = ([0] * (k - 1) + [1]) * (p - 1) + [0] * (k - 1) + [2]
    prof = mkprof(recs, types, G=p, Bg=8)
    N = 8 >> mbs_log2
    out = ev(prof, [cand([k] * p)], [ai.header(mbs_log2, p)])
    assert out["info"][0] & oracle.INFO_INVALID == 0
    mk, _ = simulate([k * f + c] * p, [k * b] * p, N)
    assert int(out["iter"][0]) == mk == (N + p - 1) * (k * (f + b) + c)
    assert len(set(int(x) for x in out["stage_T"][0, :p])) == 1


@pytest.mark.parametrize("p", [2, 3, 4, 5])
@pytest.mark.parametrize("mbs_log2", [0, 1, 3])
def test_p2p_backward_sends_match_1f1b_simulation(p, mbs_log2):
    k, f, b, c = 3, 7, 13, 5
    recs = {0: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, 0, 0, 1000],     # inner op: p2p_bwd never charged
            1: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, 0, 0, c],        # first op of stages 1..p-1
            2: lambda tpl, bb: [f, 0, b + c, 0, 0, 0, 0, 0, 0, 3000]}  # first op of stage 0
    types = [2] + [0] * (k - 1) + ([1] + [0] * (k - 1)) * (p - 1)
    prof = mkprof(recs, types, G=p, Bg=8)
    N = 8 >> mbs_log2
    out = ev(prof, [cand([k] * p)], [ai.header(mbs_log2, p)])
    assert out["info"][0] & oracle.INFO_INVALID == 0
    mk, _ = simulate([k * f] * p, [k * b + c] * p, N)
    assert int(out["iter"][0]) == mk == (N + p - 1) * (k * (f + b) + c)
    assert len(set(int(x) for x in out["stage_T"][0, :p])) == 1


# --------------------------------------------------------------------------
# R13 (in-stage tp/dp change: "an all-gather operation might be necessary between the
# two halves") against the 1F1B simulation: the collective runs on the stage's devices between
# the two halves of every microbatch, so the simulated stage takes F'_i = F_i + (changes in
# stage i) x c per microbatch. Stages with fewer changes get the same amount of extra compute,
# so the pipeline is uniform and Eq. 2 (R1) is exact -- but only if the oracle charges the
# RECEIVING op's reshard once per change per microbatch, and nothing at a stage boundary (a
# stage head whose tp/dp differs from the previous stage's last op pays a p2p, not a reshard)
# or at the op before the change.
# --------------------------------------------------------------------------
@pytest.mark.parametrize("p", [1, 2, 3, 4])
@pytest.mark.parametrize("mbs_log2", [1, 2, 3])
@pytest.mark.parametrize("changes", [(1,), (2,), (0, 1), (2, 0, 1)])
def test_reshard_matches_1f1b_simulation(p, mbs_log2, changes):
    k, f, b, c = 6, 7, 13, 5
    ch = [changes[i % len(changes)] for i in range(p)]  # tp/dp changes inside stage i
    most = max(ch)
    recs = {0: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, 1000, 0, 0],          # inner op: never charged
            1: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, c, 0, 0],             # the op after a change
            2: lambda tpl, bb: [f, 0, b, 0, 0, 0, 0, 3000, 0, 0],          # stage head: never charged
            3: lambda tpl, bb: [f + c, 0, b, 0, 0, 0, 0, 1000, 0, 0],      # compensation, 1 change
            4: lambda tpl, bb: [f + 2 * c, 0, b, 0, 0, 0, 0, 1000, 0, 0]}  # compensation, 2 changes
    types, row = [], []
    for i in range(p):
        lay = [(1, 0)] * k  # (tpl, dpl): 2 devices per stage either way (in-stage symmetry)
        recv = [2, 4][:ch[i]]  # ops that receive a new layout
        for j in range(k):
            flips = sum(1 for r in recv if j >= r)
            lay[j] = (1, 0) if flips % 2 == 0 else (0, 1)
        if i % 2 == 1:  # alternate the head's layout: a layout change across the stage boundary
            lay = [(1 - t, 1 - d) for t, d in lay]
        ty = [2] + [0] * (k - 1)
        for r in recv:
            ty[r] = 1
        if most - ch[i] > 0:
            ty[k - 1] = 3 if most - ch[i] == 1 else 4
        types += ty
        row += [ai.code(1 if j == 0 else 0, lay[j][0], lay[j][1], 0) for j in range(k)]
    prof = mkprof(recs, types, n_tp=2, n_b=8, n_dp=2, G=2 * p, Bg=8)
    N = 8 >> mbs_log2
    out = ev(prof, [row], [ai.header(mbs_log2, p)])
    assert out["info"][0] & oracle.INFO_INVALID == 0
    mk, _ = simulate([k * f + most * c] * p, [k * b] * p, N)
    assert int(out["iter"][0]) == mk == (N + p - 1) * (k * (f + b) + most * c)
    assert len(set(int(x) for x in out["stage_T"][0, :p])) == 1


# --------------------------------------------------------------------------
# readings without an independent pin: worked examples (parity unpinned beyond these)
# --------------------------------------------------------------------------
def test_p2p_and_reshard_worked_example():
    """R5: stage i pays p2p_fwd of its last op (i < p-1) and p2p_bwd of its first op
    (i > 0). R13: an in-stage tp/dp change charges the receiving op's reshard.
    Fixture and derivation: tests/golden/p2p_reshard_example.json."""
    g = _golden("p2p_reshard_example.json")

    def r(tpl, b):
        return [v if isinstance(v, int) else int(v.split("+")[0]) + tpl for v in g["record"]]
    pr = g["profile"]
    prof = mkprof({0: r}, [0] * pr["n_ops"], n_tp=pr["n_tp"], n_b=pr["n_b"], n_dp=pr["n_dp"],
                  G=pr["n_devices"], Bg=pr["global_batch"])
    row = [ai.code(*op) for op in g["row"]]
    out = ev(prof, [row], [ai.header(g["mbs_log2"], g["p"])])
    p = g["p"]
    for k in ("stage_T", "stage_comp", "stage_comm"):
        assert list(out[k][0, :p]) == g["expected"][k], k


# --------------------------------------------------------------------------
# invalid encodings
# --------------------------------------------------------------------------
def test_invalid_reasons():
    prof = mkprof({0: lambda tpl, b: [1] * 4 + [2, 1, 1, 1, 1, 1]}, [0] * 4, n_tp=3, n_b=2, n_dp=3,
                  G=4, Bg=8)
    R = {"HEAD0": 1, "NSTAGE": 2, "PRANGE": 4, "GSTAGE": 8, "GSUM": 16, "DPMBS": 32, "TABLE": 64,
         "MBS": 128, "HDR": 256}
    ok = cand([2, 2], tpdp=[(1, 0), (0, 1)])
    cases = [
        (ok, ai.header(1, 2), 0),
        ([ok[0] & 0xFE] + ok[1:], ai.header(1, 2), R["HEAD0"] | R["NSTAGE"]),
        (ok, ai.header(1, 3), R["NSTAGE"]),
        (cand([1, 1, 1, 1]), ai.header(0, 4), 0),
        (cand([1, 1, 1, 1]), ai.header(0, 5), R["NSTAGE"] | R["PRANGE"]),
        ([ok[0], ai.code(0, 0, 0, 0)] + ok[2:], ai.header(1, 2), R["GSTAGE"]),
        (cand([2, 2], tpdp=[(1, 0), (1, 0)]), ai.header(1, 2), 0),
        (cand([2, 2], tpdp=[(1, 0), (0, 0)]), ai.header(1, 2), R["GSUM"]),
        (ok, ai.header(0, 2), R["DPMBS"]),
        (cand([4], tpdp=[(0, 2)]), ai.header(2, 1), 0),
        (cand([4], tpdp=[(0, 2)]), ai.header(3, 1), 0),
        (cand([2, 2], tpdp=[(1, 0), (0, 1)]), ai.header(3, 2), R["TABLE"]),  # b = 3 >= n_b
        (cand([4], tpdp=[(3, 0)]), ai.header(0, 1), R["TABLE"] | R["GSUM"]),
        (ok, ai.header(4, 2), R["MBS"] | R["TABLE"]),
        (ok, ai.header(1, 2) | (1 << 40), R["HDR"]),
    ]
    rows = [c[0] for c in cases]
    hdrs = [c[1] for c in cases]
    out = ev(prof, rows, hdrs)
    for k, (_, _, exp) in enumerate(cases):
        info = int(out["info"][k])
        assert (info >> 18) == exp, (k, info >> 18, exp)
        assert bool(info & oracle.INFO_INVALID) == bool(exp)
        if exp:
            assert out["iter"][k] == 0 and out["max_mem"][k] == 0


# --------------------------------------------------------------------------
# selection: brute force over the exhaustively enumerated toy spaces
# --------------------------------------------------------------------------
def _brute_min(out, offset=0):
    info = out["info"].astype(np.int64)
    valid = (info & oracle.INFO_INVALID) == 0
    if not valid.any():
        return (-1, 0, -1)
    cls = ((info & oracle.INFO_OOM) != 0).astype(np.int64)
    cost = np.where(cls == 1, out["max_mem"], out["iter"]).astype(np.uint64)
    idx = np.arange(len(info), dtype=np.int64) + offset
    keys = [(int(c), int(v), int(i)) for c, v, i, ok in zip(cls, cost, idx, valid) if ok]
    return min(keys)


@pytest.mark.parametrize("name,per_op", [("toy-a", True), ("toy-b", False)])
def test_select_is_exhaustive_optimum(name, per_op):
    prof = P.WORKLOADS[name]()
    codes, hdr = ai.exhaustive(prof, per_op=per_op)
    assert len(hdr) == {"toy-a": 388800, "toy-b": 1388544}[name]
    out = oracle.evaluate(prof, codes, hdr, threads=8)
    best = oracle.select(out)
    assert best == _brute_min(out)
    # the optimum is a feasible configuration, and nothing feasible is faster
    info = out["info"]
    feas = ((info & (oracle.INFO_INVALID | oracle.INFO_OOM)) == 0)
    assert best[0] == 0 and best[1] == int(out["iter"][feas].min())
    # sharded selection with global offsets gives the same winner (§8e)
    parts = np.array_split(np.arange(len(hdr)), 5)
    res = []
    for part in parts:
        sub = {k: v[part] for k, v in out.items()}
        res.append(oracle.select(sub, global_offset=int(part[0])))
    res = [r for r in res if r[2] >= 0]
    assert min(res) == best


def test_select_orders_classes_then_cost_then_index():
    out = dict(iter=np.array([50, 10, 10, 0, 10], np.uint64),
               max_mem=np.array([5, 1, 9, 0, 9], np.uint64),
               info=np.array([oracle.INFO_OOM, oracle.INFO_OOM, 0, oracle.INFO_INVALID, 0], np.uint32))
    assert oracle.select(out) == (0, 10, 2)
    assert oracle.select(out, global_offset=100) == (0, 10, 102)
    out["info"][2] = out["info"][4] = oracle.INFO_OOM
    assert oracle.select(out) == (1, 1, 1)
    out["info"][:] = oracle.INFO_INVALID
    assert oracle.select(out)[2] == -1


# --------------------------------------------------------------------------
# Eq. 1 weight term: parameters + gradients + optimizer state. Mixed-precision
# Adam keeps fp16 weights (2 B) and gradients (2 B) plus fp32 master weights, momentum
# and variance (12 B): the textbook 16 bytes per parameter (ZeRO, Rajbhandari et al.).
# --------------------------------------------------------------------------
def test_mixed_precision_adam_is_16_bytes_per_parameter():
    rng = np.random.default_rng(21)
    for _ in range(20):
        T = int(rng.integers(1, 5))
        L = int(rng.integers(2, 9))
        params = [int(x) for x in rng.integers(1, 10 ** 6, size=T)]
        op_type = [int(x) for x in rng.integers(0, T, size=L)]
        recs = {t: (lambda tpl, b: [3, 0, 5, 0, 0, 0, 0, 0, 0, 0]) for t in range(T)}
        wm = np.array([[[4 * params[t], 12 * params[t]]] for t in range(T)], np.int64)
        p = int(rng.integers(1, min(L, 4) + 1))
        cuts = sorted(int(x) for x in rng.choice(np.arange(1, L), size=p - 1, replace=False))
        sizes = [b - a for a, b in zip([0] + cuts, cuts + [L])]
        prof = mkprof(recs, op_type, G=p, Bg=8, wmem=wm)
        out = ev(prof, [cand(sizes)], [ai.header(1, p)])
        assert out["info"][0] & oracle.INFO_INVALID == 0
        a = 0
        for i, n in enumerate(sizes):
            assert int(out["stage_mem"][0, i]) == 16 * sum(params[t] for t in op_type[a:a + n])
            a += n


# --------------------------------------------------------------------------
# Recomputation memory (R3, R4) against the memory timeline of a 1F1B stage
# (tests/memsim.py). Eq. 1 bounds the timeline from above, and equals it when the op with
# the largest transient is the stage's last op: there the recomputed op's rebuilt
# activations (act - keep) and its workspace coexist with every stashed microbatch.
# --------------------------------------------------------------------------
def test_recompute_transient_matches_memory_timeline():
    from tests.memsim import stage_memory_peak
    rng = np.random.default_rng(23)
    checked = 0
    for _ in range(60):
        p = int(rng.integers(1, 5))
        k = int(rng.integers(2, 5))
        L = p * k
        vals = []
        for j in range(L):
            act = int(rng.integers(10, 1000))
            keep = int(rng.integers(0, act + 1))
            peak = int(rng.integers(0, 200))
            vals.append((act, keep, peak))
        rc = [int(x) for x in rng.integers(0, 2, size=L)]
        for i in range(p):  # each stage's last op: recomputed, the largest transient
            j = i * k + k - 1
            act = 5000 + int(rng.integers(0, 1000))
            vals[j] = (act, int(rng.integers(0, 100)), 300 + int(rng.integers(0, 100)))
            rc[j] = 1
        recs = {j: (lambda v: (lambda tpl, b: [1, 0, 1, 0, v[0], v[1], v[2], 0, 0, 0]))(vals[j])
                for j in range(L)}
        Wt = [int(x) for x in rng.integers(0, 10 ** 4, size=L)]
        wm = np.array([[[Wt[j], 0]] for j in range(L)], np.int64)
        prof = mkprof(recs, list(range(L)), G=p, Bg=16, wmem=wm)
        mbs_log2 = int(rng.integers(0, 5))
        N = 16 >> mbs_log2
        out = ev(prof, [cand([k] * p, rc=rc)], [ai.header(mbs_log2, p)])
        assert out["info"][0] & oracle.INFO_INVALID == 0
        for i in range(p):
            ops = [vals[j] + (rc[j],) for j in range(i * k, i * k + k)]
            sim = stage_memory_peak(ops, sum(Wt[i * k:i * k + k]), p, i, N)
            assert int(out["stage_mem"][0, i]) == sim
            checked += 1
    assert checked > 100


def test_eq1_bounds_the_memory_timeline():
    """Any stage composition: the timeline never exceeds Eq. 1 (R3, R4: conservative)."""
    from tests.memsim import stage_memory_peak
    rng = np.random.default_rng(29)
    for _ in range(60):
        p = int(rng.integers(1, 5))
        k = int(rng.integers(1, 5))
        L = p * k
        vals = []
        for j in range(L):
            act = int(rng.integers(0, 1000))
            vals.append((act, int(rng.integers(0, act + 1)), int(rng.integers(0, 3000))))
        rc = [int(x) for x in rng.integers(0, 2, size=L)]
        recs = {j: (lambda v: (lambda tpl, b: [1, 0, 1, 0, v[0], v[1], v[2], 0, 0, 0]))(vals[j])
                for j in range(L)}
        prof = mkprof(recs, list(range(L)), G=p, Bg=16)
        mbs_log2 = int(rng.integers(0, 5))
        out = ev(prof, [cand([k] * p, rc=rc)], [ai.header(mbs_log2, p)])
        for i in range(p):
            ops = [vals[j] + (rc[j],) for j in range(i * k, i * k + k)]
            assert stage_memory_peak(ops, 0, p, i, 16 >> mbs_log2) <= int(out["stage_mem"][0, i])


# --------------------------------------------------------------------------
# FULL outputs (Heuristic-2's per-stage resource consumption) with every term
# present: each record field is a distinct power of ten, so the per-stage totals read as
# digit counts and a dropped or misattributed term changes a digit.
#   fwd_comp 1, fwd_comm 10, bwd_comp 100, bwd_comm 1000, reshard 1e4, p2p_fwd 1e5,
#   p2p_bwd 1e6; DP sync 1e7 per op with dp = 2 (0 with dp = 1, no data parallelism)
# --------------------------------------------------------------------------
def test_full_outputs_resource_split_fingerprint():
    prof = mkprof({0: lambda tpl, b: [1, 10, 100, 1000, 0, 0, 0, 10 ** 4, 10 ** 5, 10 ** 6]},
                  [0] * 5, n_tp=2, n_b=2, n_dp=2, G=4, Bg=8,
                  dps=[[[0, 10 ** 7], [0, 10 ** 7]]])
    # stage 0 (2 devices): op0 tp2/dp1 (head), op1 tp1/dp2 (tp/dp change: reshard), op2 tp1/dp2 rc
    # stage 1 (2 devices): op3 tp1/dp2 (head), op4 tp1/dp2 rc
    row = [ai.code(1, 1, 0, 0), ai.code(0, 0, 1, 0), ai.code(0, 0, 1, 1),
           ai.code(1, 0, 1, 0), ai.code(0, 0, 1, 1)]
    out = ev(prof, [row], [ai.header(1, 2)])  # mbs 2, N = 4
    assert out["info"][0] & oracle.INFO_INVALID == 0
    N = 4
    # compute per microbatch: 3 ops x (fwd 1 + bwd 100) + 1 recomputed forward = 304 / 203
    assert list(out["stage_comp"][0, :2]) == [N * 304, N * 203]
    # communication per microbatch: 3 x (10 + 1000) + 10 (recomputed forward collective)
    #   + 1e4 (reshard into op1) + 1e5 (p2p_fwd of op2: stage 0 sends forward)  = 113,040
    #   stage 1: 2 x 1010 + 10 + 1e6 (p2p_bwd of op3: stage 1 sends backward) = 1,002,030
    # plus the DP sync once per iteration: 2 ops with dp = 2 on each stage    = 2e7
    assert list(out["stage_comm"][0, :2]) == [N * 113040 + 2 * 10 ** 7, N * 1002030 + 2 * 10 ** 7]
    S0, S1 = 304 + 113040, 203 + 1002030
    assert list(out["stage_T"][0, :2]) == [S0 + S1 + (N - 1) * S0 + 2 * 10 ** 7,
                                           S0 + S1 + (N - 1) * S1 + 2 * 10 ** 7]


def test_heuristic1_memory_first_when_oom():
    """Heuristic-1 when the largest-memory stage is not the slowest one: out of
    memory -> the largest-memory stage; feasible -> the slowest stage."""
    # stage 0: 1 light op (memory-heavy: 3 in-flight microbatches of 40 B); stage 1: 3 slow ops
    recs = {0: lambda tpl, b: [1, 0, 1, 0, 40, 40, 0, 0, 0, 0],
            1: lambda tpl, b: [50, 0, 70, 0, 1, 1, 0, 0, 0, 0]}
    for cap, oom, neck in [(60, True, 0), (1 << 20, False, 1)]:
        prof = mkprof(recs, [0, 1, 1, 1], G=2, Bg=8, C=cap)
        out = ev(prof, [cand([1, 3])], [ai.header(1, 2)])   # N = 4, in-flight 2 / 1
        assert list(out["stage_mem"][0, :2]) == [80, 3]
        assert out["stage_T"][0, 1] > out["stage_T"][0, 0]
        assert bool(out["info"][0] & oracle.INFO_OOM) == oom
        assert out["info"][0] & 0xFF == neck


# --------------------------------------------------------------------------
# Tensor-parallel partition dimension (§4.2): an op can run under its
# alternative partition dimension (row- vs column-wise MatMul, input- vs output-channel
# convolution); choosing it reads the records profiled for that dimension in every term.
# --------------------------------------------------------------------------
DEF_FP = [1, 2, 4, 8, 16, 0, 32, 64, 128, 256]        # fc fm bc bm act keep peak rs p2pf p2pb
ALT_FP = [1000 * v for v in DEF_FP]


def _dim_prof(op_type, n_tp=2, n_dp=2, G=2, Bg=8):
    T = max(op_type) + 1
    prof = mkprof({t: (lambda tpl, b: DEF_FP) for t in range(T)}, op_type, n_tp=n_tp, n_dp=n_dp,
                  n_b=4, G=G, Bg=Bg)
    prof.rec_alt = np.zeros_like(prof.rec)
    prof.rec_alt[...] = np.array(ALT_FP, np.int64)
    return prof


@pytest.mark.parametrize("d0,d1", [(0, 0), (0, 1), (1, 0), (1, 1)])
def test_dimension_fingerprint_two_stages(d0, d1):
    """Two single-op stages: each stage's time reads its op's own dimension's compute,
    collectives and send (stage 0 pays op 0's p2p_fwd, stage 1 op 1's p2p_bwd, R5)."""
    prof = _dim_prof([0, 0])
    out = oracle.evaluate(prof, np.array([cand([1, 1])], np.uint8), np.array([ai.header(1, 2)], np.uint64),
                          full=True, dims=np.array([[d0, d1]], np.uint8))
    assert out["info"][0] & oracle.INFO_INVALID == 0
    fp = [DEF_FP, ALT_FP]
    f0, f1 = fp[d0], fp[d1]
    N = 4
    S0 = f0[0] + f0[1] + f0[2] + f0[3] + f0[8]
    S1 = f1[0] + f1[1] + f1[2] + f1[3] + f1[9]
    assert list(out["stage_T"][0, :2]) == [S0 + S1 + (N - 1) * S0, S0 + S1 + (N - 1) * S1]
    assert list(out["stage_comp"][0, :2]) == [N * (f0[0] + f0[2]), N * (f1[0] + f1[2])]
    assert list(out["stage_comm"][0, :2]) == [N * (f0[1] + f0[3] + f0[8]), N * (f1[1] + f1[3] + f1[9])]
    assert list(out["stage_mem"][0, :2]) == [min(2, N) * f0[4] + f0[6], 1 * f1[4] + f1[6]]


@pytest.mark.parametrize("d1", [0, 1])
def test_dimension_fingerprint_reshard_and_recompute(d1):
    """One stage of two ops with a tp/dp change at op 1 (R13 reshard into op 1) and op 1
    recomputed (R3, R4): the reshard, the recomputed forward and the kept /
    transient bytes all come from op 1's dimension."""
    prof = _dim_prof([0, 0])
    row = [ai.code(1, 1, 0, 0), ai.code(0, 0, 1, 1)]  # (tp2, dp1) then (tp1, dp2), op 1 recomputed
    out = oracle.evaluate(prof, np.array([row], np.uint8), np.array([ai.header(1, 1)], np.uint64),
                          full=True, dims=np.array([[0, d1]], np.uint8))
    assert out["info"][0] & oracle.INFO_INVALID == 0
    f0, f1 = DEF_FP, [DEF_FP, ALT_FP][d1]
    N = 4
    S = (f0[0] + f0[1] + f0[2] + f0[3]) + (f1[0] + f1[1] + f1[2] + f1[3]) + (f1[0] + f1[1]) + f1[7]
    assert int(out["stage_T"][0, 0]) == N * S
    assert int(out["stage_mem"][0, 0]) == f0[4] + f1[5] + max(f0[6], f1[6] + f1[4] - f1[5])


def test_dimension_choice_with_identical_records_changes_nothing():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    prof.rec_alt = prof.rec.copy()
    codes, hdr = ai.search_shaped(prof, 31, 0, 300, group_size=16)
    rng = np.random.default_rng(2)
    dims = rng.integers(0, 2, size=codes.shape, dtype=np.uint8)
    a = oracle.evaluate(prof, codes, hdr, full=True)
    b = oracle.evaluate(prof, codes, hdr, full=True, dims=dims)
    for k in a:
        assert np.array_equal(a[k], b[k]), k


def test_dimension_flip_is_local_to_its_op():
    """Flipping the dimension of op j (not a stage edge) changes stage i's per-microbatch time by
    the op's own difference d = S_alt(j) - S_def(j): T_i by N d, every other T_k by d (Eq. 2)."""
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, hdr = ai.search_shaped(prof, 33, 0, 200, group_size=16, invalid_permille=0)
    base = oracle.evaluate(prof, codes, hdr, full=True)
    rng = np.random.default_rng(4)
    checked = 0
    for c in range(len(hdr)):
        if base["info"][c] & oracle.INFO_INVALID:
            continue
        heads = np.nonzero(codes[c] & 1)[0]
        j = int(rng.integers(1, prof.n_ops - 1))
        if j in heads or (j + 1) in heads or codes[c, j] & 0x10:
            continue
        if (codes[c, j] ^ codes[c, j - 1]) & 0xEE:
            continue
        dims = np.zeros((1, prof.n_ops), np.uint8)
        dims[0, j] = 1
        new = oracle.evaluate(prof, codes[c:c + 1], hdr[c:c + 1], full=True, dims=dims)
        tpl, dpl = (int(codes[c, j]) >> 1) & 7, (int(codes[c, j]) >> 5) & 7
        b = (int(hdr[c]) & 0xFF) - dpl
        t = prof.op_type[j]
        d = int(prof.rec_alt[t, tpl, b, :4].sum()) - int(prof.rec[t, tpl, b, :4].sum())
        i = int(np.sum(codes[c, :j + 1] & 1)) - 1
        N = prof.global_batch >> (int(hdr[c]) & 0xFF)
        p = (int(hdr[c]) >> 8) & 0xFF
        for k in range(p):
            delta = int(new["stage_T"][0, k]) - int(base["stage_T"][c, k])
            assert delta == (N * d if k == i else d)
        checked += 1
    assert checked > 50


@pytest.mark.parametrize("p", [1, 2, 3, 5])
@pytest.mark.parametrize("mbs_log2", [0, 2])
def test_literal_eq2_counts_one_more_microbatch(p, mbs_log2):
    """ACESO_PIPE_LITERAL (reading R1's variant): Eq. 2 as printed -- warm-up of a
    microbatch through all stages, N steady microbatches of stage i, cool-down -- is the 1F1B
    makespan of uniform stages plus one more stage time: (N+p)(f+b)."""
    k, f_op, b_op = 2, 5, 11
    prof = mkprof({0: lambda tpl, b: [f_op, 0, b_op, 0, 1, 0, 0, 0, 0, 0]}, [0] * (p * k), G=p, Bg=8)
    N = 8 >> mbs_log2
    out = oracle.evaluate(prof, np.array([cand([k] * p)], np.uint8), np.array([ai.header(mbs_log2, p)], np.uint64),
                          literal=True)
    mk, _ = simulate([f_op * k] * p, [b_op * k] * p, N)
    assert int(out["iter"][0]) == mk + (f_op + b_op) * k == (N + p) * (f_op + b_op) * k
