"""Search driver (Alg. 1/2, Heuristic-1/2, Table 1 primitives) with a CPU
evaluator built on the oracle (tests only); the product runs it with GPUEvaluator."""
import numpy as np
import pytest

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P
from paper_conf_eurosys_liumlsmybw24_b200 import search as S


import os  # noqa: E402
import sys  # noqa: E402

sys.path.insert(0, os.path.dirname(__file__))
from oracle_evaluator import OracleEvaluator  # noqa: E402


def perf_tuple(out, i):
    return S.perf_of(int(out["info"][i]), out["iter"][i], out["max_mem"][i])


def test_primitives_keep_encodings_valid_structure():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, mbs = S.initial_config(prof, 4)
    ev = OracleEvaluator(prof)
    base = ev.evaluate(codes[None, :], np.array([S.header(mbs, 4)], np.uint64))
    prim = S.Primitives(prof, heuristic2=False)
    cands = prim.apply_all(codes, mbs, int(base["info"][0]), base["stage_comp"][0],
                           base["stage_comm"][0], base["stage_T"][0])
    assert len(cands) > 100
    cc = np.stack([c for c, _ in cands])
    hdr = np.array([S.header(int(m), int((c & 1).sum())) for c, m in cands], np.uint64)
    out = ev.evaluate(cc, hdr)
    # op moves / trades preserve the device sum and the head count: almost all valid
    valid = (out["info"] & oracle.INFO_INVALID) == 0
    assert valid.mean() > 0.9
    # every candidate differs from the base
    assert all(not (np.array_equal(c, codes) and m == mbs) for c, m in cands)


@pytest.mark.parametrize("first", ["dp", "tp"])
def test_initial_configs_are_valid(first):
    """Both device splits of the initial configuration (R28) are valid configurations with an
    even partition and the minimum microbatch; dp-first puts a stage's devices into data
    parallelism up to the profile's range, tp-first into tensor parallelism."""
    for name in ["toy-a", "gpt3-1.3b", "gpt3-13b", "t5", "wrn"]:
        prof = P.WORKLOADS[name]()
        for p in [1, 2, 4]:
            r = S.initial_config(prof, p, first)
            assert r is not None
            codes, mbs = r
            out = oracle.evaluate(prof, codes[None, :], np.array([S.header(mbs, p)], np.uint64))
            assert not out["info"][0] & oracle.INFO_INVALID, (name, p, out["info"][0] >> 18)
            assert list(np.flatnonzero(codes & 1)) == [prof.n_ops * i // p for i in range(p)]
            tpl, dpl = (codes >> 1) & 7, codes >> 5
            assert mbs == int(dpl.max())
            k = int(np.log2(prof.n_devices // p))
            if first == "tp":
                assert np.all(tpl == min(k, prof.n_tp - 1))
            else:
                assert np.all(dpl == min(k, prof.n_dp - 1))


def test_search_improves_and_is_deterministic():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    r1, st1 = S.search(prof, OracleEvaluator(prof), p_values=[2, 4], budget_s=60, max_hops=3, beam=2,
                       max_k=8, patience=4)
    r2, st2 = S.search(prof, OracleEvaluator(prof), p_values=[2, 4], budget_s=60, max_hops=3, beam=2,
                       max_k=8, patience=4)
    assert r1.perf == r2.perf and np.array_equal(r1.codes, r2.codes)
    # better than every initial configuration ("better")
    inits = []
    for p in [2, 4]:
        c, m = S.initial_config(prof, p)
        o = oracle.evaluate(prof, c[None, :], np.array([S.header(m, p)], np.uint64))
        inits.append(perf_tuple(o, 0))
    assert r1.perf < min(inits)
    assert st1["improvements"] > 0
    # the returned configuration re-evaluates to the reported performance
    o = oracle.evaluate(prof, r1.codes[None, :], np.array([S.header(r1.mbs, int((r1.codes & 1).sum()))], np.uint64))
    assert perf_tuple(o, 0) == r1.perf


def test_search_on_toy_reaches_a_feasible_near_optimum():
    """toy-A: the exhaustive optimum is known (388,800 configurations); the search
    finds a feasible configuration within 10% of it (not guaranteed to be optimal)."""
    prof = P.toy_a()
    codes, hdr = ai.exhaustive(prof, per_op=True)
    best = oracle.select(oracle.evaluate(prof, codes, hdr, threads=8))
    r, st = S.search(prof, OracleEvaluator(prof), budget_s=30, max_hops=7, beam=4)
    assert r.perf[0] == 0
    assert r.perf[1] <= best[1] * 1.10


@pytest.mark.parametrize("name", ["gpt3-1.3b", "t5", "wrn", "toy-b"])
def test_optimised_primitives_match_reference(name):
    """The generator (stage structure computed once per node, vectorised fine-tune checks)
    yields exactly the candidates of the first, one-pass-per-candidate version."""
    import importlib.util
    import os
    spec = importlib.util.spec_from_file_location(
        "_search_reference", os.path.join(os.path.dirname(__file__), "_search_reference.py"))
    R = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(R)
    prof = P.WORKLOADS[name]()
    codes, hdr = ai.search_shaped(prof, 99, 0, 60, group_size=8)
    o = oracle.evaluate(prof, codes, hdr)
    rng = np.random.default_rng(3)
    checked = 0
    for i in np.nonzero((o["info"] & oracle.INFO_INVALID) == 0)[0][:25]:
        c, mbs = codes[i], int(hdr[i] & 0xFF)
        p = int((c & 1).sum())
        G = prof.n_devices
        for h2, oom, mk in [(True, False, None), (True, True, 6), (False, False, 3)]:
            info = int(rng.integers(0, p)) | (S.INFO_OOM if oom else 0)
            comp = rng.integers(1, 1000, size=G).astype(np.uint64)
            comm = rng.integers(1, 1000, size=G).astype(np.uint64)
            stt = rng.integers(1, 1000, size=G).astype(np.uint64)
            a = S.Primitives(prof, heuristic2=h2, max_k=mk).apply_all(c, mbs, info, comp, comm, stt)
            b = R.PrimitivesReference(prof, heuristic2=h2, max_k=mk).apply_all(c, mbs, info, comp, comm, stt)
            assert len(a) == len(b)
            for (ca, ma), (cb, mb) in zip(a, b):
                assert ma == mb and np.array_equal(ca, cb)
            checked += len(a)
    assert checked > 500


@pytest.mark.parametrize("name", ["gpt3-1.3b", "t5", "wrn", "toy-b"])
def test_descriptors_expand_to_the_reference_candidates(name):
    """Primitives.describe_all (base + patches, evaluated after aceso_expand) expands to
    exactly the candidates of the reference generator, in the same order."""
    import importlib.util
    import os
    from paper_conf_eurosys_liumlsmybw24_b200 import candidates as C
    spec = importlib.util.spec_from_file_location(
        "_search_reference", os.path.join(os.path.dirname(__file__), "_search_reference.py"))
    R = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(R)
    prof = P.WORKLOADS[name]()
    codes, hdr = ai.search_shaped(prof, 98, 0, 60, group_size=8)
    o = oracle.evaluate(prof, codes, hdr)
    rng = np.random.default_rng(5)
    checked = 0
    L = prof.n_ops
    for i in np.nonzero((o["info"] & oracle.INFO_INVALID) == 0)[0][:20]:
        c, mbs = codes[i], int(hdr[i] & 0xFF)
        p = int((c & 1).sum())
        G = prof.n_devices
        for h2, oom, mk in [(True, False, None), (True, True, 5), (False, False, 3)]:
            info = int(rng.integers(0, p)) | (S.INFO_OOM if oom else 0)
            comp = rng.integers(1, 1000, size=G).astype(np.uint64)
            comm = rng.integers(1, 1000, size=G).astype(np.uint64)
            stt = rng.integers(1, 1000, size=G).astype(np.uint64)
            ref = R.PrimitivesReference(prof, heuristic2=h2, max_k=mk).apply_all(c, mbs, info, comp, comm, stt)
            cands, ranks = S.Primitives(prof, heuristic2=h2, max_k=mk).describe_all(c, mbs, info, comp, comm, stt)
            assert len(cands) == len(ref)
            bases = np.zeros((1, C.stride_of(L)), np.uint8)
            bases[0, :L] = c
            got, ghdr = C.expand_host(bases, ranks[None], cands, L)
            for k, (cr, mr) in enumerate(ref):
                assert np.array_equal(got[k], cr), (k, cands[k])
                assert int(ghdr[k] & np.uint64(0xFF)) == mr and int(ghdr[k] >> np.uint64(8)) == p
            checked += len(ref)
    assert checked > 500


def test_first_new_dedup_is_first_occurrence_against_visited():
    """_first_new (configuration dedup) equals the plain set loop: first occurrence
    in generation order of every hash not seen before; the visited array stays sorted."""
    rng = np.random.default_rng(3)
    visited_set = set()
    visited = np.zeros(0, np.uint64)
    for _ in range(6):
        hs = rng.integers(0, 50, size=200).astype(np.uint64)
        want = np.zeros(len(hs), bool)
        for i, h in enumerate(hs.tolist()):
            if h not in visited_set:
                visited_set.add(h)
                want[i] = True
        keep, visited = S._first_new(hs, visited)
        assert np.array_equal(keep, want)
        assert np.array_equal(visited, np.array(sorted(visited_set), np.uint64))


def test_heuristic2_resource_order_and_secondary_bottleneck():
    """Heuristic-2: resources by the bottleneck stage's consumption proportion;
    an OOM configuration puts memory first. The secondary bottleneck is the next
    stage of Heuristic-1's order."""
    comp = np.array([10, 30, 60], np.uint64)   # stage 1: 30% of compute
    comm = np.array([50, 40, 10], np.uint64)   # stage 1: 40% of communication
    mem = np.array([20, 50, 30], np.uint64)    # stage 1: 50% of memory
    assert S.resource_order(1, comp, comm, mem, 3, 1) == ["mem", "comm", "comp"]
    assert S.resource_order(1, comp, comm, None, 3, 1) == ["comm", "comp"]
    assert S.resource_order(S.INFO_OOM | 2, comp, comm, mem, 3, 2)[0] == "mem"
    assert S.resource_order(2, comp, comm, mem, 3, 2) == ["comp", "mem", "comm"]
    t = np.array([5, 9, 7], np.uint64)
    assert S.bottleneck_rank(1, mem, t, 3, 0) == 1
    assert S.bottleneck_rank(1, mem, t, 3, 1) == 2           # by time
    assert S.bottleneck_rank(S.INFO_OOM | 1, mem, t, 3, 1) == 2  # by memory: 50 > 30 > 20


def test_rc_attachment_is_greedy_by_activation():
    """Attached inc-rc: the k-th variant recomputes the k largest-activation
    ops of the memory bottleneck that were not recomputed; dec-rc releases smallest first."""
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, mbs = S.initial_config(prof, 4)
    heads, ends = S.stages_of(codes)
    a, e = int(heads[2]), int(ends[2])
    vs = S._rc_variants(prof, codes, mbs, S.INFO_OOM | 2, None, None)
    ks = S._greedy_counts(e - a)
    assert len(vs) == len(ks) and ks[:16] == list(range(1, 17)) and ks[-1] == e - a
    tpl, dpl = (codes[a] >> 1) & 7, (codes[a] >> 5) & 7
    act = prof.rec[prof.op_type[a:e], tpl, mbs - dpl, 4]
    prev = set()
    for k, v in zip(ks, vs):
        on = set(np.nonzero(v & 0x10)[0].tolist())
        assert len(on) == k and prev < on and all(a <= j < e for j in on)
        # the added ops are the largest activations among those not yet recomputed
        rest = sorted((act[j - a] for j in range(a, e) if j not in prev), reverse=True)
        assert sorted((act[j - a] for j in on - prev), reverse=True) == rest[:len(on - prev)]
        prev = on
    full = vs[-1]
    back = S._rc_variants(prof, full, mbs, 2, None, None)
    assert len(back) == len(ks) and not (back[-1] & 0x10).any()


def test_search_with_attachment_and_root_modes_returns_a_reproducible_configuration():
    prof = P.WORKLOADS["gpt3-13b"]()
    r, st = S.search(prof, OracleEvaluator(prof), p_values=[4, 8], budget_s=120, max_hops=2, beam=2,
                     max_k=4, patience=3, attach_rc=4)
    o = oracle.evaluate(prof, r.codes[None, :], np.array([S.header(r.mbs, int((r.codes & 1).sum()))], np.uint64))
    assert perf_tuple(o, 0) == r.perf and st["evaluated"] > 0


def test_dimension_finetune_improves_or_keeps():
    """§4.2: the greedy per-op dimension fine-tune never returns a worse
    configuration, and its result re-evaluates to the reported performance."""
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, mbs = S.initial_config(prof, 2)
    for s in range(2):  # 4 devices per stage as tp 2 x dp 2: MatMuls have two dimensions
        codes = S._recode_stage(codes, s, 1, -1)
    ev = OracleEvaluator(prof)
    base = ev.evaluate(codes[None, :], np.array([S.header(mbs, 2)], np.uint64))
    assert not base["info"][0] & oracle.INFO_INVALID
    dims, perf, st = S.finetune_dims(prof, ev, codes, mbs, max_rounds=6)
    assert perf <= perf_tuple(base, 0) and st["rounds"] >= 1
    o = oracle.evaluate(prof, codes[None, :], np.array([S.header(mbs, 2)], np.uint64), dims=dims[None, :])
    assert perf_tuple(o, 0) == perf
    assert len(st["switched"]) == int(dims.sum())


@pytest.mark.parametrize("name", ["toy-a", "gpt3-1.3b", "t5", "wrn"])
def test_megatron_grid_space(name):
    """The Megatron-LM baseline space: every configuration is valid under the
    oracle, uses global settings (one (tp, dp, recompute) for all ops, even op partition),
    covers each (p, tp, recompute, microbatch) combination once, and megatron_best returns its
    (class, cost, lowest index) optimum."""
    from paper_conf_eurosys_liumlsmybw24_b200 import exhaustive as X
    prof = P.WORKLOADS[name]()
    codes, hdr = X.megatron_grid(prof)
    L, G = prof.n_ops, prof.n_devices
    o = oracle.evaluate(prof, codes, hdr, threads=4)
    assert not np.any(o["info"] & oracle.INFO_INVALID)
    seen = set()
    for c, h in zip(codes, hdr):
        p, mbs = int(h) >> 8, int(h) & 0xFF
        heads = np.flatnonzero(c & 1)
        assert list(heads) == [L * i // p for i in range(p)]
        body = c & 0xFE
        assert np.all(body == body[0])
        tpl, dpl = (int(body[0]) >> 1) & 7, int(body[0]) >> 5
        assert p << (tpl + dpl) == G
        key = (p, tpl, (int(body[0]) >> 4) & 1, mbs)
        assert key not in seen
        seen.add(key)
    n_rc = 2
    assert len(seen) % n_rc == 0
    r = X.megatron_best(prof, OracleEvaluator(prof))
    keys = [S.perf_of(int(i), t, m) for i, t, m in zip(o["info"], o["iter"], o["max_mem"])]
    best = min((k, i) for i, k in enumerate(keys) if k[0] < 2)
    assert (r["best"]["class"], r["best"]["cost"], r["best"]["index"]) == (best[0][0], best[0][1], best[1])


def test_oom_excess_tie_break():
    """R26: the excess sum_i max(0, Mem_i - C) over a candidate's p stages, OOM candidates only."""
    C = 100
    info = np.array([(2 << 8) | S.INFO_OOM, (3 << 8) | S.INFO_OOM, (2 << 8), (2 << 8) | S.INFO_OOM | S.INFO_INVALID],
                    np.uint32)
    sm = np.array([[150, 120, 999], [101, 90, 130], [150, 150, 150], [500, 500, 500]], np.uint64)
    ex = S._oom_excess(dict(info=info, stage_mem=sm), C)
    assert list(ex) == [70, 31, 0, 0]


def test_oom_phase_fixes_a_whole_stage_per_batch():
    """With R26 the 1K-layer model's 8-stage search (initial configuration OOM: every stage
    holds its in-flight activations) becomes feasible within ten batches (five hops with their recompute attachment): each recompute move
    fixes the whole bottleneck stage instead of stopping at the next stage's memory."""
    prof = P.WORKLOADS["gpt-1k"]()
    res, st = S.search(prof, OracleEvaluator(prof), p_values=[8], budget_s=1e9, max_batches=10)
    assert res.perf[0] == 0, res.perf
