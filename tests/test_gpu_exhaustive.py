"""Exp#4 baseline (exhaustive stage-uniform space, aceso_enum_cuts + aceso_eval): the device
enumeration equals the colex statement of the header byte for byte, and the space's optimum
equals the oracle's minimum over the same configurations (toy spaces: all of them; GPT-3 1.3B:
the optimum re-evaluated by the oracle, and sampled enumeration rows)."""
import itertools

import numpy as np
import pytest
import torch

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P

pytestmark = pytest.mark.gpu
A = pytest.importorskip("paper_conf_eurosys_liumlsmybw24_b200")
from paper_conf_eurosys_liumlsmybw24_b200 import exhaustive as X  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _enumerate(prof, fam, first, n):
    dev = torch.device("cuda")
    tiled = torch.zeros(A.tiled_bytes(n, prof.n_ops), dtype=torch.uint8, device=dev)
    hd = torch.zeros(n, dtype=torch.int64, device=dev)
    A.enum_cuts(prof.n_ops, fam[0], fam[1], fam[2], first, n, tiled, hd)
    torch.cuda.synchronize()
    return tiled.cpu().numpy(), hd.cpu().numpy().view(np.uint64)


@pytest.mark.parametrize("name,p,first,n", [("toy-b", 1, 0, 1), ("toy-b", 2, 0, 9), ("toy-b", 4, 0, 84),
                                            ("gpt3-1.3b", 2, 0, 314), ("gpt3-1.3b", 4, 5_000_000, 777),
                                            ("t5", 4, 123_456, 300)])
def test_enumeration_matches_colex_statement(name, p, first, n):
    prof = P.WORKLOADS[name]()
    fam = next(f for f in X.families(prof) if f[0] == p)
    tiled, hdr = _enumerate(prof, fam, first, n)
    rows = np.stack([X.configuration(prof, fam, first + r)[0] for r in range(n)])
    assert np.array_equal(tiled, ai.tile(rows))
    assert (hdr == np.uint64(fam[2])).all()
    if p == 3 or (p <= 4 and n == A.enum_cuts_count(prof.n_ops, p)):  # the whole family: all subsets once
        cuts = {tuple(np.nonzero(r & 1)[0][1:]) for r in rows}
        assert cuts == set(itertools.combinations(range(1, prof.n_ops), p - 1))


@pytest.mark.parametrize("name", ["toy-a", "toy-b"])
def test_exhaustive_optimum_equals_oracle_minimum(name):
    prof = P.WORKLOADS[name]()
    ctx = A.Context(prof, 0)
    try:
        res = X.exhaustive_best(prof, ctx, batch=64)
        fams = X.families(prof)
        codes, hdr = [], []
        for f in fams:
            for r in range(f[3]):
                c, h = X.configuration(prof, f, r)
                codes.append(c)
                hdr.append(h)
        o = oracle.evaluate(prof, np.stack(codes), np.array(hdr, np.uint64))
        cls, cost, idx = oracle.select(o)
        assert res["explored"] == len(hdr)
        assert (res["best"]["class"], res["best"]["cost"], res["best"]["index"]) == (cls, cost, idx)
    finally:
        ctx.close()


def test_exhaustive_gpt3_optimum_reevaluated_by_oracle():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    ctx = A.Context(prof, 0)
    try:
        res = X.exhaustive_best(prof, ctx)
        assert res["explored"] == sum(f[3] for f in X.families(prof)) > 10 ** 8
        b = res["best"]
        o = oracle.evaluate(prof, res["codes"][None, :], np.array([res["hdr"]], np.uint64))
        assert int(o["info"][0]) & oracle.INFO_INVALID == 0
        cost = int(o["iter"][0]) if b["class"] == 0 else int(o["max_mem"][0])
        assert cost == b["cost"]
        # a sample of the space is no better than the reported optimum (oracle)
        fams = X.families(prof)
        rng = np.random.default_rng(7)
        rows, hs = [], []
        for _ in range(2000):
            f = fams[int(rng.integers(0, len(fams)))]
            c, h = X.configuration(prof, f, int(rng.integers(0, f[3])))
            rows.append(c)
            hs.append(h)
        os_ = oracle.evaluate(prof, np.stack(rows), np.array(hs, np.uint64), threads=8)
        ocls, ocost, _ = oracle.select(os_)
        assert (b["class"], b["cost"]) <= (ocls, ocost)
    finally:
        ctx.close()
