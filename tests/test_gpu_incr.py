"""Incremental evaluation (aceso_eval_incr): bit-exact against the
oracle on the expanded candidates, for the search driver's primitives (moves, relays,
trades, recompute, fine-tune, microbatch changes), arbitrary patches, invalid bases, FULL
mode and the fused selection."""
import numpy as np
import pytest
import torch

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P

pytestmark = pytest.mark.gpu
A = pytest.importorskip("paper_conf_eurosys_liumlsmybw24_b200")
from paper_conf_eurosys_liumlsmybw24_b200 import candidates as C  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200 import search as S  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200.api import Selection, as_u32, as_u64  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def search_batch(prof, seed, nbases=6, random_patches=0):
    """Descriptors of the search driver's primitives on valid search-shaped bases."""
    L, stride = prof.n_ops, C.stride_of(prof.n_ops)
    codes, hdr = ai.search_shaped(prof, seed, 0, 200, group_size=8)
    o = oracle.evaluate(prof, codes, hdr, full=True)
    ok = np.nonzero((o["info"] & oracle.INFO_INVALID) == 0)[0][:nbases]
    rng = np.random.default_rng(seed)
    bases = np.zeros((len(ok), stride), np.uint8)
    bhdr = np.zeros(len(ok), np.uint64)
    ranks = np.zeros((len(ok), 2, stride), np.uint16)
    chunks = []
    for bi, i in enumerate(ok):
        bases[bi, :L] = codes[i]
        bhdr[bi] = hdr[i]
        p = int((codes[i] & 1).sum())
        info = int(o["info"][i]) if rng.random() < 0.5 else int(rng.integers(0, p))
        cd, rk = S.Primitives(prof, heuristic2=False, max_k=12).describe_all(
            codes[i], int(hdr[i] & 0xFF), info, o["stage_comp"][i], o["stage_comm"][i], o["stage_T"][i])
        cd["base"] = bi
        ranks[bi] = rk
        chunks.append(cd)
    cands = np.concatenate(chunks)
    if random_patches:
        extra = np.zeros(random_patches, C.CAND_DTYPE)
        for k in range(random_patches):
            bi = int(rng.integers(0, len(ok)))
            pts = []
            for _ in range(int(rng.integers(1, 4))):
                a = int(rng.integers(0, L))
                b = int(min(L, a + rng.integers(1, 30)))
                pts.append(C.mask(a, b, int(rng.integers(0, 256)), int(rng.integers(0, 256))))
            extra[k] = C.make(bi, int(bhdr[bi] & np.uint64(0xFF)), int(bhdr[bi] >> np.uint64(8)), pts)
        cands = np.concatenate([cands, extra])
    return bases, bhdr, ranks, cands


def run_incr(ctx, bases, bhdr, ranks, cands, full=False, gofs=0, n_total=None):
    dev = torch.device("cuda")
    out, sel = ctx.eval_incr(torch.from_numpy(bases).to(dev), torch.from_numpy(bhdr.view(np.int64)).to(dev),
                             torch.from_numpy(cands.view(np.uint8)).to(dev),
                             torch.from_numpy(ranks.view(np.int16)).to(dev), n=len(cands), full=full,
                             global_offset=gofs, n_total=n_total)
    torch.cuda.synchronize()
    return out, sel


def check(prof, bases, bhdr, ranks, cands, full=False):
    ctx = A.Context(prof, 0)
    try:
        out, sel = run_incr(ctx, bases, bhdr, ranks, cands, full=full)
        codes, hdr = C.expand_host(bases, ranks, cands, prof.n_ops)
        o = oracle.evaluate(prof, codes, hdr, full=full, threads=8)
        for k, g in [("iter", as_u64(out.iter_ns)), ("max_mem", as_u64(out.max_mem)), ("info", as_u32(out.info))]:
            bad = np.nonzero(g != o[k])[0]
            assert bad.size == 0, (k, bad[:5], g[bad[:5]], o[k][bad[:5]], cands[bad[:1]])
        if full:
            valid = (o["info"] & oracle.INFO_INVALID) == 0
            p = (o["info"] >> 8) & 0xFF
            for k in ["stage_T", "stage_mem", "stage_comp", "stage_comm"]:
                g = as_u64(getattr(out, k)).reshape(out.p_max, len(cands)).T
                for c in np.nonzero(valid)[0]:
                    assert np.array_equal(g[c, :p[c]], o[k][c, :p[c]]), (k, c)
        s = Selection.from_buffer(sel)
        assert (s.cls, s.cost, s.index) == oracle.select(o)
        return o
    finally:
        ctx.close()


@pytest.mark.parametrize("name", ["gpt3-1.3b", "gpt3-13b", "t5", "wrn", "toy-b"])
def test_incremental_matches_oracle_on_search_primitives(name):
    prof = P.WORKLOADS[name]()
    o = check(prof, *search_batch(prof, 3, random_patches=300), full=True)
    prim = o["info"][:-300]  # the primitives' candidates (the random patches come last)
    assert ((prim & oracle.INFO_INVALID) == 0).mean() > 0.5


def test_incremental_1k_layers():
    prof = P.WORKLOADS["gpt-1k"]()
    check(prof, *search_batch(prof, 4, nbases=2), full=False)


def test_incremental_invalid_base_and_header_changes():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    bases, bhdr, ranks, cands = search_batch(prof, 5, nbases=3)
    bases[1, 0] &= 0xFE                    # base 1 invalid (no head at op 0)
    bhdr[2] |= np.uint64(1 << 40)           # base 2 invalid header
    cands["p"][::7] = np.maximum(1, cands["p"][::7] - 1)   # stage count differs from the base
    check(prof, bases, bhdr, ranks, cands, full=True)
