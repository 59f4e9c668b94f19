"""On-device candidate generation (aceso_expand) against the numpy
statement of the patch semantics (candidates.expand_host), and evaluation of the expanded
batch against the oracle."""
import numpy as np
import pytest
import torch

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P

pytestmark = pytest.mark.gpu
A = pytest.importorskip("paper_conf_eurosys_liumlsmybw24_b200")
from paper_conf_eurosys_liumlsmybw24_b200 import candidates as C  # noqa: E402
from paper_conf_eurosys_liumlsmybw24_b200.api import as_u32, as_u64  # noqa: E402


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def random_cands(rng, nb, L, n):
    cands = np.zeros(n, C.CAND_DTYPE)
    cands["base"] = rng.integers(0, nb, size=n)
    cands["mbs"] = rng.integers(0, 6, size=n)
    cands["p"] = rng.integers(1, 9, size=n)
    cands["n_patch"] = rng.integers(0, 7, size=n)
    for i in range(n):
        for j in range(int(cands["n_patch"][i])):
            a = int(rng.integers(0, L))
            b = int(min(L + 3, a + rng.integers(0, 40)))  # ranges may run past L (clamped)
            # the caller keeps tp/dp fields in range: at most one ADD, before any MASK
            kind = int(rng.integers(2, 4)) if j == 0 else int(rng.choice([1, 3]))
            if kind == C.PATCH_MASK:
                pt = C.mask(a, b, int(rng.integers(0, 256)), int(rng.integers(0, 256)))
            elif kind == C.PATCH_ADD:
                pt = C.add(a, b, int(rng.integers(-1, 2)), int(rng.integers(-1, 2)))
            else:
                pt = C.rank_rc(a, b, int(rng.integers(0, 300)), int(rng.integers(0, 2)), bool(rng.integers(0, 2)))
            cands["patch"][i][j] = pt
    return cands


@pytest.mark.parametrize("L", [6, 10, 16, 17, 315, 821])
def test_device_expansion_matches_host(L):
    rng = np.random.default_rng(L)
    nb, stride = 5, C.stride_of(L)
    bases = np.zeros((nb, stride), np.uint8)
    # fields kept in 1..6 so that ADD patches of +-1 stay in range
    bases[:, :L] = (rng.integers(0, 2, size=(nb, L)) | (rng.integers(1, 7, size=(nb, L)) << 1) |
                    (rng.integers(0, 2, size=(nb, L)) << 4) | (rng.integers(1, 7, size=(nb, L)) << 5)).astype(np.uint8)
    ranks = rng.integers(0, 400, size=(nb, 2, stride)).astype(np.uint16)
    cands = random_cands(rng, nb, L, 1000)
    codes_h, hdr_h = C.expand_host(bases, ranks, cands, L)
    dev = torch.device("cuda")
    tb = torch.from_numpy(bases).to(dev)
    rk = torch.from_numpy(ranks.view(np.int16)).to(dev)
    cd = torch.from_numpy(cands.view(np.uint8)).to(dev)
    tiled = torch.zeros(A.tiled_bytes(1000, L), dtype=torch.uint8, device=dev)
    hdr = torch.empty(1000, dtype=torch.int64, device=dev)
    from paper_conf_eurosys_liumlsmybw24_b200 import _lib as Lb
    from paper_conf_eurosys_liumlsmybw24_b200.api import _ptr, _stream
    rc = Lb.load().aceso_expand(_ptr(tb), _ptr(rk), nb, L, _ptr(cd), 1000, _ptr(tiled), _ptr(hdr), _stream(None))
    assert rc == 0
    torch.cuda.synchronize()
    assert np.array_equal(tiled.cpu().numpy(), ai.tile(codes_h))
    assert np.array_equal(hdr.cpu().numpy().view(np.uint64), hdr_h)


def test_expanded_batch_evaluates_like_the_oracle():
    """Context.expand feeding aceso_eval: a search-like batch (op moves, tp/dp trades, rc)."""
    prof = P.WORKLOADS["gpt3-1.3b"]()
    ctx = A.Context(prof, 0)
    L, stride = prof.n_ops, C.stride_of(prof.n_ops)
    codes, hdr = ai.search_shaped(prof, 5, 0, 8, group_size=8)
    bases = np.zeros((8, stride), np.uint8)
    bases[:, :L] = codes
    rng = np.random.default_rng(9)
    ranks = np.tile(np.arange(stride, dtype=np.uint16), (8, 2, 1))
    cands = np.zeros(3000, C.CAND_DTYPE)
    for i in range(3000):
        b = int(rng.integers(0, 8))
        heads = np.flatnonzero(codes[b] & 1)
        pts = []
        if len(heads) > 1 and rng.random() < 0.5:  # move the first k ops of a stage forward
            s = int(rng.integers(1, len(heads)))
            a = int(heads[s])
            e = int(heads[s + 1]) if s + 1 < len(heads) else L
            k = int(rng.integers(1, max(2, e - a)))
            if k < e - a:
                pts = [C.mask(a, a + k, 0x10, codes[b][a - 1] & 0xEE), C.mask(a + k, a + k + 1, 0xFE, 1)]
        if rng.random() < 0.3:
            pts.append(C.rank_rc(0, L, int(rng.integers(0, L)), 0, False))
        cands[i] = C.make(b, int(hdr[b] & 0xFF), int((hdr[b] >> np.uint64(8)) & np.uint64(0xFF)), pts)
    dev = torch.device("cuda")
    tiled, hd = ctx.expand(torch.from_numpy(bases).to(dev), torch.from_numpy(cands.view(np.uint8)).to(dev),
                           torch.from_numpy(ranks.view(np.int16)).to(dev), n=3000)
    out, _ = ctx.eval(tiled, hd, n=3000, full=False, select=False)
    torch.cuda.synchronize()
    ch, hh = C.expand_host(bases, ranks, cands, L)
    o = oracle.evaluate(prof, ch, hh, threads=8)
    assert np.array_equal(as_u64(out.iter_ns), o["iter"])
    assert np.array_equal(as_u64(out.max_mem), o["max_mem"])
    assert np.array_equal(as_u32(out.info), o["info"])
    ctx.close()
