"""GPU parity of the tensor-parallel partition dimension (§4.2): candidates with
a dimension plane (aceso_eval_dims) against the oracle with the same per-op choices, bit-exact
on every output and the selection."""
import numpy as np
import pytest
import torch

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P

pytestmark = pytest.mark.gpu

A = pytest.importorskip("paper_conf_eurosys_liumlsmybw24_b200")
from paper_conf_eurosys_liumlsmybw24_b200.api import AcesoError, Selection, as_u32, as_u64  # noqa: E402

SEED = 20240422


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _run(ctx, prof, codes, hdr, dims, full=True, device_pack=False):
    n = len(hdr)
    tiled = torch.from_numpy(ai.tile(codes)).cuda()
    hd = torch.from_numpy(np.ascontiguousarray(hdr, np.uint64).view(np.int64)).cuda()
    if dims is None:
        plane = None
    elif device_pack:
        plane = ctx.pack_dims(torch.from_numpy(np.ascontiguousarray(dims, np.uint8)).cuda())
    else:
        plane = torch.from_numpy(ai.tile_dims(dims)).cuda()
    out, sel = ctx.eval(tiled, hd, n=n, full=full, select=True, dims=plane)
    torch.cuda.synchronize()
    g = dict(iter=as_u64(out.iter_ns), max_mem=as_u64(out.max_mem), info=as_u32(out.info))
    if full:
        for k in ["stage_T", "stage_mem", "stage_comp", "stage_comm"]:
            g[k] = as_u64(getattr(out, k)).reshape(out.p_max, n).T
    return g, Selection.from_buffer(sel)


def _compare(ctx, prof, codes, hdr, dims, full=True, device_pack=False):
    g, sel = _run(ctx, prof, codes, hdr, dims, full, device_pack)
    o = oracle.evaluate(prof, codes, hdr, full=full, threads=8, dims=dims)
    for k in ["iter", "max_mem", "info"]:
        bad = np.nonzero(g[k] != o[k])[0]
        assert bad.size == 0, (k, bad[:5], g[k][bad[:5]], o[k][bad[:5]])
    if full:
        valid = (o["info"] & oracle.INFO_INVALID) == 0
        p = (o["info"] >> 8) & 0xFF
        for k in ["stage_T", "stage_mem", "stage_comp", "stage_comm"]:
            for c in np.nonzero(valid)[0]:
                assert np.array_equal(g[k][c, :p[c]], o[k][c, :p[c]]), (k, c)
    assert (sel.cls, sel.cost, sel.index) == oracle.select(o)
    return g, o


@pytest.mark.parametrize("name", ["gpt3-1.3b", "t5", "wrn", "toy-b", "gpt3-13b"])
def test_dimension_plane_parity(name):
    prof = P.WORKLOADS[name]()
    ctx = A.Context(prof, 0)
    try:
        rng = np.random.default_rng(7)
        codes, hdr = ai.search_shaped(prof, SEED + 90, 0, 1777, group_size=16)
        dims = (rng.random(codes.shape) < 0.3).astype(np.uint8)
        g, o = _compare(ctx, prof, codes, hdr, dims)
        assert ((o["info"] & oracle.INFO_INVALID) == 0).mean() > 0.9
        _compare(ctx, prof, codes[:301], hdr[:301], dims[:301], full=False, device_pack=True)
        dcodes, dhdr = ai.dense_random(prof, SEED + 91, 0, 500)
        _compare(ctx, prof, dcodes, dhdr, (rng.random(dcodes.shape) < 0.5).astype(np.uint8))
        rcodes = rng.integers(0, 256, size=(200, prof.n_ops), dtype=np.uint8)
        rhdr = rng.integers(0, 1 << 16, size=200, dtype=np.uint64)
        _compare(ctx, prof, rcodes, rhdr, rng.integers(0, 256, size=rcodes.shape, dtype=np.uint8))
    finally:
        ctx.close()


def test_all_default_dimensions_equal_plain_eval():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    ctx = A.Context(prof, 0)
    try:
        codes, hdr = ai.search_shaped(prof, SEED + 92, 0, 999, group_size=16)
        a, sa = _run(ctx, prof, codes, hdr, None)
        b, sb = _run(ctx, prof, codes, hdr, np.zeros_like(codes))
        for k in a:
            assert np.array_equal(a[k], b[k]), k
        assert (sa.cls, sa.cost, sa.index) == (sb.cls, sb.cost, sb.index)
    finally:
        ctx.close()


def test_device_pack_matches_host_plane():
    prof = P.WORKLOADS["wrn"]()
    ctx = A.Context(prof, 0)
    try:
        rng = np.random.default_rng(9)
        dims = rng.integers(0, 3, size=(70, prof.n_ops), dtype=np.uint8)
        plane = ctx.pack_dims(torch.from_numpy(dims).cuda())
        torch.cuda.synchronize()
        assert np.array_equal(plane.cpu().numpy()[:ai.dims_bytes(70, prof.n_ops)], ai.tile_dims(dims))
    finally:
        ctx.close()


def test_dimension_plane_errors():
    prof = P.WORKLOADS["toy-a"]()
    prof.rec_alt = None
    ctx = A.Context(prof, 0)
    try:
        codes, hdr = ai.search_shaped(prof, SEED, 0, 10)
        with pytest.raises(AcesoError, match="rec_alt"):
            _run(ctx, prof, codes, hdr, np.zeros_like(codes))
    finally:
        ctx.close()
    wide = P.jittered(P.WORKLOADS["toy-a"](), 3, 0, scale=1 << 9)
    wide.rec_alt = wide.rec.copy()
    ctx = A.Context(wide, 0)
    try:
        codes, hdr = ai.search_shaped(wide, SEED, 0, 10)
        with pytest.raises(AcesoError, match="32-bit"):
            _run(ctx, wide, codes, hdr, np.zeros_like(codes))
    finally:
        ctx.close()
