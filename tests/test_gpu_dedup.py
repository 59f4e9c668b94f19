"""Configuration dedup on the device (aceso_hash, aceso_dedup)
against the numpy statement of include/aceso.h (tests/hash_reference.py)."""
import os
import sys

import numpy as np
import pytest
import torch

import aceso_inputs as ai
from aceso_inputs import profiles as P

sys.path.insert(0, os.path.dirname(__file__))
from hash_reference import VisitedReference, config_hash  # noqa: E402

pytestmark = pytest.mark.gpu
A = pytest.importorskip("paper_conf_eurosys_liumlsmybw24_b200")


@pytest.fixture(scope="module", autouse=True)
def _need_gpu():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def device_hash(codes, hdr, L):
    tiled = torch.from_numpy(ai.tile(codes)).cuda()
    hd = torch.from_numpy(np.ascontiguousarray(hdr, np.uint64).view(np.int64)).cuda()
    h = A.hash_candidates(tiled, hd, L)
    torch.cuda.synchronize()
    return h.cpu().numpy().view(np.uint64)


@pytest.mark.parametrize("name", ["toy-a", "toy-b", "gpt3-1.3b", "gpt3-13b", "t5", "wrn", "gpt-1k"])
def test_hash_matches_reference(name):
    prof = P.WORKLOADS[name]()
    n = 97 if name == "gpt-1k" else 3001
    codes, hdr = ai.search_shaped(prof, 7, 0, n, group_size=16)
    assert np.array_equal(device_hash(codes, hdr, prof.n_ops), config_hash(codes, hdr))


def test_hash_every_length_and_ignores_padding():
    rng = np.random.default_rng(2)
    for L in list(range(1, 40)) + [63, 64, 65, 127, 128, 129]:
        codes = rng.integers(0, 256, size=(70, L), dtype=np.uint8)
        hdr = rng.integers(0, 1 << 62, size=70, dtype=np.uint64)
        tiled = ai.tile(codes)
        # garbage in the tiled padding bytes must not change the hash
        nch = (L + 15) // 16
        t = tiled.reshape(-1, nch, 32, 16)
        if L % 16:
            t[:, -1, :, L % 16:] = 0xA5
        hd = torch.from_numpy(hdr.view(np.int64)).cuda()
        h = A.hash_candidates(torch.from_numpy(tiled).cuda(), hd, L)
        assert np.array_equal(h.cpu().numpy().view(np.uint64), config_hash(codes, hdr)), L


def test_visited_set_first_occurrence_across_calls():
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, hdr = ai.search_shaped(prof, 11, 0, 4000, group_size=64)
    rng = np.random.default_rng(4)
    vs = A.VisitedSet(1 << 14)
    ref = VisitedReference()
    seen_rows = []
    for call in range(4):
        idx = rng.integers(0, 4000, size=2500)  # repeats inside and across calls
        c, h = codes[idx], hdr[idx]
        hs = device_hash(c, h, prof.n_ops)
        dup = vs.insert(torch.from_numpy(hs.view(np.int64)).cuda())
        torch.cuda.synchronize()
        assert not vs.overflowed()
        assert np.array_equal(dup.cpu().numpy(), ref.insert(hs)), call
        seen_rows.append(idx)
    # distinct configurations map to distinct hashes here (no false duplicates)
    all_idx = np.unique(np.concatenate(seen_rows))
    rows = {codes[i].tobytes() + hdr[i].tobytes() for i in all_idx}
    assert len(rows) == len(set(config_hash(codes[all_idx], hdr[all_idx]).tolist()))


def test_visited_set_overflow_is_reported():
    vs = A.VisitedSet(64)
    hs = torch.arange(1, 200, dtype=torch.int64, device="cuda") * 7919
    vs.insert(hs)
    torch.cuda.synchronize()
    assert vs.overflowed()


def test_search_device_visited_set_equals_host_statement_through_growth():
    """search.DeviceVisited (aceso_dedup inside the search driver, rebuilt 4x larger before
    its load factor passes 1/2) keeps exactly what the host statement _first_new keeps, batch
    after batch, with repeats inside a batch and across batches and several table rebuilds."""
    from paper_conf_eurosys_liumlsmybw24_b200 import search as S
    rng = np.random.default_rng(11)
    pool = rng.integers(1, 2**63, 5000, dtype=np.int64).view(np.uint64)
    dv = S.DeviceVisited(0, slots=64)
    hv = S._HostVisited()
    for b in range(12):
        hs = pool[rng.integers(0, 300 + 400 * b, int(rng.integers(1, 900)))]
        r = dict(hash=hs, hash_dev=torch.from_numpy(hs.view(np.int64)).cuda())
        assert np.array_equal(dv.first_new(r), hv.first_new(r)), b
    assert dv.vs.slots > 64 and dv.count == len(hv.h)
