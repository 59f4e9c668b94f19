"""CPU evaluator for the search driver built on the oracle (test infrastructure): the same
interface as search.GPUEvaluator (evaluate, evaluate_cands), with host expansion of the
candidate descriptors and the numpy statement of the configuration hash."""
import os
import sys

import oracle

sys.path.insert(0, os.path.dirname(__file__))
from hash_reference import config_hash  # noqa: E402


class OracleEvaluator:
    def __init__(self, prof):
        self.prof = prof
        self.evaluated = 0

    def evaluate(self, codes, hdr, dims=None, hashes=False):
        self.evaluated += len(hdr)
        r = oracle.evaluate(self.prof, codes, hdr, full=True, threads=8, dims=dims)
        if hashes:
            r["hash"] = config_hash(codes, hdr)
        return r

    def evaluate_cands(self, bases, ranks, cands):
        from paper_conf_eurosys_liumlsmybw24_b200 import candidates as C
        codes, hdr = C.expand_host(bases, ranks, cands, self.prof.n_ops)
        r = self.evaluate(codes, hdr)
        r["hash"] = config_hash(codes, hdr)
        return r
