"""Mutation check of the oracle pins (CPU): each plausible one-line mistake in
oracle/aceso_oracle.c — a dropped term, a wrong index, an off-by-one, a flipped
comparison — must make tests/test_oracle_pins.py fail. The mutant is compiled into a
temporary library and the pins run against it (ACESO_ORACLE_LIB).

P:Lnn = PAPER.md line; R# = reading in DESIGN.md §3.
"""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "oracle", "aceso_oracle.c")

# (name, passage, exact source text, replacement)
MUTATIONS = [
    ("eq1-drop-optimizer", "Eq. 1 M_opt, P:L229",
     "+\n             (u64)P->wmem[((int64_t)t * P->n_tp + tpl[j]) * 2 + 1];", ";"),
    ("eq1-drop-param-grad", "Eq. 1 M_param + M_grad, P:L229",
     "u64 Wj = (u64)P->wmem[((int64_t)t * P->n_tp + tpl[j]) * 2 + 0] +", "u64 Wj = "),
    ("r3-drop-recompute-transient", "R3/R4, P:L232-234",
     "u64 ej = peak + (rc[j] ? (act - keep) : 0);", "u64 ej = peak;"),
    ("r3-no-keep", "R3, P:L232", "u64 Aj = rc[j] ? keep : act;", "u64 Aj = act;"),
    ("r3-keep-swapped", "R3, P:L232", "u64 Aj = rc[j] ? keep : act;", "u64 Aj = rc[j] ? act : keep;"),
    ("r7-recompute-comp-only", "R7, P:L241",
     "u64 Bp = bc + bm + (rc[j] ? F : 0);", "u64 Bp = bc + bm + (rc[j] ? fc : 0);"),
    ("r7-no-recompute", "P:L241", "u64 Bp = bc + bm + (rc[j] ? F : 0);", "u64 Bp = bc + bm;"),
    ("full-comp-no-recompute", "Heuristic-2 resources, P:L206-210",
     "comp[i] += fc + bc + (rc[j] ? fc : 0);", "comp[i] += fc + bc;"),
    ("full-comm-no-recompute", "Heuristic-2 resources, P:L206-210",
     "comm[i] += fm + bm + (rc[j] ? fm : 0) + rs;", "comm[i] += fm + bm + rs;"),
    ("full-comm-no-reshard", "Heuristic-2 resources, R13",
     "comm[i] += fm + bm + (rc[j] ? fm : 0) + rs;", "comm[i] += fm + bm + (rc[j] ? fm : 0);"),
    ("full-comm-no-dp-sync", "Heuristic-2 resources, R6",
     "if (sK) sK[i] = N * comm[i] + Dd[i];", "if (sK) sK[i] = N * comm[i];"),
    ("full-comp-per-microbatch", "Heuristic-2 resources (N microbatches)",
     "if (sC) sC[i] = N * comp[i];", "if (sC) sC[i] = comp[i];"),
    ("full-comm-no-p2p", "R5 in the comm share",
     "      S[i] += v;\n      comm[i] += v;\n    }\n    if (i > 0) {",
     "      S[i] += v;\n    }\n    if (i > 0) {"),
    ("eq2-N-not-N-1", "Eq. 2 / R1, P:L238", "u64 Ti = sumS + (N - 1) * S[i] + Dd[i];",
     "u64 Ti = sumS + N * S[i] + Dd[i];"),
    ("eq2-drop-sum", "Eq. 2 / R1, P:L238", "u64 Ti = sumS + (N - 1) * S[i] + Dd[i];",
     "u64 Ti = S[i] + (N - 1) * S[i] + Dd[i];"),
    ("eq2-drop-dp-sync", "R6, P:L94", "u64 Ti = sumS + (N - 1) * S[i] + Dd[i];",
     "u64 Ti = sumS + (N - 1) * S[i];"),
    ("dp-sync-summed", "R6, P:L94", "u64 Ti = sumS + (N - 1) * S[i] + Dd[i];",
     "u64 Ti = sumS + (N - 1) * S[i] + Dd[0];"),
    ("eq1-inflight-off-by-one", "Eq. 1 / R2, P:L229",
     "u64 inflight = (u64)(p - i) < N ? (u64)(p - i) : N;",
     "u64 inflight = (u64)(p - i - 1) < N ? (u64)(p - i - 1) : N;"),
    ("eq1-inflight-no-min", "R2", "u64 inflight = (u64)(p - i) < N ? (u64)(p - i) : N;",
     "u64 inflight = (u64)(p - i);"),
    ("r4-extra-summed", "R4, P:L234", "if (ej > E[i]) E[i] = ej;", "E[i] += ej;"),
    ("r10-oom-ge", "R10", "if (Mi > (u64)P->C) oom = 1;", "if (Mi >= (u64)P->C) oom = 1;"),
    ("r11-argmax-last-tie", "Heuristic-1 ties, R11",
     "if (i == 0 || Ti > iter) { iter = Ti; argT = i; }",
     "if (i == 0 || Ti >= iter) { iter = Ti; argT = i; }"),
    ("h1-always-time", "Heuristic-1, P:L155", "unsigned bottleneck = oom ? argM : argT;",
     "unsigned bottleneck = argT;"),
    ("r8-b-from-tp", "R8, P:L188", "int b = (int)mbs_log2 - dpl[j];", "int b = (int)mbs_log2 - tpl[j];"),
    ("lookup-dps-transposed", "P:L94 DP sync lookup",
     "u64 dj = (u64)P->dps[((int64_t)t * P->n_tp + tpl[j]) * P->n_dp + dpl[j]];",
     "u64 dj = (u64)P->dps[((int64_t)t * P->n_tp + dpl[j]) * P->n_dp + tpl[j]];"),
    ("r5-drop-p2p-fwd", "R5, P:L241", "if (i + 1 < p) {", "if (0) {"),
    ("r5-p2p-bwd-of-last-op", "R5, P:L241",
     "int t = P->op_type[first];\n      u64 v = rec_field(P, dim[first], t, tpl[first], (int)mbs_log2 - dpl[first], P2P_BWD);",
     "int t = P->op_type[last];\n      u64 v = rec_field(P, dim[last], t, tpl[last], (int)mbs_log2 - dpl[last], P2P_BWD);"),
    ("r13-drop-reshard", "R13, P:L261",
     "rs = rec_field(P, dim[j], t, tpl[j], b, RESHARD);", "rs = 0;"),
    ("r13-reshard-at-stage-heads", "R13, P:L261 (a stage boundary is a p2p, not a reshard)",
     "if (j > 0 && !head[j] && (tpl[j] != tpl[j - 1] || dpl[j] != dpl[j - 1]))",
     "if (j > 0 && (tpl[j] != tpl[j - 1] || dpl[j] != dpl[j - 1]))"),
    ("r13-reshard-on-every-op", "R13, P:L261 (only at a tp/dp change)",
     "if (j > 0 && !head[j] && (tpl[j] != tpl[j - 1] || dpl[j] != dpl[j - 1]))",
     "if (j > 0 && !head[j])"),
    ("r13-sender-pays", "R13, P:L261 (the receiving op's record)",
     "rs = rec_field(P, dim[j], t, tpl[j], b, RESHARD);",
     "rs = rec_field(P, dim[j - 1], P->op_type[j - 1], tpl[j - 1], (int)mbs_log2 - dpl[j - 1], RESHARD);"),
    ("r13-reshard-once-per-iteration", "R13 + Eq. 2 (per microbatch)",
     "    S[i] += F + Bp + rs;", "    S[i] += F + Bp;\n    Dd[i] += rs;"),
    ("r9-no-gsum-check", "R9, P:L151", "if (gsum != (u64)P->G) reasons |= O_R_GSUM;", ";"),
    ("dim-ignored-for-compute", "TP dimension, P:L263-265",
     "u64 fc = rec_field(P, dim[j], t, tpl[j], b, FWD_COMP);", "u64 fc = rec_field(P, 0, t, tpl[j], b, FWD_COMP);"),
    ("dim-ignored-for-memory", "TP dimension, P:L263-265",
     "u64 act = rec_field(P, dim[j], t, tpl[j], b, ACT);", "u64 act = rec_field(P, 0, t, tpl[j], b, ACT);"),
    ("dim-ignored-for-reshard", "TP dimension + R13",
     "rs = rec_field(P, dim[j], t, tpl[j], b, RESHARD);", "rs = rec_field(P, 0, t, tpl[j], b, RESHARD);"),
    ("dim-ignored-for-p2p-fwd", "TP dimension + R5",
     "u64 v = rec_field(P, dim[last], t, tpl[last], (int)mbs_log2 - dpl[last], P2P_FWD);",
     "u64 v = rec_field(P, 0, t, tpl[last], (int)mbs_log2 - dpl[last], P2P_FWD);"),
    ("dim-of-previous-op", "TP dimension, P:L263-265",
     "dim[j] = dims ? (dims[j] != 0) : 0;", "dim[j] = dims ? (dims[j > 0 ? j - 1 : 0] != 0) : 0;"),
    ("literal-eq2-ignored", "R1 variant, P:L238-241", "if (P->literal) Ti += S[i];", ";"),
    ("select-tie-highest-index", "R11 (selection)", "else better = g < best_idx;",
     "else better = g > best_idx;"),
    ("select-oom-before-feasible", "P:L138 better", "else if (k != best_cls) better = k < best_cls;",
     "else if (k != best_cls) better = k > best_cls;"),
]


@pytest.mark.parametrize("name,passage,old,new", MUTATIONS, ids=[m[0] for m in MUTATIONS])
def test_pins_reject_mutant(tmp_path, name, passage, old, new):
    src = open(SRC).read()
    assert src.count(old) == 1, f"mutation site of {name} not unique / not found"
    mut = tmp_path / "mutant.c"
    mut.write_text(src.replace(old, new))
    lib = tmp_path / "libmutant.so"
    subprocess.check_call(["gcc", "-O1", "-w", "-shared", "-fPIC", "-pthread", "-o", str(lib), str(mut)])
    env = dict(os.environ, ACESO_ORACLE_LIB=str(lib))
    r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_oracle_pins.py")],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode != 0, f"mutant {name} ({passage}) passes every pin:\n{r.stdout[-2000:]}"


def test_pins_pass_unmutated(tmp_path):
    """Baseline of the check above: the unmodified source, built the same way, passes."""
    lib = tmp_path / "liboriginal.so"
    subprocess.check_call(["gcc", "-O1", "-w", "-shared", "-fPIC", "-pthread", "-o", str(lib), SRC])
    env = dict(os.environ, ACESO_ORACLE_LIB=str(lib))
    r = subprocess.run([sys.executable, "-m", "pytest", "-x", "-q", "-p", "no:cacheprovider",
                        os.path.join(ROOT, "tests", "test_oracle_pins.py")],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:]
