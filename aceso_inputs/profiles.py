"""Synthetic op-cost profiles shaped like the paper's workloads (input synthesis only).

Aceso profiles every operator under each partition and the collective times per
group size; real profiling needs the real models on real GPUs
and is out of scope, so these tables are derived analytically from the model
dimensions of Table 2 on a V100-like device: compute from
FLOPs at an efficiency curve, memory-bound ops from bytes at HBM bandwidth,
tensor/data-parallel collectives and pipeline sends from an alpha-beta model
(NVLink inside 8 devices, 100 Gb/s InfiniBand beyond).

This module holds none of the method's arithmetic (no Eq. 1/2, no lookup by a
configuration, no selection): it only fills the profile tables consumed by
both the oracle and the CUDA library. Every number is an integer (ns, bytes).

Record fields, per (type, tpl, b) — restated from DESIGN.md §2:
  fwd_comp, fwd_comm, bwd_comp, bwd_comm, act, keep, peak, reshard, p2p_fwd, p2p_bwd
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

NF = 10
U32 = (1 << 32) - 1
GiB = 1 << 30


@dataclasses.dataclass
class Profile:
    name: str
    op_type: np.ndarray  # uint16 [L]
    type_names: list
    rec: np.ndarray  # int64 [T, n_tp, n_b, NF]
    wmem: np.ndarray  # int64 [T, n_tp, 2]
    dps: np.ndarray  # int64 [T, n_tp, n_dp]
    n_devices: int
    mem_capacity: int
    global_batch: int
    # records of each type's alternative tensor-parallel partition dimension (§4.2, P:L263-265:
    # row- vs column-wise MatMul, input- vs output-channel convolution); None: no alternative
    rec_alt: np.ndarray | None = None

    @property
    def n_ops(self):
        return int(self.op_type.shape[0])

    @property
    def n_types(self):
        return int(self.rec.shape[0])

    @property
    def n_tp(self):
        return int(self.rec.shape[1])

    @property
    def n_b(self):
        return int(self.rec.shape[2])

    @property
    def n_dp(self):
        return int(self.dps.shape[2])

    def rc_rank(self) -> np.ndarray:
        """Per-op rank (0 = largest) of its type's activation bytes at tp=1, b=1.

        Used by the candidate generator's greedy recomputation primitive
        (recompute the operators with the largest activation size)."""
        act = self.rec[:, 0, 0, 4].astype(np.float64)
        order = np.argsort(-act, kind="stable")
        rank_of_type = np.empty(self.n_types, dtype=np.int64)
        rank_of_type[order] = np.arange(self.n_types)
        return np.minimum(rank_of_type[self.op_type.astype(np.int64)], 254).astype(np.uint8)


# ----------------------------------------------------------------------------
# device / network model (V100-32GB cluster)
# ----------------------------------------------------------------------------
@dataclasses.dataclass
class Hw:
    mm_peak: float = 125e12  # fp16 tensor-core FLOP/s
    mm_eff: float = 0.70
    mm_half: float = 4e9  # FLOPs at which efficiency is half of mm_eff
    hbm: float = 900e9 * 0.8
    launch_f: float = 6e-6
    launch_b: float = 12e-6
    nvlink: float = 120e9
    ib: float = 12.5e9
    alpha: float = 8e-6


def _mm_time(hw, flops):
    if flops <= 0:
        return 0.0
    eff = hw.mm_eff * flops / (flops + hw.mm_half)
    return flops / (hw.mm_peak * eff)


def _allreduce(hw, nbytes, g, cross_node):
    if g <= 1 or nbytes <= 0:
        return 0.0
    bw = hw.ib if cross_node else hw.nvlink
    return 2.0 * (g - 1) / g * nbytes / bw + 2 * (g - 1) * hw.alpha


def _allgather(hw, nbytes, g, cross_node):
    if g <= 1 or nbytes <= 0:
        return 0.0
    bw = hw.ib if cross_node else hw.nvlink
    return (g - 1) / g * nbytes / bw + (g - 1) * hw.alpha


def _ns(sec):
    return int(round(sec * 1e9))


@dataclasses.dataclass
class OpCost:
    """Per-op quantities for one (tp, b): seconds and bytes."""
    flops: float = 0.0  # forward matmul FLOPs (per GPU)
    mbytes: float = 0.0  # forward memory traffic (per GPU)
    tp_fwd_bytes: float = 0.0  # forward all-reduce payload over tp
    tp_bwd_bytes: float = 0.0  # backward all-reduce payload over tp
    tp_fwd_gather: float = 0.0  # forward all-gather payload over tp
    act: float = 0.0  # bytes kept for backward
    keep_frac: float = 0.25  # fraction kept when recomputed
    out: float = 0.0  # output bytes (per GPU)
    inp: float = 0.0  # input bytes, full (for reshard / p2p)
    params: float = 0.0  # parameters per GPU
    workspace: float = 0.0
    # tensor-parallel partition dimension: "col" (MatMul split along its output
    # features: input replicated, output sharded), "row" (split along its input features:
    # input sharded, partial outputs all-reduced), "out" / "in" (convolution output / input
    # channels); "" = no alternative dimension
    part: str = ""


def _alternative(c: OpCost, tp: int) -> OpCost:
    """The op's cost under its other partition dimension (Megatron's column/row pairing for
    MatMul, output/input channels for convolution)."""
    import dataclasses as dc
    if c.part == "col":  # -> row-wise: input sharded, partial outputs all-reduced forward
        return dc.replace(c, act=c.act / tp, out=c.out * tp, tp_fwd_bytes=c.tp_fwd_bytes + c.out * tp,
                          tp_bwd_bytes=0.0, part="row")
    if c.part == "row":  # -> column-wise: input replicated, output gathered, input grads all-reduced
        return dc.replace(c, act=c.act * tp, out=c.out / tp, tp_fwd_bytes=0.0, tp_fwd_gather=c.out,
                          tp_bwd_bytes=c.tp_bwd_bytes + c.act * tp, part="col")
    if c.part == "out":  # -> input channels: input sharded, partial outputs all-reduced
        return dc.replace(c, act=c.act / tp, out=c.out * tp, tp_fwd_gather=0.0, tp_fwd_bytes=c.out * tp,
                          tp_bwd_bytes=0.0, part="in")
    return c


def _mem(x):
    """Exact byte count (integer): no allocator rounding, so memory values carry no common
    power-of-two factor the library could rely on."""
    return int(math.ceil(x))


def _record(hw, c: OpCost, tp, n_dev):
    cross_tp = tp > 8
    f_comp = hw.launch_f + _mm_time(hw, c.flops) + c.mbytes / hw.hbm
    b_comp = hw.launch_b + 2.0 * _mm_time(hw, c.flops) + 1.5 * c.mbytes / hw.hbm
    f_comm = _allreduce(hw, c.tp_fwd_bytes, tp, cross_tp) + _allgather(hw, c.tp_fwd_gather, tp, cross_tp)
    b_comm = _allreduce(hw, c.tp_bwd_bytes, tp, cross_tp) + _allgather(hw, c.tp_fwd_gather, tp, cross_tp)
    act = _mem(c.act)
    keep = min(act, _mem(c.act * c.keep_frac))
    peak = _mem(c.out + c.workspace)
    reshard = _allgather(hw, c.inp, 2 * tp, 2 * tp > 8)
    p2p_bw = hw.nvlink if n_dev <= 8 else hw.ib
    p2p_f = hw.alpha + c.out / p2p_bw
    p2p_b = hw.alpha + c.inp / tp / p2p_bw
    return [_ns(f_comp), _ns(f_comm), _ns(b_comp), _ns(b_comm), act, keep, peak, _ns(reshard),
            _ns(p2p_f), _ns(p2p_b)]


def _build(name, ops, type_of, n_devices, global_batch, n_b_max, hw, bytes_per_param, opt_per_param,
           grad_bytes_per_param, mem_capacity):
    """ops: list of type keys (model order); type_of: key -> fn(b, tp) -> OpCost."""
    keys = []
    idx = {}
    op_type = np.empty(len(ops), dtype=np.uint16)
    for j, k in enumerate(ops):
        if k not in idx:
            idx[k] = len(keys)
            keys.append(k)
        op_type[j] = idx[k]
    K = int(math.log2(n_devices)) + 1
    n_tp = n_dp = K
    T = len(keys)
    # per-GPU batch choices b = 2^0 .. 2^(n_b-1); the largest n_b <= n_b_max whose times fit
    # the ABI's 32-bit nanosecond fields (include/aceso.h range rules; memory values are 64-bit)
    n_b = n_b_max
    while True:
        rec = np.zeros((T, n_tp, n_b, NF), dtype=np.int64)
        rec_alt = np.zeros((T, n_tp, n_b, NF), dtype=np.int64)
        for t, k in enumerate(keys):
            for tpl in range(n_tp):
                for b in range(n_b):
                    c = type_of[k](1 << b, 1 << tpl)
                    rec[t, tpl, b] = _record(hw, c, 1 << tpl, n_devices)
                    # tp = 1: nothing is partitioned, both dimensions cost the same
                    rec_alt[t, tpl, b] = (_record(hw, _alternative(c, 1 << tpl), 1 << tpl, n_devices)
                                          if tpl > 0 else rec[t, tpl, b])
        times = np.concatenate([rec, rec_alt])[..., [0, 1, 2, 3, 7, 8, 9]]
        if times.max() <= U32 or n_b == 1:
            break
        n_b -= 1
    assert np.concatenate([rec, rec_alt])[..., [0, 1, 2, 3, 7, 8, 9]].max() <= U32, name
    assert (rec_alt[..., 5] <= rec_alt[..., 4]).all()
    wmem = np.zeros((T, n_tp, 2), dtype=np.int64)
    dps = np.zeros((T, n_tp, n_dp), dtype=np.int64)
    for t, k in enumerate(keys):
        for tpl in range(n_tp):
            prm = type_of[k](1, 1 << tpl).params
            wmem[t, tpl, 0] = _mem(prm * bytes_per_param)
            wmem[t, tpl, 1] = _mem(prm * opt_per_param)
            for dpl in range(n_dp):
                dp = 1 << dpl
                dps[t, tpl, dpl] = _ns(_allreduce(hw, prm * grad_bytes_per_param, dp,
                                                  (1 << tpl) * dp > 8))
    assert dps.max() <= U32, name
    return Profile(name=name, op_type=op_type, type_names=[str(k) for k in keys], rec=rec, wmem=wmem,
                   dps=dps, n_devices=n_devices, mem_capacity=int(mem_capacity),
                   global_batch=int(global_batch), rec_alt=rec_alt)


# ----------------------------------------------------------------------------
# transformer (GPT-3 / T5 / 1K-layer) op costs; 13 ops per layer (R17)
# ----------------------------------------------------------------------------
def _xf_ops(h, a, ff, inner, s, V, dtype_b=2.0, s_kv=None):
    """Returns dict kind -> fn(b, tp) -> OpCost for one transformer shape."""
    s_kv = s if s_kv is None else s_kv
    ws = 32 * 2 ** 20  # cuBLAS workspace

    def ln(b, tp):
        t = b * s
        return OpCost(mbytes=4 * t * h * dtype_b, act=t * h * dtype_b, keep_frac=1.0,
                      out=t * h * dtype_b, inp=t * h * dtype_b, params=2 * h)

    def qkv(b, tp):
        t = b * s
        return OpCost(flops=2 * t * h * 3 * inner / tp, mbytes=(t * h + 3 * t * inner / tp) * dtype_b,
                      tp_bwd_bytes=t * h * dtype_b, act=t * h * dtype_b, keep_frac=1.0,
                      out=3 * t * inner * dtype_b / tp, inp=t * h * dtype_b,
                      params=(3 * h * inner + 3 * inner) / tp, workspace=ws, part="col")

    def xq(b, tp):  # cross-attention q (decoder) + kv (encoder output)
        t, tk = b * s, b * s_kv
        return OpCost(flops=2 * (t * h * inner + 2 * tk * h * inner) / tp,
                      mbytes=(t * h + tk * h + 3 * t * inner / tp) * dtype_b,
                      tp_bwd_bytes=(t + tk) * h * dtype_b, act=(t + tk) * h * dtype_b, keep_frac=1.0,
                      out=(t + 2 * tk) * inner * dtype_b / tp, inp=t * h * dtype_b,
                      params=3 * h * inner / tp, workspace=ws, part="col")

    def score(b, tp):
        t = b * s
        e = b * (a / tp) * s * s_kv
        return OpCost(flops=2 * b * s * s_kv * inner / tp, mbytes=(2 * t * inner / tp + e) * dtype_b,
                      act=2 * t * inner * dtype_b / tp, keep_frac=0.0, out=e * dtype_b,
                      inp=2 * t * inner * dtype_b, workspace=ws)

    def softmax(b, tp):
        e = b * (a / tp) * s * s_kv
        return OpCost(mbytes=2 * e * dtype_b, act=e * dtype_b, keep_frac=0.0, out=e * dtype_b,
                      inp=e * dtype_b * tp)

    def dropout(b, tp):
        e = b * (a / tp) * s * s_kv
        return OpCost(mbytes=e * (2 * dtype_b + 1), act=e * 1.0, keep_frac=0.0, out=e * dtype_b,
                      inp=e * dtype_b * tp)

    def context(b, tp):
        t = b * s
        e = b * (a / tp) * s * s_kv
        return OpCost(flops=2 * b * s * s_kv * inner / tp, mbytes=(e + 2 * t * inner / tp) * dtype_b,
                      act=(e + t * inner / tp) * dtype_b, keep_frac=0.125, out=t * inner * dtype_b / tp,
                      inp=e * dtype_b * tp, workspace=ws)

    def outproj(b, tp):
        t = b * s
        return OpCost(flops=2 * t * inner * h / tp, mbytes=(t * inner / tp + t * h) * dtype_b,
                      tp_fwd_bytes=t * h * dtype_b, act=t * inner * dtype_b / tp, keep_frac=0.5,
                      out=t * h * dtype_b, inp=t * inner * dtype_b, params=inner * h / tp + h,
                      workspace=ws, part="row")

    def resid(b, tp):
        t = b * s
        return OpCost(mbytes=t * h * (3 * dtype_b + 1), act=t * h * 1.0, keep_frac=0.0,
                      out=t * h * dtype_b, inp=t * h * dtype_b)

    def fc1(b, tp):
        t = b * s
        return OpCost(flops=2 * t * h * ff / tp, mbytes=(t * h + t * ff / tp) * dtype_b,
                      tp_bwd_bytes=t * h * dtype_b, act=t * h * dtype_b, keep_frac=1.0,
                      out=t * ff * dtype_b / tp, inp=t * h * dtype_b, params=(h * ff + ff) / tp,
                      workspace=ws, part="col")

    def gelu(b, tp):
        t = b * s
        return OpCost(mbytes=2 * t * ff * dtype_b / tp, act=t * ff * dtype_b / tp, keep_frac=0.0,
                      out=t * ff * dtype_b / tp, inp=t * ff * dtype_b)

    def fc2(b, tp):
        t = b * s
        return OpCost(flops=2 * t * ff * h / tp, mbytes=(t * ff / tp + t * h) * dtype_b,
                      tp_fwd_bytes=t * h * dtype_b, act=t * ff * dtype_b / tp, keep_frac=0.5,
                      out=t * h * dtype_b, inp=t * ff * dtype_b, params=ff * h / tp + h, workspace=ws,
                      part="row")

    def emb(b, tp):
        t = b * s
        return OpCost(mbytes=2 * t * h * dtype_b, tp_fwd_bytes=t * h * dtype_b, act=t * 4.0,
                      keep_frac=1.0, out=t * h * dtype_b, inp=t * 4.0, params=V * h / tp)

    def head(b, tp):
        t = b * s
        return OpCost(flops=2 * t * h * V / tp, mbytes=(t * h + 2 * t * V / tp * 2) * dtype_b,
                      tp_fwd_bytes=t * 12.0, act=t * h * dtype_b + t * V * 4.0 / tp, keep_frac=0.25,
                      out=t * V * 4.0 / tp, inp=t * h * dtype_b, params=0.0, workspace=ws, part="col")

    return dict(ln=ln, qkv=qkv, xq=xq, score=score, softmax=softmax, dropout=dropout, context=context,
                outproj=outproj, resid=resid, fc1=fc1, gelu=gelu, fc2=fc2, emb=emb, head=head)


GPT_LAYER = ["ln", "qkv", "score", "softmax", "dropout", "context", "outproj", "resid",
             "ln", "fc1", "gelu", "fc2", "resid"]
# distinct type per position inside the layer (13 types) so both residuals/lns
# are separate profile entries, as a per-op profiler would record them
GPT_LAYER_KEYS = ["ln1", "qkv", "score", "softmax", "dropout", "context", "outproj", "resid1",
                  "ln2", "fc1", "gelu", "fc2", "resid2"]

GPT3_SIZES = {  # params: (layers, hidden, heads) — GPT-3 family [3], Table 2
    "0.35B": (24, 1024, 16),
    "1.3B": (24, 2048, 16),
    "2.6B": (32, 2560, 32),
    "6.7B": (32, 4096, 32),
    "13B": (40, 5120, 40),
}


def gpt(size="1.3B", n_devices=8, layers=None, hidden=None, heads=None, seq=2048, vocab=51200,
        global_batch=1024, mem_capacity=32 * GiB, n_b_max=6, name=None):
    nl, h, a = GPT3_SIZES.get(size, (None, None, None))
    nl = layers if layers is not None else nl
    h = hidden if hidden is not None else h
    a = heads if heads is not None else a
    fns = _xf_ops(h, a, 4 * h, h, seq, vocab)
    ops, type_of = ["emb"], {"emb": fns["emb"]}
    for _ in range(nl):
        for kind, key in zip(GPT_LAYER, GPT_LAYER_KEYS):
            ops.append(key)
            type_of[key] = fns[kind]
    ops += ["final_ln", "head"]
    type_of["final_ln"] = fns["ln"]
    type_of["head"] = fns["head"]
    return _build(name or f"gpt3-{size}-{n_devices}dev", ops, type_of, n_devices, global_batch,
                  n_b_max, Hw(), 4.0, 12.0, 2.0, mem_capacity)


def gpt_1k(n_devices=64, layers=1000, hidden=512, heads=8, seq=2048, n_b_max=6):
    """1K-layer GPT on 64 devices (scalability case; DeepNet-like dims [47])."""
    return gpt(size="1k", n_devices=n_devices, layers=layers, hidden=hidden, heads=heads, seq=seq,
               n_b_max=n_b_max, name=f"gpt-{layers}L-{n_devices}dev")


T5_ENC = GPT_LAYER
T5_DEC = ["ln", "qkv", "score", "softmax", "dropout", "context", "outproj", "resid",
          "ln", "xq", "score", "softmax", "dropout", "context", "outproj", "resid",
          "ln", "fc1", "gelu", "fc2", "resid"]


def t5(n_devices=16, enc_layers=24, dec_layers=24, d_model=1024, inner=16384, heads=128,
       ff=65536, seq_enc=2048, seq_dec=512, vocab=32128, global_batch=1024,
       mem_capacity=32 * GiB, n_b_max=6):
    """T5 (~11B: d_model 1024, 128 heads x 128, d_ff 65536 [40]); encoder seq 2048,
    decoder seq 512."""
    fe = _xf_ops(d_model, heads, ff, inner, seq_enc, vocab)
    fd = _xf_ops(d_model, heads, ff, inner, seq_dec, vocab)
    fx = _xf_ops(d_model, heads, ff, inner, seq_dec, vocab, s_kv=seq_enc)
    ops, type_of = ["enc_emb"], {"enc_emb": fe["emb"]}
    for _ in range(enc_layers):
        for pos, kind in enumerate(T5_ENC):
            k = f"enc_{pos}_{kind}"
            ops.append(k)
            type_of[k] = fe[kind]
    ops.append("enc_final_ln")
    type_of["enc_final_ln"] = fe["ln"]
    ops.append("dec_emb")
    type_of["dec_emb"] = fd["emb"]
    for _ in range(dec_layers):
        for pos, kind in enumerate(T5_DEC):
            k = f"dec_{pos}_{kind}"
            ops.append(k)
            cross = 9 <= pos <= 15
            type_of[k] = (fx if cross else fd)[kind]
    ops += ["dec_final_ln", "head"]
    type_of["dec_final_ln"] = fd["ln"]
    type_of["head"] = fd["head"]
    return _build(f"t5-11B-{n_devices}dev", ops, type_of, n_devices, global_batch, n_b_max, Hw(),
                  4.0, 12.0, 2.0, mem_capacity)


# ----------------------------------------------------------------------------
# Wide-ResNet (FP32, batch 1536, 224x224): bottleneck blocks [3,4,23,3]
# ----------------------------------------------------------------------------
def wrn(n_devices=16, width=480, blocks=(3, 4, 23, 3), global_batch=1536, mem_capacity=32 * GiB,
        n_b_max=6):
    hw = Hw(mm_peak=15.7e12, mm_eff=0.75, mm_half=2e9)  # V100 FP32
    fb = 4.0  # fp32 bytes
    ws = 64 * 2 ** 20

    def conv(cin, cout, k, stride, H):
        Ho = H // stride

        def f(b, tp):
            out = b * cout * Ho * Ho * fb / tp
            inp = b * cin * H * H * fb
            return OpCost(flops=2 * b * Ho * Ho * cout * cin * k * k / tp, mbytes=inp + out,
                          tp_fwd_gather=inp if k > 1 else 0.0, tp_bwd_bytes=inp, act=inp,
                          keep_frac=0.5, out=out, inp=inp, params=cin * cout * k * k / tp,
                          workspace=ws, part="out")
        return f

    def elt(C, H, kind):
        def f(b, tp):
            n = b * C * H * H / tp
            mult = {"bn": 3.0, "relu": 2.0, "add": 3.0, "pool": 2.0}[kind]
            return OpCost(mbytes=mult * n * fb, act=n * fb, keep_frac=0.25 if kind != "add" else 0.0,
                          out=n * fb, inp=n * fb * tp, params=2 * C / tp if kind == "bn" else 0.0)
        return f

    def fc(cin, ncls):
        def f(b, tp):
            return OpCost(flops=2 * b * cin * ncls / tp, mbytes=(b * cin + b * ncls / tp) * fb,
                          tp_fwd_bytes=b * ncls * fb, act=b * cin * fb, keep_frac=1.0,
                          out=b * ncls * fb / tp, inp=b * cin * fb, params=cin * ncls / tp)
        return f

    def loss(b, tp):
        return OpCost(mbytes=b * 1000 * fb * 3, tp_fwd_bytes=b * 12.0, act=b * 1000 * fb, keep_frac=0.0,
                      out=b * 4.0, inp=b * 1000 * fb)

    ops, type_of = [], {}

    def add(key, fn):
        ops.append(key)
        type_of.setdefault(key, fn)

    stem = width // 4 if width >= 256 else 64  # stem channels
    add(f"conv7_3_{stem}", conv(3, stem, 7, 2, 224))
    add(f"bn_{stem}_112", elt(stem, 112, "bn"))
    add(f"relu_{stem}_112", elt(stem, 112, "relu"))
    add(f"pool_{stem}_112", elt(stem, 56, "pool"))
    cin, H = stem, 56
    for g, nblk in enumerate(blocks):
        w = 2 * width * (1 << g)  # inner width (wide factor 2)
        cout = 4 * width * (1 << g)
        for blk in range(nblk):
            stride = 2 if (blk == 0 and g > 0) else 1
            Ho = H // stride
            if blk == 0:
                add(f"ds_conv_{cin}_{cout}_{H}_{stride}", conv(cin, cout, 1, stride, H))
                add(f"ds_bn_{cout}_{Ho}", elt(cout, Ho, "bn"))
            add(f"c1_{cin}_{w}_{H}", conv(cin, w, 1, 1, H))
            add(f"bn_{w}_{H}", elt(w, H, "bn"))
            add(f"relu_{w}_{H}", elt(w, H, "relu"))
            add(f"c2_{w}_{w}_{H}_{stride}", conv(w, w, 3, stride, H))
            add(f"bn_{w}_{Ho}", elt(w, Ho, "bn"))
            add(f"relu_{w}_{Ho}", elt(w, Ho, "relu"))
            add(f"c3_{w}_{cout}_{Ho}", conv(w, cout, 1, 1, Ho))
            add(f"bn3_{cout}_{Ho}", elt(cout, Ho, "bn"))
            add(f"add_{cout}_{Ho}", elt(cout, Ho, "add"))
            add(f"relu3_{cout}_{Ho}", elt(cout, Ho, "relu"))
            cin, H = cout, Ho
    add(f"avgpool_{cin}", elt(cin, 1, "pool"))
    add(f"fc_{cin}", fc(cin, 1000))
    add("loss", loss)
    return _build(f"wrn-{n_devices}dev", ops, type_of, n_devices, global_batch, n_b_max, hw,
                  8.0, 8.0, 4.0, mem_capacity)


# ----------------------------------------------------------------------------
# toy models (exhaustively enumerable, BASELINE.json configs[0])
# ----------------------------------------------------------------------------
def toy_a(mem_capacity=None):
    """4-layer GPT on 4 devices, one op per layer: emb + 4 layer-ops + head (L=6, T=3)."""
    h, a, s = 1024, 16, 512
    fns = _xf_ops(h, a, 4 * h, h, s, 51200)

    def layer(b, tp):  # a whole transformer layer as one op
        parts = [fns[k](b, tp) for k in GPT_LAYER]
        return OpCost(flops=sum(p.flops for p in parts), mbytes=sum(p.mbytes for p in parts),
                      tp_fwd_bytes=sum(p.tp_fwd_bytes for p in parts),
                      tp_bwd_bytes=sum(p.tp_bwd_bytes for p in parts),
                      act=sum(p.act for p in parts), keep_frac=0.1, out=parts[-1].out,
                      inp=parts[0].inp, params=sum(p.params for p in parts),
                      workspace=max(p.workspace for p in parts))
    ops = ["emb", "layer", "layer", "layer", "layer", "head"]
    type_of = {"emb": fns["emb"], "layer": layer, "head": fns["head"]}
    return _build("toy-a", ops, type_of, 4, 16, 3, Hw(), 4.0, 12.0, 2.0,
                  mem_capacity if mem_capacity is not None else 5 * GiB // 4)


def toy_b(mem_capacity=None):
    """4-layer GPT on 4 devices, two ops per layer: emb + 4 x (attn, mlp) + head (L=10, T=4)."""
    h, a, s = 1024, 16, 512
    fns = _xf_ops(h, a, 4 * h, h, s, 51200)

    def group(kinds):
        def f(b, tp):
            parts = [fns[k](b, tp) for k in kinds]
            return OpCost(flops=sum(p.flops for p in parts), mbytes=sum(p.mbytes for p in parts),
                          tp_fwd_bytes=sum(p.tp_fwd_bytes for p in parts),
                          tp_bwd_bytes=sum(p.tp_bwd_bytes for p in parts),
                          act=sum(p.act for p in parts), keep_frac=0.1, out=parts[-1].out,
                          inp=parts[0].inp, params=sum(p.params for p in parts),
                          workspace=max(p.workspace for p in parts))
        return f
    ops = ["emb"] + ["attn", "mlp"] * 4 + ["head"]
    type_of = {"emb": fns["emb"], "attn": group(GPT_LAYER[:8]), "mlp": group(GPT_LAYER[8:]),
               "head": fns["head"]}
    return _build("toy-b", ops, type_of, 4, 8, 3, Hw(), 4.0, 12.0, 2.0,
                  mem_capacity if mem_capacity is not None else 5 * GiB // 4)


def from_tables(name, op_type, rec, wmem, dps, n_devices, mem_capacity, global_batch):
    """Hand-built profile (tests)."""
    return Profile(name=name, op_type=np.asarray(op_type, dtype=np.uint16), type_names=[],
                   rec=np.asarray(rec, dtype=np.int64), wmem=np.asarray(wmem, dtype=np.int64),
                   dps=np.asarray(dps, dtype=np.int64), n_devices=int(n_devices),
                   mem_capacity=int(mem_capacity), global_batch=int(global_batch))


def jittered(prof: Profile, seed: int, shift: int = 0, scale: int = 1) -> Profile:
    """Copy of `prof` whose memory values (act, keep, peak, param+grad, optimizer) are offset
    by seeded odd multiples of 2^shift bytes, times `scale` (tests: memory values with no
    common power-of-two factor above 2^shift, and values beyond 32-bit units). keep <= act is
    kept. Input synthesis only: no model arithmetic."""
    rng = np.random.default_rng(seed)
    rec = prof.rec.copy()
    wm = prof.wmem.copy()
    unit = 1 << shift

    def odd(shape):
        return (2 * rng.integers(0, 64, size=shape) + 1) * unit

    act = rec[..., 4] * scale + odd(rec.shape[:-1])
    keep = np.minimum(rec[..., 5] * scale + odd(rec.shape[:-1]), act)
    keep = keep - keep % unit
    rec[..., 4] = act
    rec[..., 5] = keep
    rec[..., 6] = rec[..., 6] * scale + odd(rec.shape[:-1])
    wm = wm * scale + odd(wm.shape)
    return Profile(name=f"{prof.name}-jit{shift}x{scale}", op_type=prof.op_type.copy(),
                   type_names=list(prof.type_names), rec=rec, wmem=wm, dps=prof.dps.copy(),
                   n_devices=prof.n_devices, mem_capacity=prof.mem_capacity * scale,
                   global_batch=prof.global_batch)


# BASELINE.json configs -> profile builders (configs[0..4])
WORKLOADS = {
    "toy-a": toy_a,
    "toy-b": toy_b,
    "gpt3-1.3b": lambda: gpt("1.3B", 8),
    "gpt3-13b": lambda: gpt("13B", 32),
    "t5": lambda: t5(16),
    "wrn": lambda: wrn(16),
    "gpt-1k": lambda: gpt_1k(64),
}
