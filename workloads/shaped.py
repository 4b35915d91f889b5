"""Synthetic training-step DAGs shaped like the paper's workloads.

The paper's DAGs come from TensorFlow profiles that are not available (PAPER.md L127,
L218-226 §3.3 Table 1), so these generators build op-level training graphs with the
same *shape*: a forward graph of layer templates, its backward mirror (one gradient op
per differentiable input, AddN where an output feeds several consumers, saved
activations as forward->backward skip edges), one ApplyAdam per weight, and small
"satellite" ops (Shape/Reshape/Identity/Const, the bulk of a TF graph) until the op
count matches the Table 1 row.  Op durations follow the Table 1 bucket mix of the
anchor row (<10us / 10-100us / >100us), log-uniform inside a bucket; edge sizes are
activation/weight tensor sizes of the paper's hyper-parameters (L297-301).

Nothing here computes a schedule or a makespan.
"""

from __future__ import annotations

from collections import defaultdict
from typing import Dict, List, Sequence

import numpy as np

from .dag import Graph
from .rng import SplitMix64

# Table 1: op counts (<10us, 10-100us, >100us)
TABLE1 = {
    "transformer6": (14511, 4119, 763),
    "rnnlm2": (3401, 973, 240),
    "nasnet4": (14191, 1677, 1033),
    "nmt2": (21243, 8114, 703),
}

BUCKETS_NS = ((1_000, 10_000), (10_000, 100_000), (100_000, 3_000_000))

# role -> cost score (heavier roles get the long-duration buckets first)
HEAVY = {"MatMul": 100.0, "Conv2D": 120.0, "BatchMatMul": 60.0, "FusedBatchNorm": 12.0,
         "Softmax": 8.0, "ApplyAdam": 6.0, "AddN": 5.0, "ConcatV2": 4.0, "MaxPool": 10.0,
         "AvgPool": 8.0, "SoftmaxXent": 15.0, "Gather": 10.0, "Tanh": 3.0, "Sigmoid": 3.0}
GRAD_FACTOR = 1.6           # gradient ops of heavy roles cost more than the forward op
SATELLITE_ROLES = ("Shape", "Reshape", "Identity", "Const", "Cast", "StridedSlice",
                   "BroadcastGradientArgs", "Sum", "ExpandDims")


class Builder:
    """Accumulates ops and edges in creation order (creation order is topological)."""

    def __init__(self, name: str, seed: int):
        self.name = name
        self.rng = SplitMix64(seed)
        self.roles: List[str] = []
        self.layer: List[int] = []
        self.out_bytes: List[int] = []
        self.score: List[float] = []
        self.needs_grad: List[bool] = []
        self.inputs: List[List[int]] = []
        self.src: List[int] = []
        self.dst: List[int] = []
        self.ebytes: List[int] = []
        self.forward_end = 0

    @property
    def n(self) -> int:
        return len(self.roles)

    def op(self, role: str, layer: int, out_bytes: int, inputs: Sequence[int] = (),
           grad: bool = True, score: float = None) -> int:
        v = self.n
        self.roles.append(role)
        self.layer.append(layer)
        self.out_bytes.append(int(out_bytes))
        base = role.replace("Grad", "").replace("BackpropInput", "").replace("BackpropFilter", "")
        s = HEAVY.get(base, 1.0) if score is None else score
        if role.endswith("Grad") or "Backprop" in role:
            s *= GRAD_FACTOR
        self.score.append(s * (1.0 + 0.3 * self.rng.uniform()))
        self.needs_grad.append(grad)
        self.inputs.append(list(inputs))
        for u in inputs:
            self.edge(u, v)
        return v

    def edge(self, u: int, v: int, nbytes: int = None):
        self.src.append(u)
        self.dst.append(v)
        self.ebytes.append(self.out_bytes[u] if nbytes is None else int(nbytes))

    # --- common layer pieces -------------------------------------------------------------
    def var(self, layer: int, nbytes: int) -> int:
        return self.op("VariableV2", layer, nbytes, (), grad=True, score=0.2)

    def const(self, layer: int, nbytes: int = 4) -> int:
        return self.op("Const", layer, nbytes, (), grad=False, score=0.1)

    def dense(self, x: int, layer: int, act_bytes: int, w_bytes: int, bias=True) -> int:
        w = self.var(layer, w_bytes)
        y = self.op("MatMul", layer, act_bytes, (x, w))
        if bias:
            b = self.var(layer, max(4, w_bytes // 1024))
            y = self.op("BiasAdd", layer, act_bytes, (y, b))
        return y

    def layernorm(self, x: int, layer: int, nbytes: int) -> int:
        mu = self.op("Mean", layer, nbytes // 1024 + 4, (x,))
        d = self.op("Sub", layer, nbytes, (x, mu))
        sq = self.op("Square", layer, nbytes, (d,))
        var = self.op("Mean", layer, nbytes // 1024 + 4, (sq,))
        eps = self.op("Add", layer, nbytes // 1024 + 4, (var,))
        rs = self.op("Rsqrt", layer, nbytes // 1024 + 4, (eps,))
        y = self.op("Mul", layer, nbytes, (d, rs))
        g = self.var(layer, 4096)
        y = self.op("Mul", layer, nbytes, (y, g))
        b = self.var(layer, 4096)
        return self.op("Add", layer, nbytes, (y, b))

    # --- backward mirror ---------------------------------------------------------------------
    def backward(self, loss: int, unary_saves_output=("Relu", "Tanh", "Sigmoid", "Softmax")):
        """Reverse-mode mirror of the forward graph built so far (TF gradients() shape)."""
        self.forward_end = self.n
        fwd_inputs = [list(x) for x in self.inputs]
        grads_to: Dict[int, List[int]] = defaultdict(list)
        seed = self.op("OnesLike", self.layer[loss], self.out_bytes[loss], (loss,), grad=False)
        grads_to[loss].append(seed)
        for f in range(self.forward_end - 1, -1, -1):
            if not self.needs_grad[f] or not grads_to.get(f):
                continue
            contribs = grads_to[f]
            if len(contribs) == 1:
                g = contribs[0]
            else:
                g = self.op("AddN", self.layer[f], self.out_bytes[f], contribs, grad=False)
            if self.roles[f] == "VariableV2":
                self.op("ApplyAdam", self.layer[f], 4, (f, g, self._adam_lr), grad=False)
                continue
            ins = [u for u in dict.fromkeys(fwd_inputs[f]) if self.needs_grad[u]]
            role = self.roles[f]
            for u in ins:
                saved = [w for w in dict.fromkeys(fwd_inputs[f]) if w != u]
                if role in unary_saves_output:
                    saved = [f]
                if role == "Conv2D":
                    grole = "Conv2DBackpropFilter" if self.roles[u] == "VariableV2" \
                        else "Conv2DBackpropInput"
                else:
                    grole = role + "Grad"
                b = self.op(grole, self.layer[f], self.out_bytes[u], [g] + saved, grad=False)
                grads_to[u].append(b)

    def start_backward_helpers(self, layer: int):
        self._adam_lr = self.const(layer, 4)

    # --- satellites --------------------------------------------------------------------------
    def pad_satellites(self, target_n: int, m_over_n: float = 1.5):
        """Insert small TF-style ops (Shape/Reshape/Identity/Const, ...) until n == target_n.

        Patterns keep the graph acyclic: a satellite reads only an existing op u and feeds
        only a consumer v of u (or reads nothing).  Pattern choice steers m/n to m_over_n."""
        r = self.rng
        base_edges = len(self.src)
        if target_n < self.n:
            raise ValueError(f"{self.name}: core graph has {self.n} ops > target {target_n}")
        while self.n < target_n:
            e = r.below(base_edges)
            u, v = self.src[e], self.dst[e]
            cur_ratio = len(self.src) / max(1, self.n)
            kind = r.below(3) if cur_ratio >= m_over_n else 3 + r.below(2)
            layer = self.layer[v]
            sb = 4 + r.below(256)
            if kind == 0:            # Const -> v
                c = self.op(SATELLITE_ROLES[3], layer, sb, (), grad=False, score=0.1)
                self.edge(c, v)
            elif kind == 1:          # u -> Identity -> v
                self.op("Identity", layer, sb, (u,), grad=False, score=0.15)
                self.edge(self.n - 1, v)
            elif kind == 2:          # u -> Shape  (dangling shape query, sink)
                self.op("Shape", layer, sb, (u,), grad=False, score=0.1)
            elif self.n + 2 <= target_n:   # u -> Shape -> Reshape(u) -> v
                s = self.op("Shape", layer, sb, (u,), grad=False, score=0.1)
                rr = self.op("Reshape", layer, self.out_bytes[u] if r.chance(0.1) else sb,
                             (u, s), grad=False, score=0.2)
                self.edge(rr, v, sb)
            else:                    # u -> StridedSlice -> v
                self.op("StridedSlice", layer, sb, (u,), grad=False, score=0.15)
                self.edge(self.n - 1, v)

    # --- finalise ----------------------------------------------------------------------------
    def finish(self, anchor: str, meta: dict) -> Graph:
        n = self.n
        counts = TABLE1[anchor]
        tot = sum(counts)
        n_hi = int(round(n * counts[2] / tot))
        n_mid = int(round(n * counts[1] / tot))
        order = sorted(range(n), key=lambda v: -self.score[v])
        bucket = np.zeros(n, dtype=np.int64)
        for rank, v in enumerate(order):
            bucket[v] = 2 if rank < n_hi else (1 if rank < n_hi + n_mid else 0)
        p = np.zeros(n, dtype=np.int64)
        r = SplitMix64(self.rng.next_u64())
        for v in range(n):
            lo, hi = BUCKETS_NS[int(bucket[v])]
            p[v] = r.log_uniform_int(lo, hi)
        g = Graph(self.name, n, p, np.asarray(self.src, dtype=np.int32),
                  np.asarray(self.dst, dtype=np.int32), np.asarray(self.ebytes, dtype=np.int64),
                  layer=np.asarray(self.layer, dtype=np.int32), roles=list(self.roles),
                  meta=dict(meta, anchor=anchor, forward_ops=self.forward_end))
        return g


# ---------------------------------------------------------------------------------------
# Transformer (Transformer, 6 layers, hidden 1024, 16 heads, batch 32)
# ---------------------------------------------------------------------------------------
def transformer(seed: int = 1003, n_target: int = 19393, enc_layers: int = 6,
                dec_layers: int = 6, heads: int = 16) -> Graph:
    b = Builder("transformer", seed)
    act = 32 * 32 * 1024 * 4                      # 4 MB activations (SURVEY §8(d) Bytes)
    head_act = act // heads
    score_bytes = 32 * 32 * 32 * 4
    w = 1024 * 1024 * 4
    n_layers = enc_layers + dec_layers
    last = n_layers - 1

    def attention(xq, xkv, layer, mask):
        q = b.dense(xq, layer, act, w)
        k = b.dense(xkv, layer, act, w)
        v = b.dense(xkv, layer, act, w)
        outs = []
        for _ in range(heads):
            qh = b.op("StridedSlice", layer, head_act, (q,))
            kh = b.op("StridedSlice", layer, head_act, (k,))
            vh = b.op("StridedSlice", layer, head_act, (v,))
            s = b.op("BatchMatMul", layer, score_bytes, (qh, kh))
            s = b.op("Mul", layer, score_bytes, (s,))
            s = b.op("Add", layer, score_bytes, (s, mask))
            a = b.op("Softmax", layer, score_bytes, (s,))
            a = b.op("Dropout", layer, score_bytes, (a,))
            outs.append(b.op("BatchMatMul", layer, head_act, (a, vh)))
        c = b.op("ConcatV2", layer, act, outs)
        o = b.dense(c, layer, act, w)
        o = b.op("Dropout", layer, act, (o,))
        o = b.op("Add", layer, act, (o, xq))
        return b.layernorm(o, layer, act)

    def ffn(x, layer):
        h = b.dense(x, layer, 4 * act, 4 * w)
        h = b.op("Relu", layer, 4 * act, (h,))
        h = b.op("Dropout", layer, 4 * act, (h,))
        o = b.dense(h, layer, act, 4 * w)
        o = b.op("Dropout", layer, act, (o,))
        o = b.op("Add", layer, act, (o, x))
        return b.layernorm(o, layer, act)

    def embed(layer):
        tab = b.var(layer, 32000 * 1024 * 4 // 64)
        ids = b.const(layer, 32 * 32 * 4)
        e = b.op("Gather", layer, act, (tab, ids))
        e = b.op("Mul", layer, act, (e,))
        pos = b.const(layer, act)
        return b.op("Add", layer, act, (e, pos))

    src_mask = b.const(0, score_bytes)
    x = embed(0)
    for l in range(enc_layers):
        x = attention(x, x, l, src_mask)
        x = ffn(x, l)
    enc_top = x
    tgt_mask = b.const(enc_layers, score_bytes)
    y = embed(enc_layers)
    for l in range(enc_layers, n_layers):
        y = attention(y, y, l, tgt_mask)
        y = attention(y, enc_top, l, src_mask)     # cross-attention fans out from enc_top
        y = ffn(y, l)
    logits = b.dense(y, last, act * 4, 4 * w)
    labels = b.const(last, 32 * 32 * 4)
    loss = b.op("SoftmaxXent", last, 4, (logits, labels))
    b.start_backward_helpers(last)
    b.backward(loss)
    b.pad_satellites(n_target, 1.5)
    return b.finish("transformer6", {"enc_layers": enc_layers, "dec_layers": dec_layers,
                                      "heads": heads, "n_layers": n_layers})


# ---------------------------------------------------------------------------------------
# Inception-V3 topology with the NASNet-4 size and cost mix (Table 1)
# ---------------------------------------------------------------------------------------
def inception_v3(seed: int = 1001, n_target: int = 16901) -> Graph:
    b = Builder("inception_v3", seed)
    batch = 32

    def fm(h, c):
        return batch * h * h * c * 4           # CNN feature maps: 32 x H x W x C x 4 (L301)

    def conv_unit(x, layer, h, cin, cout, k=3):
        wv = b.var(layer, k * k * cin * cout * 4)
        y = b.op("Conv2D", layer, fm(h, cout), (x, wv))
        gamma = b.var(layer, cout * 4)
        beta = b.var(layer, cout * 4)
        y = b.op("FusedBatchNorm", layer, fm(h, cout), (y, gamma, beta))
        return b.op("Relu", layer, fm(h, cout), (y,))

    def module_a(x, layer, h, cin):
        b1 = conv_unit(x, layer, h, cin, 64, 1)
        b2 = conv_unit(conv_unit(x, layer, h, cin, 48, 1), layer, h, 48, 64, 5)
        b3 = conv_unit(conv_unit(conv_unit(x, layer, h, cin, 64, 1), layer, h, 64, 96),
                       layer, h, 96, 96)
        p = b.op("AvgPool", layer, fm(h, cin), (x,))
        b4 = conv_unit(p, layer, h, cin, 64, 1)
        return b.op("ConcatV2", layer, fm(h, 288), (b1, b2, b3, b4))

    def reduction_a(x, layer, h, cin):
        b1 = conv_unit(x, layer, h // 2, cin, 384)
        b2 = conv_unit(conv_unit(conv_unit(x, layer, h, cin, 64, 1), layer, h, 64, 96),
                       layer, h // 2, 96, 96)
        p = b.op("MaxPool", layer, fm(h // 2, cin), (x,))
        return b.op("ConcatV2", layer, fm(h // 2, 768), (b1, b2, p))

    def module_c(x, layer, h, cin, c7):
        b1 = conv_unit(x, layer, h, cin, 192, 1)
        t = conv_unit(x, layer, h, cin, c7, 1)
        t = conv_unit(t, layer, h, c7, c7, 7)
        b2 = conv_unit(t, layer, h, c7, 192, 7)
        t = conv_unit(x, layer, h, cin, c7, 1)
        for _ in range(3):
            t = conv_unit(t, layer, h, c7, c7, 7)
        b3 = conv_unit(t, layer, h, c7, 192, 7)
        p = b.op("AvgPool", layer, fm(h, cin), (x,))
        b4 = conv_unit(p, layer, h, cin, 192, 1)
        return b.op("ConcatV2", layer, fm(h, 768), (b1, b2, b3, b4))

    def reduction_b(x, layer, h, cin):
        b1 = conv_unit(conv_unit(x, layer, h, cin, 192, 1), layer, h // 2, 192, 320)
        t = conv_unit(x, layer, h, cin, 192, 1)
        t = conv_unit(t, layer, h, 192, 192, 7)
        t = conv_unit(t, layer, h, 192, 192, 7)
        b2 = conv_unit(t, layer, h // 2, 192, 192)
        p = b.op("MaxPool", layer, fm(h // 2, cin), (x,))
        return b.op("ConcatV2", layer, fm(h // 2, 1280), (b1, b2, p))

    def module_e(x, layer, h, cin):
        b1 = conv_unit(x, layer, h, cin, 320, 1)
        t = conv_unit(x, layer, h, cin, 384, 1)
        b2 = b.op("ConcatV2", layer, fm(h, 768), (conv_unit(t, layer, h, 384, 384, 3),
                                                   conv_unit(t, layer, h, 384, 384, 3)))
        t = conv_unit(conv_unit(x, layer, h, cin, 448, 1), layer, h, 448, 384)
        b3 = b.op("ConcatV2", layer, fm(h, 768), (conv_unit(t, layer, h, 384, 384, 3),
                                                   conv_unit(t, layer, h, 384, 384, 3)))
        p = b.op("AvgPool", layer, fm(h, cin), (x,))
        b4 = conv_unit(p, layer, h, cin, 192, 1)
        return b.op("ConcatV2", layer, fm(h, 2048), (b1, b2, b3, b4))

    img = b.const(0, fm(299, 3))
    layer = 0
    x = conv_unit(img, layer, 149, 3, 32)
    x = conv_unit(x, layer, 147, 32, 32)
    x = conv_unit(x, layer, 147, 32, 64)
    x = b.op("MaxPool", layer, fm(73, 64), (x,))
    x = conv_unit(x, layer, 73, 64, 80, 1)
    x = conv_unit(x, layer, 71, 80, 192)
    x = b.op("MaxPool", layer, fm(35, 192), (x,))
    cin = 192
    for _ in range(3):
        layer += 1
        x = module_a(x, layer, 35, cin)
        cin = 288
    layer += 1
    x = reduction_a(x, layer, 35, 288)
    for c7 in (128, 160, 160, 192):
        layer += 1
        x = module_c(x, layer, 17, 768, c7)
    layer += 1
    x = reduction_b(x, layer, 17, 768)
    cin = 1280
    for _ in range(2):
        layer += 1
        x = module_e(x, layer, 8, cin)
        cin = 2048
    layer += 1
    x = b.op("AvgPool", layer, batch * 2048 * 4, (x,))
    x = b.op("Dropout", layer, batch * 2048 * 4, (x,))
    logits = b.dense(x, layer, batch * 1000 * 4, 2048 * 1000 * 4)
    labels = b.const(layer, batch * 4)
    loss = b.op("SoftmaxXent", layer, 4, (logits, labels))
    b.start_backward_helpers(layer)
    b.backward(loss)
    b.pad_satellites(n_target, 1.5)
    return b.finish("nasnet4", {"n_layers": layer + 1})


# ---------------------------------------------------------------------------------------
# NMT seq2seq: 4-layer LSTM encoder-decoder with Bahdanau attention (PAPER.md L297,
# SURVEY §8(d)); hidden 1024, batch 128 -> 512 KB states.
# ---------------------------------------------------------------------------------------
def nmt(seed: int = 1002, n_target: int = 30060, layers: int = 4, steps: int = 36) -> Graph:
    b = Builder("nmt4", seed)
    hid = 128 * 1024 * 4                          # 512 KB state
    gates = 4 * hid
    wbytes = 2 * 1024 * 4 * 1024 * 4              # [2H, 4H] fp32 = 32 MB
    T = steps
    last = layers - 1

    def lstm_cell(x, h, c, W, bias, layer):
        xh = b.op("ConcatV2", layer, 2 * hid, (x, h))
        z = b.op("MatMul", layer, gates, (xh, W))
        z = b.op("BiasAdd", layer, gates, (z, bias))
        sp = b.op("Split", layer, gates, (z,))
        i = b.op("Sigmoid", layer, hid, (sp,))
        f = b.op("Sigmoid", layer, hid, (sp,))
        o = b.op("Sigmoid", layer, hid, (sp,))
        gg = b.op("Tanh", layer, hid, (sp,))
        fc = b.op("Mul", layer, hid, (f, c))
        ig = b.op("Mul", layer, hid, (i, gg))
        c2 = b.op("Add", layer, hid, (fc, ig))
        tc = b.op("Tanh", layer, hid, (c2,))
        h2 = b.op("Mul", layer, hid, (o, tc))
        return h2, c2

    def stack(prefix_layer0, seq_inputs, layer_base):
        Ws = [b.var(min(l, last), wbytes) for l in range(layers)]
        Bs = [b.var(min(l, last), 4 * 1024 * 4) for l in range(layers)]
        h0 = b.const(0, hid)
        hs = [h0] * layers
        cs = [h0] * layers
        tops = []
        for t in range(T):
            x = seq_inputs[t]
            for l in range(layers):
                hs[l], cs[l] = lstm_cell(x, hs[l], cs[l], Ws[l], Bs[l], l)
                x = hs[l]
            tops.append(x)
        return tops

    emb_enc = b.var(0, 32000 * 1024 * 4 // 64)
    enc_in = [b.op("Gather", 0, hid, (emb_enc, b.const(0, 512))) for _ in range(T)]
    enc_tops = stack(0, enc_in, 0)
    mem = b.op("Pack", last, T * hid, enc_tops)          # attention memory: fan-in T
    keys = b.dense(mem, last, T * hid, 1024 * 1024 * 4, bias=False)

    emb_dec = b.var(0, 32000 * 1024 * 4 // 64)
    Wd = [b.var(l, wbytes) for l in range(layers)]
    Bd = [b.var(l, 4 * 1024 * 4) for l in range(layers)]
    Wq = b.var(last, 1024 * 1024 * 4)
    Wa = b.var(last, 2048 * 1024 * 4)
    Wp = b.var(last, 1024 * 32000 * 4 // 16)
    h0 = b.const(0, hid)
    hs = [h0] * layers
    cs = [h0] * layers
    att = h0
    losses = []
    for t in range(T):
        e = b.op("Gather", 0, hid, (emb_dec, b.const(0, 512)))
        x = b.op("ConcatV2", 0, 2 * hid, (e, att))          # input feeding
        for l in range(layers):
            hs[l], cs[l] = lstm_cell(x, hs[l], cs[l], Wd[l], Bd[l], l)
            x = hs[l]
        q = b.op("MatMul", last, hid, (x, Wq))
        sc = b.op("BatchMatMul", last, 128 * T * 4, (q, keys))
        a = b.op("Softmax", last, 128 * T * 4, (sc,))
        ctx = b.op("BatchMatMul", last, hid, (a, mem))
        cat = b.op("ConcatV2", last, 2 * hid, (ctx, x))
        att = b.op("Tanh", last, hid, (b.op("MatMul", last, hid, (cat, Wa)),))
        logits = b.op("MatMul", last, 128 * 2000 * 4, (att, Wp))
        lab = b.const(last, 512)
        losses.append(b.op("SoftmaxXent", last, 512, (logits, lab)))
    loss = b.op("AddN", last, 4, losses, grad=True)
    b.start_backward_helpers(last)
    b.backward(loss)
    b.pad_satellites(n_target, 1.5)
    return b.finish("nmt2", {"layers": layers, "steps": T, "n_layers": layers})


# ---------------------------------------------------------------------------------------
# statistics every generator reports (SURVEY §8(d) "Structural targets")
# ---------------------------------------------------------------------------------------
def stats(g: Graph) -> dict:
    n, m = g.n, g.m
    indeg = np.bincount(g.dst, minlength=n)
    outdeg = np.bincount(g.src, minlength=n)
    p = g.p
    b0 = int(np.sum(p < 10_000))
    b1 = int(np.sum((p >= 10_000) & (p < 100_000)))
    b2 = int(np.sum(p >= 100_000))
    # height H(v) (Def 3.4): level-wise Kahn, sources at height 1
    h = np.ones(n, dtype=np.int64)
    succ = [[] for _ in range(n)]
    deg = indeg.copy()
    for s, d in zip(g.src.tolist(), g.dst.tolist()):
        succ[s].append(d)
    frontier = [v for v in range(n) if deg[v] == 0]
    height = 0
    while frontier:
        height += 1
        nxt = []
        for v in frontier:
            h[v] = height
            for w in succ[v]:
                deg[w] -= 1
                if deg[w] == 0:
                    nxt.append(w)
        frontier = nxt
    return {"n": n, "m": m, "m_over_n": round(m / max(1, n), 3),
            "max_in": int(indeg.max()) if n else 0, "max_out": int(outdeg.max()) if n else 0,
            "height": height, "sum_p_ns": int(p.sum()),
            "mix_pct": [round(100 * b0 / n, 2), round(100 * b1 / n, 2), round(100 * b2 / n, 2)],
            "sum_bytes": int(g.nbytes.sum())}
