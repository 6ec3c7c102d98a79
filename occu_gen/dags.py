"""Synthetic DL computation graphs shaped like the paper's workloads.

The paper represents a DL model as a DAG of operators (P49, Fig. 1), built from
ONNX (P95, P239), for the Table II families (P165-P187).  Its dataset is not
available, so this module builds ONNX-granularity forward graphs per family and
expands them into *training* graphs:

* one backward node per forward op, fed by reversed (bwd-typed) edges;
* a saved-activation edge fwd(u) -> bwd(u) (fwd-typed);
* one loss node between the last forward op and its backward node;
* one parameter-update node per parameter tensor, fed by its op's backward
  node (bwd-typed).

Node order is topological: forward ops, loss, then backward ops in reverse
forward order, each followed by its update nodes.  Hyperparameters (batch,
input channels, sequence length, GPU) change features, never topology.

This module holds none of the GNN's arithmetic; shapes/FLOPs here are inputs.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

# ---- operator vocabulary (>30 types, P239) -> one-hot slot -----------------
OP_TYPES = [
    "Conv", "BatchNorm", "Relu", "MaxPool", "AvgPool", "GlobalAveragePool", "Add",
    "Gemm", "MatMul", "Flatten", "Reshape", "Transpose", "Softmax", "ReduceMean",
    "Sub", "Pow", "Sqrt", "Div", "Mul", "Erf", "Tanh", "Sigmoid", "Concat", "Shape",
    "Gather", "Unsqueeze", "Slice", "Dropout", "LRN", "Split", "Where", "Cast",
    "Constant", "Pad", "Identity", "LayerNormalization", "Squeeze", "Loss",
    "Update", "Expand",
]
OP_INDEX = {t: i for i, t in enumerate(OP_TYPES)}
assert len(OP_TYPES) == 40

ROLE_FWD, ROLE_BWD, ROLE_UPDATE, ROLE_LOSS = 0, 1, 2, 3


@dataclass
class Op:
    type: str
    inputs: list
    out_shape: tuple
    hp: tuple = ()                # op hyperparameters (kernel, stride, ...)
    params: list = field(default_factory=list)   # parameter tensor shapes
    flops: float = 0.0
    temp: float = 0.0             # temporary workspace elements


def numel(shape) -> int:
    n = 1
    for s in shape:
        n *= int(s)
    return n


class Builder:
    """Forward-graph builder; shapes are symbolic in the model config."""

    def __init__(self, hp: dict):
        self.ops: list[Op] = []
        self.hp = hp

    def add(self, type_, inputs, out_shape, hp=(), params=(), flops=None, temp=0.0):
        inputs = [i for i in inputs if i is not None]
        if flops is None:
            flops = float(numel(out_shape))
        self.ops.append(Op(type_, list(inputs), tuple(int(s) for s in out_shape),
                           tuple(hp), list(params), float(flops), float(temp)))
        return len(self.ops) - 1

    def shape(self, i):
        return self.ops[i].out_shape

    # --- CNN ops -----------------------------------------------------------
    def conv(self, x, k, r, stride=1, pad=None, groups=1, bias=False):
        n, c, h, w = self.shape(x)
        if pad is None:
            pad = r // 2
        p = (h + 2 * pad - r) // stride + 1
        q = (w + 2 * pad - r) // stride + 1
        # P131: FLOPs = 2*K*C*R*S*N*P*Q (per group: C/groups input channels)
        fl = 2.0 * k * (c // groups) * r * r * n * p * q
        params = [(k, c // groups, r, r)] + ([(k,)] if bias else [])
        return self.add("Conv", [x], (n, k, p, q), (r, r, stride, pad, 1, groups, c, k),
                        params, fl, temp=float(c // groups * r * r * p * q))

    def bn(self, x):
        c = self.shape(x)[1]
        return self.add("BatchNorm", [x], self.shape(x), (c,), [(c,), (c,)],
                        4.0 * numel(self.shape(x)))

    def relu(self, x):
        return self.add("Relu", [x], self.shape(x))

    def pool(self, x, kind, r, stride, pad=0):
        n, c, h, w = self.shape(x)
        p = (h + 2 * pad - r) // stride + 1
        q = (w + 2 * pad - r) // stride + 1
        return self.add(kind, [x], (n, c, p, q), (r, r, stride, pad), (),
                        float(n * c * p * q * r * r))

    def gap(self, x):
        n, c, h, w = self.shape(x)
        return self.add("GlobalAveragePool", [x], (n, c, 1, 1), (), (), float(n * c * h * w))

    def flatten(self, x):
        s = self.shape(x)
        return self.add("Flatten", [x], (s[0], numel(s[1:])))

    def linear(self, x, out, bias=True, op="Gemm"):
        s = self.shape(x)
        m = numel(s[:-1])
        k = s[-1]
        # P133: GEMM FLOPs 2*M*N*K
        params = [(out, k)] + ([(out,)] if bias else [])
        return self.add(op, [x], tuple(s[:-1]) + (out,), (k, out), params, 2.0 * m * out * k)

    def add2(self, a, b):
        return self.add("Add", [a, b], self.shape(a))

    # --- transformer ops (ONNX granularity) -------------------------------
    def const(self):
        return self.add("Constant", [], (1,))

    def onnx_reshape(self, x, new_shape):
        """Reshape with the ONNX dynamic-shape subgraph:
        Shape -> (Constant, Gather, Unsqueeze) x2, Constant x2 -> Concat -> Reshape."""
        sh = self.add("Shape", [x], (len(self.shape(x)),))
        parts = []
        for _ in range(2):
            g = self.add("Gather", [sh, self.const()], (1,))
            parts.append(self.add("Unsqueeze", [g], (1,)))
        parts += [self.const(), self.const()]
        cat = self.add("Concat", parts, (len(new_shape),))
        return self.add("Reshape", [x, cat], new_shape)

    def layernorm(self, x, decomposed=True):
        s = self.shape(x)
        h = s[-1]
        if not decomposed:
            return self.add("LayerNormalization", [x], s, (h,), [(h,), (h,)], 8.0 * numel(s))
        red = tuple(s[:-1]) + (1,)
        m = self.add("ReduceMean", [x], red)
        d = self.add("Sub", [x, m], s)
        p = self.add("Pow", [d, self.const()], s)
        v = self.add("ReduceMean", [p], red)
        e = self.add("Add", [v, self.const()], red)
        q = self.add("Sqrt", [e], red)
        n = self.add("Div", [d, q], s)
        g = self.add("Mul", [n], s, (), [(h,)])
        return self.add("Add", [g], s, (), [(h,)])

    def gelu(self, x):
        s = self.shape(x)
        a = self.add("Div", [x, self.const()], s)
        b = self.add("Erf", [a], s)
        c = self.add("Add", [b, self.const()], s)
        d = self.add("Mul", [x, c], s)
        return self.add("Mul", [d, self.const()], s)

    def onnx_linear(self, x, out, cast=True):
        """MatMul + separate bias Add, with autocast Casts on the operands (AMP training)."""
        if cast:
            x = self.add("Cast", [x], self.shape(x))
        y = self.linear(x, out, bias=False, op="MatMul")
        if cast:
            y = self.add("Cast", [y], self.shape(y))
        return self.add("Add", [y], self.shape(y), (), [(out,)])

    def attention(self, x, heads, shape_ops=True):
        b, t, h = self.shape(x)
        dh = h // heads
        proj = []
        for _ in range(3):
            y = self.onnx_linear(x, h) if shape_ops else self.linear(x, h, bias=True, op="MatMul")
            if shape_ops:
                y = self.onnx_reshape(y, (b, t, heads, dh))
            else:
                y = self.add("Reshape", [y], (b, t, heads, dh))
            y = self.add("Transpose", [y], (b, heads, t, dh))
            proj.append(y)
        q, k, v = proj
        kt = self.add("Transpose", [k], (b, heads, dh, t))
        s = self.add("MatMul", [q, kt], (b, heads, t, t), (dh,), (), 2.0 * b * heads * t * t * dh)
        s = self.add("Div", [s, self.const()], (b, heads, t, t))
        s = self.add("Add", [s], (b, heads, t, t))            # mask
        s = self.add("Softmax", [s], (b, heads, t, t), (), (), 5.0 * b * heads * t * t)
        s = self.add("Dropout", [s], (b, heads, t, t))
        o = self.add("MatMul", [s, v], (b, heads, t, dh), (t,), (), 2.0 * b * heads * t * t * dh)
        o = self.add("Transpose", [o], (b, t, heads, dh))
        if shape_ops:
            o = self.onnx_reshape(o, (b, t, h))
        else:
            o = self.add("Reshape", [o], (b, t, h))
            return self.linear(o, h, bias=True, op="MatMul")
        return self.onnx_linear(o, h)

    def ffn(self, x, h, mult, onnx=True):
        if onnx:
            return self.onnx_linear(self.gelu(self.onnx_linear(x, h * mult)), h)
        return self.linear(self.gelu(self.linear(x, h * mult, op="MatMul")), h, op="MatMul")

    def encoder_block(self, x, heads, ffn_mult=4, pre_ln=False, shape_ops=True, decomposed_ln=True):
        h = self.shape(x)[-1]
        if pre_ln:
            y = self.layernorm(x, decomposed_ln)
            y = self.attention(y, heads, shape_ops)
            y = self.add("Dropout", [y], self.shape(y))
            x = self.add2(x, y)
            y = self.layernorm(x, decomposed_ln)
            y = self.ffn(y, h, ffn_mult, shape_ops)
            y = self.add("Dropout", [y], self.shape(y))
            return self.add2(x, y)
        y = self.attention(x, heads, shape_ops)
        y = self.add("Dropout", [y], self.shape(y))
        x = self.layernorm(self.add2(x, y), decomposed_ln)
        y = self.ffn(x, h, ffn_mult, shape_ops)
        y = self.add("Dropout", [y], self.shape(y))
        return self.layernorm(self.add2(x, y), decomposed_ln)


# ---------------------------------------------------------------------------
# Families (Table II, P165-P187).  hp keys: batch, cin, seq, hw.
# ---------------------------------------------------------------------------

def _img(b: Builder):
    n, c, hw = b.hp["batch"], b.hp["cin"], b.hp.get("hw", 224)
    return b.add("Identity", [], (n, c, hw, hw))


def lenet5(b: Builder):
    b.hp = dict(b.hp, hw=32)
    x = _img(b)
    x = b.pool(b.relu(b.conv(x, 6, 5, pad=0, bias=True)), "MaxPool", 2, 2)
    x = b.pool(b.relu(b.conv(x, 16, 5, pad=0, bias=True)), "MaxPool", 2, 2)
    x = b.flatten(x)
    x = b.relu(b.linear(x, 120))
    x = b.relu(b.linear(x, 84))
    x = b.linear(x, 10)
    return b.add("Softmax", [x], b.shape(x))


def alexnet(b: Builder):
    x = _img(b)
    x = b.relu(b.conv(x, 64, 11, 4, 2, bias=True))
    x = b.add("LRN", [x], b.shape(x))
    x = b.pool(x, "MaxPool", 3, 2)
    x = b.relu(b.conv(x, 192, 5, 1, 2, bias=True))
    x = b.add("LRN", [x], b.shape(x))
    x = b.pool(x, "MaxPool", 3, 2)
    x = b.relu(b.conv(x, 384, 3, bias=True))
    x = b.relu(b.conv(x, 256, 3, bias=True))
    x = b.relu(b.conv(x, 256, 3, bias=True))
    x = b.pool(x, "MaxPool", 3, 2)
    x = b.flatten(x)
    for w in (4096, 4096):
        x = b.add("Dropout", [x], b.shape(x))
        x = b.relu(b.linear(x, w))
    return b.linear(x, 1000)


def _vgg(cfg):
    def build(b: Builder):
        x = _img(b)
        for v in cfg:
            if v == "M":
                x = b.pool(x, "MaxPool", 2, 2)
            else:
                x = b.relu(b.conv(x, v, 3, bias=True))
        x = b.flatten(x)
        for w in (4096, 4096):
            x = b.add("Dropout", [b.relu(b.linear(x, w))], (b.shape(x)[0], w))
        return b.linear(x, 1000)
    return build


vgg11 = _vgg([64, "M", 128, "M", 256, 256, "M", 512, 512, "M", 512, 512, "M"])
vgg13 = _vgg([64, 64, "M", 128, 128, "M", 256, 256, "M", 512, 512, "M", 512, 512, "M"])
vgg16 = _vgg([64, 64, "M", 128, 128, "M", 256, 256, 256, "M", 512, 512, 512, "M",
              512, 512, 512, "M"])


def _resnet(blocks, bottleneck):
    def build(b: Builder):
        x = _img(b)
        x = b.pool(b.relu(b.bn(b.conv(x, 64, 7, 2, 3))), "MaxPool", 3, 2, 1)
        cin = 64
        for stage, nb in enumerate(blocks):
            width = 64 * 2 ** stage
            out = width * 4 if bottleneck else width
            for i in range(nb):
                stride = 2 if (i == 0 and stage > 0) else 1
                idn = x
                if bottleneck:
                    y = b.relu(b.bn(b.conv(x, width, 1, 1, 0)))
                    y = b.relu(b.bn(b.conv(y, width, 3, stride)))
                    y = b.bn(b.conv(y, out, 1, 1, 0))
                else:
                    y = b.relu(b.bn(b.conv(x, width, 3, stride)))
                    y = b.bn(b.conv(y, width, 3, 1))
                if stride != 1 or cin != out:
                    idn = b.bn(b.conv(x, out, 1, stride, 0))
                x = b.relu(b.add2(y, idn))
                cin = out
        x = b.flatten(b.gap(x))
        return b.linear(x, 1000)
    return build


resnet18 = _resnet([2, 2, 2, 2], False)
resnet34 = _resnet([3, 4, 6, 3], False)
resnet50 = _resnet([3, 4, 6, 3], True)


def convnext_b(b: Builder):
    x = _img(b)
    x = b.conv(x, 128, 4, 4, 0, bias=True)
    x = b.add("Transpose", [x], b.shape(x))
    x = b.layernorm(x, decomposed=False)
    dims, depths = [128, 256, 512, 1024], [3, 3, 27, 3]
    for s, (dim, dep) in enumerate(zip(dims, depths)):
        if s > 0:
            x = b.layernorm(x, decomposed=False)
            x = b.conv(x, dim, 2, 2, 0, bias=True)
        for _ in range(dep):
            y = b.conv(x, dim, 7, 1, 3, groups=dim, bias=True)
            n_, c_, h_, w_ = b.shape(y)
            y = b.add("Transpose", [y], (n_, h_, w_, c_))
            y = b.layernorm(y, decomposed=False)
            y = b.linear(y, 4 * dim, op="MatMul")
            y = b.gelu(y)
            y = b.linear(y, dim, op="MatMul")
            y = b.add("Mul", [y], b.shape(y), (), [(dim,)])
            y = b.add("Transpose", [y], (n_, c_, h_, w_))
            x = b.add2(x, y)
    x = b.flatten(b.gap(x))
    x = b.layernorm(x, decomposed=False)
    return b.linear(x, 1000)


def _rnn(kind):
    def build(b: Builder):
        n, t, hid = b.hp["batch"], b.hp["seq"], 256
        x = b.add("Identity", [], (t, n, 128))
        h = b.add("Constant", [], (n, hid))
        c = b.add("Constant", [], (n, hid)) if kind == "lstm" else None
        outs = []
        for step in range(min(t, 16)):                  # unrolled window of the sequence
            xs = b.add("Slice", [x], (n, 128))
            gates = 4 if kind == "lstm" else 1
            a = b.linear(xs, gates * hid, bias=True)
            r = b.linear(h, gates * hid, bias=False)
            z = b.add2(a, r)
            if kind == "lstm":
                sp = b.add("Split", [z], (n, hid))
                i_ = b.add("Sigmoid", [sp], (n, hid))
                f_ = b.add("Sigmoid", [sp], (n, hid))
                g_ = b.add("Tanh", [sp], (n, hid))
                o_ = b.add("Sigmoid", [sp], (n, hid))
                c = b.add2(b.add("Mul", [f_, c], (n, hid)), b.add("Mul", [i_, g_], (n, hid)))
                h = b.add("Mul", [o_, b.add("Tanh", [c], (n, hid))], (n, hid))
            else:
                h = b.add("Tanh", [z], (n, hid))
            outs.append(b.add("Unsqueeze", [h], (1, n, hid)))
        y = b.add("Concat", outs, (len(outs), n, hid))
        y = b.add("Gather", [y], (n, hid))
        return b.linear(y, 10)
    return build


lstm = _rnn("lstm")
rnn = _rnn("rnn")


def _vit(depth, dim, heads, patch):
    def build(b: Builder):
        n, c = b.hp["batch"], b.hp["cin"]
        x = _img(b)
        x = b.conv(x, dim, patch, patch, 0, bias=True)
        t = (224 // patch) ** 2
        x = b.add("Flatten", [x], (n, dim, t))
        x = b.add("Transpose", [x], (n, t, dim))
        cls = b.add("Expand", [], (n, 1, dim), (), [(1, 1, dim)])
        x = b.add("Concat", [cls, x], (n, t + 1, dim))
        x = b.add("Add", [x], (n, t + 1, dim), (), [(1, t + 1, dim)])
        for _ in range(depth):
            x = b.encoder_block(x, heads, pre_ln=True, shape_ops=True)
        x = b.layernorm(x)
        x = b.add("Gather", [x], (n, dim))
        return b.linear(x, 1000)
    return build


vit_t = _vit(12, 192, 3, 16)
vit_s = _vit(12, 384, 6, 16)
clip_vit_b32 = _vit(12, 768, 12, 32)
clip_vit_b16 = _vit(12, 768, 12, 16)


def swin_s(b: Builder):
    n = b.hp["batch"]
    x = _img(b)
    x = b.conv(x, 96, 4, 4, 0, bias=True)
    x = b.add("Transpose", [b.add("Flatten", [x], (n, 96, 3136))], (n, 3136, 96))
    x = b.layernorm(x)
    dims, depths, heads = [96, 192, 384, 768], [2, 2, 18, 2], [3, 6, 12, 24]
    t = 3136
    for s in range(4):
        if s > 0:
            t //= 4
            x = b.add("Reshape", [x], (n, t, 4 * dims[s - 1]))
            x = b.layernorm(x)
            x = b.linear(x, dims[s], bias=False, op="MatMul")
        for _ in range(depths[s]):
            # window partition / reverse around the attention block
            x = b.add("Reshape", [x], (n * max(t // 49, 1), min(t, 49), dims[s]))
            x = b.encoder_block(x, heads[s], pre_ln=True, shape_ops=False)
            x = b.add("Reshape", [x], (n, t, dims[s]))
    x = b.layernorm(x)
    x = b.add("ReduceMean", [x], (n, 768))
    return b.linear(x, 1000)


def maxvit_t(b: Builder):
    n = b.hp["batch"]
    x = _img(b)
    x = b.relu(b.bn(b.conv(x, 64, 3, 2, 1)))
    x = b.conv(x, 64, 3, 1, 1)
    dims, depths = [64, 128, 256, 512], [2, 2, 5, 2]
    for s in range(4):
        for i in range(depths[s]):
            stride = 2 if i == 0 else 1
            # MBConv
            y = b.bn(x)
            y = b.gelu(b.bn(b.conv(y, dims[s] * 4, 1, 1, 0)))
            y = b.gelu(b.bn(b.conv(y, dims[s] * 4, 3, stride, 1, groups=dims[s] * 4)))
            se = b.gap(y)
            se = b.add("Sigmoid", [b.conv(b.add("Relu", [b.conv(se, dims[s], 1, 1, 0, bias=True)],
                                                   (n, dims[s], 1, 1)), dims[s] * 4, 1, 1, 0,
                                            bias=True)], (n, dims[s] * 4, 1, 1))
            y = b.add("Mul", [y, se], b.shape(y))
            y = b.conv(y, dims[s], 1, 1, 0, bias=True)
            if stride != 1 or b.shape(x)[1] != dims[s]:
                x = b.conv(b.pool(x, "AvgPool", 2, stride), dims[s], 1, 1, 0, bias=True)
            x = b.add2(x, y)
            nn_, cc, hh, ww = b.shape(x)
            tt = hh * ww
            for _part in ("block", "grid"):
                z = b.add("Reshape", [x], (nn_ * max(tt // 49, 1), min(tt, 49), cc))
                z = b.encoder_block(z, max(cc // 32, 1), pre_ln=True, shape_ops=False)
                x = b.add("Reshape", [z], (nn_, cc, hh, ww))
    x = b.flatten(b.gap(x))
    x = b.layernorm(x)
    return b.linear(x, 1000)


# ---------------------------------------------------------------------------
# BERT / GPT-2 as the paper's largest graphs (P239: up to 2,664 nodes): the torch.onnx export
# of the Hugging Face modules in training mode under AMP autocast, constant folding off.
# Relative to the compact ONNX-style blocks above this adds what such an export contains:
# autocast Casts on every Linear operand (input, weight, bias) and around the fp32 ops
# (Softmax, LayerNorm), opset-13+ axes / ratio / training-mode inputs as Constant nodes
# (Unsqueeze, ReduceMean, Dropout), HF's `x.size()[:-1] + (...)` shape arithmetic
# (Shape -> Slice -> Concat -> Reshape), GPT-2's Conv1D (view -> addmm -> view), its causal
# mask slice (Shape / Gather / Sub / Slice / Where) per layer and its tanh GELU.  DESIGN.md R43.
# ---------------------------------------------------------------------------
class _HF:
    def __init__(self, b: Builder):
        self.b = b

    def const(self):
        return self.b.const()

    def cast(self, x, shape=None):
        return self.b.add("Cast", [x], self.b.shape(x) if shape is None else shape)

    def unsq(self, x, shape):
        return self.b.add("Unsqueeze", [x, self.const()], shape)

    def slice_(self, x, shape):
        # Slice(data, starts, ends, axes, steps)
        return self.b.add("Slice", [x, self.const(), self.const(), self.const(), self.const()], shape)

    def size_reshape(self, x, new_shape, keep):
        """HF shape arithmetic: x.size()[:keep] + (extra...) -> Reshape."""
        b = self.b
        sh = b.add("Shape", [x], (len(b.shape(x)),))
        head = self.slice_(sh, (keep,))
        extra = [self.const() for _ in range(len(new_shape) - keep)]
        cat = b.add("Concat", [head] + extra, (len(new_shape),))
        return b.add("Reshape", [x, cat], new_shape)

    def linear(self, x, out):
        """nn.Linear under autocast: Cast(x), Cast(W), Cast(b) -> MatMul (transposed weight)
        -> Add(bias)."""
        b = self.b
        s = b.shape(x)
        k = s[-1]
        xc = self.cast(x)
        wc = b.add("Cast", [], (out, k), (), [(out, k)])
        wt = b.add("Transpose", [wc], (k, out))
        y = b.add("MatMul", [xc, wt], tuple(s[:-1]) + (out,), (k, out), (),
                  2.0 * numel(s[:-1]) * out * k)
        bc = b.add("Cast", [], (out,), (), [(out,)])
        return b.add("Add", [y, bc], b.shape(y))

    def conv1d(self, x, out):
        """GPT-2 Conv1D: size_out = x.size()[:-1] + (nf,); x.view(-1, x.size(-1)) ->
        addmm(bias, x, W) (Gemm) -> view(size_out); autocast Casts on the operands."""
        b = self.b
        s = b.shape(x)
        k = s[-1]
        m = numel(s[:-1])
        sh = b.add("Shape", [x], (len(s),))
        last = b.add("Gather", [sh, self.const()], (1,))
        u = self.unsq(last, (1,))
        cat = b.add("Concat", [self.const(), u], (2,))
        flat = b.add("Reshape", [x, cat], (m, k))
        xc = self.cast(flat)
        wc = b.add("Cast", [], (k, out), (), [(k, out)])
        bc = b.add("Cast", [], (out,), (), [(out,)])
        g = b.add("Gemm", [bc, xc, wc], (m, out), (k, out), (), 2.0 * m * out * k)
        sh2 = b.add("Shape", [x], (len(s),))
        head = self.slice_(sh2, (len(s) - 1,))
        cat2 = b.add("Concat", [head, self.const()], (len(s),))
        return b.add("Reshape", [g, cat2], tuple(s[:-1]) + (out,))

    def dropout(self, x):
        # training-mode Dropout(data, ratio, training_mode) -> (output, mask)
        return self.b.add("Dropout", [x, self.const(), self.const()], self.b.shape(x))

    def layernorm(self, x):
        """LayerNorm autocast to fp32, decomposed (opset < 17), axes as Constant inputs."""
        b = self.b
        s = b.shape(x)
        h = s[-1]
        red = tuple(s[:-1]) + (1,)
        xf = self.cast(x)
        m = b.add("ReduceMean", [xf, self.const()], red)
        d = b.add("Sub", [xf, m], s)
        p = b.add("Pow", [d, self.const()], s)
        v = b.add("ReduceMean", [p, self.const()], red)
        e = b.add("Add", [v, self.const()], red)
        q = b.add("Sqrt", [e], red)
        n = b.add("Div", [d, q], s)
        g = b.add("Mul", [n], s, (), [(h,)])
        return b.add("Add", [g], s, (), [(h,)])

    def softmax(self, x):
        xf = self.cast(x)
        y = self.b.add("Softmax", [xf], self.b.shape(x), (), (), 5.0 * numel(self.b.shape(x)))
        return self.cast(y)

    def gelu_erf(self, x):
        b = self.b
        s = b.shape(x)
        a = b.add("Div", [x, self.const()], s)
        e = b.add("Erf", [a], s)
        c = b.add("Add", [e, self.const()], s)
        d = b.add("Mul", [x, c], s)
        return b.add("Mul", [d, self.const()], s)

    def gelu_tanh(self, x):
        """gelu_new: 0.5·x·(1 + tanh(sqrt(2/π)·(x + 0.044715·x³)))."""
        b = self.b
        s = b.shape(x)
        p3 = b.add("Pow", [x, self.const()], s)
        m1 = b.add("Mul", [p3, self.const()], s)
        a1 = b.add("Add", [x, m1], s)
        m2 = b.add("Mul", [a1, self.const()], s)
        t = b.add("Tanh", [m2], s)
        a2 = b.add("Add", [t, self.const()], s)
        m3 = b.add("Mul", [x, self.const()], s)
        return b.add("Mul", [m3, a2], s)

    def attention(self, x, heads, mask, causal):
        b = self.b
        n, t, h = b.shape(x)
        dh = h // heads
        if causal:                                  # c_attn: one Conv1D, then split
            qkv = self.conv1d(x, 3 * h)
            sp = b.add("Split", [qkv, self.const()], (n, t, h))
            parts = [sp, b.add("Identity", [sp], (n, t, h)), b.add("Identity", [sp], (n, t, h))]
        else:
            parts = [self.linear(x, h) for _ in range(3)]
        heads_ = []
        for y in parts:
            y = self.size_reshape(y, (n, t, heads, dh), 2)
            heads_.append(b.add("Transpose", [y], (n, heads, t, dh)))
        q, k, v = heads_
        kt = b.add("Transpose", [k], (n, heads, dh, t))
        sc = b.add("MatMul", [q, kt], (n, heads, t, t), (dh,), (), 2.0 * n * heads * t * t * dh)
        sc = b.add("Div", [sc, self.const()], (n, heads, t, t))
        if causal:                                  # bias[:, :, k-q:k, :k], torch.where(...)
            shq = b.add("Shape", [q], (4,))
            ql = b.add("Gather", [shq, self.const()], (1,))
            shk = b.add("Shape", [k], (4,))
            kl = b.add("Gather", [shk, self.const()], (1,))
            st = b.add("Sub", [kl, ql], (1,))
            s1 = b.add("Slice", [self.const(), self.unsq(st, (1,)), self.unsq(kl, (1,)),
                                 self.const(), self.const()], (1, 1, t, 1024))
            s2 = b.add("Slice", [s1, self.const(), self.unsq(kl, (1,)), self.const(), self.const()],
                       (1, 1, t, t))
            cm = b.add("Cast", [s2], (1, 1, t, t))
            fill = b.add("Cast", [self.const()], (1,))
            sc = b.add("Where", [cm, sc, fill], (n, heads, t, t))
        sc = b.add("Add", [sc, mask], (n, heads, t, t))
        pr = self.dropout(self.softmax(sc))
        o = b.add("MatMul", [pr, v], (n, heads, t, dh), (t,), (), 2.0 * n * heads * t * t * dh)
        o = b.add("Transpose", [o], (n, t, heads, dh))
        o = self.size_reshape(o, (n, t, h), 2)
        return self.conv1d(o, h) if causal else self.linear(o, h)

    def block(self, x, heads, mask, causal):
        b = self.b
        h = b.shape(x)[-1]
        if causal:                                   # GPT-2: pre-LN
            y = self.attention(self.layernorm(x), heads, mask, True)
            x = b.add2(x, self.dropout(y))
            y = self.conv1d(self.gelu_tanh(self.conv1d(self.layernorm(x), 4 * h)), h)
            return b.add2(x, self.dropout(y))
        y = self.dropout(self.attention(x, heads, mask, False))
        x = self.layernorm(b.add2(y, x))
        y = self.dropout(self.linear(self.gelu_erf(self.linear(x, 4 * h)), h))
        return self.layernorm(b.add2(y, x))


def _bert(depth, dim, heads, causal=False):
    def build(b: Builder):
        hf = _HF(b)
        n, t = b.hp["batch"], b.hp["seq"]
        ids = b.add("Identity", [], (n, t))
        sh = b.add("Shape", [ids], (2,))
        ln_ = b.add("Gather", [sh, b.const()], (1,))
        pos = hf.slice_(ln_, (1, t))
        tok = b.add("Gather", [ids], (n, t, dim), (), [(30522 if not causal else 50257, dim)])
        pe = b.add("Gather", [pos], (1, t, dim), (), [(512 if not causal else 1024, dim)])
        x = b.add2(tok, pe)
        if not causal:
            tt = b.add("Gather", [b.add("Identity", [], (n, t))], (n, t, dim), (), [(2, dim)])
            x = hf.dropout(hf.layernorm(b.add2(x, tt)))
        else:
            x = hf.dropout(x)
        # extended attention mask: (1 - mask[:, None, None, :]) * finfo.min, in the model dtype
        am = b.add("Identity", [], (n, t))
        mask = hf.unsq(hf.unsq(am, (n, 1, t)), (n, 1, 1, t))
        mask = hf.cast(mask)
        mask = b.add("Sub", [b.const(), mask], (n, 1, 1, t))
        mask = b.add("Mul", [mask, b.const()], (n, 1, 1, t))
        for _ in range(depth):
            x = hf.block(x, heads, mask, causal)
        if causal:
            x = hf.layernorm(x)
            return b.linear(x, 50257, bias=False, op="MatMul")
        x = b.add("Gather", [x, b.const()], (n, dim))
        x = b.add("Tanh", [hf.linear(x, dim)], (n, dim))
        return hf.linear(hf.dropout(x), 2)
    return build


distilbert = _bert(6, 768, 12)
bert_base = _bert(12, 768, 12)
gpt2 = _bert(12, 768, 12, causal=True)


def clip_rn50(b: Builder):
    return _resnet([3, 4, 6, 3], True)(b)


FAMILIES = {
    "convnext_b": convnext_b, "resnet18": resnet18, "resnet34": resnet34,
    "resnet50": resnet50, "vgg11": vgg11, "vgg13": vgg13, "vgg16": vgg16,
    "alexnet": alexnet, "lenet5": lenet5, "lstm": lstm, "rnn": rnn,
    "vit_t": vit_t, "vit_s": vit_s, "swin_s": swin_s, "maxvit_t": maxvit_t,
    "distilbert": distilbert, "gpt2": gpt2, "clip_rn50": clip_rn50,
    "clip_vit_b32": clip_vit_b32, "clip_vit_b16": clip_vit_b16,
    "bert_base": bert_base,
}
CNN = {"convnext_b", "resnet18", "resnet34", "resnet50", "vgg11", "vgg13", "vgg16",
       "alexnet", "lenet5", "clip_rn50"}
RNN = {"lstm", "rnn"}
TRANSFORMER = set(FAMILIES) - CNN - RNN


def default_hp(family: str) -> dict:
    if family in RNN:
        return {"batch": 128, "seq": 64, "cin": 1}
    if family in TRANSFORMER:
        return {"batch": 16, "seq": 512, "cin": 3}
    return {"batch": 16, "cin": 3}


def build_forward(family: str, hp: dict | None = None) -> Builder:
    hp = dict(default_hp(family), **(hp or {}))
    b = Builder(hp)
    FAMILIES[family](b)
    return b


@dataclass
class TrainGraph:
    """A training DAG: local int32 COO plus per-node/edge descriptors."""
    family: str
    num_nodes: int
    src: np.ndarray            # int32 [m]
    dst: np.ndarray            # int32 [m]
    node_op: np.ndarray        # int32 [n] index into OP_TYPES
    node_role: np.ndarray      # int32 [n]
    node_fwd: np.ndarray       # int32 [n] forward op index (or -1)
    node_param: np.ndarray     # int32 [n] param slot for update nodes (or -1)
    edge_bwd: np.ndarray       # int8 [m] 1 if backward-typed
    edge_fwd_src: np.ndarray   # int32 [m] forward op whose tensor the edge carries
    fwd: Builder = None
    param_shapes: list = None

    @property
    def num_edges(self) -> int:
        return int(self.src.size)


def expand_training(family: str, fb: Builder) -> TrainGraph:
    ops = fb.ops
    nf = len(ops)
    param_owner = []                     # (op index, shape)
    for i, op in enumerate(ops):
        for s in op.params:
            param_owner.append((i, s))
    # node ids: fwd 0..nf-1, loss nf, then bwd in reverse order + their updates
    loss = nf
    bwd_id = {}
    upd_ids = {}
    nxt = nf + 1
    by_op = {}
    for k, (i, _) in enumerate(param_owner):
        by_op.setdefault(i, []).append(k)
    for i in range(nf - 1, -1, -1):
        bwd_id[i] = nxt
        nxt += 1
        for k in by_op.get(i, []):
            upd_ids[k] = nxt
            nxt += 1
    n = nxt
    node_op = np.zeros(n, np.int32)
    node_role = np.zeros(n, np.int32)
    node_fwd = np.full(n, -1, np.int32)
    node_param = np.full(n, -1, np.int32)
    for i, op in enumerate(ops):
        node_op[i] = OP_INDEX[op.type]
        node_role[i] = ROLE_FWD
        node_fwd[i] = i
        node_op[bwd_id[i]] = OP_INDEX[op.type]
        node_role[bwd_id[i]] = ROLE_BWD
        node_fwd[bwd_id[i]] = i
    node_op[loss] = OP_INDEX["Loss"]
    node_role[loss] = ROLE_LOSS
    node_fwd[loss] = nf - 1
    for k, (i, _) in enumerate(param_owner):
        u = upd_ids[k]
        node_op[u] = OP_INDEX["Update"]
        node_role[u] = ROLE_UPDATE
        node_fwd[u] = i
        node_param[u] = k
    src, dst, eb, ets = [], [], [], []
    for v, op in enumerate(ops):
        for u in op.inputs:
            src.append(u); dst.append(v); eb.append(0); ets.append(u)          # forward dataflow
    for v, op in enumerate(ops):
        for u in op.inputs:
            src.append(bwd_id[v]); dst.append(bwd_id[u]); eb.append(1); ets.append(u)  # gradient
    for i in range(nf):
        src.append(i); dst.append(bwd_id[i]); eb.append(0); ets.append(i)      # saved activation
    src.append(nf - 1); dst.append(loss); eb.append(0); ets.append(nf - 1)
    src.append(loss); dst.append(bwd_id[nf - 1]); eb.append(1); ets.append(nf - 1)
    for k, (i, _) in enumerate(param_owner):
        src.append(bwd_id[i]); dst.append(upd_ids[k]); eb.append(1); ets.append(i)
    return TrainGraph(family, n, np.asarray(src, np.int32), np.asarray(dst, np.int32),
                      node_op, node_role, node_fwd, node_param,
                      np.asarray(eb, np.int8), np.asarray(ets, np.int32), fb,
                      [s for _, s in param_owner])


def is_dag(num_nodes: int, src: np.ndarray, dst: np.ndarray) -> bool:
    """Kahn's algorithm; self-loops or cycles -> False."""
    indeg = np.zeros(num_nodes, np.int64)
    np.add.at(indeg, dst, 1)
    adj = [[] for _ in range(num_nodes)]
    for s, t in zip(src.tolist(), dst.tolist()):
        adj[s].append(t)
    stack = [u for u in range(num_nodes) if indeg[u] == 0]
    seen = 0
    while stack:
        u = stack.pop()
        seen += 1
        for t in adj[u]:
            indeg[t] -= 1
            if indeg[t] == 0:
                stack.append(t)
    return seen == num_nodes


_TOPO_CACHE: dict = {}


def training_graph(family: str, hp: dict | None = None) -> TrainGraph:
    """Training DAG for a family; topology is independent of ``hp``."""
    key = (family, tuple(sorted((hp or {}).items())))
    if key not in _TOPO_CACHE:
        _TOPO_CACHE[key] = expand_training(family, build_forward(family, hp))
    return _TOPO_CACHE[key]


def relabel(g: TrainGraph, perm: np.ndarray) -> TrainGraph:
    """Graph with node u renamed perm[u] (node arrays permuted accordingly)."""
    inv = np.argsort(perm)
    return TrainGraph(g.family, g.num_nodes, perm[g.src].astype(np.int32),
                      perm[g.dst].astype(np.int32), g.node_op[inv], g.node_role[inv],
                      g.node_fwd[inv], g.node_param[inv], g.edge_bwd, g.edge_fwd_src,
                      g.fwd, g.param_shapes)
