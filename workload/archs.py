"""Model architectures of the paper's evaluation mix, as plain layer lists.

NEUTRAL MODULE: this file is *input description* shared by the oracle (``oracle/``)
and the CUDA path (``paper_conf_sosp_ngd023_b200/``).  It holds no arithmetic of the
method (no convolution, no pooling, no scheduling) -- only the graph of layers and
their static shapes, the same way a model file handed to ``paella_register_model``
would.  Its correctness is pinned independently by ``tests/test_oracle_infer.py``,
which checks the oracle's forward over this graph against torchvision's own model
definitions (pin P-inf-1).

Paper: Table 2 (PAPER.md P1268-1281) lists ResNet-18/34/50, MobileNetV2,
SqueezeNet1.1, DenseNet(-121), GoogLeNet and InceptionV3 "from repositories of
pre-trained models such as the ONNX Model Zoo" (P1367-1369).  Reading C1-Q1
(DESIGN.md): the torchvision definitions, batch 1, 224x224 (Inception 299x299).
The toy model is BASELINE.json configs[0] ("3-layer conv+MLP toy model").

BatchNorm is never a node: synthetic weights are generated already folded
(SURVEY.md §8(c) C1 step 4).  DenseNet's pre-activation BN+ReLU, which cannot be
folded into the following conv, is a per-input-channel ``prologue`` (scale, shift,
ReLU) on the consuming conv / global-average-pool.

Node dict keys:
  id, op, name, inputs (list of node ids), out (C, H, W), plus op attributes:
  conv    : cin, cout, kh, kw, sh, sw, ph, pw, groups, act, bias, residual, prologue
  maxpool : k, s, p, ceil
  avgpool : k, s, p                      (count_include_pad=True)
  gap     : prologue                     (global average pool -> (C,1,1))
  fc      : cin, cout, act
  concat  : (channel concat of inputs, in order)
  input   : (fp32 NCHW image, batch 1)
"""
from __future__ import annotations

import math

ACTS = ("none", "relu", "relu6")


def _conv_out(n, k, s, p):
    return (n + 2 * p - k) // s + 1


def _pool_out(n, k, s, p, ceil):
    # PyTorch rule (torch.nn.MaxPool2d docs): ceil mode drops a last window that
    # starts inside the right padding.
    if not ceil:
        return (n + 2 * p - k) // s + 1
    o = -(-(n + 2 * p - k) // s) + 1
    if (o - 1) * s >= n + p:
        o -= 1
    return o


class Graph:
    """A model as a topologically ordered list of nodes."""

    def __init__(self, name, in_shape, num_classes):
        self.name = name
        self.num_classes = num_classes
        self.nodes = []
        self.input = self._add("input", "input", [], tuple(in_shape))

    # -- construction helpers ------------------------------------------------
    def _add(self, op, name, inputs, out, **attrs):
        nid = len(self.nodes)
        node = dict(id=nid, op=op, name=name, inputs=list(inputs), out=tuple(out))
        node.update(attrs)
        self.nodes.append(node)
        return nid

    def shape(self, nid):
        return self.nodes[nid]["out"]

    def conv(self, x, cout, k, s=1, p=0, groups=1, act="relu", bias=True,
             residual=None, prologue=False, name=None):
        kh, kw = (k, k) if isinstance(k, int) else k
        sh, sw = (s, s) if isinstance(s, int) else s
        ph, pw = (p, p) if isinstance(p, int) else p
        c, h, w = self.shape(x)
        assert act in ACTS and c % groups == 0 and cout % groups == 0
        oh, ow = _conv_out(h, kh, sh, ph), _conv_out(w, kw, sw, pw)
        if residual is not None:
            assert self.shape(residual) == (cout, oh, ow), (name, self.shape(residual))
        return self._add("conv", name or f"conv{len(self.nodes)}", [x], (cout, oh, ow),
                         cin=c, cout=cout, kh=kh, kw=kw, sh=sh, sw=sw, ph=ph, pw=pw,
                         groups=groups, act=act, bias=bias, residual=residual,
                         prologue=prologue)

    def maxpool(self, x, k, s, p=0, ceil=False, name=None):
        c, h, w = self.shape(x)
        return self._add("maxpool", name or f"maxpool{len(self.nodes)}", [x],
                         (c, _pool_out(h, k, s, p, ceil), _pool_out(w, k, s, p, ceil)),
                         k=k, s=s, p=p, ceil=ceil)

    def avgpool(self, x, k, s, p=0, name=None):
        c, h, w = self.shape(x)
        return self._add("avgpool", name or f"avgpool{len(self.nodes)}", [x],
                         (c, _pool_out(h, k, s, p, False), _pool_out(w, k, s, p, False)),
                         k=k, s=s, p=p)

    def gap(self, x, prologue=False, name=None):
        c, _, _ = self.shape(x)
        return self._add("gap", name or f"gap{len(self.nodes)}", [x], (c, 1, 1),
                         prologue=prologue)

    def spin(self, x, us, name=None):
        """Synthetic kernel of the HoL microbenchmark (Fig. 2, P431-445): one block that
        stays resident `us` microseconds and copies its input (identity)."""
        return self._add("spin", name or f"spin{len(self.nodes)}", [x], self.shape(x), us=us)

    def fc(self, x, cout, act="none", name=None):
        c, h, w = self.shape(x)
        return self._add("fc", name or f"fc{len(self.nodes)}", [x], (cout, 1, 1),
                         cin=c * h * w, cout=cout, act=act)

    def concat(self, xs, name=None):
        shapes = [self.shape(x) for x in xs]
        h, w = shapes[0][1:]
        assert all(s[1:] == (h, w) for s in shapes)
        return self._add("concat", name or f"concat{len(self.nodes)}", xs,
                         (sum(s[0] for s in shapes), h, w))

    # -- queries ---------------------------------------------------------------
    @property
    def output(self):
        return len(self.nodes) - 1

    def weight_nodes(self):
        """conv/fc nodes in execution order (the LSUV order, C1 step 3)."""
        return [n for n in self.nodes if n["op"] in ("conv", "fc")]

    def prologue_nodes(self):
        return [n for n in self.nodes if n.get("prologue")]

    def param_shapes(self):
        """name -> shape of every parameter tensor (weights are [cout, cin/g, kh, kw])."""
        out = {}
        for n in self.nodes:
            if n["op"] == "conv":
                out[n["name"] + ".weight"] = (n["cout"], n["cin"] // n["groups"], n["kh"], n["kw"])
                out[n["name"] + ".bias"] = (n["cout"],)
            elif n["op"] == "fc":
                out[n["name"] + ".weight"] = (n["cout"], n["cin"])
                out[n["name"] + ".bias"] = (n["cout"],)
            if n.get("prologue"):
                c = self.shape(n["inputs"][0])[0]
                out[n["name"] + ".pro_scale"] = (c,)
                out[n["name"] + ".pro_shift"] = (c,)
        return out

    def flops(self):
        f = 0
        for n in self.nodes:
            if n["op"] == "conv":
                c, h, w = n["out"]
                f += 2 * c * h * w * (n["cin"] // n["groups"]) * n["kh"] * n["kw"]
            elif n["op"] == "fc":
                f += 2 * n["cin"] * n["cout"]
        return f


# ---------------------------------------------------------------------------
# The models
# ---------------------------------------------------------------------------

def toy():
    """BASELINE.json configs[0]: conv3x3(3->16,s1,p1)+bias+ReLU -> maxpool 2x2 s2 ->
    FC 4096->128 + ReLU -> FC 128->10; input 1x3x32x32."""
    g = Graph("toy", (3, 32, 32), 10)
    x = g.conv(g.input, 16, 3, 1, 1, act="relu", name="conv1")
    x = g.maxpool(x, 2, 2, 0, name="pool1")
    x = g.fc(x, 128, act="relu", name="fc1")
    g.fc(x, 10, act="none", name="fc2")
    return g


def hol_synthetic(n_kernels=8, spin_us=300):
    """Fig. 2's synthetic job (P431-445): a chain of `n_kernels` kernels, each ONE block
    of 128 threads resident for `spin_us` us, on a 1x1 input of 8 channels (identity
    copies), closed by a global average pool over the single pixel (8 outputs)."""
    g = Graph(f"hol{n_kernels}x{spin_us}", (8, 1, 1), 8)
    x = g.input
    for i in range(n_kernels):
        x = g.spin(x, spin_us, name=f"spin{i}")
    g.gap(x, name="out")
    return g


def _resnet(name, block, layers):
    g = Graph(name, (3, 224, 224), 1000)
    x = g.conv(g.input, 64, 7, 2, 3, name="conv1")
    x = g.maxpool(x, 3, 2, 1, name="maxpool")
    inplanes = 64
    for li, (planes, nblocks) in enumerate(zip((64, 128, 256, 512), layers)):
        for b in range(nblocks):
            stride = 2 if (b == 0 and li > 0) else 1
            pre = f"layer{li + 1}.{b}"
            exp = 1 if block == "basic" else 4
            identity = x
            if stride != 1 or inplanes != planes * exp:
                identity = g.conv(x, planes * exp, 1, stride, 0, act="none",
                                  name=pre + ".downsample.0")
            if block == "basic":
                y = g.conv(x, planes, 3, stride, 1, name=pre + ".conv1")
                x = g.conv(y, planes, 3, 1, 1, residual=identity, name=pre + ".conv2")
            else:  # bottleneck v1.5: stride on the 3x3
                y = g.conv(x, planes, 1, 1, 0, name=pre + ".conv1")
                y = g.conv(y, planes, 3, stride, 1, name=pre + ".conv2")
                x = g.conv(y, planes * 4, 1, 1, 0, residual=identity, name=pre + ".conv3")
            inplanes = planes * exp
    x = g.gap(x, name="avgpool")
    g.fc(x, 1000, name="fc")
    return g


def resnet18():
    return _resnet("resnet18", "basic", (2, 2, 2, 2))


def resnet34():
    return _resnet("resnet34", "basic", (3, 4, 6, 3))


def resnet50():
    return _resnet("resnet50", "bottleneck", (3, 4, 6, 3))


def mobilenet_v2():
    g = Graph("mobilenet_v2", (3, 224, 224), 1000)
    x = g.conv(g.input, 32, 3, 2, 1, act="relu6", name="features.0.0")
    cin = 32
    idx = 1
    for t, c, n, s in ((1, 16, 1, 1), (6, 24, 2, 2), (6, 32, 3, 2), (6, 64, 4, 2),
                       (6, 96, 3, 1), (6, 160, 3, 2), (6, 320, 1, 1)):
        for i in range(n):
            stride = s if i == 0 else 1
            hidden = int(round(cin * t))
            pre = f"features.{idx}.conv"
            y = x
            j = 0
            if t != 1:
                y = g.conv(y, hidden, 1, 1, 0, act="relu6", name=f"{pre}.{j}.0")
                j += 1
            y = g.conv(y, hidden, 3, stride, 1, groups=hidden, act="relu6", name=f"{pre}.{j}.0")
            j += 1
            res = x if (stride == 1 and cin == c) else None
            x = g.conv(y, c, 1, 1, 0, act="none", residual=res, name=f"{pre}.{j}")
            cin = c
            idx += 1
    x = g.conv(x, 1280, 1, 1, 0, act="relu6", name=f"features.{idx}.0")
    x = g.gap(x, name="avgpool")
    g.fc(x, 1000, name="classifier.1")
    return g


def squeezenet1_1():
    g = Graph("squeezenet1_1", (3, 224, 224), 1000)
    x = g.conv(g.input, 64, 3, 2, 0, name="features.0")
    x = g.maxpool(x, 3, 2, 0, ceil=True, name="features.2")

    def fire(x, idx, sq, e1, e3):
        s = g.conv(x, sq, 1, 1, 0, name=f"features.{idx}.squeeze")
        a = g.conv(s, e1, 1, 1, 0, name=f"features.{idx}.expand1x1")
        b = g.conv(s, e3, 3, 1, 1, name=f"features.{idx}.expand3x3")
        return g.concat([a, b], name=f"features.{idx}.cat")

    x = fire(x, 3, 16, 64, 64)
    x = fire(x, 4, 16, 64, 64)
    x = g.maxpool(x, 3, 2, 0, ceil=True, name="features.5")
    x = fire(x, 6, 32, 128, 128)
    x = fire(x, 7, 32, 128, 128)
    x = g.maxpool(x, 3, 2, 0, ceil=True, name="features.8")
    x = fire(x, 9, 48, 192, 192)
    x = fire(x, 10, 48, 192, 192)
    x = fire(x, 11, 64, 256, 256)
    x = fire(x, 12, 64, 256, 256)
    x = g.conv(x, 1000, 1, 1, 0, act="relu", name="classifier.1")
    g.gap(x, name="classifier.3")
    return g


def densenet121():
    g = Graph("densenet121", (3, 224, 224), 1000)
    x = g.conv(g.input, 64, 7, 2, 3, name="features.conv0")  # + norm0 + relu0 folded
    x = g.maxpool(x, 3, 2, 1, name="features.pool0")
    growth, bn_size = 32, 4
    nfeat = 64
    for bi, nl in enumerate((6, 12, 24, 16)):
        feats = [x]
        for li in range(nl):
            pre = f"features.denseblock{bi + 1}.denselayer{li + 1}"
            inp = feats[0] if len(feats) == 1 else g.concat(feats, name=pre + ".cat")
            # norm1+relu1 = prologue; conv1 + norm2 folded; relu2
            y = g.conv(inp, bn_size * growth, 1, 1, 0, act="relu", prologue=True, name=pre + ".conv1")
            y = g.conv(y, growth, 3, 1, 1, act="none", bias=False, name=pre + ".conv2")
            feats.append(y)
        x = g.concat(feats, name=f"features.denseblock{bi + 1}.cat")
        nfeat += nl * growth
        if bi != 3:
            pre = f"features.transition{bi + 1}"
            y = g.conv(x, nfeat // 2, 1, 1, 0, act="none", bias=False, prologue=True, name=pre + ".conv")
            x = g.avgpool(y, 2, 2, 0, name=pre + ".pool")
            nfeat //= 2
    x = g.gap(x, prologue=True, name="features.norm5")  # norm5 + relu + GAP
    g.fc(x, 1000, name="classifier")
    return g


def inception_v3():
    g = Graph("inception_v3", (3, 299, 299), 1000)
    C = g.conv
    x = C(g.input, 32, 3, 2, 0, name="Conv2d_1a_3x3.conv")
    x = C(x, 32, 3, 1, 0, name="Conv2d_2a_3x3.conv")
    x = C(x, 64, 3, 1, 1, name="Conv2d_2b_3x3.conv")
    x = g.maxpool(x, 3, 2, 0, name="maxpool1")
    x = C(x, 80, 1, 1, 0, name="Conv2d_3b_1x1.conv")
    x = C(x, 192, 3, 1, 0, name="Conv2d_4a_3x3.conv")
    x = g.maxpool(x, 3, 2, 0, name="maxpool2")

    def inc_a(x, m, pf):
        b1 = C(x, 64, 1, name=f"{m}.branch1x1.conv")
        b5 = C(x, 48, 1, name=f"{m}.branch5x5_1.conv")
        b5 = C(b5, 64, 5, 1, 2, name=f"{m}.branch5x5_2.conv")
        b3 = C(x, 64, 1, name=f"{m}.branch3x3dbl_1.conv")
        b3 = C(b3, 96, 3, 1, 1, name=f"{m}.branch3x3dbl_2.conv")
        b3 = C(b3, 96, 3, 1, 1, name=f"{m}.branch3x3dbl_3.conv")
        bp = g.avgpool(x, 3, 1, 1, name=f"{m}.avgpool")
        bp = C(bp, pf, 1, name=f"{m}.branch_pool.conv")
        return g.concat([b1, b5, b3, bp], name=f"{m}.cat")

    def inc_b(x, m):
        b3 = C(x, 384, 3, 2, 0, name=f"{m}.branch3x3.conv")
        bd = C(x, 64, 1, name=f"{m}.branch3x3dbl_1.conv")
        bd = C(bd, 96, 3, 1, 1, name=f"{m}.branch3x3dbl_2.conv")
        bd = C(bd, 96, 3, 2, 0, name=f"{m}.branch3x3dbl_3.conv")
        bp = g.maxpool(x, 3, 2, 0, name=f"{m}.maxpool")
        return g.concat([b3, bd, bp], name=f"{m}.cat")

    def inc_c(x, m, c7):
        b1 = C(x, 192, 1, name=f"{m}.branch1x1.conv")
        b7 = C(x, c7, 1, name=f"{m}.branch7x7_1.conv")
        b7 = C(b7, c7, (1, 7), 1, (0, 3), name=f"{m}.branch7x7_2.conv")
        b7 = C(b7, 192, (7, 1), 1, (3, 0), name=f"{m}.branch7x7_3.conv")
        bd = C(x, c7, 1, name=f"{m}.branch7x7dbl_1.conv")
        bd = C(bd, c7, (7, 1), 1, (3, 0), name=f"{m}.branch7x7dbl_2.conv")
        bd = C(bd, c7, (1, 7), 1, (0, 3), name=f"{m}.branch7x7dbl_3.conv")
        bd = C(bd, c7, (7, 1), 1, (3, 0), name=f"{m}.branch7x7dbl_4.conv")
        bd = C(bd, 192, (1, 7), 1, (0, 3), name=f"{m}.branch7x7dbl_5.conv")
        bp = g.avgpool(x, 3, 1, 1, name=f"{m}.avgpool")
        bp = C(bp, 192, 1, name=f"{m}.branch_pool.conv")
        return g.concat([b1, b7, bd, bp], name=f"{m}.cat")

    def inc_d(x, m):
        b3 = C(x, 192, 1, name=f"{m}.branch3x3_1.conv")
        b3 = C(b3, 320, 3, 2, 0, name=f"{m}.branch3x3_2.conv")
        b7 = C(x, 192, 1, name=f"{m}.branch7x7x3_1.conv")
        b7 = C(b7, 192, (1, 7), 1, (0, 3), name=f"{m}.branch7x7x3_2.conv")
        b7 = C(b7, 192, (7, 1), 1, (3, 0), name=f"{m}.branch7x7x3_3.conv")
        b7 = C(b7, 192, 3, 2, 0, name=f"{m}.branch7x7x3_4.conv")
        bp = g.maxpool(x, 3, 2, 0, name=f"{m}.maxpool")
        return g.concat([b3, b7, bp], name=f"{m}.cat")

    def inc_e(x, m):
        b1 = C(x, 320, 1, name=f"{m}.branch1x1.conv")
        b3 = C(x, 384, 1, name=f"{m}.branch3x3_1.conv")
        b3a = C(b3, 384, (1, 3), 1, (0, 1), name=f"{m}.branch3x3_2a.conv")
        b3b = C(b3, 384, (3, 1), 1, (1, 0), name=f"{m}.branch3x3_2b.conv")
        bd = C(x, 448, 1, name=f"{m}.branch3x3dbl_1.conv")
        bd = C(bd, 384, 3, 1, 1, name=f"{m}.branch3x3dbl_2.conv")
        bda = C(bd, 384, (1, 3), 1, (0, 1), name=f"{m}.branch3x3dbl_3a.conv")
        bdb = C(bd, 384, (3, 1), 1, (1, 0), name=f"{m}.branch3x3dbl_3b.conv")
        bp = g.avgpool(x, 3, 1, 1, name=f"{m}.avgpool")
        bp = C(bp, 192, 1, name=f"{m}.branch_pool.conv")
        return g.concat([b1, b3a, b3b, bda, bdb, bp], name=f"{m}.cat")

    x = inc_a(x, "Mixed_5b", 32)
    x = inc_a(x, "Mixed_5c", 64)
    x = inc_a(x, "Mixed_5d", 64)
    x = inc_b(x, "Mixed_6a")
    x = inc_c(x, "Mixed_6b", 128)
    x = inc_c(x, "Mixed_6c", 160)
    x = inc_c(x, "Mixed_6d", 160)
    x = inc_c(x, "Mixed_6e", 192)
    x = inc_d(x, "Mixed_7a")
    x = inc_e(x, "Mixed_7b")
    x = inc_e(x, "Mixed_7c")
    x = g.gap(x, name="avgpool")
    g.fc(x, 1000, name="fc")
    return g


MODELS = {
    "toy": toy,
    "resnet18": resnet18,
    "resnet34": resnet34,
    "resnet50": resnet50,
    "mobilenet_v2": mobilenet_v2,
    "squeezenet1_1": squeezenet1_1,
    "densenet121": densenet121,
    "inception_v3": inception_v3,
}

#: seed offset per model ("model weights seed 0 (+ model index)")
MODEL_INDEX = {name: i for i, name in enumerate(MODELS)}


def build(name):
    return MODELS[name]()
