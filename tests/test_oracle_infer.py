"""Pins for oracle C1 (float64 inference) -- SURVEY.md §8(c) P-inf-1..3.

P-inf-1: torchvision's own model definitions, float64 CPU, with the same synthetic
parameters (BN set to the identity-plus-bias that the folded weights stand for)
must equal the numpy oracle to 1e-9 relative.  This also pins the shared layer
lists in workload/archs.py (a wrong stride/pad/branch order fails it).
P-inf-2: direct nested-loop conv / pool on tiny tensors for every variant used.
P-inf-3: closed forms.
"""
import itertools

import numpy as np
import pytest
import torch

from oracle import infer
from oracle.bf16 import round_bf16
from workload import archs, rng

torch.set_default_dtype(torch.float64)


def _tv_model(name):
    import torchvision.models as tvm
    if name == "inception_v3":
        return tvm.inception_v3(weights=None, aux_logits=False, transform_input=False, init_weights=False)
    return getattr(tvm, name)(weights=None)


def _load_into_torchvision(g, params, m):
    mods = dict(m.named_modules())
    order = [k for k, _ in m.named_modules()]
    used = set()
    for n in g.nodes:
        if n["op"] == "conv" or n["op"] == "fc":
            mod = mods[n["name"]]
            w = torch.from_numpy(params[n["name"] + ".weight"].astype(np.float64))
            b = torch.from_numpy(params[n["name"] + ".bias"].astype(np.float64))
            with torch.no_grad():
                mod.weight.copy_(w.reshape(mod.weight.shape))
                if mod.bias is not None:
                    mod.bias.copy_(b)
                elif n["op"] == "conv" and n["bias"]:
                    # the BN right after this conv is the folded one
                    nxt = order[order.index(n["name"]) + 1]
                    bn = mods[nxt]
                    assert isinstance(bn, torch.nn.BatchNorm2d), (n["name"], nxt)
                    bn.weight.fill_(1.0)
                    bn.bias.copy_(b)
                    bn.running_mean.zero_()
                    bn.running_var.fill_(1.0 - bn.eps)
                    used.add(nxt)
                else:
                    assert not np.any(params[n["name"] + ".bias"])
        if n.get("prologue"):
            nm = n["name"]
            if nm.endswith(".conv1"):
                bnname = nm[:-len(".conv1")] + ".norm1"
            elif nm.endswith(".conv"):
                bnname = nm[:-len(".conv")] + ".norm"
            else:
                bnname = nm
            bn = mods[bnname]
            with torch.no_grad():
                bn.weight.copy_(torch.from_numpy(params[nm + ".pro_scale"].astype(np.float64)))
                bn.bias.copy_(torch.from_numpy(params[nm + ".pro_shift"].astype(np.float64)))
                bn.running_mean.zero_()
                bn.running_var.fill_(1.0 - bn.eps)
            used.add(bnname)
    bns = [k for k, v in mods.items() if isinstance(v, torch.nn.BatchNorm2d)]
    assert set(bns) == used, set(bns) ^ used


@pytest.mark.parametrize("name", ["resnet18", "mobilenet_v2", "squeezenet1_1", "resnet50",
                                  "densenet121", "inception_v3", "resnet34"])
def test_pin_torchvision_float64(name):
    g = archs.build(name)
    params = rng.model_params(g)
    m = _tv_model(name).double().eval()
    _load_into_torchvision(g, params, m)
    x = round_bf16(rng.image(g, 0))
    with torch.no_grad():
        ref = m(torch.from_numpy(x.astype(np.float64))).numpy().reshape(-1)
    out = infer.forward(g, params, x, dtype="fp32")
    np.testing.assert_allclose(out, ref, rtol=1e-9, atol=1e-9 * np.abs(ref).max())
    # LSUV makes logits O(1) ("logits std ~ 1.0")
    assert 0.2 < np.std(out) < 5.0


def test_toy_against_torch():
    g = archs.toy()
    params = rng.model_params(g)
    x = rng.image(g, 3)
    t = torch.from_numpy(x.astype(np.float64))
    P = {k: torch.from_numpy(v.astype(np.float64)) for k, v in params.items()}
    y = torch.relu(torch.nn.functional.conv2d(t, P["conv1.weight"], P["conv1.bias"], 1, 1))
    y = torch.nn.functional.max_pool2d(y, 2, 2).flatten()
    y = torch.relu(P["fc1.weight"] @ y + P["fc1.bias"])
    y = P["fc2.weight"] @ y + P["fc2.bias"]
    np.testing.assert_allclose(infer.forward(g, params, x, dtype="fp32"), y.numpy(), rtol=1e-12, atol=1e-12)
    assert sum(int(np.prod(v.shape)) for v in params.values()) == 448 + 524416 + 1290


# --- P-inf-2: brute force -----------------------------------------------------

def _direct_conv(x, w, b, s, p, groups):
    c, h, wd = x.shape
    co, cig, kh, kw = w.shape
    oh = (h + 2 * p[0] - kh) // s[0] + 1
    ow = (wd + 2 * p[1] - kw) // s[1] + 1
    y = np.zeros((co, oh, ow))
    cog = co // groups
    for o in range(co):
        gi = o // cog
        for i, j in itertools.product(range(oh), range(ow)):
            acc = b[o]
            for ci in range(cig):
                for a in range(kh):
                    for bb in range(kw):
                        hi = i * s[0] + a - p[0]
                        wi = j * s[1] + bb - p[1]
                        if 0 <= hi < h and 0 <= wi < wd:
                            acc += w[o, ci, a, bb] * x[gi * cig + ci, hi, wi]
            y[o, i, j] = acc
    return y


CONV_VARIANTS = [((7, 7), (2, 2), (3, 3), 1), ((3, 3), (1, 1), (1, 1), 1), ((3, 3), (2, 2), (1, 1), 1),
                 ((3, 3), (2, 2), (0, 0), 1), ((3, 3), (1, 1), (0, 0), 1), ((1, 1), (1, 1), (0, 0), 1),
                 ((1, 1), (2, 2), (0, 0), 1), ((5, 5), (1, 1), (2, 2), 1), ((1, 7), (1, 1), (0, 3), 1),
                 ((7, 1), (1, 1), (3, 0), 1), ((1, 3), (1, 1), (0, 1), 1), ((3, 1), (1, 1), (1, 0), 1),
                 ((3, 3), (1, 1), (1, 1), 4), ((3, 3), (2, 2), (1, 1), 4), ((3, 3), (1, 1), (1, 1), 2)]


@pytest.mark.parametrize("k,s,p,groups", CONV_VARIANTS)
def test_conv_brute_force(k, s, p, groups):
    r = np.random.default_rng(7)
    cin, cout = 4, 4 if groups > 1 else 3
    x = r.standard_normal((cin, 9, 8))
    w = r.standard_normal((cout, cin // groups) + k)
    b = r.standard_normal(cout)
    np.testing.assert_allclose(infer.conv2d(x, w, b, s, p, groups), _direct_conv(x, w, b, s, p, groups),
                               rtol=1e-12, atol=1e-12)


def _direct_pool(x, k, s, p, kind, ceil=False):
    c, h, w = x.shape
    oh, ow = infer.pool_out(h, k, s, p, ceil), infer.pool_out(w, k, s, p, ceil)
    y = np.zeros((c, oh, ow))
    for ch, i, j in itertools.product(range(c), range(oh), range(ow)):
        vals = []
        for a, bb in itertools.product(range(k), range(k)):
            hi, wi = i * s + a - p, j * s + bb - p
            inside = 0 <= hi < h and 0 <= wi < w
            vals.append(x[ch, hi, wi] if inside else (-np.inf if kind == "max" else 0.0))
        y[ch, i, j] = max(vals) if kind == "max" else sum(vals) / (k * k)
    return y


@pytest.mark.parametrize("k,s,p,ceil", [(3, 2, 1, False), (3, 2, 0, False), (3, 2, 0, True), (2, 2, 0, False)])
@pytest.mark.parametrize("h", [7, 8, 10, 11])
def test_maxpool_brute_force(k, s, p, ceil, h):
    x = np.random.default_rng(h).standard_normal((3, h, h + 1))
    np.testing.assert_array_equal(infer.maxpool2d(x, k, s, p, ceil), _direct_pool(x, k, s, p, "max", ceil))
    t = torch.nn.functional.max_pool2d(torch.from_numpy(x)[None], k, s, p, ceil_mode=ceil)[0].numpy()
    np.testing.assert_array_equal(infer.maxpool2d(x, k, s, p, ceil), t)


@pytest.mark.parametrize("k,s,p", [(3, 1, 1), (2, 2, 0)])
def test_avgpool_brute_force(k, s, p):
    x = np.random.default_rng(1).standard_normal((3, 9, 7))
    np.testing.assert_allclose(infer.avgpool2d(x, k, s, p), _direct_pool(x, k, s, p, "avg"), rtol=1e-12)


def test_squeezenet_ceil_sizes():
    # ceil_mode happens not to change SqueezeNet sizes: 111->55->27->13
    assert [infer.pool_out(n, 3, 2, 0, True) for n in (111, 55, 27)] == [55, 27, 13]
    assert infer.pool_out(6, 3, 2, 0, True) == 3 and infer.pool_out(6, 3, 2, 0, False) == 2


# --- P-inf-3: closed forms ----------------------------------------------------

def test_onehot_kernel_is_shift():
    x = np.random.default_rng(2).standard_normal((2, 6, 6))
    w = np.zeros((2, 2, 3, 3))
    w[0, 0, 0, 2] = 1.0   # y0[i,j] = x0[i-1, j+1]
    w[1, 1, 1, 1] = 1.0   # identity
    y = infer.conv2d(x, w, np.zeros(2), (1, 1), (1, 1))
    np.testing.assert_array_equal(y[1], x[1])
    np.testing.assert_array_equal(y[0, 1:, :-1], x[0, :-1, 1:])
    assert np.all(y[0, 0, :] == 0) and np.all(y[0, :, -1] == 0)


def test_avgpool_count_include_pad_constant():
    c = 2.5
    y = infer.avgpool2d(np.full((1, 5, 5), c), 3, 1, 1)
    assert y[0, 0, 0] == pytest.approx(c * 4 / 9) and y[0, 0, 2] == pytest.approx(c * 6 / 9)
    assert y[0, 2, 2] == pytest.approx(c)


def test_fc_identity_relu6_gap_ramp():
    x = np.arange(12.0).reshape(12, 1, 1) - 3
    np.testing.assert_array_equal(infer.fc(x, np.eye(12), np.zeros(12)), x.reshape(-1))
    np.testing.assert_array_equal(infer.act(np.array([-1.0, 3.0, 6.0, 9.0]), "relu6"), [0, 3, 6, 6])
    ramp = np.arange(20.0).reshape(1, 4, 5)
    assert infer.gap(ramp)[0, 0, 0] == pytest.approx(9.5)


def test_lsuv_unit_std():
    g = archs.resnet18()
    P = rng.model_params(g)
    vals = infer.forward(g, P, rng.calibration_input(g).astype(np.float32), dtype="fp32", return_all=True)
    # the first conv's output (pre-activation) is ~unit std on the calibration input;
    # after its ReLU the std is below 1 and strictly positive
    first = g.weight_nodes()[0]["id"]
    assert 0.3 < np.std(vals[first]) < 1.0
