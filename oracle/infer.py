"""ORACLE (test infrastructure) -- C1: float64 inference, the plain definition.

SURVEY.md §8(c) C1 gives the operator definitions this file writes out; the paper
itself (PAPER.md P1268-1281, Table 2) only names the models.  Every tensor is
float64 NCHW with batch 1; every function is a direct restatement of the
definition with at most one library primitive (a matmul) per step.

    conv2d   y[co,oh,ow] = b[co] + sum_{ci in grp(co),kh,kw} W[co,ci',kh,kw] *
                           x[ci, oh*s_h+kh-p_h, ow*s_w+kw-p_w]      (zero padding)
    maxpool  max over the window, padding = -inf, PyTorch ceil_mode rule
    avgpool  sum over the window / (k*k)   (count_include_pad=True)
    gap      mean over H*W
    fc       y = W x + b
    act      relu = max(x,0); relu6 = min(max(x,0),6)
    prologue (DenseNet pre-activation BN+ReLU): relu(scale[c]*x[c] + shift[c])
    residual added after bias, before the activation (torchvision order)
    concat   along channels, in input order

The output is the logits (no softmax).  Pinned by tests/test_oracle_infer.py
against torchvision's float64 CPU forward (P-inf-1), a direct nested-loop conv/pool
(P-inf-2) and closed forms (P-inf-3).
"""
from __future__ import annotations

import numpy as np
from numpy.lib.stride_tricks import as_strided

from .bf16 import round_bf16


def act(x, kind):
    if kind == "none":
        return x
    if kind == "relu":
        return np.maximum(x, 0.0)
    if kind == "relu6":
        return np.minimum(np.maximum(x, 0.0), 6.0)
    raise ValueError(kind)


def _windows(xp, kh, kw, sh, sw, oh, ow):
    """View (C, kh, kw, oh, ow) of the padded input xp (C, Hp, Wp)."""
    c = xp.shape[0]
    s0, s1, s2 = xp.strides
    return as_strided(xp, shape=(c, kh, kw, oh, ow), strides=(s0, s1, s2, s1 * sh, s2 * sw),
                      writeable=False)


def conv2d(x, w, b, stride, pad, groups=1):
    """x (C,H,W), w (Co, C/g, kh, kw), b (Co,) -> (Co, OH, OW).  Cross-correlation."""
    c, h, wd = x.shape
    co, cig, kh, kw = w.shape
    sh, sw = stride
    ph, pw = pad
    oh = (h + 2 * ph - kh) // sh + 1
    ow = (wd + 2 * pw - kw) // sw + 1
    xp = np.zeros((c, h + 2 * ph, wd + 2 * pw))
    xp[:, ph:ph + h, pw:pw + wd] = x
    win = _windows(xp, kh, kw, sh, sw, oh, ow)            # (C, kh, kw, oh, ow)
    cog = co // groups
    # im2col per group: (g, cig*kh*kw, oh*ow); weights (g, cog, cig*kh*kw)
    cols = win.reshape(groups, cig * kh * kw, oh * ow)
    wm = w.reshape(groups, cog, cig * kh * kw)
    y = np.matmul(wm, cols).reshape(co, oh, ow)
    return y + b[:, None, None]


def pool_out(n, k, s, p, ceil):
    if not ceil:
        return (n + 2 * p - k) // s + 1
    o = -(-(n + 2 * p - k) // s) + 1
    if (o - 1) * s >= n + p:   # last window must start inside input or left padding
        o -= 1
    return o


def maxpool2d(x, k, s, p, ceil=False):
    c, h, w = x.shape
    oh, ow = pool_out(h, k, s, p, ceil), pool_out(w, k, s, p, ceil)
    # pad right enough for ceil-mode windows that run past the input
    hp = max(h + 2 * p, (oh - 1) * s + k)
    wp = max(w + 2 * p, (ow - 1) * s + k)
    xp = np.full((c, hp, wp), -np.inf)
    xp[:, p:p + h, p:p + w] = x
    return _windows(xp, k, k, s, s, oh, ow).max(axis=(1, 2))


def avgpool2d(x, k, s, p):
    """count_include_pad=True: divisor is always k*k."""
    c, h, w = x.shape
    oh, ow = pool_out(h, k, s, p, False), pool_out(w, k, s, p, False)
    xp = np.zeros((c, h + 2 * p, w + 2 * p))
    xp[:, p:p + h, p:p + w] = x
    return _windows(xp, k, k, s, s, oh, ow).sum(axis=(1, 2)) / (k * k)


def gap(x):
    return x.mean(axis=(1, 2), keepdims=True)


def fc(x, w, b):
    return w @ x.reshape(-1) + b


def prologue(x, scale, shift):
    return np.maximum(scale[:, None, None] * x + shift[:, None, None], 0.0)


def forward(g, params, image, dtype="bf16", return_all=False):
    """Run graph ``g`` (workload.archs.Graph) in float64.

    image: fp32 NCHW (1,C,H,W) as the client supplies it.  dtype='bf16' applies the
    ingest RNE rounding to the input (reading C1-Q7); 'fp32' uses it as is.
    Returns the logits (num_classes,) float64, or every node's value if return_all.
    """
    x0 = np.asarray(image, dtype=np.float32)[0]
    if dtype == "bf16":
        x0 = round_bf16(x0)
    vals = {}
    P = {k: np.asarray(v, dtype=np.float64) for k, v in params.items()}
    for n in g.nodes:
        op = n["op"]
        ins = [vals[i] for i in n["inputs"]]
        if op == "input":
            y = x0.astype(np.float64)
        elif op == "conv":
            x = ins[0]
            if n["prologue"]:
                x = prologue(x, P[n["name"] + ".pro_scale"], P[n["name"] + ".pro_shift"])
            y = conv2d(x, P[n["name"] + ".weight"], P[n["name"] + ".bias"],
                       (n["sh"], n["sw"]), (n["ph"], n["pw"]), n["groups"])
            if n["residual"] is not None:
                y = y + vals[n["residual"]]
            y = act(y, n["act"])
        elif op == "maxpool":
            y = maxpool2d(ins[0], n["k"], n["s"], n["p"], n["ceil"])
        elif op == "avgpool":
            y = avgpool2d(ins[0], n["k"], n["s"], n["p"])
        elif op == "gap":
            x = ins[0]
            if n["prologue"]:
                x = prologue(x, P[n["name"] + ".pro_scale"], P[n["name"] + ".pro_shift"])
            y = gap(x)
        elif op == "fc":
            y = act(fc(ins[0], P[n["name"] + ".weight"], P[n["name"] + ".bias"]), n["act"])
            y = y.reshape(-1, 1, 1)
        elif op == "concat":
            y = np.concatenate(ins, axis=0)
        elif op == "spin":          # Fig. 2 synthetic kernel: occupies the GPU, computes nothing
            y = ins[0]
        else:
            raise ValueError(op)
        assert y.shape == n["out"], (n["name"], y.shape, n["out"])
        vals[n["id"]] = y
    if return_all:
        return vals
    return vals[g.output].reshape(-1)


def lsuv_scales(g, raw_params, calib):
    """C1 step 3 (LSUV): in execution order, divide each conv/FC's W and b by the std
    of that layer's output (after bias, before residual add and activation) on the
    calibration input, every earlier layer already rescaled.  One float64 forward in
    node order: when a weight layer is reached its output std fixes its factor, the
    layer is rescaled and the forward continues with the rescaled output.
    Returns {layer name: factor}."""
    P = {k: np.asarray(v, dtype=np.float64) for k, v in raw_params.items()}
    scales = {}
    vals = {}
    for n in g.nodes:
        op = n["op"]
        ins = [vals[i] for i in n["inputs"]]
        if op == "input":
            y = np.asarray(calib, dtype=np.float64)[0]
        elif op in ("conv", "fc"):
            x = ins[0]
            if n.get("prologue"):
                x = prologue(x, P[n["name"] + ".pro_scale"], P[n["name"] + ".pro_shift"])
            w, b = P[n["name"] + ".weight"], P[n["name"] + ".bias"]
            if op == "conv":
                pre = conv2d(x, w, b, (n["sh"], n["sw"]), (n["ph"], n["pw"]), n["groups"])
            else:
                pre = fc(x, w, b).reshape(-1, 1, 1)
            s = 1.0 / float(np.std(pre))
            scales[n["name"]] = s
            y = pre * s
            if op == "conv" and n["residual"] is not None:
                y = y + vals[n["residual"]]
            y = act(y, n["act"])
        elif op == "maxpool":
            y = maxpool2d(ins[0], n["k"], n["s"], n["p"], n["ceil"])
        elif op == "avgpool":
            y = avgpool2d(ins[0], n["k"], n["s"], n["p"])
        elif op == "gap":
            x = ins[0]
            if n["prologue"]:
                x = prologue(x, P[n["name"] + ".pro_scale"], P[n["name"] + ".pro_shift"])
            y = gap(x)
        elif op == "concat":
            y = np.concatenate(ins, axis=0)
        vals[n["id"]] = y
    return scales
