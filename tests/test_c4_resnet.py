"""Pin the oracle on the C4 (ResNet-50 v1.5 inference-shaped) program, mini size.

Layer by layer, the oracle's output of every launch is checked against numpy
float64 arithmetic applied to the oracle's own input of that launch, within the
rigorous bound of a sequential fp32 FMA accumulation of n terms:
|fl - exact| <= (n + 2) * 2^-24 * (sum |w x| + |b|) (Higham, gamma_n).  ReLU,
max-pool and the residual add are exact functions of their inputs up to one
rounding.  The shapes are ResNet-50's: 72 launches, 53 convolutions.
"""
import numpy as np
import pytest

import oracle as O
from fi_inputs import resnet as R

U = 2.0 ** -24


@pytest.fixture(scope="module")
def c4mini():
    prog = R.c4(full=False)
    g = O.Golden(prog)
    return prog, g, g.final_image()


def _act(prog, img, name):
    b = prog.buffer(name)
    return img[int(b["off"]):int(b["off"]) + int(b["size"])].view("<f4")


def test_shape_is_resnet50(c4mini):
    prog, g, _ = c4mini
    kinds = [k for _, k, _ in prog.meta["layers"]]
    assert len(prog.instances) == 72
    assert kinds.count("conv") == 53 and kinds.count("add") == 16
    assert kinds.count("maxpool") == kinds.count("avgpool") == kinds.count("fc") == 1
    c = g.counts()
    assert (c[:, 7] == c[:, 0] + c[:, 1] + c[:, 2] + c[:, 5]).all()       # Table II identities
    assert (c[:, 6] == c[:, 7] + c[:, 3]).all()


def test_layers_match_float64_within_fma_bound(c4mini):
    prog, g, img = c4mini
    shapes = {}
    # input image (zero-bordered by 3)
    b = prog.buffer("image")
    hw = prog.meta["hw"]
    shapes["image"] = (3, hw, hw, 3)
    for name, kind, m in prog.meta["layers"]:
        if kind == "conv":
            C, H, W, pad = shapes[m["x"]]
            x = _act(prog, img, m["x"]).reshape(C, H + 2 * pad, W + 2 * pad).astype(np.float64)
            k, s = m["k"], m["stride"]
            w = _act(prog, img, name + ".w").astype(np.float64)
            Cout = w.size // (C * k * k)
            w = w.reshape(C, k, k, Cout)
            bias = _act(prog, img, name + ".b").astype(np.float64)
            Ho, Wo = (H + 2 * pad - k) // s + 1, (W + 2 * pad - k) // s + 1
            acc = np.zeros((Cout, Ho, Wo))
            mag = np.zeros((Cout, Ho, Wo))
            for ky in range(k):
                for kx in range(k):
                    patch = x[:, ky:ky + s * (Ho - 1) + 1:s, kx:kx + s * (Wo - 1) + 1:s]
                    acc += np.einsum("chw,co->ohw", patch, w[:, ky, kx, :])
                    mag += np.einsum("chw,co->ohw", np.abs(patch), np.abs(w[:, ky, kx, :]))
            want = acc + bias[:, None, None]
            bound = (C * k * k + 2) * U * (mag + np.abs(bias)[:, None, None]) + 1e-30
            if m["relu"]:
                want = np.maximum(want, 0.0)
            # consumer padding of this activation: from the buffer size
            yb = _act(prog, img, name)
            pad_o = int(round((np.sqrt(yb.size / Cout) - Ho) / 2))
            y = yb.reshape(Cout, Ho + 2 * pad_o, Wo + 2 * pad_o).astype(np.float64)
            inner = y[:, pad_o:pad_o + Ho, pad_o:pad_o + Wo]
            assert (np.abs(inner - want) <= bound).all(), name
            border = y.copy()
            border[:, pad_o:pad_o + Ho, pad_o:pad_o + Wo] = 0
            assert (border == 0).all(), name
            shapes[name] = (Cout, Ho, Wo, pad_o)
        elif kind == "maxpool":
            C, H, W, pad = shapes[m["x"]]
            x = _act(prog, img, m["x"]).reshape(C, H + 2, W + 2)
            Ho, Wo = H // 2, W // 2
            want = np.max([x[:, ky:ky + 2 * Ho:2, kx:kx + 2 * Wo:2] for ky in range(3) for kx in range(3)], axis=0)
            assert np.array_equal(_act(prog, img, name).reshape(C, Ho, Wo), want)
            shapes[name] = (C, Ho, Wo, 0)
        elif kind == "add":
            C, H, W, _ = shapes[m["a"]]
            a, bb = _act(prog, img, m["a"]), _act(prog, img, m["b"])
            want = np.maximum(a + bb, np.float32(0))                    # one f32 rounding, then ReLU
            assert np.array_equal(_act(prog, img, name), want), name
            shapes[name] = (C, H, W, 0)
        elif kind == "avgpool":
            C, H, W, _ = shapes[m["x"]]
            x = _act(prog, img, m["x"]).reshape(C, H * W).astype(np.float64)
            want = x.sum(axis=1) / (H * W)
            bound = (H * W + 3) * U * np.abs(x).sum(axis=1) / (H * W) + 1e-30
            assert (np.abs(_act(prog, img, name) - want) <= bound).all()
            shapes[name] = (C, 1, 1, 0)
        elif kind == "fc":
            x = _act(prog, img, "avgpool").astype(np.float64)
            w = _act(prog, img, "fc.w").astype(np.float64).reshape(x.size, 1000)
            bias = _act(prog, img, "fc.b").astype(np.float64)
            want = x @ w + bias
            bound = (x.size + 2) * U * (np.abs(x) @ np.abs(w) + np.abs(bias))
            assert (np.abs(_act(prog, img, "logits") - want) <= bound).all()


def test_full_size_shape():
    prog = R.c4(full=True)
    assert len(prog.instances) == 72 and prog.n_warps == 265696
    conv1 = prog.buffer("conv1")
    assert int(conv1["size"]) == 4 * 64 * 114 * 114               # 64 x 112 x 112, zero border 1 for max-pool
    assert int(prog.buffer("logits")["size"]) == 4000
