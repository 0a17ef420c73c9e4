"""C4: ResNet-50 v1.5 inference-shaped program (BASELINE.json configs[3]).

Input format only: mini-SASS kernels and a launch schedule with the shape of
ResNet-50 v1.5 inference at batch 1 — conv1 7x7/2 + maxpool 3x3/2, 16
bottlenecks (3-4-6-3; stride on the 3x3, v1.5), 4 downsample 1x1 convs, 16
residual add+ReLU kernels, global average pool, FC 2048 -> 1000: 53 + 16 + 3 =
72 launches.  Direct convolution, 4 output channels per thread (one LDG of the
input pixel and one LDG.128 of 4 weights per tap, 4 FFMAs), BN folded into the
weights and bias, ReLU as FMNMX with +0.  Activations are CHW with a zero
border as wide as the consumer's padding (SSA buffers start zeroed, so the
border is free), weights [Cin][kh][kw][Cout].  Thread -> (channel group, row,
column) uses multiply-high division by constants, as compilers emit it.

`width` scales every channel count (64 at full size), `hw` the input side (224).
Weights He-uniform-like: exact f32 grid values scaled by a power of two near
sqrt(6 / fan_in).
"""
from __future__ import annotations

import math

import numpy as np

from . import isa
from .isa import Asm, RZ
from .program import ProgramBuilder, Program, ptr_words, f32_data

C4_DATA_SEED = 0xD0000004
C4_CAMPAIGN_SEED = 0xC0000004
ONE = 31                                    # register holding 1 (pointer bumps)


def magic(d: int, n_max: int) -> tuple[int, int]:
    """(M, s) with floor(n / d) == (n * M) >> (32 + s) for 0 <= n < n_max, checked."""
    if d & (d - 1) == 0:
        return 0, d.bit_length() - 1                   # power of two: plain shift (M = 0 flags it)
    for s in range(0, 32):
        M = -(-(1 << (32 + s)) // d)
        if M >= 1 << 32:
            break
        n = np.arange(n_max, dtype=np.uint64)
        if np.array_equal((n * np.uint64(M)) >> np.uint64(32 + s), n // np.uint64(d)):
            return M, s
    raise ValueError(f"no magic number for d={d}")


def _divmod(s: Asm, q: int, r: int, n: int, d: int, n_max: int, tmp: int):
    """q = n / d, r = n % d (registers; tmp, tmp+1 scratch)."""
    M, sh = magic(d, n_max)
    if M == 0:
        s.shf(q, n, imm=sh, mode=isa.SHF_R_U32)
    else:
        s.imad_wide(tmp, n, imm=M, c=RZ, unsigned=True)
        s.shf(q, tmp + 1, imm=sh, mode=isa.SHF_R_U32)
    s.imad(r, q, imm=(-d) & 0xFFFFFFFF, c=n)


def conv_code(kh, kw, stride, Hp_in, Wp_in, Cout, Hout, Wout, Hp_out, Wp_out, pad_out, relu, total) -> np.ndarray:
    """cbank: in(0) w(8) bias(16) out(24) Cin(32)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)                                 # t
    s.isetp(0, 0, imm=total, cmp=isa.GE, unsigned=True)
    s.exit(guard=0)
    _divmod(s, 3, 13, 0, Wout, total, 28)              # R3 = t / W, R13 = x
    _divmod(s, 15, 14, 3, Hout, total // Wout + 1, 28)  # R15 = cog, R14 = y
    s.mov(ONE, imm=1)
    s.imad(1, 14, imm=stride * Wp_in, c=RZ)
    s.imad(1, 13, imm=stride, c=1)                     # receptive-field origin (padded coords)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 1, imm=4, c=4, unsigned=True)       # input pointer
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 15, imm=16, c=6, unsigned=True)     # weight pointer (4 channels)
    for a in range(4):
        s.mov(8 + a, imm=0)
    s.ldc(12, 32)                                      # Cin
    s.label("ci")
    for ky in range(kh):
        for kx in range(kw):
            s.ldg(16, 4, off=4 * (ky * Wp_in + kx))
            s.ldg(20, 6, off=4 * (ky * kw + kx) * Cout, width=isa.W128)
            for a in range(4):
                s.ffma(8 + a, 16, 20 + a, 8 + a)
    s.imad_wide(4, ONE, imm=4 * Hp_in * Wp_in, c=4, unsigned=True)
    s.imad_wide(6, ONE, imm=4 * kh * kw * Cout, c=6, unsigned=True)
    s.iadd3(12, 12, imm=0xFFFFFFFF)
    s.isetp(0, 12, imm=0, cmp=isa.GT)
    s.bra("ci", guard=0)
    s.ldc(26, 16, wide=True)
    s.imad_wide(26, 15, imm=16, c=26, unsigned=True)
    s.ldg(20, 26, width=isa.W128)                      # folded-BN bias
    for a in range(4):
        s.fadd(8 + a, 8 + a, 20 + a)
        if relu:
            s.fmnmx(8 + a, 8 + a, RZ, is_max=True)
    s.imad(2, 15, imm=4 * Hp_out, c=14)
    s.iadd3(2, 2, imm=pad_out)
    s.imad(2, 2, imm=Wp_out, c=13)
    s.iadd3(2, 2, imm=pad_out)
    s.ldc(24, 24, wide=True)
    s.imad_wide(24, 2, imm=4, c=24, unsigned=True)
    for a in range(4):
        s.stg(24, 8 + a, off=4 * a * Hp_out * Wp_out)
    s.exit()
    return s.assemble()


def add_relu_code(total) -> np.ndarray:
    """out = max(a + b, +0) elementwise; cbank: a(0) b(8) out(16)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.isetp(0, 0, imm=total, cmp=isa.GE, unsigned=True)
    s.exit(guard=0)
    for i, off in enumerate((0, 8, 16)):
        s.ldc(4 + 2 * i, off, wide=True)
        s.imad_wide(4 + 2 * i, 0, imm=4, c=4 + 2 * i, unsigned=True)
    s.ldg(10, 4)
    s.ldg(11, 6)
    s.fadd(10, 10, 11)
    s.fmnmx(10, 10, RZ, is_max=True)
    s.stg(8, 10)
    s.exit()
    return s.assemble()


def maxpool_code(C, Hp_in, Wp_in, Hout, Wout, total) -> np.ndarray:
    """3x3 / 2 over a zero-bordered ReLU output (max with +0 padding == -inf padding
    for inputs >= 0); cbank: in(0) out(8)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.isetp(0, 0, imm=total, cmp=isa.GE, unsigned=True)
    s.exit(guard=0)
    _divmod(s, 3, 13, 0, Wout, total, 28)
    _divmod(s, 15, 14, 3, Hout, total // Wout + 1, 28)   # R15 = c
    s.imad(1, 15, imm=Hp_in, c=RZ)
    s.imad(1, 14, imm=2, c=1)
    s.imad(1, 1, imm=Wp_in, c=RZ)
    s.imad(1, 13, imm=2, c=1)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 1, imm=4, c=4, unsigned=True)
    s.ldg(8, 4)
    for ky in range(3):
        for kx in range(3):
            if ky or kx:
                s.ldg(9, 4, off=4 * (ky * Wp_in + kx))
                s.fmnmx(8, 8, 9, is_max=True)
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 0, imm=4, c=6, unsigned=True)
    s.stg(6, 8)
    s.exit()
    return s.assemble()


def avgpool_code(C, HW, scale_bits) -> np.ndarray:
    """out[c] = (sum of the HW values of channel c, in order) * (1/HW); cbank: in(0) out(8)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.isetp(0, 0, imm=C, cmp=isa.GE, unsigned=True)
    s.exit(guard=0)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 0, imm=4 * HW, c=4, unsigned=True)
    s.mov(8, imm=0)
    for i in range(HW):
        s.ldg(9, 4, off=4 * i)
        s.fadd(8, 8, 9)
    s.mov(10, imm=scale_bits)
    s.fmul(8, 8, 10)
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 0, imm=4, c=6, unsigned=True)
    s.stg(6, 8)
    s.exit()
    return s.assemble()


def fc_code(K, N) -> np.ndarray:
    """logits[o] = bias[o] + sum_k x[k] * w[k][o] (k ascending); cbank: x(0) w(8) bias(16) out(24)."""
    assert K % 4 == 0
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.isetp(0, 0, imm=N, cmp=isa.GE, unsigned=True)
    s.exit(guard=0)
    s.mov(ONE, imm=1)
    s.ldc(4, 0, wide=True)                            # x
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 0, imm=4, c=6, unsigned=True)      # w column o
    s.ldc(26, 16, wide=True)
    s.imad_wide(26, 0, imm=4, c=26, unsigned=True)
    s.ldg(8, 26)                                      # acc = bias[o]
    s.mov(12, imm=K // 4)
    s.label("k")
    s.ldg(16, 4, width=isa.W128)                      # x[k..k+3]
    for a in range(4):
        s.ldg(20 + a, 6, off=4 * N * a)
    for a in range(4):
        s.ffma(8, 16 + a, 20 + a, 8)
    s.imad_wide(4, ONE, imm=16, c=4, unsigned=True)
    s.imad_wide(6, ONE, imm=16 * N, c=6, unsigned=True)
    s.iadd3(12, 12, imm=0xFFFFFFFF)
    s.isetp(0, 12, imm=0, cmp=isa.GT)
    s.bra("k", guard=0)
    s.ldc(24, 24, wide=True)
    s.imad_wide(24, 0, imm=4, c=24, unsigned=True)
    s.stg(24, 8)
    s.exit()
    return s.assemble()


class _Net:
    def __init__(self, width: int, hw: int, seed: int):
        self.pb = ProgramBuilder(f"resnet50_w{width}_hw{hw}")
        self.rng_seed = seed
        self.kern = {}
        self.n_inst = 0
        self.layers = []                              # (name, kind, meta) for the numpy pin

    def kernel(self, key, maker):
        if key not in self.kern:
            self.kern[key] = self.pb.add_kernel(f"{key[0]}_{len(self.kern)}", maker(), nregs=40)
        return self.kern[key]

    def data(self, n, scale_exp):
        self.rng_seed += 1
        return (f32_data(self.rng_seed, n) * np.float32(2.0 ** scale_exp)).astype(np.float32)

    def act(self, name, C, H, W, pad, output=False):
        Hp, Wp = H + 2 * pad, W + 2 * pad
        va = self.pb.add_buffer(name, 4 * C * Hp * Wp, writer=self.n_inst, output=output, dtype=isa.DT_F32)
        return dict(name=name, va=va, C=C, H=H, W=W, pad=pad, Hp=Hp, Wp=Wp)

    def conv(self, name, x, Cout, k, stride, relu, pad_out):
        assert x["pad"] == k // 2 and Cout % 4 == 0
        Hout = (x["H"] + 2 * (k // 2) - k) // stride + 1
        Wout = (x["W"] + 2 * (k // 2) - k) // stride + 1
        fan_in = x["C"] * k * k
        w = self.data(x["C"] * k * k * Cout, round(math.log2(math.sqrt(6.0 / fan_in))))
        b = self.data(Cout, -4)
        wva = self.pb.add_buffer(name + ".w", 4 * w.size, w, dtype=isa.DT_F32)
        bva = self.pb.add_buffer(name + ".b", 4 * b.size, b, dtype=isa.DT_F32)
        y = self.act(name, Cout, Hout, Wout, pad_out)
        total = Cout // 4 * Hout * Wout
        kid = self.kernel(("conv", k, stride, x["Hp"], x["Wp"], Cout, Hout, Wout, y["Hp"], y["Wp"], pad_out, relu),
                          lambda: conv_code(k, k, stride, x["Hp"], x["Wp"], Cout, Hout, Wout, y["Hp"], y["Wp"],
                                            pad_out, relu, total))
        self.pb.add_instance(kid, (total + 255) // 256, 256,
                             ptr_words(x["va"]) + ptr_words(wva) + ptr_words(bva) + ptr_words(y["va"]) + [x["C"]])
        self.n_inst += 1
        self.layers.append((name, "conv", dict(x=x["name"], y=name, k=k, stride=stride, relu=relu)))
        return y

    def add_relu(self, name, a, b):
        assert a["pad"] == 0 and b["pad"] == 0 and (a["C"], a["H"]) == (b["C"], b["H"])
        y = self.act(name, a["C"], a["H"], a["W"], 0)
        total = a["C"] * a["H"] * a["W"]
        kid = self.kernel(("add", total), lambda: add_relu_code(total))
        self.pb.add_instance(kid, (total + 255) // 256, 256, ptr_words(a["va"]) + ptr_words(b["va"]) + ptr_words(y["va"]))
        self.n_inst += 1
        self.layers.append((name, "add", dict(a=a["name"], b=b["name"])))
        return y


def resnet50(width: int = 64, hw: int = 224, seed: int = C4_DATA_SEED) -> Program:
    """ResNet-50 v1.5 inference at batch 1; width 64 / hw 224 is C4."""
    net = _Net(width, hw, seed)
    pb = net.pb
    img = net.data(3 * (hw + 6) * (hw + 6), 0).reshape(3, hw + 6, hw + 6)
    img[:, :3, :] = 0
    img[:, -3:, :] = 0
    img[:, :, :3] = 0
    img[:, :, -3:] = 0
    x = dict(name="image", va=pb.add_buffer("image", img.nbytes, img, dtype=isa.DT_F32), C=3, H=hw, W=hw, pad=3,
             Hp=hw + 6, Wp=hw + 6)
    c1 = net.conv("conv1", x, width, 7, 2, True, 1)
    H, W = c1["H"] // 2, c1["W"] // 2
    p = net.act("maxpool", width, H, W, 0)
    total = width * H * W
    kid = net.kernel(("maxpool", width, H), lambda: maxpool_code(width, c1["Hp"], c1["Wp"], H, W, total))
    pb.add_instance(kid, (total + 255) // 256, 256, ptr_words(c1["va"]) + ptr_words(p["va"]))
    net.n_inst += 1
    net.layers.append(("maxpool", "maxpool", dict(x="conv1")))
    x = p
    for li, (blocks, mid, stride) in enumerate([(3, width, 1), (4, 2 * width, 2), (6, 4 * width, 2),
                                                (3, 8 * width, 2)]):
        out_c = 4 * mid
        for bi in range(blocks):
            s = stride if bi == 0 else 1
            nm = f"l{li + 1}b{bi}"
            a = net.conv(nm + ".a", x, mid, 1, 1, True, 1)
            b = net.conv(nm + ".b", a, mid, 3, s, True, 0)
            c = net.conv(nm + ".c", b, out_c, 1, 1, False, 0)
            sc = net.conv(nm + ".down", x, out_c, 1, s, False, 0) if bi == 0 else x
            x = net.add_relu(nm + ".out", c, sc)
    C, HW = x["C"], x["H"] * x["W"]
    g = pb.add_buffer("avgpool", 4 * C, writer=net.n_inst, dtype=isa.DT_F32)
    kid = net.kernel(("avgpool", C, HW), lambda: avgpool_code(C, HW, isa.f32_bits(np.float32(1.0) / np.float32(HW))))
    pb.add_instance(kid, (C + 255) // 256, 256, ptr_words(x["va"]) + ptr_words(g))
    net.n_inst += 1
    net.layers.append(("avgpool", "avgpool", dict(x=x["name"])))
    wfc = net.data(C * 1000, round(math.log2(math.sqrt(6.0 / C))))
    bfc = net.data(1000, -4)
    wva = pb.add_buffer("fc.w", 4 * wfc.size, wfc, dtype=isa.DT_F32)
    bva = pb.add_buffer("fc.b", 4 * bfc.size, bfc, dtype=isa.DT_F32)
    out = pb.add_buffer("logits", 4 * 1000, writer=net.n_inst, output=True, dtype=isa.DT_F32)
    kid = net.kernel(("fc", C), lambda: fc_code(C, 1000))
    pb.add_instance(kid, (1000 + 255) // 256, 256, ptr_words(g) + ptr_words(wva) + ptr_words(bva) + ptr_words(out))
    net.n_inst += 1
    net.layers.append(("fc", "fc", dict(x="avgpool")))
    prog = pb.build(config="C4", width=width, hw=hw)
    prog.meta["layers"] = net.layers
    return prog


def c4(full: bool = True) -> Program:
    """C4 (full: width 64, 224x224); mini-C4 for parity: width 8, 32x32."""
    return resnet50() if full else resnet50(width=8, hw=32)
