"""C5: mixed HPC suite shaped after Table IV, SURVEY §8(d).

Input format only.  Five programs, each a few static kernels launched many
times with SSA buffers per step:
  stencil  3-D 7-point Jacobi, FP32, zero (Dirichlet) halo           2 static / 101 dynamic
  lbm      D3Q19 lattice Boltzmann (BGK, pull streaming, periodic), FP64   3 / 3*steps
  md       Lennard-Jones molecular dynamics, all pairs + cutoff, velocity Verlet, FP64   3 / 3*steps
  ep       embarrassingly parallel: LCG pairs, acceptance + annulus tallies, FP64 + int
  cg       the C3 conjugate-gradient generator at another size
Full sizes give ~1e9 counted thread-instructions per program; `mini` sizes are
the oracle parity cases.
"""
from __future__ import annotations

import numpy as np

from . import isa
from .isa import Asm, RZ
from .program import ProgramBuilder, Program, ptr_words, f32_data, f64_data

C5_DATA_SEED = 0xD0000005
C5_CAMPAIGN_SEED = 0xC0000005


def _tid(s: Asm, total: int):
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.isetp(0, 0, imm=total, cmp=isa.GE, unsigned=True)
    s.exit(guard=0)


# ---------------------------------------------------------------------------
# 3-D 7-point stencil (FP32): u' = c0 u + c1 (sum of the 6 neighbours); halo 0
# ---------------------------------------------------------------------------
def stencil_code(n: int) -> np.ndarray:
    """Thread per interior point of an n^3 grid stored (n+2)^3; cbank: u(0) u'(8) c0(16) c1(20)."""
    assert n & (n - 1) == 0
    lg = n.bit_length() - 1
    P = n + 2
    s = Asm()
    _tid(s, n * n * n)
    s.lop3(3, 0, RZ, RZ, 0xC0, imm=n - 1)              # x
    s.shf(4, 0, imm=lg, mode=isa.SHF_R_U32)
    s.lop3(5, 4, RZ, RZ, 0xC0, imm=n - 1)              # y
    s.shf(6, 0, imm=2 * lg, mode=isa.SHF_R_U32)        # z
    s.imad(7, 6, imm=P, c=5)                           # z*P + y   (interior offset +1 folded below)
    s.imad(7, 7, imm=P, c=3)                           # (z*P + y)*P + x
    s.iadd3(7, 7, imm=P * P + P + 1)                   # + halo
    s.ldc(8, 0, wide=True)
    s.imad_wide(8, 7, imm=4, c=8, unsigned=True)
    s.ldg(12, 8)
    for q, off in enumerate((-1, 1, -P, P, -P * P, P * P)):
        s.ldg(13 + q, 8, off=4 * off)
    s.fadd(19, 13, 14)
    s.fadd(19, 19, 15)
    s.fadd(19, 19, 16)
    s.fadd(19, 19, 17)
    s.fadd(19, 19, 18)
    s.ldc(20, 16)
    s.ldc(21, 20)
    s.fmul(12, 12, 20)
    s.ffma(12, 19, 21, 12)
    s.ldc(10, 8, wide=True)
    s.imad_wide(10, 7, imm=4, c=10, unsigned=True)
    s.stg(10, 12)
    s.exit()
    return s.assemble()


def sumsq_code(n_words: int) -> np.ndarray:
    """One CTA of 256 threads: per-thread strided sums of squares, then a SHFL
    tree and a per-warp store; cbank: u(0) out(8).  (The second static kernel.)"""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 0, imm=4, c=4, unsigned=True)
    s.mov(8, imm=0)
    s.mov(9, imm=(n_words + 255) // 256)
    s.mov(31, imm=1)
    s.mov(10, imm=0)                                   # index
    s.label("l")
    s.iadd3(11, 10, 0)                                 # i = k*256 + tid
    s.isetp(1, 11, imm=n_words, cmp=isa.LT, unsigned=True)
    s.ldg(12, 4, guard=1)
    s.ffma(8, 12, 12, 8, guard=1)
    s.imad_wide(4, 31, imm=1024, c=4, unsigned=True)
    s.iadd3(10, 10, imm=256)
    s.iadd3(9, 9, imm=0xFFFFFFFF)
    s.isetp(0, 9, imm=0, cmp=isa.GT)
    s.bra("l", guard=0)
    for sh in (16, 8, 4, 2, 1):
        s.shfl(13, 8, imm=sh, mode=isa.SHFL_BFLY)
        s.fadd(8, 8, 13)
    s.ldc(6, 8, wide=True)
    s.shf(14, 0, imm=5, mode=isa.SHF_R_U32)
    s.imad_wide(6, 14, imm=4, c=6, unsigned=True)
    s.lop3(15, 0, RZ, RZ, 0xC0, imm=31)
    s.isetp(2, 15, imm=0, cmp=isa.EQ)
    s.stg(6, 8, guard=2)
    s.exit()
    return s.assemble()


def stencil(n: int = 128, iters: int = 100, seed: int = C5_DATA_SEED) -> Program:
    P = n + 2
    pb = ProgramBuilder(f"stencil{n}_it{iters}")
    ks = pb.add_kernel("stencil7", stencil_code(n), nregs=32)
    kr = pb.add_kernel("sumsq", sumsq_code(P * P * P), nregs=32)
    u0 = np.zeros((P, P, P), dtype=np.float32)
    u0[1:-1, 1:-1, 1:-1] = f32_data(seed, n * n * n).reshape(n, n, n)
    u = pb.add_buffer("u0", 4 * P ** 3, u0, dtype=isa.DT_F32)
    c0, c1 = isa.f32_bits(0.25), isa.f32_bits(0.125)
    for it in range(iters):
        un = pb.add_buffer(f"u{it + 1}", 4 * P ** 3, writer=it, output=it == iters - 1, dtype=isa.DT_F32)
        pb.add_instance(ks, (n ** 3 + 255) // 256, 256, ptr_words(u) + ptr_words(un) + [c0, c1])
        u = un
    out = pb.add_buffer("sumsq", 4 * 8, writer=iters, output=True, dtype=isa.DT_F32)
    pb.add_instance(kr, 1, 256, ptr_words(u) + ptr_words(out))
    return pb.build(config="C5-stencil", n=n, iters=iters)


# ---------------------------------------------------------------------------
# D3Q19 lattice Boltzmann (FP64): BGK collision, pull streaming, periodic box
# ---------------------------------------------------------------------------
D3Q19 = [(0, 0, 0)] + [(1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)] + \
        [(sx, sy, 0) for sx in (1, -1) for sy in (1, -1)] + [(sx, 0, sz) for sx in (1, -1) for sz in (1, -1)] + \
        [(0, sy, sz) for sy in (1, -1) for sz in (1, -1)]
D3Q19_W = [1 / 3] + [1 / 18] * 6 + [1 / 36] * 12
FQ = 32                                                # f_q in R[FQ + 2q]


def _cell_xyz(s: Asm, n: int):
    lg = n.bit_length() - 1
    s.lop3(3, 0, RZ, RZ, 0xC0, imm=n - 1)              # x
    s.shf(4, 0, imm=lg, mode=isa.SHF_R_U32)
    s.lop3(4, 4, RZ, RZ, 0xC0, imm=n - 1)              # y
    s.shf(5, 0, imm=2 * lg, mode=isa.SHF_R_U32)        # z


def _moments(s: Asm):
    """rho -> R70, jx, jy, jz -> R72, R74, R76 from f_q."""
    s.dadd(70, FQ, FQ + 2)
    for q in range(2, 19):
        s.dadd(70, 70, FQ + 2 * q)
    for a, reg in enumerate((72, 74, 76)):
        terms = [(q, D3Q19[q][a]) for q in range(19) if D3Q19[q][a]]
        q0, c0 = terms[0]
        q1, c1 = terms[1]
        s.dadd(reg, FQ + 2 * q0, FQ + 2 * q1, nega=c0 < 0, negb=c1 < 0)
        for q, c in terms[2:]:
            s.dadd(reg, reg, FQ + 2 * q, negb=c < 0)


def lbm_collide_code(n: int) -> np.ndarray:
    """cbank: f_old(0) f_new(8) 1.0(16) 3.0(24) 4.5(32) 1.5(40) -omega(48) w0(56) w1(64) w2(72)."""
    N = n ** 3
    s = Asm()
    _tid(s, N)
    _cell_xyz(s, n)
    s.ldc(14, 0, wide=True)
    for q, (cx, cy, cz) in enumerate(D3Q19):
        # source cell x - c (periodic)
        s.iadd3(7, 3, imm=(-cx) & 0xFFFFFFFF)
        s.lop3(7, 7, RZ, RZ, 0xC0, imm=n - 1)
        s.iadd3(8, 4, imm=(-cy) & 0xFFFFFFFF)
        s.lop3(8, 8, RZ, RZ, 0xC0, imm=n - 1)
        s.iadd3(9, 5, imm=(-cz) & 0xFFFFFFFF)
        s.lop3(9, 9, RZ, RZ, 0xC0, imm=n - 1)
        s.imad(10, 9, imm=n, c=8)
        s.imad(10, 10, imm=n, c=7)
        s.iadd3(10, 10, imm=q * N)
        s.imad_wide(12, 10, imm=8, c=14, unsigned=True)
        s.ldg(FQ + 2 * q, 12, width=isa.W64)
    _moments(s)
    for r, off in ((78, 16), (80, 24), (82, 32), (84, 40), (86, 48), (88, 56), (90, 64), (92, 72)):
        s.ldc(r, off, wide=True)
    s.mufu_rcp64(94, 70)                               # 1 / rho (correctly rounded)
    for reg in (72, 74, 76):
        s.dmul(reg, reg, 94)                           # u
    s.dmul(96, 72, 72)
    s.dfma(96, 74, 74, 96)
    s.dfma(96, 76, 76, 96)
    s.dmul(96, 96, 84)                                 # 1.5 |u|^2
    for r, w in ((98, 88), (100, 90), (102, 92)):
        s.dmul(r, w, 70)                               # w_q rho
    s.ldc(10, 8, wide=True)
    s.imad_wide(12, 0, imm=8, c=10, unsigned=True)     # &f_new[0][cell]
    for q, c in enumerate(D3Q19):
        nz = [(a, v) for a, v in enumerate(c) if v]
        ureg = (72, 74, 76)
        if not nz:
            s.mov(104, imm=0)
            s.mov(105, imm=0)
        elif len(nz) == 1:
            a, v = nz[0]
            s.dadd(104, ureg[a], RZ, nega=v < 0)
        else:
            (a0, v0), (a1, v1) = nz
            s.dadd(104, ureg[a0], ureg[a1], nega=v0 < 0, negb=v1 < 0)
        s.dfma(106, 104, 82, 80)                       # 4.5 cu + 3
        s.dfma(106, 106, 104, 78)                      # 1 + 3 cu + 4.5 cu^2
        s.dadd(106, 106, 96, negb=True)
        s.dmul(106, 106, 98 if q == 0 else (100 if q < 7 else 102))   # f_eq
        s.dadd(108, FQ + 2 * q, 106, negb=True)
        s.dfma(108, 86, 108, FQ + 2 * q)               # f - omega (f - f_eq)
        s.stg(12, 108, off=8 * q * N, width=isa.W64)
    s.exit()
    return s.assemble()


def lbm_moments_code(n: int) -> np.ndarray:
    """rho, jx, jy, jz per cell; cbank: f(0) out(8)  (out = [4][N] f64)."""
    N = n ** 3
    s = Asm()
    _tid(s, N)
    s.ldc(6, 0, wide=True)
    s.imad_wide(12, 0, imm=8, c=6, unsigned=True)
    for q in range(19):
        s.ldg(FQ + 2 * q, 12, off=8 * q * N, width=isa.W64)
    _moments(s)
    s.ldc(6, 8, wide=True)
    s.imad_wide(12, 0, imm=8, c=6, unsigned=True)
    for a, reg in enumerate((70, 72, 74, 76)):
        s.stg(12, reg, off=8 * a * N, width=isa.W64)
    s.exit()
    return s.assemble()


def lbm_init_code(n: int) -> np.ndarray:
    """f_q = w_q rho0 (fluid at rest, density perturbation); cbank: rho0(0) f(8) w0(16) w1(24) w2(32)."""
    N = n ** 3
    s = Asm()
    _tid(s, N)
    s.ldc(6, 0, wide=True)
    s.imad_wide(6, 0, imm=8, c=6, unsigned=True)
    s.ldg(8, 6, width=isa.W64)
    for r, off in ((10, 16), (12, 24), (14, 32)):
        s.ldc(r, off, wide=True)
        s.dmul(r, r, 8)
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 0, imm=8, c=6, unsigned=True)
    for q in range(19):
        s.stg(6, 10 if q == 0 else (12 if q < 7 else 14), off=8 * q * N, width=isa.W64)
    s.exit()
    return s.assemble()


def _f64_words(x: float) -> list[int]:
    b = int(np.array([x], dtype="<f8").view("<u8")[0])
    return [b & 0xFFFFFFFF, b >> 32]


def lbm(n: int = 32, steps: int = 120, every: int = 10, tau: float = 0.8, seed: int = C5_DATA_SEED + 1) -> Program:
    N = n ** 3
    pb = ProgramBuilder(f"lbm_d3q19_{n}_s{steps}")
    ki = pb.add_kernel("lbm_init", lbm_init_code(n), nregs=40)
    kc = pb.add_kernel("lbm_stream_collide", lbm_collide_code(n), nregs=112)
    km = pb.add_kernel("lbm_moments", lbm_moments_code(n), nregs=80)
    rho0 = (1.0 + 0.01 * f64_data(seed, N)).astype(np.float64)
    r0 = pb.add_buffer("rho0", 8 * N, rho0, dtype=isa.DT_F64)
    w = [_f64_words(v) for v in (D3Q19_W[0], D3Q19_W[1], D3Q19_W[7])]
    k = 0
    f = pb.add_buffer("f0", 8 * 19 * N, writer=k, dtype=isa.DT_F64)
    pb.add_instance(ki, (N + 255) // 256, 256, ptr_words(r0) + ptr_words(f) + w[0] + w[1] + w[2])
    k += 1
    consts = _f64_words(1.0) + _f64_words(3.0) + _f64_words(4.5) + _f64_words(1.5) + _f64_words(-1.0 / tau)
    for st in range(steps):
        fn = pb.add_buffer(f"f{st + 1}", 8 * 19 * N, writer=k, output=st == steps - 1, dtype=isa.DT_F64)
        pb.add_instance(kc, (N + 255) // 256, 256, ptr_words(f) + ptr_words(fn) + consts + w[0] + w[1] + w[2])
        k += 1
        f = fn
        if (st + 1) % every == 0 or st == steps - 1:
            m = pb.add_buffer(f"m{st + 1}", 8 * 4 * N, writer=k, output=st == steps - 1, dtype=isa.DT_F64)
            pb.add_instance(km, (N + 255) // 256, 256, ptr_words(f) + ptr_words(m))
            k += 1
    return pb.build(config="C5-lbm", n=n, steps=steps, tau=tau)


# ---------------------------------------------------------------------------
# Lennard-Jones molecular dynamics (FP64), all pairs with cutoff, velocity Verlet
# ---------------------------------------------------------------------------
def md_force_code(N: int) -> np.ndarray:
    """f_i = sum_j 24 (2 s^6 - 1) s^6 / r^2 d (j ascending, r < rc, minimum image),
    pe_i = sum_j 4 s^6 (s^6 - 1), s^6 = r^-6.  cbank: x y z (0, 8, 16) f (24: [3][N]) pe (32)
    L (40) L/2 (48) rc^2 (56) 24 (64) 2 (72) 1 (80) 4 (88)."""
    s = Asm()
    _tid(s, N)
    s.mov(31, imm=1)
    for a, off in enumerate((0, 8, 16)):
        s.ldc(4 + 2 * a, off, wide=True)                # base pointers R4, R6, R8
    for a in range(3):
        s.imad_wide(10, 0, imm=8, c=4 + 2 * a, unsigned=True)
        s.ldg(32 + 2 * a, 10, width=isa.W64)           # x_i, y_i, z_i -> R32, R34, R36
    for r, off in ((40, 40), (42, 48), (44, 56), (46, 64), (48, 72), (50, 80), (52, 88)):
        s.ldc(r, off, wide=True)
    for r in (54, 56, 58, 60):                         # fx fy fz pe
        s.mov(r, imm=0)
        s.mov(r + 1, imm=0)
    s.mov(12, imm=0)                                   # j
    s.label("j")
    s.isetp(1, 12, 0, cmp=isa.EQ)
    s.bra("next", guard=1)
    for a in range(3):
        s.ldg(62 + 2 * a, 4 + 2 * a, width=isa.W64)    # x_j
        s.dadd(68 + 2 * a, 32 + 2 * a, 62 + 2 * a, negb=True)   # d = x_i - x_j
        s.dsetp(2, 68 + 2 * a, 42, cmp=isa.GT)
        s.dadd(68 + 2 * a, 68 + 2 * a, 40, negb=True, guard=2)  # d > L/2: d -= L
        s.dadd(74, 42, RZ, nega=True)                  # -L/2
        s.dsetp(3, 68 + 2 * a, 74, cmp=isa.LT)
        s.dadd(68 + 2 * a, 68 + 2 * a, 40, guard=3)    # d < -L/2: d += L
    s.dmul(76, 68, 68)
    s.dfma(76, 70, 70, 76)
    s.dfma(76, 72, 72, 76)                             # r^2
    s.dsetp(4, 76, 44, cmp=isa.GE)
    s.bra("next", guard=4)
    s.mufu_rcp64(78, 76)                               # 1 / r^2
    s.dmul(80, 78, 78)
    s.dmul(80, 80, 78)                                 # s6
    s.dfma(82, 80, 48, 50, negc=True)                  # 2 s6 - 1
    s.dmul(82, 82, 80)
    s.dmul(82, 82, 46)
    s.dmul(82, 82, 78)                                 # fr
    s.dfma(54, 82, 68, 54)
    s.dfma(56, 82, 70, 56)
    s.dfma(58, 82, 72, 58)
    s.dadd(84, 80, 50, negb=True)                      # s6 - 1
    s.dmul(84, 84, 80)
    s.dfma(60, 84, 52, 60)                             # pe += 4 s6 (s6 - 1)
    s.label("next")
    for a in range(3):
        s.imad_wide(4 + 2 * a, 31, imm=8, c=4 + 2 * a, unsigned=True)
    s.iadd3(12, 12, imm=1)
    s.isetp(0, 12, imm=N, cmp=isa.LT, unsigned=True)
    s.bra("j", guard=0)
    s.ldc(10, 24, wide=True)
    s.imad_wide(10, 0, imm=8, c=10, unsigned=True)
    for a in range(3):
        s.stg(10, 54 + 2 * a, off=8 * a * N, width=isa.W64)
    s.ldc(10, 32, wide=True)
    s.imad_wide(10, 0, imm=8, c=10, unsigned=True)
    s.stg(10, 60, width=isa.W64)
    s.exit()
    return s.assemble()


def md_kick_drift_code(N: int, drift: bool) -> np.ndarray:
    """v' = v + (dt/2) f; with drift also x' = x + dt v', wrapped into [0, L).
    cbank: v(0: [3][N]) f(8) v'(16) dt/2(24) x(32) x'(40) dt(48) L(56)."""
    s = Asm()
    _tid(s, N)
    s.ldc(20, 24, wide=True)
    if drift:
        s.ldc(22, 48, wide=True)
        s.ldc(24, 56, wide=True)
    for a in range(3):
        for r, off in ((4, 0), (6, 8), (8, 16)):
            s.ldc(r, off, wide=True)
            s.imad_wide(r, 0, imm=8, c=r, unsigned=True)
        s.ldg(10, 4, off=8 * a * N, width=isa.W64)
        s.ldg(12, 6, off=8 * a * N, width=isa.W64)
        s.dfma(10, 12, 20, 10)
        s.stg(8, 10, off=8 * a * N, width=isa.W64)
        if drift:
            s.ldc(14, 32, wide=True)
            s.imad_wide(14, 0, imm=8, c=14, unsigned=True)
            s.ldg(16, 14, off=8 * a * N, width=isa.W64)
            s.dfma(16, 10, 22, 16)
            s.dsetp(1, 16, 24, cmp=isa.GE)
            s.dadd(16, 16, 24, negb=True, guard=1)
            s.dsetp(2, 16, RZ, cmp=isa.LT)
            s.dadd(16, 16, 24, guard=2)
            s.ldc(14, 40, wide=True)
            s.imad_wide(14, 0, imm=8, c=14, unsigned=True)
            s.stg(14, 16, off=8 * a * N, width=isa.W64)
    s.exit()
    return s.assemble()


def md(m: int = 12, steps: int = 17, dt: float = 0.002, seed: int = C5_DATA_SEED + 2) -> Program:
    """N = m^3 particles on a jittered cubic lattice at density ~0.8; 1 + 3 * steps launches."""
    N = m ** 3
    a = (1 / 0.8) ** (1 / 3)
    Lb = m * a
    rc = min(2.5, Lb / 2 - 0.01)
    g = np.stack(np.meshgrid(np.arange(m), np.arange(m), np.arange(m), indexing="ij"), 0).reshape(3, N)
    x0 = ((g + 0.5) * a + 0.05 * a * f64_data(seed, 3 * N).reshape(3, N)).astype(np.float64)
    v0 = (0.1 * f64_data(seed + 1, 3 * N)).astype(np.float64)
    pb = ProgramBuilder(f"md_lj_{N}_s{steps}")
    kf = pb.add_kernel("lj_force", md_force_code(N), nregs=90)
    kd = pb.add_kernel("kick_drift", md_kick_drift_code(N, True), nregs=32)
    kk = pb.add_kernel("kick", md_kick_drift_code(N, False), nregs=32)
    fw = lambda v: _f64_words(v)  # noqa: E731
    consts_f = fw(Lb) + fw(Lb / 2) + fw(rc * rc) + fw(24.0) + fw(2.0) + fw(1.0) + fw(4.0)
    x = pb.add_buffer("x0", 8 * 3 * N, x0, dtype=isa.DT_F64)
    v = pb.add_buffer("v0", 8 * 3 * N, v0, dtype=isa.DT_F64)
    k = 0

    def force(xb, tag, last):
        nonlocal k
        f = pb.add_buffer(f"f{tag}", 8 * 3 * N, writer=k, output=last, dtype=isa.DT_F64)
        pe = pb.add_buffer(f"pe{tag}", 8 * N, writer=k, output=last, dtype=isa.DT_F64)
        pb.add_instance(kf, (N + 127) // 128, 128,
                        ptr_words(xb) + ptr_words(xb + 8 * N) + ptr_words(xb + 16 * N) + ptr_words(f) + ptr_words(pe)
                        + consts_f)
        k += 1
        return f

    f = force(x, 0, False)
    for st in range(steps):
        last = st == steps - 1
        vh = pb.add_buffer(f"vh{st + 1}", 8 * 3 * N, writer=k, dtype=isa.DT_F64)
        xn = pb.add_buffer(f"x{st + 1}", 8 * 3 * N, writer=k, output=last, dtype=isa.DT_F64)
        pb.add_instance(kd, (N + 255) // 256, 256, ptr_words(v) + ptr_words(f) + ptr_words(vh) + fw(dt / 2)
                        + ptr_words(x) + ptr_words(xn) + fw(dt) + fw(Lb))
        k += 1
        f = force(xn, st + 1, last)
        vn = pb.add_buffer(f"v{st + 1}", 8 * 3 * N, writer=k, output=last, dtype=isa.DT_F64)
        pb.add_instance(kk, (N + 255) // 256, 256, ptr_words(vh) + ptr_words(f) + ptr_words(vn) + fw(dt / 2))
        k += 1
        x, v = xn, vn
    return pb.build(config="C5-md", N=N, steps=steps, L=Lb, rc=rc, dt=dt)


# ---------------------------------------------------------------------------
# EP-like (FP64 + integer): LCG pairs, acceptance test, annulus tallies
# ---------------------------------------------------------------------------
def ep_gen_code(threads: int, pairs: int) -> np.ndarray:
    """Per thread: `pairs` draws (u1, u2) from a 32-bit LCG, X = 2 u1 - 1, Y = 2 u2 - 1,
    t = X^2 + Y^2; accepted (t <= 1): count, tally t into 4 rings by thresholds
    1/4, 1/2, 3/4, and sums sx += X t, sy += Y t.  cbank: out(0: [threads][8] u32
    count q0 q1 q2 q3 pad sx sy... as words) seed(8)."""
    s = Asm()
    _tid(s, threads)
    s.ldc(3, 8)
    s.imad(4, 0, imm=2654435761, c=3)                  # x = t * golden + seed
    for r in range(10, 20):
        s.mov(r, imm=0)                                # counters R10..R14, sx R16:17, sy R18:19
    s.mov(20, imm=isa.f32_bits(2.0 ** -32))
    s.mov(5, imm=pairs)
    s.mov(22, imm=0)
    s.mov(23, imm=0x3FF00000)                          # 1.0
    s.mov(24, imm=0)
    s.mov(25, imm=0x3FD00000)                          # 0.25
    s.mov(26, imm=0)
    s.mov(27, imm=0x3FE00000)                          # 0.5
    s.mov(28, imm=0)
    s.mov(29, imm=0x3FE80000)                          # 0.75
    s.mov(30, imm=0)
    s.mov(31, imm=0x40000000)                          # 2.0
    s.label("p")
    for reg in (32, 34):
        s.imad(4, 4, imm=1664525, c=RZ)
        s.iadd3(4, 4, imm=1013904223)
        s.i2f(6, 4, unsigned=True)
        s.fmul(6, 6, 20)                               # u in [0, 1) (f32)
        s.f2f_f64_f32(reg, 6)
        s.dfma(reg, reg, 30, 22, negc=True)            # 2u - 1
    s.dmul(36, 32, 32)
    s.dfma(36, 34, 34, 36)                             # t
    s.dsetp(1, 36, 22, cmp=isa.GT)
    s.bra("skip", guard=1)
    s.iadd3(10, 10, imm=1)
    s.dsetp(2, 36, 24, cmp=isa.LT)
    s.iadd3(11, 11, imm=1, guard=2)
    s.dsetp(2, 36, 26, cmp=isa.LT)
    s.iadd3(12, 12, imm=1, guard=2)
    s.dsetp(2, 36, 28, cmp=isa.LT)
    s.iadd3(13, 13, imm=1, guard=2)
    s.dfma(16, 32, 36, 16)
    s.dfma(18, 34, 36, 18)
    s.label("skip")
    s.iadd3(5, 5, imm=0xFFFFFFFF)
    s.isetp(0, 5, imm=0, cmp=isa.GT)
    s.bra("p", guard=0)
    s.ldc(6, 0, wide=True)
    s.imad_wide(6, 0, imm=32, c=6, unsigned=True)
    s.stg(6, 10, width=isa.W128)                       # count, r1, r2, r3
    s.stg(6, 16, off=16, width=isa.W128)               # sx, sy
    s.exit()
    return s.assemble()


def ep_reduce_code(threads: int) -> np.ndarray:
    """Sum the per-thread records of one chunk: 32 lanes stride the records, then a
    SHFL tree (f64 sums as two 32-bit shuffles); one warp.  cbank: in(0) out(8)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.mov(35, imm=1)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 0, imm=32, c=4, unsigned=True)
    for r in range(10, 20):
        s.mov(r, imm=0)
    s.mov(21, imm=(threads + 31) // 32)
    s.label("r")
    s.ldg(24, 4, width=isa.W128)
    s.ldg(28, 4, off=16, width=isa.W128)
    for q in range(4):
        s.iadd3(10 + q, 10 + q, 24 + q)
    s.dadd(16, 16, 28)
    s.dadd(18, 18, 30)
    s.imad_wide(4, 35, imm=32 * 32, c=4, unsigned=True)
    s.iadd3(21, 21, imm=0xFFFFFFFF)
    s.isetp(0, 21, imm=0, cmp=isa.GT)
    s.bra("r", guard=0)
    for sh in (16, 8, 4, 2, 1):
        for q in range(4):
            s.shfl(24 + q, 10 + q, imm=sh, mode=isa.SHFL_BFLY)
            s.iadd3(10 + q, 10 + q, 24 + q)
        for r in (16, 18):
            s.shfl(28, r, imm=sh, mode=isa.SHFL_BFLY)
            s.shfl(29, r + 1, imm=sh, mode=isa.SHFL_BFLY)
            s.dadd(r, r, 28)
    s.isetp(1, 0, imm=0, cmp=isa.NE)
    s.exit(guard=1)
    s.ldc(6, 8, wide=True)
    s.stg(6, 10, width=isa.W128)
    s.stg(6, 16, off=16, width=isa.W128)
    s.exit()
    return s.assemble()


def ep(threads: int = 16384, pairs: int = 512, chunks: int = 4, seed: int = C5_DATA_SEED + 3) -> Program:
    """chunks x (generate, reduce): 2 static / 2 * chunks dynamic."""
    assert threads % 32 == 0
    pb = ProgramBuilder(f"ep_{threads}x{pairs}x{chunks}")
    kg = pb.add_kernel("ep_gen", ep_gen_code(threads, pairs), nregs=40)
    kr = pb.add_kernel("ep_reduce", ep_reduce_code(threads), nregs=40)
    k = 0
    for c in range(chunks):
        rec = pb.add_buffer(f"rec{c}", 32 * threads, writer=k, dtype=isa.DT_U32)
        pb.add_instance(kg, (threads + 255) // 256, 256, ptr_words(rec) + [(seed + 7919 * c) & 0xFFFFFFFF])
        k += 1
        out = pb.add_buffer(f"tally{c}", 32, writer=k, output=True, dtype=isa.DT_U32)
        pb.add_instance(kr, 1, 32, ptr_words(rec) + ptr_words(out))
        k += 1
    return pb.build(config="C5-ep", threads=threads, pairs=pairs, chunks=chunks, seed=seed)


# ---------------------------------------------------------------------------
def c5(full: bool = True) -> list[Program]:
    """The five C5 programs (full sizes ~1e9 counted thread-instructions each; mini
    sizes are oracle parity cases)."""
    from .programs import cg_program
    if full:
        return [stencil(128, 100), lbm(32, 120, 10), md(12, 17), ep(16384, 512, 4), cg_program(256, 256, 200)]
    return [stencil(8, 6), lbm(4, 6, 3), md(3, 3), ep(256, 16, 2), cg_program(32, 8, 3)]
