"""Seeded synthetic programs C1, C2 (+ mini sizes) and fuzz programs.

Shapes follow SURVEY.md §8(d) / App. A.5 and BASELINE.json `configs`:
  C1  vector add c = a + b, n = 1024 FP32, 4 CTAs x 256 threads, one instance.
  C2  SGEMM C = A.B (A stored K-major, B row-major), 128x128 CTA tile,
      8x8 micro-tile per thread; 4096^3 at full size, 256^3 as "mini-C2".
Fuzz programs are random straight-line/branchy kernels used to cross-check the
two interpreters opcode by opcode.
"""
from __future__ import annotations

import numpy as np

from . import isa
from .isa import Asm, RZ, PT, NEG
from .program import ProgramBuilder, Program, ptr_words, f32_data, f64_data, u32_data

DATA_SEED = {1: 0xD0000001, 2: 0xD0000002, 3: 0xD0000003}
CAMPAIGN_SEED = {1: 0xC0000001, 2: 0xC0000002, 3: 0xC0000003}


# ---------------------------------------------------------------------------
# C1: vector add (App. A.5 listing, 18 static instructions)
# ---------------------------------------------------------------------------
def c1_code() -> np.ndarray:
    s = Asm()
    s.s2r(0, isa.SR_TID)                      # 0
    s.s2r(1, isa.SR_CTAID)                    # 1
    s.s2r(2, isa.SR_NTID)                     # 2
    s.imad(0, 1, 2, 0)                        # 3  gid = ctaid*ntid + tid
    s.ldc(3, 24)                              # 4  n
    s.isetp(0, 0, 3, cmp=isa.GE)              # 5  P0 = gid >= n
    s.exit(guard=0)                           # 6  @P0 EXIT
    s.ldc(4, 0, wide=True)                    # 7  a
    s.imad_wide(4, 0, imm=4, c=4)             # 8
    s.ldc(6, 8, wide=True)                    # 9  b
    s.imad_wide(6, 0, imm=4, c=6)             # 10
    s.ldg(8, 4)                               # 11
    s.ldg(9, 6)                               # 12
    s.ldc(10, 16, wide=True)                  # 13 c
    s.imad_wide(10, 0, imm=4, c=10)           # 14
    s.fadd(8, 8, 9)                           # 15
    s.stg(10, 8)                              # 16
    s.exit()                                  # 17
    return s.assemble()


def vector_add(n: int = 1024, grid: int = 4, block: int = 256, seed: int = DATA_SEED[1]) -> Program:
    pb = ProgramBuilder(f"vecadd_n{n}")
    k = pb.add_kernel("vecadd", c1_code(), nregs=12)
    a = pb.add_buffer("a", 4 * n, f32_data(seed, n), dtype=isa.DT_F32)
    b = pb.add_buffer("b", 4 * n, f32_data(seed + 1, n), dtype=isa.DT_F32)
    c = pb.add_buffer("c", 4 * n, writer=0, output=True, dtype=isa.DT_F32)
    pb.add_instance(k, grid, block, ptr_words(a) + ptr_words(b) + ptr_words(c) + [n])
    return pb.build(config="C1", n=n, grid=grid, block=block)


def c1() -> Program:
    return vector_add()


def vector_add_f64(n: int = 512, grid: int = 2, block: int = 256, seed: int = DATA_SEED[1] + 64) -> Program:
    """c = a + b in FP64 (LDG.64, DADD, STG.64): an f64 output buffer for the
    C-12 secondary numeric classification (an element is a register pair)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)                      # 0
    s.s2r(1, isa.SR_CTAID)                    # 1
    s.s2r(2, isa.SR_NTID)                     # 2
    s.imad(0, 1, 2, 0)                        # 3  gid
    s.ldc(3, 24)                              # 4  n
    s.isetp(0, 0, 3, cmp=isa.GE)              # 5
    s.exit(guard=0)                           # 6
    s.ldc(4, 0, wide=True)                    # 7  a
    s.imad_wide(4, 0, imm=8, c=4)             # 8
    s.ldc(6, 8, wide=True)                    # 9  b
    s.imad_wide(6, 0, imm=8, c=6)             # 10
    s.ldg(8, 4, width=isa.W64)                # 11 R8:R9
    s.ldg(10, 6, width=isa.W64)               # 12 R10:R11
    s.ldc(12, 16, wide=True)                  # 13 c
    s.imad_wide(12, 0, imm=8, c=12)           # 14
    s.dadd(8, 8, 10)                          # 15 R8:R9
    s.stg(12, 8, width=isa.W64)               # 16
    s.exit()                                  # 17
    pb = ProgramBuilder(f"vecadd_f64_n{n}")
    k = pb.add_kernel("vecadd_f64", s.assemble(), nregs=14)
    a = pb.add_buffer("a", 8 * n, f64_data(seed, n), dtype=isa.DT_F64)
    b = pb.add_buffer("b", 8 * n, f64_data(seed + 1, n), dtype=isa.DT_F64)
    c = pb.add_buffer("c", 8 * n, writer=0, output=True, dtype=isa.DT_F64)
    pb.add_instance(k, grid, block, ptr_words(a) + ptr_words(b) + ptr_words(c) + [n])
    return pb.build(config="vecadd_f64", n=n, grid=grid, block=block)


# ---------------------------------------------------------------------------
# C2: SGEMM, 128x128 CTA tile, 8x8 per thread (App. A.5)
# ---------------------------------------------------------------------------
ACC0, AFR, BFR = 8, 72, 80
PA, PB, KCNT, SA, SB, TMP = 88, 90, 92, 93, 94, 95


def sgemm_code(n_ctas_x: int) -> np.ndarray:
    assert n_ctas_x & (n_ctas_x - 1) == 0
    lg = n_ctas_x.bit_length() - 1
    AND = 0xC0                                 # LOP3 lut for a & b
    s = Asm()
    s.s2r(0, isa.SR_TID)                       # 0
    s.s2r(1, isa.SR_CTAID)                     # 1
    s.lop3(2, 0, RZ, RZ, AND, imm=15)          # 2  tx
    s.shf(3, 0, imm=4, mode=isa.SHF_R_U32)     # 3  ty
    s.lop3(4, 1, RZ, RZ, AND, imm=n_ctas_x - 1)  # 4  bx
    s.shf(5, 1, imm=lg, mode=isa.SHF_R_U32)    # 5  by
    s.imad(6, 5, imm=128, c=RZ)                # 6
    s.imad(6, 3, imm=8, c=6)                   # 7  m0
    s.imad(7, 4, imm=128, c=RZ)                # 8
    s.imad(7, 2, imm=8, c=7)                   # 9  n0
    s.ldc(PA, 0, wide=True)                    # 10 A
    s.imad_wide(PA, 6, imm=4, c=PA, unsigned=True)   # 11
    s.ldc(PB, 8, wide=True)                    # 12 B
    s.imad_wide(PB, 7, imm=4, c=PB, unsigned=True)   # 13
    s.ldc(KCNT, 24)                            # 14 K
    s.ldc(SA, 28)                              # 15 M*4
    s.ldc(SB, 32)                              # 16 N*4
    s.label("loop")                            # 17
    s.ldg(AFR, PA, 0, isa.W128)
    s.ldg(AFR + 4, PA, 16, isa.W128)
    s.ldg(BFR, PB, 0, isa.W128)
    s.ldg(BFR + 4, PB, 16, isa.W128)
    for i in range(8):
        for j in range(8):
            r = ACC0 + 8 * i + j
            s.ffma(r, AFR + i, BFR + j, r)
    s.imad_wide(PA, SA, imm=1, c=PA, unsigned=True)
    s.imad_wide(PB, SB, imm=1, c=PB, unsigned=True)
    s.iadd3(KCNT, KCNT, imm=0xFFFFFFFF)
    s.isetp(0, KCNT, imm=0, cmp=isa.GT)
    s.bra("loop", guard=0)
    s.ldc(PA, 16, wide=True)                   # C
    s.ldc(TMP, 36)                             # N
    s.imad(TMP, 6, TMP, 7)                     # m0*N + n0
    s.imad_wide(PA, TMP, imm=4, c=PA, unsigned=True)
    for i in range(8):
        s.stg(PA, ACC0 + 8 * i, 0, isa.W128)
        s.stg(PA, ACC0 + 8 * i + 4, 16, isa.W128)
        s.imad_wide(PA, SB, imm=1, c=PA, unsigned=True)
    s.exit()
    return s.assemble()


def sgemm(M: int, N: int, K: int, seed: int = DATA_SEED[2]) -> Program:
    assert M % 128 == 0 and N % 128 == 0 and K >= 1
    nx = N // 128
    pb = ProgramBuilder(f"sgemm_{M}x{N}x{K}")
    k = pb.add_kernel("sgemm_128x128", sgemm_code(nx), nregs=96)
    a = pb.add_buffer("A", 4 * K * M, f32_data(seed, K * M), dtype=isa.DT_F32)      # A^T: [K][M]
    b = pb.add_buffer("B", 4 * K * N, f32_data(seed + 1, K * N), dtype=isa.DT_F32)  # [K][N]
    c = pb.add_buffer("C", 4 * M * N, writer=0, output=True, dtype=isa.DT_F32)      # [M][N]
    pb.add_instance(k, (M // 128) * nx, 256,
                    ptr_words(a) + ptr_words(b) + ptr_words(c) + [K, 4 * M, 4 * N, N])
    return pb.build(config="C2", M=M, N=N, K=K)


def c2(full: bool = True) -> Program:
    return sgemm(4096, 4096, 4096) if full else sgemm(256, 256, 256)


# ---------------------------------------------------------------------------
# Fuzz programs (random opcode mixes, divergence, SHFL, special FP values)
# ---------------------------------------------------------------------------
SPECIAL_F32 = [0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000, 0xFFC00001,
               0x00000001, 0x807FFFFF, 0x3F800000, 0xBF800000, 0x4B000000, 0xCF000000,
               0x4F000000, 0x7F7FFFFF, 0x34000000, 0x3EFFFFFF]
SPECIAL_F64_HI = [0x00000000, 0x80000000, 0x7FF00000, 0xFFF00000, 0x7FF80000, 0x3FF00000,
                  0xBFF00000, 0x00000001, 0x41E00000, 0xC1E00000, 0x47EFFFFF, 0x36A00000]

NWORK = 16      # working registers R0..R15 (pairs inside)
R_GID, R_PIN, R_POUT, R_TMP, R_CNT = 20, 22, 24, 26, 27


def _fuzz_body(rng: np.random.Generator, s: Asm, n_ops: int, allow_branch=True):
    """Random ops on R0..R15 / P0..P5; forward branches only."""
    def r():
        return int(rng.integers(0, NWORK))

    def pr():
        return int(rng.integers(0, NWORK // 2)) * 2

    def g():
        x = rng.random()
        if x < 0.75:
            return PT
        return int(rng.integers(0, 6)) | (NEG if rng.random() < 0.5 else 0)

    def imm_or_none():
        return int(rng.integers(0, 2**32)) if rng.random() < 0.3 else None

    pending = []
    for n in range(n_ops):
        for lbl in [p for p in pending if p[1] == n]:
            s.label(lbl[0])
        k = int(rng.integers(0, 27))
        if k == 0:
            s.mov(r(), b=r(), imm=imm_or_none(), guard=g())
        elif k == 1:
            s.iadd3(r(), r(), r(), r(), imm=imm_or_none(), nega=rng.random() < 0.3,
                    negb=rng.random() < 0.3, carry=int(rng.integers(0, 6)) if rng.random() < 0.3 else PT, guard=g())
        elif k == 2:
            s.imad(r(), r(), r(), r(), imm=imm_or_none(), guard=g())
        elif k == 3:
            s.imad_wide(pr(), r(), r(), c=pr() if rng.random() < 0.7 else RZ, imm=imm_or_none(),
                        unsigned=rng.random() < 0.5, guard=g())
        elif k == 4:
            im = int(rng.integers(0, 40)) if rng.random() < 0.5 else None
            s.shf(r(), r(), r(), imm=im, mode=int(rng.integers(0, 3)), guard=g())
        elif k == 5:
            s.lop3(r(), r(), r(), r(), int(rng.integers(0, 256)), guard=g())
        elif k == 6:
            s.sel(r(), r(), r(), int(rng.integers(0, 8)) | (NEG if rng.random() < 0.3 else 0), guard=g())
        elif k == 7:
            s.isetp(int(rng.integers(0, 6)), r(), r(), cmp=int(rng.integers(0, 6)), imm=imm_or_none(),
                    unsigned=rng.random() < 0.5, guard=g())
        elif k == 8:
            s.fsetp(int(rng.integers(0, 6)), r(), r(), cmp=int(rng.integers(0, 6)), guard=g())
        elif k == 9:
            s.dsetp(int(rng.integers(0, 6)), pr(), pr(), cmp=int(rng.integers(0, 6)), guard=g())
        elif k in (10, 11, 12):
            op = [s.fadd, s.fmul, s.ffma][k - 10]
            args = (r(), r(), r()) if k < 12 else (r(), r(), r(), r())
            op(*args, nega=rng.random() < 0.3, negb=rng.random() < 0.3, negc=rng.random() < 0.3, guard=g())
        elif k == 13:
            s.fmnmx(r(), r(), r(), is_max=rng.random() < 0.5, guard=g())
        elif k in (14, 15, 16):
            op = [s.dadd, s.dmul, s.dfma][k - 14]
            args = (pr(), pr(), pr()) if k < 16 else (pr(), pr(), pr(), pr())
            op(*args, nega=rng.random() < 0.3, negb=rng.random() < 0.3, negc=rng.random() < 0.3, guard=g())
        elif k == 17:
            s.i2f(r(), r(), unsigned=rng.random() < 0.5, guard=g())
        elif k == 18:
            s.f2i(r(), r(), guard=g())
        elif k == 19:
            s.f2f_f64_f32(pr(), r(), guard=g())
        elif k == 20:
            s.f2f_f32_f64(r(), pr(), guard=g())
        elif k in (21, 22):
            im = int(rng.integers(0, 40)) if rng.random() < 0.6 else None
            s.shfl(r(), r(), r(), imm=im, mode=int(rng.integers(0, 4)), guard=g())
        elif k == 23:
            s.imnmx(r(), r(), r(), is_max=rng.random() < 0.5, unsigned=rng.random() < 0.5, guard=g())
        elif k == 24 and allow_branch and n + 2 < n_ops:
            # forward branch on a (usually lane-divergent) predicate
            lbl = f"L{n}"
            tgt = n + 1 + int(rng.integers(1, min(6, n_ops - n)))
            pending.append((lbl, tgt))
            s.bra(lbl, guard=int(rng.integers(0, 6)) | (NEG if rng.random() < 0.5 else 0))
        elif k == 25:
            s.s2r(r(), int(rng.integers(0, 6)), guard=g())
        else:
            s.nop(guard=g())
    for lbl in [p for p in pending if p[1] >= n_ops]:
        s.label(lbl[0])


F32_SPECIALS = np.array([0x7FC00000, 0xFFC00000, 0x7F800001, 0xFF812345, 0x7FFFFFFF, 0x7FA5A5A5, 0x7F800000,
                         0xFF800000, 0x00000000, 0x80000000, 0x00000001, 0x807FFFFF, 0x7F7FFFFF, 0x3F800000,
                         0xBF800000, 0x00800000], dtype=np.uint32)


def ffma_runs(seed: int = 5, grid: int = 2, block: int = 96) -> Program:
    """Straight runs of unguarded FFMAs (the emulator's FFMA batch path) over
    special f32 values: NaNs with payloads and both signs, infinities, signed
    zeros, denormals, extremes.  Independent batches, dependent chains, and a
    run that reads a register written earlier in it."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 0, imm=64, c=4, unsigned=True)
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 0, imm=96, c=6, unsigned=True)
    for q in range(4):
        s.ldg(8 + 4 * q, 4, off=16 * q, width=isa.W128)
    for q in range(8):                                 # independent: R24..R31
        s.ffma(24 + q, 8 + q, 9 + q, 10 + q)
    for q in range(8):                                 # chain through R32
        s.ffma(32, 32 if q else 12, 16 + q, 24 + q)
    for q in range(8):                                 # reads results of this run: R33..R39
        s.ffma(33 + (q % 7), 24 + q, 32, 33 + ((q + 3) % 7))
    for q in range(6):
        s.stg(6, 24 + 4 * q, off=16 * q, width=isa.W128)
    s.exit()
    n = grid * block
    rng = np.random.Generator(np.random.PCG64(seed))
    x = rng.integers(0, 2**32, size=16 * n, dtype=np.uint64).astype(np.uint32)
    pick = rng.random(16 * n) < 0.5
    x[pick] = F32_SPECIALS[rng.integers(0, len(F32_SPECIALS), int(pick.sum()))]
    pb = ProgramBuilder(f"ffma_runs_{seed}")
    k = pb.add_kernel("ffma_runs", s.assemble(), nregs=44)
    xb = pb.add_buffer("X", 64 * n, x.view(np.float32), dtype=isa.DT_U32)
    yb = pb.add_buffer("Y", 96 * n, writer=0, output=True, dtype=isa.DT_U32)
    pb.add_instance(k, grid, block, ptr_words(xb) + ptr_words(yb))
    return pb.build(config="ffma_runs", n=n)


def fuzz_program(seed: int, n_ops: int = 120, grid: int = 2, block: int = 80, loop_iters: int = 3) -> Program:
    """Random kernel: load 16 words per thread (special FP values mixed in), run
    a random op mix (optionally inside a counted loop), store the 16 registers
    and the 6 predicates.  block=80 gives a partial third warp per CTA."""
    rng = np.random.Generator(np.random.PCG64(seed))
    nthr = grid * block
    words = u32_data(seed ^ 0x5EED, nthr * NWORK)
    sp = rng.random(words.size) < 0.25
    words[sp] = rng.choice(np.array(SPECIAL_F32, dtype=np.uint32), size=int(sp.sum()))
    hi = (np.arange(words.size) % 2 == 1) & (rng.random(words.size) < 0.2)
    words[hi] = rng.choice(np.array(SPECIAL_F64_HI, dtype=np.uint32), size=int(hi.sum()))

    s = Asm()
    s.s2r(R_GID, isa.SR_TID)
    s.s2r(R_TMP, isa.SR_CTAID)
    s.s2r(R_TMP + 1, isa.SR_NTID)
    s.imad(R_GID, R_TMP, R_TMP + 1, R_GID)
    s.ldc(R_PIN, 0, wide=True)
    s.imad_wide(R_PIN, R_GID, imm=4 * NWORK, c=R_PIN, unsigned=True)
    for i in range(0, NWORK, 4):
        s.ldg(i, R_PIN, 4 * i, isa.W128)
    if loop_iters > 1:
        s.mov(R_CNT, imm=loop_iters)
        s.label("top")
    _fuzz_body(rng, s, n_ops)
    if loop_iters > 1:
        s.iadd3(R_CNT, R_CNT, imm=0xFFFFFFFF)
        s.isetp(6, R_CNT, imm=0, cmp=isa.GT)
        s.bra("top", guard=6)
    s.ldc(R_POUT, 8, wide=True)
    s.imad_wide(R_POUT, R_GID, imm=4 * (NWORK + 4), c=R_POUT, unsigned=True)
    for i in range(0, NWORK, 4):
        s.stg(R_POUT, i, 4 * i, isa.W128)
    # predicates -> one word (SEL per predicate, accumulate with IMAD)
    s.mov(R_TMP, imm=0)
    for p in range(6):
        s.sel(R_TMP + 1, RZ, RZ, p, imm=1 << p)   # P ? RZ : (1<<p)
        s.iadd3(R_TMP, R_TMP, R_TMP + 1)
    s.stg(R_POUT, R_TMP, 4 * NWORK)
    s.stg(R_POUT, R_GID, 4 * NWORK + 4)
    s.exit()

    pb = ProgramBuilder(f"fuzz_{seed}")
    k = pb.add_kernel("fuzz", s.assemble(), nregs=32)
    xin = pb.add_buffer("X", 4 * nthr * NWORK, words)
    yout = pb.add_buffer("Y", 4 * nthr * (NWORK + 4), writer=0, output=True)
    pb.add_instance(k, grid, block, ptr_words(xin) + ptr_words(yout))
    return pb.build(config="fuzz", seed=seed)


def multi_instance_chain(n_inst: int = 3, n: int = 256, block: int = 64, seed: int = 77, shrink: int = 0) -> Program:
    """y_{i+1} = y_i * s + x (FP32) over n_inst launches of one static kernel, each
    writing a new SSA buffer version.  Exercises multi-instance profiling,
    kernel_count, and (oracle full mode) downstream propagation.  With shrink > 0
    launch i only updates the first n - shrink*i elements (the rest exit early),
    so instances of the same static kernel have different counts (approximate
    profiling)."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.ldc(3, 24)
    s.isetp(0, 0, 3, cmp=isa.GE)
    s.exit(guard=0)
    s.ldc(4, 0, wide=True)
    s.imad_wide(4, 0, imm=4, c=4, unsigned=True)
    s.ldc(6, 8, wide=True)
    s.imad_wide(6, 0, imm=4, c=6, unsigned=True)
    s.ldc(10, 16, wide=True)
    s.imad_wide(10, 0, imm=4, c=10, unsigned=True)
    s.ldg(8, 4)
    s.ldg(9, 6)
    s.ldc(12, 28)
    s.ffma(8, 9, 12, 8)
    s.stg(10, 8)
    s.exit()
    code = s.assemble()
    pb = ProgramBuilder(f"chain_{n_inst}")
    k = pb.add_kernel("axpy_chain", code, nregs=12)
    x = pb.add_buffer("x", 4 * n, f32_data(seed, n), dtype=isa.DT_F32)
    y = pb.add_buffer("y0", 4 * n, f32_data(seed + 1, n), dtype=isa.DT_F32)
    grid = (n + block - 1) // block
    for i in range(n_inst):
        ynew = pb.add_buffer(f"y{i + 1}", 4 * n, writer=i, output=(i == n_inst - 1), dtype=isa.DT_F32)
        pb.add_instance(k, grid, block, ptr_words(x) + ptr_words(y) + ptr_words(ynew) + [n - shrink * i, isa.f32_bits(0.5)])
        y = ynew
    return pb.build(config="chain", n_inst=n_inst, n=n)


# ---------------------------------------------------------------------------
# C3: library-style FP64 conjugate gradient on a 2-D 5-point Laplacian
# (mirrors 354.cg's many small kernels, ~5,000 dynamic instances)
# ---------------------------------------------------------------------------
def _vec_prologue(s: Asm, n_off: int, exit_out: bool = True):
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)                             # i = ctaid*ntid + tid
    s.ldc(3, n_off)
    if exit_out:
        s.isetp(0, 0, 3, cmp=isa.GE)
        s.exit(guard=0)


def cg_spmv_code(nx: int) -> np.ndarray:
    """Ap = A p, A = 4I - shifts (Dirichlet): neighbour loads predicated on the
    boundary (partial active masks on boundary rows).  cbank: p, Ap, n, nx-1,
    log2 nx, ny-1, 4.0."""
    s = Asm()
    _vec_prologue(s, 16)
    s.ldc(5, 20)                                   # nx - 1
    s.ldc(6, 24)                                   # log2 nx
    s.lop3(7, 0, 5, RZ, 0xC0)                      # ix = i & (nx-1)
    s.shf(8, 0, 6, mode=isa.SHF_R_U32)             # iy = i >> log2 nx
    s.ldc(10, 0, wide=True)
    s.imad_wide(10, 0, imm=8, c=10, unsigned=True)
    s.ldg(12, 10, 0, isa.W64)
    s.ldc(16, 32, wide=True)                       # 4.0
    s.dmul(14, 12, 16)
    s.isetp(1, 7, imm=0, cmp=isa.GT)
    s.ldg(18, 10, -8, isa.W64, guard=1)
    s.dadd(14, 14, 18, negb=True, guard=1)
    s.isetp(2, 7, 5, cmp=isa.LT)
    s.ldg(18, 10, 8, isa.W64, guard=2)
    s.dadd(14, 14, 18, negb=True, guard=2)
    s.isetp(3, 8, imm=0, cmp=isa.GT)
    s.ldg(18, 10, -8 * nx, isa.W64, guard=3)
    s.dadd(14, 14, 18, negb=True, guard=3)
    s.ldc(9, 28)                                   # ny - 1
    s.isetp(4, 8, 9, cmp=isa.LT)
    s.ldg(18, 10, 8 * nx, isa.W64, guard=4)
    s.dadd(14, 14, 18, negb=True, guard=4)
    s.ldc(20, 8, wide=True)
    s.imad_wide(20, 0, imm=8, c=20, unsigned=True)
    s.stg(20, 14, 0, isa.W64)
    s.exit()
    return s.assemble()


def cg_dot_partial_code() -> np.ndarray:
    """part[warp] = sum over the warp of a[i]*b[i] (SHFL.BFLY tree on f64 pairs).
    cbank: a, b, part, n."""
    s = Asm()
    _vec_prologue(s, 24, exit_out=False)
    s.mov(10, imm=0)
    s.mov(11, imm=0)
    s.isetp(0, 0, 3, cmp=isa.LT)
    s.ldc(12, 0, wide=True, guard=0)
    s.imad_wide(12, 0, imm=8, c=12, unsigned=True, guard=0)
    s.ldg(14, 12, 0, isa.W64, guard=0)
    s.ldc(16, 8, wide=True, guard=0)
    s.imad_wide(16, 0, imm=8, c=16, unsigned=True, guard=0)
    s.ldg(18, 16, 0, isa.W64, guard=0)
    s.dmul(10, 14, 18, guard=0)
    for d in (16, 8, 4, 2, 1):
        s.shfl(20, 10, imm=d, mode=isa.SHFL_BFLY)
        s.shfl(21, 11, imm=d, mode=isa.SHFL_BFLY)
        s.dadd(10, 10, 20)
    s.s2r(4, isa.SR_LANEID)
    s.isetp(1, 4, imm=0, cmp=isa.EQ)
    s.shf(5, 0, imm=5, mode=isa.SHF_R_U32)         # global warp index
    s.ldc(22, 16, wide=True)
    s.imad_wide(22, 5, imm=8, c=22, unsigned=True, guard=1)
    s.stg(22, 10, 0, isa.W64, guard=1)
    s.exit()
    return s.assemble()


def cg_dot_final_code() -> np.ndarray:
    """out = sum of np partials: one warp, strided loop (lanes leave it at
    different trip counts), SHFL.BFLY tree.  cbank: part, out, np."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.mov(10, imm=0)
    s.mov(11, imm=0)
    s.ldc(3, 16)
    s.ldc(12, 0, wide=True)
    s.label("loop")
    s.isetp(0, 0, 3, cmp=isa.GE)
    s.bra("done", guard=0)
    s.imad_wide(14, 0, imm=8, c=12, unsigned=True)
    s.ldg(16, 14, 0, isa.W64)
    s.dadd(10, 10, 16)
    s.iadd3(0, 0, imm=32)
    s.bra("loop")
    s.label("done")
    for d in (16, 8, 4, 2, 1):
        s.shfl(20, 10, imm=d, mode=isa.SHFL_BFLY)
        s.shfl(21, 11, imm=d, mode=isa.SHFL_BFLY)
        s.dadd(10, 10, 20)
    s.s2r(4, isa.SR_LANEID)
    s.isetp(1, 4, imm=0, cmp=isa.EQ)
    s.ldc(18, 8, wide=True)
    s.stg(18, 10, 0, isa.W64, guard=1)
    s.exit()
    return s.assemble()


def cg_scalar_code() -> np.ndarray:
    """out = num * rcp(den) in lane 0 (alpha = rr/pAp, beta = rr'/rr).
    cbank: num, den, out."""
    s = Asm()
    s.s2r(0, isa.SR_LANEID)
    s.isetp(0, 0, imm=0, cmp=isa.NE)
    s.exit(guard=0)
    s.ldc(2, 0, wide=True)
    s.ldg(4, 2, 0, isa.W64)
    s.ldc(6, 8, wide=True)
    s.ldg(8, 6, 0, isa.W64)
    s.mufu_rcp64(10, 8)
    s.dmul(12, 4, 10)
    s.ldc(14, 16, wide=True)
    s.stg(14, 12, 0, isa.W64)
    s.exit()
    return s.assemble()


def cg_axpy_code(neg: bool) -> np.ndarray:
    """out = (+-alpha) * p + x.  cbank: x, p, alpha, out, n."""
    s = Asm()
    _vec_prologue(s, 32)
    s.ldc(2, 16, wide=True)
    s.ldg(4, 2, 0, isa.W64)
    s.ldc(6, 0, wide=True)
    s.imad_wide(6, 0, imm=8, c=6, unsigned=True)
    s.ldg(8, 6, 0, isa.W64)
    s.ldc(10, 8, wide=True)
    s.imad_wide(10, 0, imm=8, c=10, unsigned=True)
    s.ldg(12, 10, 0, isa.W64)
    s.dfma(14, 4, 12, 8, nega=neg)
    s.ldc(16, 24, wide=True)
    s.imad_wide(16, 0, imm=8, c=16, unsigned=True)
    s.stg(16, 14, 0, isa.W64)
    s.exit()
    return s.assemble()


def _f64_words(x: float) -> list[int]:
    b = int(np.array([x], dtype="<f8").view("<u8")[0])
    return [b & 0xFFFFFFFF, b >> 32]


def cg_program(nx: int = 512, ny: int = 256, iters: int = 500, seed: int = DATA_SEED[3]) -> Program:
    """CG for A x = b (x0 = 0, r0 = p0 = b), 10 launches per iteration, every
    vector / partial / scalar a new SSA buffer version; output = the final x."""
    assert nx & (nx - 1) == 0 and (nx * ny) % 256 == 0
    n = nx * ny
    nparts = n // 32
    pb = ProgramBuilder(f"cg_{nx}x{ny}_it{iters}")
    K = {}
    for name, code in (("spmv_lap5", cg_spmv_code(nx)), ("dot_partial_b", cg_dot_partial_code()),
                       ("dot_final_b", cg_dot_final_code()), ("dot_partial_pAp", cg_dot_partial_code()),
                       ("dot_final_pAp", cg_dot_final_code()), ("scalar_alpha", cg_scalar_code()),
                       ("axpy_x", cg_axpy_code(False)), ("axpy_r", cg_axpy_code(True)),
                       ("dot_partial_rr", cg_dot_partial_code()), ("dot_final_rr", cg_dot_final_code()),
                       ("scalar_beta", cg_scalar_code()), ("xpay_p", cg_axpy_code(False))):
        K[name] = pb.add_kernel(name, code, nregs=24)
    grid = n // 256
    lg = nx.bit_length() - 1

    def newbuf(name, nbytes, output=False):
        return pb.add_buffer(name, nbytes, writer=len(pb.instances), output=output, dtype=isa.DT_F64)

    def dot(kp, kf, a, b, tag):
        part = newbuf(f"part_{tag}", 8 * nparts)
        pb.add_instance(K[kp], grid, 256, ptr_words(a) + ptr_words(b) + ptr_words(part) + [n])
        out = newbuf(f"dot_{tag}", 8)
        pb.add_instance(K[kf], 1, 32, ptr_words(part) + ptr_words(out) + [nparts])
        return out

    b = pb.add_buffer("b", 8 * n, f64_data(seed, n), dtype=isa.DT_F64)
    x = pb.add_buffer("x0", 8 * n, dtype=isa.DT_F64)                 # zeros, never written
    r = p = b
    rr = dot("dot_partial_b", "dot_final_b", r, r, "rr0")
    for it in range(iters):
        ap = newbuf(f"Ap{it}", 8 * n)
        pb.add_instance(K["spmv_lap5"], grid, 256, ptr_words(p) + ptr_words(ap) + [n, nx - 1, lg, ny - 1] +
                        _f64_words(4.0))
        pap = dot("dot_partial_pAp", "dot_final_pAp", p, ap, f"pAp{it}")
        alpha = newbuf(f"alpha{it}", 8)
        pb.add_instance(K["scalar_alpha"], 1, 32, ptr_words(rr) + ptr_words(pap) + ptr_words(alpha))
        last = it == iters - 1
        xn = newbuf(f"x{it + 1}", 8 * n, output=last)
        pb.add_instance(K["axpy_x"], grid, 256, ptr_words(x) + ptr_words(p) + ptr_words(alpha) + ptr_words(xn) + [n])
        rn = newbuf(f"r{it + 1}", 8 * n)
        pb.add_instance(K["axpy_r"], grid, 256, ptr_words(r) + ptr_words(ap) + ptr_words(alpha) + ptr_words(rn) + [n])
        rrn = dot("dot_partial_rr", "dot_final_rr", rn, rn, f"rr{it + 1}")
        beta = newbuf(f"beta{it}", 8)
        pb.add_instance(K["scalar_beta"], 1, 32, ptr_words(rrn) + ptr_words(rr) + ptr_words(beta))
        pn = newbuf(f"p{it + 1}", 8 * n)
        pb.add_instance(K["xpay_p"], grid, 256, ptr_words(rn) + ptr_words(p) + ptr_words(beta) + ptr_words(pn) + [n])
        x, r, p, rr = xn, rn, pn, rrn
    return pb.build(config="C3", nx=nx, ny=ny, iters=iters, n=n)


def c3(full: bool = True) -> Program:
    return cg_program(512, 256, 500) if full else cg_program(32, 16, 6)


def scatter_chain(n_inst: int = 4, n: int = 256, block: int = 64, seed: int = 91) -> Program:
    """x_{i+1}[perm_i[j]] = 0.5 * x_i[j] + 1 and perm_{i+1}[j] = perm_i[j] over n_inst
    launches: data-dependent store addresses, so a corrupted index makes a warp
    store where another warp (or another buffer) does — wild stores whose order
    C-14 fixes — or fault (DUE), in later launches too."""
    s = Asm()
    s.s2r(0, isa.SR_TID)
    s.s2r(1, isa.SR_CTAID)
    s.s2r(2, isa.SR_NTID)
    s.imad(0, 1, 2, 0)
    s.ldc(3, 32)
    s.isetp(0, 0, 3, cmp=isa.GE)
    s.exit(guard=0)
    s.ldc(4, 0, wide=True)                             # perm_i
    s.imad_wide(4, 0, imm=4, c=4, unsigned=True)
    s.ldc(6, 8, wide=True)                             # x_i
    s.imad_wide(6, 0, imm=4, c=6, unsigned=True)
    s.ldg(12, 4)                                       # p = perm_i[j]
    s.ldg(13, 6)                                       # v = x_i[j]
    s.ldc(14, 36)                                      # 0.5
    s.ldc(15, 40)                                      # 1.0
    s.ffma(13, 13, 14, 15)
    s.ldc(8, 16, wide=True)                            # x_{i+1}
    s.imad_wide(8, 12, imm=4, c=8, unsigned=True)
    s.stg(8, 13)
    s.ldc(10, 24, wide=True)                           # perm_{i+1}
    s.imad_wide(10, 0, imm=4, c=10, unsigned=True)
    s.stg(10, 12)
    s.exit()
    rng = np.random.Generator(np.random.PCG64(seed))
    pb = ProgramBuilder(f"scatter_chain_{n_inst}")
    k = pb.add_kernel("scatter", s.assemble(), nregs=16)
    perm = pb.add_buffer("perm0", 4 * n, rng.permutation(n).astype(np.uint32).view(np.float32), dtype=isa.DT_U32)
    x = pb.add_buffer("x0", 4 * n, f32_data(seed, n), dtype=isa.DT_F32)
    grid = (n + block - 1) // block
    for i in range(n_inst):
        last = i == n_inst - 1
        xn = pb.add_buffer(f"x{i + 1}", 4 * n, writer=i, output=last, dtype=isa.DT_F32)
        pn = pb.add_buffer(f"perm{i + 1}", 4 * n, writer=i, output=last, dtype=isa.DT_U32)
        pb.add_instance(k, grid, block, ptr_words(perm) + ptr_words(x) + ptr_words(xn) + ptr_words(pn)
                        + [n, isa.f32_bits(0.5), isa.f32_bits(1.0)])
        perm, x = pn, xn
    return pb.build(config="scatter_chain", n_inst=n_inst, n=n)
