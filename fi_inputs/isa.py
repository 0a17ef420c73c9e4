"""Mini-SASS instruction *encoding* (the input format only).

This module is part of the seeded input generators shared by the oracle and
the CUDA path.  It fixes how a synthetic program is written down (opcode
numbers, operand fields, modifier bits) and nothing else: it holds none of the
method's arithmetic — no instruction-group classification (Table II,
PAPER.md:94-104), no destination-slot rule, no execution semantics.  Those are
implemented independently in ``oracle/`` and in the CUDA library, from the
semantics written out in DESIGN.md §3.

Static instruction, 16 bytes, little endian:

    byte 0  op      opcode number (below)
    byte 1  guard   bits 0-2 predicate index (7 = PT), bit 3 negate
    byte 2  d0      first destination (GP register, or predicate for *SETP)
    byte 3  d1      IADD3 carry-out predicate (7 = none)
    byte 4  a       source a
    byte 5  b       source b (or the immediate when MOD_BIMM is set)
    byte 6  c       source c (SEL: predicate index, bit 3 negate)
    byte 7  mod     opcode modifiers
    bytes 8-11  imm   u32 immediate
    bytes 12-15 ext   u32 (LOP3 truth table in the low byte)
"""
from __future__ import annotations

import numpy as np

# ---- opcode numbers -------------------------------------------------------
NOP, EXIT, BRA, MOV, S2R, IADD3, IMAD, IMAD_WIDE, SHF, LOP3, SEL = range(11)
ISETP, FSETP, DSETP, FADD, FMUL, FFMA, FMNMX, DADD, DMUL, DFMA = range(11, 21)
LDG, LDC, STG, I2F, F2I, F2F_F64_F32, F2F_F32_F64, SHFL, IMNMX = range(21, 30)
MUFU_RCP64 = 30
N_OPCODES = 31

OPNAMES = [
    "NOP", "EXIT", "BRA", "MOV", "S2R", "IADD3", "IMAD", "IMAD.WIDE", "SHF", "LOP3", "SEL",
    "ISETP", "FSETP", "DSETP", "FADD", "FMUL", "FFMA", "FMNMX", "DADD", "DMUL", "DFMA",
    "LDG", "LDC", "STG", "I2F", "F2I", "F2F.F64.F32", "F2F.F32.F64", "SHFL", "IMNMX", "MUFU.RCP64",
]

RZ = 127          # zero register: reads 0, writes discarded
PT = 7            # true predicate: reads 1, writes discarded
NEG = 8           # guard / SEL predicate negate bit

# ---- modifier bits --------------------------------------------------------
MOD_BIMM = 0x80   # operand b is `imm`
# FADD/FMUL/FFMA/DADD/DMUL/DFMA: negate a/b/c ; IADD3: negate a/b
MOD_NEGA, MOD_NEGB, MOD_NEGC = 0x01, 0x02, 0x04
# IMAD.WIDE / I2F / ISETP / IMNMX unsigned
MOD_U32_WIDE = 0x01     # IMAD.WIDE.U32, I2F.U32
MOD_CMP_U32 = 0x08      # ISETP / IMNMX unsigned
# comparison codes (ISETP/FSETP/DSETP mod bits 0-2)
LT, LE, GT, GE, EQ, NE = range(6)
# SHF mode (mod bits 0-1)
SHF_L, SHF_R_U32, SHF_R_S32 = 0, 1, 2
# FMNMX / IMNMX
MOD_MAX = 0x01
# LDG/STG width (mod bits 0-1): 4, 8, 16 bytes
W32, W64, W128 = 0, 1, 2
# LDC width
MOD_LDC64 = 0x01
# SHFL mode (mod bits 0-1)
SHFL_IDX, SHFL_BFLY, SHFL_DOWN, SHFL_UP = 0, 1, 2, 3
# S2R special registers (imm)
SR_TID, SR_CTAID, SR_NTID, SR_NCTAID, SR_LANEID, SR_WARPID = range(6)

# ---- record / buffer format constants ----------------
VA_BASE = 0x00007F0000000000
ALLOC_ALIGN = 256
BUF_OUTPUT = 0x1
DT_U32, DT_F32, DT_F64 = 0, 1, 2

INSN_DTYPE = np.dtype([
    ("op", "u1"), ("guard", "u1"), ("d0", "u1"), ("d1", "u1"),
    ("a", "u1"), ("b", "u1"), ("c", "u1"), ("mod", "u1"),
    ("imm", "<u4"), ("ext", "<u4"),
])
assert INSN_DTYPE.itemsize == 16


def insn(op, d0=RZ, a=RZ, b=RZ, c=RZ, *, d1=PT, mod=0, imm=0, ext=0, guard=PT):
    """One encoded instruction as a tuple for INSN_DTYPE."""
    return (op, guard, d0, d1, a, b, c, mod, imm & 0xFFFFFFFF, ext & 0xFFFFFFFF)


def f32_bits(x: float) -> int:
    return int(np.array([x], dtype="<f4").view("<u4")[0])


class Asm:
    """Tiny assembler: appends encoded instructions, resolves labels."""

    def __init__(self):
        self.rows: list[tuple] = []
        self.labels: dict[str, int] = {}
        self.fixups: list[tuple[int, str]] = []

    @property
    def pc(self) -> int:
        return len(self.rows)

    def label(self, name: str):
        self.labels[name] = self.pc

    def emit(self, op, **kw):
        self.rows.append(insn(op, **kw))
        return self

    # mnemonics ----------------------------------------------------------
    def nop(self, guard=PT):
        return self.emit(NOP, guard=guard)

    def exit(self, guard=PT):
        return self.emit(EXIT, guard=guard)

    def bra(self, target: str, guard=PT):
        self.fixups.append((self.pc, target))
        return self.emit(BRA, guard=guard)

    def mov(self, d, b=None, imm=None, guard=PT):
        if imm is not None:
            return self.emit(MOV, d0=d, mod=MOD_BIMM, imm=imm, guard=guard)
        return self.emit(MOV, d0=d, b=b, guard=guard)

    def s2r(self, d, sr, guard=PT):
        return self.emit(S2R, d0=d, imm=sr, guard=guard)

    def iadd3(self, d, a, b=RZ, c=RZ, imm=None, nega=False, negb=False, carry=PT, guard=PT):
        mod = (MOD_NEGA if nega else 0) | (MOD_NEGB if negb else 0)
        if imm is not None:
            mod |= MOD_BIMM
        return self.emit(IADD3, d0=d, d1=carry, a=a, b=b, c=c, mod=mod, imm=imm or 0, guard=guard)

    def imad(self, d, a, b=RZ, c=RZ, imm=None, guard=PT):
        mod = MOD_BIMM if imm is not None else 0
        return self.emit(IMAD, d0=d, a=a, b=b, c=c, mod=mod, imm=imm or 0, guard=guard)

    def imad_wide(self, d, a, b=RZ, c=RZ, imm=None, unsigned=False, guard=PT):
        mod = (MOD_BIMM if imm is not None else 0) | (MOD_U32_WIDE if unsigned else 0)
        return self.emit(IMAD_WIDE, d0=d, a=a, b=b, c=c, mod=mod, imm=imm or 0, guard=guard)

    def shf(self, d, a, b=RZ, imm=None, mode=SHF_L, guard=PT):
        mod = (MOD_BIMM if imm is not None else 0) | mode
        return self.emit(SHF, d0=d, a=a, b=b, mod=mod, imm=imm or 0, guard=guard)

    def lop3(self, d, a, b, c, lut, imm=None, guard=PT):
        mod = MOD_BIMM if imm is not None else 0
        return self.emit(LOP3, d0=d, a=a, b=b, c=c, ext=lut, mod=mod, imm=imm or 0, guard=guard)

    def sel(self, d, a, b, p, imm=None, guard=PT):
        mod = MOD_BIMM if imm is not None else 0
        return self.emit(SEL, d0=d, a=a, b=b, c=p, mod=mod, imm=imm or 0, guard=guard)

    def isetp(self, p, a, b=RZ, cmp=LT, imm=None, unsigned=False, guard=PT):
        mod = cmp | (MOD_CMP_U32 if unsigned else 0) | (MOD_BIMM if imm is not None else 0)
        return self.emit(ISETP, d0=p, a=a, b=b, mod=mod, imm=imm or 0, guard=guard)

    def fsetp(self, p, a, b, cmp=LT, guard=PT):
        return self.emit(FSETP, d0=p, a=a, b=b, mod=cmp, guard=guard)

    def dsetp(self, p, a, b, cmp=LT, guard=PT):
        return self.emit(DSETP, d0=p, a=a, b=b, mod=cmp, guard=guard)

    def _fp(self, op, d, a, b, c=RZ, nega=False, negb=False, negc=False, imm=None, guard=PT):
        mod = (MOD_NEGA if nega else 0) | (MOD_NEGB if negb else 0) | (MOD_NEGC if negc else 0)
        if imm is not None:
            mod |= MOD_BIMM
        return self.emit(op, d0=d, a=a, b=b, c=c, mod=mod, imm=imm or 0, guard=guard)

    def fadd(self, d, a, b, **kw):
        return self._fp(FADD, d, a, b, **kw)

    def fmul(self, d, a, b, **kw):
        return self._fp(FMUL, d, a, b, **kw)

    def ffma(self, d, a, b, c, **kw):
        return self._fp(FFMA, d, a, b, c, **kw)

    def fmnmx(self, d, a, b, is_max=False, guard=PT):
        return self.emit(FMNMX, d0=d, a=a, b=b, mod=MOD_MAX if is_max else 0, guard=guard)

    def dadd(self, d, a, b, **kw):
        return self._fp(DADD, d, a, b, **kw)

    def dmul(self, d, a, b, **kw):
        return self._fp(DMUL, d, a, b, **kw)

    def dfma(self, d, a, b, c, **kw):
        return self._fp(DFMA, d, a, b, c, **kw)

    def ldg(self, d, a, off=0, width=W32, guard=PT):
        return self.emit(LDG, d0=d, a=a, mod=width, imm=off, guard=guard)

    def ldc(self, d, byte_off, wide=False, guard=PT):
        return self.emit(LDC, d0=d, mod=MOD_LDC64 if wide else 0, imm=byte_off, guard=guard)

    def stg(self, a, b, off=0, width=W32, guard=PT):
        return self.emit(STG, a=a, b=b, mod=width, imm=off, guard=guard)

    def i2f(self, d, a, unsigned=False, guard=PT):
        return self.emit(I2F, d0=d, a=a, mod=MOD_U32_WIDE if unsigned else 0, guard=guard)

    def f2i(self, d, a, guard=PT):
        return self.emit(F2I, d0=d, a=a, guard=guard)

    def f2f_f64_f32(self, d, a, guard=PT):
        return self.emit(F2F_F64_F32, d0=d, a=a, guard=guard)

    def f2f_f32_f64(self, d, a, guard=PT):
        return self.emit(F2F_F32_F64, d0=d, a=a, guard=guard)

    def shfl(self, d, a, b=RZ, imm=None, mode=SHFL_IDX, guard=PT):
        mod = mode | (MOD_BIMM if imm is not None else 0)
        return self.emit(SHFL, d0=d, a=a, b=b, mod=mod, imm=imm or 0, guard=guard)

    def imnmx(self, d, a, b, is_max=False, unsigned=False, guard=PT):
        mod = (MOD_MAX if is_max else 0) | (MOD_CMP_U32 if unsigned else 0)
        return self.emit(IMNMX, d0=d, a=a, b=b, mod=mod, guard=guard)

    def mufu_rcp64(self, d, a, guard=PT):
        return self.emit(MUFU_RCP64, d0=d, a=a, guard=guard)

    def assemble(self) -> np.ndarray:
        code = np.array(self.rows, dtype=INSN_DTYPE)
        for pc, name in self.fixups:
            code["imm"][pc] = self.labels[name]
        return code
