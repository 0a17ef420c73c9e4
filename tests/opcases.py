"""Per-opcode conformance programs with independently computed expectations.

Each case is a one-warp-per-32-threads kernel: thread t loads 8 words
X[t*8 .. t*8+7] into R0..R7, runs the instruction(s) under test, and stores
R8..R11 and a predicate word to Y[t*8 ..].  The expected Y is computed here
from numpy's IEEE arithmetic (a library routine) or exact rational arithmetic
(FFMA/DFMA: Fraction, rounded to nearest-even by hand), and from Python
integers for the integer ops — following the semantics written in DESIGN.md §3
(C-13 for NaN / FTZ / F2I / FMNMX readings).  Used by the oracle pins (CPU) and
again by the GPU parity tests.
"""
from __future__ import annotations

import math
from fractions import Fraction

import numpy as np

from fi_inputs import isa
from fi_inputs.isa import Asm, RZ, PT, NEG
from fi_inputs.program import ProgramBuilder, ptr_words

QNAN32, QNAN64 = 0x7FFFFFFF, 0x7FFFFFFFFFFFFFFF
M32 = 0xFFFFFFFF
SPEC32 = [0x00000000, 0x80000000, 0x7F800000, 0xFF800000, 0x7FC00000, 0xFFC00001, 0x00000001,
          0x807FFFFF, 0x00800000, 0x3F800000, 0xBF800000, 0x4B000000, 0xCF000000, 0x4F000000,
          0x7F7FFFFF, 0x34000000, 0x3EFFFFFF, 0x4EFFFFFF, 0xCF000001]
SPEC64 = [0x0, 0x8000000000000000, 0x7FF0000000000000, 0xFFF0000000000000, 0x7FF8000000000000,
          0x1, 0x3FF0000000000000, 0xBFF0000000000000, 0x7FEFFFFFFFFFFFFF, 0x0010000000000000,
          0x41E0000000000000, 0xC1E0000000000000, 0x3CA0000000000000]
NTHREADS = 64


def build(rows, words: np.ndarray, name="opcase"):
    """rows: encoded insns operating on R0..R7 (inputs) -> R8..R11, P0..P5."""
    s = Asm()
    s.s2r(20, isa.SR_TID)
    s.s2r(21, isa.SR_CTAID)
    s.s2r(22, isa.SR_NTID)
    s.imad(20, 21, 22, 20)
    s.ldc(24, 0, wide=True)
    s.imad_wide(24, 20, imm=32, c=24, unsigned=True)
    s.ldg(0, 24, 0, isa.W128)
    s.ldg(4, 24, 16, isa.W128)
    s.rows.extend(rows)
    s.ldc(26, 8, wide=True)
    s.imad_wide(26, 20, imm=32, c=26, unsigned=True)
    s.stg(26, 8, 0, isa.W128)
    s.mov(12, imm=0)
    for p in range(6):
        s.sel(13, RZ, RZ, p | NEG, imm=1 << p)        # !P ? 0 : bit -> (P ? bit : 0) via negate
        s.iadd3(12, 12, 13)
    s.stg(26, 12, 16)
    s.exit()
    pb = ProgramBuilder(name)
    k = pb.add_kernel(name, s.assemble(), nregs=32)
    n = words.shape[0]
    x = pb.add_buffer("X", 32 * n, words.astype("<u4"))
    y = pb.add_buffer("Y", 32 * n, writer=0, output=True)
    pb.add_instance(k, n // 32, 32, ptr_words(x) + ptr_words(y))
    return pb.build(config="opcase")


# ---------------------------------------------------------------------------
# exact arithmetic helpers
# ---------------------------------------------------------------------------
def f32(b):
    return float(np.array([b], dtype="<u4").view("<f4")[0])


def f64(b):
    return float(np.array([b], dtype="<u8").view("<f8")[0])


def bits32(x: float) -> int:
    v = np.array([x], dtype="<f4")
    return QNAN32 if np.isnan(v[0]) else int(v.view("<u4")[0])


def bits64(x: float) -> int:
    v = np.array([x], dtype="<f8")
    return QNAN64 if np.isnan(v[0]) else int(v.view("<u8")[0])


def round_fraction(x: Fraction, mant: int, emin: int, emax: int):
    """Round exact nonzero x to a binary format with `mant` fraction bits,
    round-to-nearest-even.  Returns (sign, biased_exp, fraction), or
    (sign, None, None) on overflow to infinity."""
    sign = 1 if x < 0 else 0
    a = -x if x < 0 else x
    e = a.numerator.bit_length() - a.denominator.bit_length()   # 2^e <= a < 2^(e+1)
    if Fraction(2) ** e > a:
        e -= 1
    elif Fraction(2) ** (e + 1) <= a:
        e += 1
    e = max(e, emin)                               # subnormals share emin's quantum
    q = a / Fraction(2) ** (e - mant)
    n = q.numerator // q.denominator
    r = q - n
    if r > Fraction(1, 2) or (r == Fraction(1, 2) and n % 2 == 1):
        n += 1
    if n >= 2 ** (mant + 1):                       # carry into the next binade
        n //= 2
        e += 1
    if e > emax:
        return sign, None, None
    if n < 2 ** mant:                              # subnormal
        return sign, 0, n
    return sign, e - emin + 1, n - 2 ** mant


def exact_fma(a, b, c, fmt):
    """fma(a, b, c) correctly rounded; fmt = 32 or 64; operands as Python floats."""
    mant, emin, emax, total = (23, -126, 127, 32) if fmt == 32 else (52, -1022, 1023, 64)
    if any(math.isnan(v) for v in (a, b, c)):
        return QNAN32 if fmt == 32 else QNAN64
    prod_inf = math.isinf(a) or math.isinf(b)
    if prod_inf:
        if a == 0 or b == 0:
            return QNAN32 if fmt == 32 else QNAN64
        ps = math.copysign(1, a) * math.copysign(1, b)
        if math.isinf(c) and math.copysign(1, c) != ps:
            return QNAN32 if fmt == 32 else QNAN64
        return _pack(0 if ps > 0 else 1, None, total, mant)
    if math.isinf(c):
        return _pack(0 if c > 0 else 1, None, total, mant)
    p = Fraction(a) * Fraction(b)
    x = p + Fraction(c)
    if x == 0:
        psign = (math.copysign(1, a) * math.copysign(1, b)) < 0
        neg = (p == 0 and c == 0 and psign and math.copysign(1, c) < 0)
        return (1 << (total - 1)) if neg else 0
    sign, be, fr = round_fraction(x, mant, emin, emax)
    if be is None:
        return _pack(sign, None, total, mant)
    return (sign << (total - 1)) | (be << mant) | fr


def _pack(sign, _, total, mant):
    exp_all = (1 << (total - 1 - mant)) - 1
    return (sign << (total - 1)) | (exp_all << mant)


# ---------------------------------------------------------------------------
# cases: (name, rows, words[NTHREADS, 8], expected fn(words) -> Y[NTHREADS, 8])
# ---------------------------------------------------------------------------
def rand_words(rng, spec=SPEC32, p=0.3):
    w = rng.integers(0, 2**32, size=(NTHREADS, 8), dtype=np.uint64).astype(np.uint32)
    m = rng.random(w.shape) < p
    w[m] = rng.choice(np.array(spec, dtype=np.uint32), size=int(m.sum()))
    return w


def rand_words64(rng, p=0.3):
    w = rng.integers(0, 2**32, size=(NTHREADS, 8), dtype=np.uint64).astype(np.uint32)
    # make pairs (0,1),(2,3),(4,5) special sometimes
    for pr in (0, 2, 4):
        m = rng.random(NTHREADS) < p
        v = rng.choice(np.array(SPEC64, dtype=np.uint64), size=NTHREADS)
        w[m, pr] = (v[m] & M32).astype(np.uint32)
        w[m, pr + 1] = (v[m] >> np.uint64(32)).astype(np.uint32)
    # moderate-magnitude doubles so FMA paths are exercised without overflow
    for pr in (0, 2, 4):
        m = rng.random(NTHREADS) < 0.4
        v = np.array([bits64(float(x)) for x in rng.standard_normal(NTHREADS)], dtype=np.uint64)
        w[m, pr] = (v[m] & M32).astype(np.uint32)
        w[m, pr + 1] = (v[m] >> np.uint64(32)).astype(np.uint32)
    return w


def out_words(r8=None, r9=None, r10=None, r11=None, pw=0):
    return [r8 or 0, r9 or 0, r10 or 0, r11 or 0, pw, 0, 0, 0]


def _pair(w, i):
    return int(w[i]) | (int(w[i + 1]) << 32)


def _fmnmx(a, b, is_max):
    x, y = f32(a), f32(b)
    if math.isnan(x) and math.isnan(y):
        return QNAN32
    if math.isnan(x):
        return b
    if math.isnan(y):
        return a
    if x == y:
        xneg = a >> 31
        if is_max:
            return b if xneg else a
        return a if xneg else b
    if is_max:
        return a if x > y else b
    return a if x < y else b


def _cmp(x, y, c):
    return [x < y, x <= y, x > y, x >= y, x == y, x != y][c]


def _s32(x):
    return x - (1 << 32) if x >> 31 else x


def _lop3(a, b, c, lut):
    r = 0
    for i in range(8):
        if (lut >> i) & 1:
            r |= (a if i & 4 else ~a) & (b if i & 2 else ~b) & (c if i & 1 else ~c)
    return r & M32


def _f2i(a):
    x = f32(a)
    if math.isnan(x):
        return 0
    if x >= 2147483648.0:
        return 0x7FFFFFFF
    if x < -2147483648.0:
        return 0x80000000
    return int(x) & M32        # int() truncates toward zero


def cases(seed=0):
    rng = np.random.Generator(np.random.PCG64(seed))
    A = Asm
    out = []

    def add(name, rows, words, fn):
        exp = np.array([fn(w, t) for t, w in enumerate(words)], dtype=np.uint64).astype(np.uint32)
        out.append((name, rows, words, exp))

    def rows_of(f):
        s = A()
        f(s)
        return s.rows

    # FP32 binary ops with negation modifiers
    for opname, op in (("FADD", np.add), ("FMUL", np.multiply)):
        for mod in range(4):
            w = rand_words(rng)
            em = getattr(A(), opname.lower())
            rows = rows_of(lambda s, em=opname.lower(), mod=mod: getattr(s, em)(8, 0, 1, nega=bool(mod & 1), negb=bool(mod & 2)))
            def fn(w, t, op=op, mod=mod):
                a = np.array([w[0] ^ (0x80000000 if mod & 1 else 0)], "<u4").view("<f4")
                b = np.array([w[1] ^ (0x80000000 if mod & 2 else 0)], "<u4").view("<f4")
                with np.errstate(all="ignore"):
                    return out_words(bits32(op(a, b)[0]))
            add(f"{opname}.m{mod}", rows, w, fn)
    # FFMA (exact rational rounding)
    for mod in (0, 1, 2, 4, 7):
        w = rand_words(rng)
        rows = rows_of(lambda s, mod=mod: s.ffma(8, 0, 1, 2, nega=bool(mod & 1), negb=bool(mod & 2), negc=bool(mod & 4)))
        def fn(w, t, mod=mod):
            a = f32(int(w[0]) ^ (0x80000000 if mod & 1 else 0))
            b = f32(int(w[1]) ^ (0x80000000 if mod & 2 else 0))
            c = f32(int(w[2]) ^ (0x80000000 if mod & 4 else 0))
            return out_words(exact_fma(a, b, c, 32))
        add(f"FFMA.m{mod}", rows, w, fn)
    # FFMA with small-integer-scaled operands where fma != mul+add
    w = rng.integers(0, 2**32, size=(NTHREADS, 8), dtype=np.uint64).astype(np.uint32)
    for t in range(NTHREADS):
        a = 1.0 + (t + 1) * 2.0**-23
        w[t, 0] = bits32(a)
        w[t, 1] = bits32(a)
        w[t, 2] = bits32(-float(np.float32(a * a)))
    add("FFMA.fused", rows_of(lambda s: s.ffma(8, 0, 1, 2)), w,
        lambda w, t: out_words(exact_fma(f32(w[0]), f32(w[1]), f32(w[2]), 32)))
    # FMNMX
    for is_max in (False, True):
        w = rand_words(rng, p=0.6)
        w[:8, 0] = [0, 0x80000000, 0, 0x80000000, 0x7FC00000, 0x7FC00000, 0x3F800000, 0xFFC00001]
        w[:8, 1] = [0x80000000, 0, 0, 0x80000000, 0x7FC00001, 0x3F800000, 0x7FC00000, 0xBF800000]
        add(f"FMNMX.{'max' if is_max else 'min'}", rows_of(lambda s, m=is_max: s.fmnmx(8, 0, 1, is_max=m)), w,
            lambda w, t, m=is_max: out_words(_fmnmx(int(w[0]), int(w[1]), m)))
    # FP64
    for opname, op in (("DADD", np.add), ("DMUL", np.multiply)):
        for mod in (0, 1, 2, 3):
            w = rand_words64(rng)
            rows = rows_of(lambda s, em=opname.lower(), mod=mod: getattr(s, em)(8, 0, 2, nega=bool(mod & 1), negb=bool(mod & 2)))
            def fn(w, t, op=op, mod=mod):
                a = np.array([_pair(w, 0) ^ ((1 << 63) if mod & 1 else 0)], "<u8").view("<f8")
                b = np.array([_pair(w, 2) ^ ((1 << 63) if mod & 2 else 0)], "<u8").view("<f8")
                with np.errstate(all="ignore"):
                    r = bits64(op(a, b)[0])
                return out_words(r & M32, r >> 32)
            add(f"{opname}.m{mod}", rows, w, fn)
    for mod in (0, 4, 3):
        w = rand_words64(rng)
        rows = rows_of(lambda s, mod=mod: s.dfma(8, 0, 2, 4, nega=bool(mod & 1), negb=bool(mod & 2), negc=bool(mod & 4)))
        def fn(w, t, mod=mod):
            a = f64(_pair(w, 0) ^ ((1 << 63) if mod & 1 else 0))
            b = f64(_pair(w, 2) ^ ((1 << 63) if mod & 2 else 0))
            c = f64(_pair(w, 4) ^ ((1 << 63) if mod & 4 else 0))
            r = exact_fma(a, b, c, 64)
            return out_words(r & M32, r >> 32)
        add(f"DFMA.m{mod}", rows, w, fn)
    # compares
    for c in range(6):
        w = rand_words(rng, p=0.5)
        w[::3, 1] = w[::3, 0]
        add(f"ISETP.s.{c}", rows_of(lambda s, c=c: s.isetp(0, 0, 1, cmp=c)), w,
            lambda w, t, c=c: out_words(pw=int(_cmp(_s32(int(w[0])), _s32(int(w[1])), c))))
        add(f"ISETP.u.{c}", rows_of(lambda s, c=c: s.isetp(1, 0, 1, cmp=c, unsigned=True)), w,
            lambda w, t, c=c: out_words(pw=int(_cmp(int(w[0]), int(w[1]), c)) << 1))
        add(f"FSETP.{c}", rows_of(lambda s, c=c: s.fsetp(2, 0, 1, cmp=c)), w,
            lambda w, t, c=c: out_words(pw=(int(not (math.isnan(f32(w[0])) or math.isnan(f32(w[1])))
                                                 and _cmp(f32(w[0]), f32(w[1]), c)) << 2)))
        w2 = rand_words64(rng)
        w2[::4, 2:4] = w2[::4, 0:2]
        add(f"DSETP.{c}", rows_of(lambda s, c=c: s.dsetp(5, 0, 2, cmp=c)), w2,
            lambda w, t, c=c: out_words(pw=(int(not (math.isnan(f64(_pair(w, 0))) or math.isnan(f64(_pair(w, 2))))
                                                 and _cmp(f64(_pair(w, 0)), f64(_pair(w, 2)), c)) << 5)))
    # MUFU.RCP64: correctly rounded 1/x (Python float division is IEEE RN)
    w2 = rand_words64(rng)
    def rcp(w, t):
        x = f64(_pair(w, 0))
        if x == 0.0:
            r = bits64(math.copysign(math.inf, x))
        elif math.isnan(x):
            r = QNAN64
        else:
            r = bits64(1.0 / x)
        return out_words(r & M32, r >> 32)
    add("MUFU.RCP64", rows_of(lambda s: s.mufu_rcp64(8, 0)), w2, rcp)
    # conversions
    w = rand_words(rng, p=0.5)
    w[:6, 0] = [0x7FFFFFFF, 0x80000000, 0xFFFFFFFF, 16777217, 0x4F000000, 0xCF000001]
    add("I2F.s32", rows_of(lambda s: s.i2f(8, 0)), w,
        lambda w, t: out_words(bits32(np.float32(np.int32(np.uint32(w[0]).view(np.int32))))))
    add("I2F.u32", rows_of(lambda s: s.i2f(8, 0, unsigned=True)), w,
        lambda w, t: out_words(bits32(np.float32(np.uint32(w[0])))))
    add("F2I", rows_of(lambda s: s.f2i(8, 0)), w, lambda w, t: out_words(_f2i(int(w[0]))))
    def f2f64(w, t):
        r = bits64(float(np.float64(np.array([w[0]], "<u4").view("<f4")[0])))
        return out_words(r & M32, r >> 32)
    add("F2F.F64.F32", rows_of(lambda s: s.f2f_f64_f32(8, 0)), w, f2f64)
    w2 = rand_words64(rng)
    add("F2F.F32.F64", rows_of(lambda s: s.f2f_f32_f64(8, 0)), w2,
        lambda w, t: out_words(bits32(np.array([_pair(w, 0)], "<u8").view("<f8").astype("<f4")[0])))
    # integer ALU
    w = rand_words(rng, p=0.2)
    for neg in range(4):
        add(f"IADD3.carry.n{neg}", rows_of(lambda s, neg=neg: s.iadd3(8, 0, 1, 2, nega=bool(neg & 1), negb=bool(neg & 2), carry=3)), w,
            lambda w, t, neg=neg: (lambda sm: out_words(sm & M32, pw=int((sm >> 32) != 0) << 3))(
                ((-int(w[0])) & M32 if neg & 1 else int(w[0])) + ((-int(w[1])) & M32 if neg & 2 else int(w[1])) + int(w[2])))
    add("IADD3.imm", rows_of(lambda s: s.iadd3(8, 0, imm=0xFFFFFFF0, c=2)), w,
        lambda w, t: out_words((int(w[0]) + 0xFFFFFFF0 + int(w[2])) & M32))
    add("IMAD", rows_of(lambda s: s.imad(8, 0, 1, 2)), w, lambda w, t: out_words((int(w[0]) * int(w[1]) + int(w[2])) & M32))
    add("IMAD.WIDE.s", rows_of(lambda s: s.imad_wide(8, 0, 1, 2)), w,
        lambda w, t: (lambda r: out_words(r & M32, r >> 32))((_s32(int(w[0])) * _s32(int(w[1])) + _pair(w, 2)) % 2**64))
    add("IMAD.WIDE.u", rows_of(lambda s: s.imad_wide(8, 0, 1, 2, unsigned=True)), w,
        lambda w, t: (lambda r: out_words(r & M32, r >> 32))((int(w[0]) * int(w[1]) + _pair(w, 2)) % 2**64))
    add("IMAD.WIDE.rz", rows_of(lambda s: s.imad_wide(8, 0, imm=0xFFFFFFFE, c=RZ)), w,
        lambda w, t: (lambda r: out_words(r & M32, r >> 32))((_s32(int(w[0])) * -2) % 2**64))
    ws = w.copy()
    ws[:, 1] = rng.integers(0, 40, size=NTHREADS)
    for mode in range(3):
        def shf(w, t, mode=mode):
            a, sh = int(w[0]), min(int(w[1]), 32)
            if mode == 0:
                return out_words(0 if sh >= 32 else (a << sh) & M32)
            if mode == 1:
                return out_words(0 if sh >= 32 else a >> sh)
            return out_words((_s32(a) >> min(sh, 31)) & M32 if sh < 32 else (M32 if a >> 31 else 0))
        add(f"SHF.{mode}", rows_of(lambda s, mode=mode: s.shf(8, 0, 1, mode=mode)), ws, shf)
    for lut in (0x00, 0xFF, 0xC0, 0xFC, 0x3C, 0x96, 0xE8, 0x1B, int(rng.integers(0, 256))):
        add(f"LOP3.{lut:02x}", rows_of(lambda s, lut=lut: s.lop3(8, 0, 1, 2, lut)), w,
            lambda w, t, lut=lut: out_words(_lop3(int(w[0]), int(w[1]), int(w[2]), lut)))
    for um in range(4):
        def mnmx(w, t, um=um):
            a, b = int(w[0]), int(w[1])
            if um & 2:
                v = max(a, b) if um & 1 else min(a, b)
            else:
                v = (max(_s32(a), _s32(b)) if um & 1 else min(_s32(a), _s32(b))) & M32
            return out_words(v)
        add(f"IMNMX.{um}", rows_of(lambda s, um=um: s.imnmx(8, 0, 1, is_max=bool(um & 1), unsigned=bool(um & 2))), w, mnmx)
    # SEL on a data-dependent predicate; MOV; S2R
    add("SEL", rows_of(lambda s: (s.isetp(4, 0, 1, cmp=isa.LT, unsigned=True), s.sel(8, 0, 1, 4), s.sel(9, 0, 1, 4 | NEG))), w,
        lambda w, t: out_words(int(w[0]) if int(w[0]) < int(w[1]) else int(w[1]),
                               int(w[1]) if int(w[0]) < int(w[1]) else int(w[0]),
                               pw=int(int(w[0]) < int(w[1])) << 4))
    add("MOV", rows_of(lambda s: (s.mov(8, b=3), s.mov(9, imm=0xDEADBEEF), s.mov(10, b=RZ))), w,
        lambda w, t: out_words(int(w[3]), 0xDEADBEEF, 0))
    add("S2R", rows_of(lambda s: (s.s2r(8, isa.SR_TID), s.s2r(9, isa.SR_CTAID), s.s2r(10, isa.SR_LANEID),
                                  s.s2r(11, isa.SR_NCTAID))), w,
        lambda w, t: out_words(t % 32, t // 32, t % 32, NTHREADS // 32))
    # SHFL (reads the source lane's register)
    wl = w.copy()
    wl[:, 1] = rng.integers(0, 64, size=NTHREADS)
    for mode in range(4):
        def shfl(w, t, mode=mode, W=wl):
            lane, base = t % 32, t - t % 32
            b = int(w[1])
            src = [b & 31, lane ^ (b & 31), lane + b if lane + b <= 31 else lane, lane - b if lane - b >= 0 else lane][mode]
            return out_words(int(W[base + src, 0]))
        add(f"SHFL.{mode}", rows_of(lambda s, mode=mode: s.shfl(8, 0, 1, mode=mode)), wl, shfl)
    add("SHFL.imm", rows_of(lambda s: s.shfl(8, 0, imm=5, mode=isa.SHFL_BFLY)), wl,
        lambda w, t, W=wl: out_words(int(W[t - t % 32 + ((t % 32) ^ 5), 0])))
    # guarded execution: only lanes where P0 (= R0 < R1 unsigned) execute
    add("GUARD", rows_of(lambda s: (s.isetp(0, 0, 1, cmp=isa.LT, unsigned=True), s.mov(8, b=2, guard=0),
                                    s.mov(9, b=3, guard=0 | NEG))), w,
        lambda w, t: out_words(int(w[2]) if int(w[0]) < int(w[1]) else 0, 0 if int(w[0]) < int(w[1]) else int(w[3]),
                               pw=int(int(w[0]) < int(w[1]))))
    # register RZ / PT discards
    add("RZPT", rows_of(lambda s: (s.mov(RZ, b=0), s.isetp(PT, 0, 1, cmp=isa.EQ), s.mov(8, b=RZ))), w,
        lambda w, t: out_words(0))
    return out
