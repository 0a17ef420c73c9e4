// sem.cuh — the opcode semantics of DESIGN.md §3.2 (readings C-7, C-13), ONE copy
// for both CUDA engines: emu.cuh (the shared-memory interpreter) includes it, and
// build.py embeds its text ahead of jit_prelude.cuh, so the JIT's step mode and
// the helpers its generated code calls are the same functions.  Self-contained:
// no includes (NVRTC compiles it as part of the generated program).
// Independent of oracle/ (the CPU oracle implements §3.2 on its own).
#pragma once

namespace fisem {

typedef unsigned int u32;
typedef int i32;
typedef unsigned long long u64;
typedef long long i64;

// opcode numbers of the input format
enum : u32 {
    NOP = 0, EXIT, BRA, MOV, S2R, IADD3, IMAD, IMAD_WIDE, SHF, LOP3, SEL,
    ISETP, FSETP, DSETP, FADD, FMUL, FFMA, FMNMX, DADD, DMUL, DFMA,
    LDG, LDC, STG, I2F, F2I, F2F_F64_F32, F2F_F32_F64, SHFL, IMNMX, MUFU_RCP64
};
constexpr u32 kQNaN32 = 0x7FFFFFFFu;                 // C-13: every NaN result canonicalised
constexpr u64 kQNaN64 = 0x7FFFFFFFFFFFFFFFull;

__device__ __forceinline__ float u2f(u32 x) { return __uint_as_float(x); }
__device__ __forceinline__ u32 fbits(float f) { return f != f ? kQNaN32 : __float_as_uint(f); }
__device__ __forceinline__ double u2d(u64 x) { return __longlong_as_double((long long)x); }
__device__ __forceinline__ u64 dbits(double d) { return d != d ? kQNaN64 : (u64)__double_as_longlong(d); }
__device__ __forceinline__ u64 pair(u32 lo, u32 hi) { return (u64)lo | ((u64)hi << 32); }

// FMNMX: IEEE minNum / maxNum with -0 < +0 (C-13)
__device__ __forceinline__ u32 fmnmx(u32 a, u32 b, bool mx) {
    const float x = u2f(a), y = u2f(b);
    const bool xn = x != x, yn = y != y;
    if (xn && yn) return kQNaN32;
    if (xn) return b;
    if (yn) return a;
    if (x == y) {
        const bool xneg = a >> 31;
        return mx ? (xneg ? b : a) : (xneg ? a : b);
    }
    return mx ? (x > y ? a : b) : (x < y ? a : b);
}

// comparisons LT LE GT GE EQ NE (mod & 7); floating point ones are ordered
__device__ __forceinline__ bool cmp_f(double x, double y, u32 c) {
    if (x != x || y != y) return false;
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}
__device__ __forceinline__ bool cmp_s(i32 x, i32 y, u32 c) {
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}
__device__ __forceinline__ bool cmp_u(u32 x, u32 y, u32 c) {
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}

// F2I: round toward zero, saturating, NaN -> 0 (C-13)
__device__ __forceinline__ u32 f2i(u32 a) {
    const float f = u2f(a);
    if (f != f) return 0;
    if (f >= 2147483648.0f) return 0x7FFFFFFFu;
    if (f < -2147483648.0f) return 0x80000000u;
    return (u32)__float2int_rz(f);
}

// LOP3: bit i of lut selects the minterm (i&4 ? a : ~a) & (i&2 ? b : ~b) & (i&1 ? c : ~c)
__device__ __forceinline__ u32 lop3(u32 a, u32 b, u32 c, u32 lut) {
    u32 r = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const u32 t = ((i & 4) ? a : ~a) & ((i & 2) ? b : ~b) & ((i & 1) ? c : ~c);
        r |= ((lut >> i) & 1u) ? t : 0u;
    }
    return r;
}

// SHF: s = min(b, 32); m = 0 a << s, 1 a >> s logical, 2 a >> s arithmetic
__device__ __forceinline__ u32 shf(u32 a, u32 bv, u32 m) {
    const u32 s = bv > 32 ? 32 : bv;
    if (m == 0) return s >= 32 ? 0u : a << s;
    if (m == 1) return s >= 32 ? 0u : a >> s;
    return (u32)((i32)a >> (s >= 32 ? 31 : s));
}

// SHFL source lane: IDX b&31, BFLY lane^(b&31), DOWN lane+b (> 31: own lane), UP lane-b (< 0: own lane)
__device__ __forceinline__ u32 shfl_src(u32 lane, u32 bv, u32 m) {
    i64 src;
    switch (m & 3) {
        case 0: src = bv & 31; break;
        case 1: src = lane ^ (bv & 31); break;
        case 2: src = (i64)lane + (i64)bv; if (src > 31) src = lane; break;
        default: src = (i64)lane - (i64)bv; if (src < 0) src = lane; break;
    }
    return (u32)src;
}

// guard: predicate bits 0-2 (7 = PT), bit 3 negates
__device__ __forceinline__ bool guard_of(u32 guard, u32 preds) {
    const u32 gs = guard & 7;
    return (((gs == 7) ? 1u : ((preds >> gs) & 1u)) ^ ((guard >> 3) & 1u)) != 0;
}

// One lane's column of a warp's shared-memory register file: rows of 32 lanes ×
// 4 B, register r at byte offset 128 r; the zero row (RZ, indices >= n_regs) at zb.
struct RegFile {
    char* Rb;              // (char*)(R + lane)
    u32* R;                // row 0, lane 0
    u32 zb;                // byte offset of the zero row
    __device__ __forceinline__ u32 rd(u32 o) const { return *reinterpret_cast<const u32*>(Rb + o); }
    __device__ __forceinline__ u64 rd64(u32 o) const { return (u64)rd(o) | ((u64)rd(min(o + 128u, zb)) << 32); }
    __device__ __forceinline__ void wr(u32 o, u32 v) const {
        if (o < zb) *reinterpret_cast<u32*>(Rb + o) = v;
    }
};

struct LaneCtx {
    u32 lane, cta, wic, block, grid, cbank_len;
    const u32* cb;                                   // the instance's constant bank
};

// One "plain" instruction (everything but BRA / EXIT / LDG / STG) in this lane,
// on a pre-decoded instruction D = {op | mod<<16 | pb<<24, a | b<<16, c | d<<16,
// imm} with register byte offsets.  All lanes call it together (SHFL reads the
// source lane's register even if that lane does not execute); `ex` = executes here.
__device__ __forceinline__ void exec_plain(const RegFile& F, const LaneCtx& L, const uint4 D, const bool ex,
                                           u32& preds) {
    const u32 op = D.x & 0xFF, mod = (D.x >> 16) & 0xFF, pb = D.x >> 24;
    const u32 ia = D.y & 0xFFFF, ib = D.y >> 16, ic = D.z & 0xFFFF, id = D.z >> 16;
    const u32 imm = D.w;
    const u32 bv = (mod & 0x80) ? imm : F.rd(ib);
    switch (op) {
        case FFMA: {                                 // fused (C-13); operands negated by mod bits 0/1/2
            const float x = u2f(F.rd(ia) ^ (mod << 31)), y = u2f(bv ^ ((mod & 2) << 30)),
                        z = u2f(F.rd(ic) ^ ((mod & 4) << 29));
            const u32 r = fbits(__fmaf_rn(x, y, z));
            if (ex) F.wr(id, r);
            break;
        }
        case MOV: if (ex) F.wr(id, bv); break;
        case S2R: {
            u32 v = 0;
            switch (imm) {
                case 0: v = L.wic * 32 + L.lane; break; case 1: v = L.cta; break; case 2: v = L.block; break;
                case 3: v = L.grid; break; case 4: v = L.lane; break; case 5: v = L.wic; break;
            }
            if (ex) F.wr(id, v);
            break;
        }
        case IADD3: {                                // 64-bit sum; carry-out to predicate pb
            const u32 a = F.rd(ia), c = F.rd(ic);
            const u32 x = (mod & 1) ? 0u - a : a, y = (mod & 2) ? 0u - bv : bv;
            const u64 s = (u64)x + y + c;
            if (ex) {
                F.wr(id, (u32)s);
                if (pb != 7) preds = (preds & ~(1u << pb)) | ((u32)((s >> 32) != 0) << pb);
            }
            break;
        }
        case IMAD: if (ex) F.wr(id, F.rd(ia) * bv + F.rd(ic)); break;
        case IMAD_WIDE: {                            // signed (unsigned if mod & 1) 32x32 -> 64, plus pair(c)
            const u32 a = F.rd(ia);
            const u64 prod = (mod & 1) ? (u64)a * (u64)bv : (u64)((i64)(i32)a * (i64)(i32)bv);
            const u64 r = prod + F.rd64(ic);
            if (ex) { F.wr(id, (u32)r); F.wr(id + 128, (u32)(r >> 32)); }
            break;
        }
        case SHF: { const u32 v = shf(F.rd(ia), bv, mod & 3); if (ex) F.wr(id, v); break; }
        case LOP3: if (ex) F.wr(id, lop3(F.rd(ia), bv, F.rd(ic), pb)); break;
        case SEL: {
            const u32 p = pb & 7;
            const bool s = (((p == 7) ? 1u : ((preds >> p) & 1u)) ^ ((pb >> 3) & 1u)) != 0;
            if (ex) F.wr(id, s ? F.rd(ia) : bv);
            break;
        }
        case ISETP: case FSETP: case DSETP: {
            bool v;
            const u32 c = mod & 7;
            if (op == ISETP) v = (mod & 8) ? cmp_u(F.rd(ia), bv, c) : cmp_s((i32)F.rd(ia), (i32)bv, c);
            else if (op == FSETP) v = cmp_f((double)u2f(F.rd(ia)), (double)u2f(F.rd(ib)), c);
            else v = cmp_f(u2d(F.rd64(ia)), u2d(F.rd64(ib)), c);
            if (ex && pb != 7) preds = (preds & ~(1u << pb)) | ((u32)v << pb);
            break;
        }
        case FADD: case FMUL: {                      // never contracted (C-13)
            const float x = u2f(F.rd(ia) ^ (mod << 31)), y = u2f(bv ^ ((mod & 2) << 30));
            const float r = op == FADD ? __fadd_rn(x, y) : __fmul_rn(x, y);
            if (ex) F.wr(id, fbits(r));
            break;
        }
        case FMNMX: if (ex) F.wr(id, fmnmx(F.rd(ia), bv, mod & 1)); break;
        case DADD: case DMUL: case DFMA: {
            const double x = u2d(F.rd64(ia) ^ ((u64)(mod & 1) << 63));
            const double y = u2d(F.rd64(ib) ^ ((u64)(mod & 2) << 62));
            const double z = u2d(F.rd64(ic) ^ ((u64)(mod & 4) << 61));
            const double r = op == DADD ? __dadd_rn(x, y) : op == DMUL ? __dmul_rn(x, y) : __fma_rn(x, y, z);
            const u64 b = dbits(r);
            if (ex) { F.wr(id, (u32)b); F.wr(id + 128, (u32)(b >> 32)); }
            break;
        }
        case LDC: {                                  // constant bank word(s), 0 past its end
            const u32 w0 = imm >> 2;
            if (ex) {
                F.wr(id, w0 < L.cbank_len ? __ldg(&L.cb[w0]) : 0u);
                if (mod & 1) F.wr(id + 128, w0 + 1 < L.cbank_len ? __ldg(&L.cb[w0 + 1]) : 0u);
            }
            break;
        }
        case I2F: if (ex) F.wr(id, fbits((mod & 1) ? __uint2float_rn(F.rd(ia)) : __int2float_rn((int)F.rd(ia)))); break;
        case F2I: if (ex) F.wr(id, f2i(F.rd(ia))); break;
        case F2F_F64_F32: {
            const u64 b = dbits((double)u2f(F.rd(ia)));
            if (ex) { F.wr(id, (u32)b); F.wr(id + 128, (u32)(b >> 32)); }
            break;
        }
        case F2F_F32_F64: if (ex) F.wr(id, fbits(__double2float_rn(u2d(F.rd64(ia))))); break;
        case SHFL: {
            const u32 src = shfl_src(L.lane, bv, mod & 3);
            __syncwarp();
            const u32 v = *reinterpret_cast<const u32*>(reinterpret_cast<const char*>(F.R + src) + ia);
            __syncwarp();
            if (ex) F.wr(id, v);
            break;
        }
        case MUFU_RCP64: {                           // 1/x in f64, round to nearest
            const u64 b = dbits(__drcp_rn(u2d(F.rd64(ia))));
            if (ex) { F.wr(id, (u32)b); F.wr(id + 128, (u32)(b >> 32)); }
            break;
        }
        case IMNMX: {                                // signed (unsigned if mod & 8) min / max (mod & 1)
            const u32 a = F.rd(ia);
            u32 v;
            if (mod & 8) v = (mod & 1) ? max(a, bv) : min(a, bv);
            else v = (u32)((mod & 1) ? max((i32)a, (i32)bv) : min((i32)a, (i32)bv));
            if (ex) F.wr(id, v);
            break;
        }
        default: break;                              // NOP
    }
}

}  // namespace fisem
