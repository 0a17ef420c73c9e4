// emu.cuh — warp-per-warp mini-SASS emulator, sm_100a.
//
// One CUDA warp emulates one synthetic warp: CUDA lane λ is synthetic lane λ,
// so per-lane state (pc, live, predicates) lives in registers and warp-level
// decisions (min-PC scheduling, active / pred masks) are single REDUX / VOTE
// instructions.  The 32-bit register file is a [n_regs+1][32] u32 array in
// shared memory (row n_regs is all zeros and serves RZ and any index >= n_regs),
// so every register access is one bank-conflict-free LDS/STS.
//
// Memory follows DESIGN.md §3.5: loads of instance k read the golden final
// image where the buffer's writer < k and zero where writer >= k (equivalent to
// the state before k under SSA), so neither the golden passes nor injection
// replicas ever snapshot memory.
//
// Modes:
//   EMU_LEN    golden pass 1: stores go to the image; count steps and stored words
//   EMU_TRACE  golden pass 2: write trace records (App. A.3) and the golden store log
//   EMU_INJ    injection replica: corrupt one destination after
//              the site's instruction; log stores after the site; faults end the run
#pragma once
#include "common.cuh"

namespace fi {

constexpr uint32_t kFull = 0xFFFFFFFFu;
enum EmuMode { EMU_LEN = 0, EMU_TRACE = 1, EMU_INJ = 2 };

struct EmuProg {
    const fi_insn* code;
    const fi_kernel* kern;
    const fi_instance* inst;
    const uint32_t* cbank;
    const fi_buffer* buf;
    const uint32_t* gran;
    uint64_t image_bytes;
    uint32_t n_regs;
    uint32_t n_inst;
};

inline EmuProg make_emu_prog(const fi_program* p) {
    return EmuProg{p->code, p->kern, p->inst, p->cbank, p->buf, p->gran, p->image_bytes, p->n_regs, p->n_inst};
}

struct HookIn { uint32_t step, lane, kind, reg, bfm, mask, pc; };

struct EmuOut {
    uint32_t steps = 0, fault = 0, fault_pc = 0, nstore = 0;
    uint32_t before = 0, after = 0, mask = 0;
    bool fired = false, bad = false;
};

// instance of global warp w (binary search over warp_begin)
__device__ __forceinline__ uint32_t instance_of_warp(const fi_instance* inst, uint32_t n_inst, uint32_t w) {
    uint32_t lo = 0, hi = n_inst;                 // find last k with warp_begin <= w
    while (hi - lo > 1) {
        uint32_t mid = (lo + hi) >> 1;
        if (__ldg(&inst[mid].warp_begin) <= w) lo = mid; else hi = mid;
    }
    return lo;
}

__device__ __forceinline__ float u2f(uint32_t x) { return __uint_as_float(x); }
__device__ __forceinline__ uint32_t fbits(float f) { return f != f ? kQNaN32 : __float_as_uint(f); }
__device__ __forceinline__ double u2d(uint64_t x) { return __longlong_as_double((long long)x); }
__device__ __forceinline__ uint64_t dbits(double d) { return d != d ? kQNaN64 : (uint64_t)__double_as_longlong(d); }

__device__ __forceinline__ uint32_t dev_fmnmx(uint32_t a, uint32_t b, bool mx) {
    float x = u2f(a), y = u2f(b);
    bool xn = x != x, yn = y != y;
    if (xn && yn) return kQNaN32;
    if (xn) return b;
    if (yn) return a;
    if (x == y) {                                   // +0 / -0: -0 < +0 (C-13)
        bool xneg = a >> 31;
        return mx ? (xneg ? b : a) : (xneg ? a : b);
    }
    return mx ? (x > y ? a : b) : (x < y ? a : b);
}

__device__ __forceinline__ bool dev_cmp_f(double x, double y, uint32_t c) {
    if (x != x || y != y) return false;             // ordered compares
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}
template <class T>
__device__ __forceinline__ bool dev_cmp_i(T x, T y, uint32_t c) {
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}

__device__ __forceinline__ uint32_t dev_f2i(uint32_t a) {
    float f = u2f(a);
    if (f != f) return 0;
    if (f >= 2147483648.0f) return 0x7FFFFFFFu;
    if (f < -2147483648.0f) return 0x80000000u;
    return (uint32_t)__float2int_rz(f);
}

__device__ __forceinline__ uint32_t dev_lop3(uint32_t a, uint32_t b, uint32_t c, uint32_t lut) {
    // bit i of lut selects the minterm (i&4 ? a : ~a) & (i&2 ? b : ~b) & (i&1 ? c : ~c)
    uint32_t r = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        uint32_t t = ((i & 4) ? a : ~a) & ((i & 2) ? b : ~b) & ((i & 1) ? c : ~c);
        r |= ((lut >> i) & 1u) ? t : 0u;
    }
    return r;
}

// 0 ok, 1 misaligned, 2 unmapped (C-15).  On success *bid = buffer id.
__device__ __forceinline__ uint32_t check_access(const EmuProg& P, uint64_t va, uint32_t w, uint32_t* bid) {
    if (va & (w - 1)) return 1;
    uint64_t off = va - kVaBase;
    if (va < kVaBase || off >= P.image_bytes) return 2;
    uint32_t b = __ldg(&P.gran[off >> 8]);
    if (b == kNoBuf) return 2;
    uint64_t end = __ldg(&P.buf[b].off) + __ldg(&P.buf[b].size);
    if (off + w > end) return 2;
    *bid = b;
    return 0;
}

template <int MODE>
__device__ __noinline__ EmuOut emulate(const EmuProg P, uint8_t* img_w, const uint8_t* img,
                                       uint32_t k, uint32_t cta, uint32_t wic, uint32_t* __restrict__ R,
                                       uint32_t watchdog, fi_record* __restrict__ rec_out,
                                       fi_store* __restrict__ st_out, uint32_t st_cap, HookIn hook) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const fi_instance in = P.inst[k];
    const fi_kernel kn = P.kern[in.kernel];
    const fi_insn* __restrict__ code = P.code + kn.code_off;
    const uint32_t* __restrict__ cb = P.cbank + in.cbank_off;
    const uint32_t zr = P.n_regs;

    for (uint32_t r = 0; r <= zr; ++r) R[r * 32 + lane] = 0u;
    uint32_t nl = in.block - wic * 32;
    bool live = lane < (nl > 32 ? 32u : nl);
    uint32_t pc = 0, preds = 0;
    EmuOut o;
    uint32_t step = 0, nst = 0;
    uint4 recbuf = make_uint4(0, 0, 0, 0);
    __syncwarp();

#define RROW(r) ((r) < zr ? (r) : zr)
#define RD(r) R[RROW(r) * 32 + lane]
#define WR(r, v) do { if ((r) < zr) R[(r) * 32 + lane] = (v); } while (0)
#define RD64(r) ((uint64_t)RD(r) | ((uint64_t)RD((r) + 1) << 32))

    for (;;) {
        const uint32_t lm = __ballot_sync(kFull, live);
        if (!lm) break;
        const uint32_t pcm = __reduce_min_sync(kFull, live ? pc : 0xFFFFFFFFu);
        if (step >= watchdog) { o.fault = 3; o.fault_pc = pcm; break; }
        if (pcm >= kn.code_len) { o.fault = 4; o.fault_pc = pcm; break; }
        const bool act = live && pc == pcm;
        const uint32_t active = __ballot_sync(kFull, act);
        const uint4 raw = __ldg(reinterpret_cast<const uint4*>(code + pcm));
        const uint32_t op = raw.x & 0xFF, guard = (raw.x >> 8) & 0xFF, d0 = (raw.x >> 16) & 0xFF, d1 = raw.x >> 24;
        const uint32_t ra = raw.y & 0xFF, rb = (raw.y >> 8) & 0xFF, rc = (raw.y >> 16) & 0xFF, mod = raw.y >> 24;
        const uint32_t imm = raw.z, ext = raw.w;
        const uint32_t gsel = guard & 7;
        const bool pv = (((gsel == 7) ? 1u : ((preds >> gsel) & 1u)) ^ ((guard >> 3) & 1u)) != 0;
        const uint32_t pred = __ballot_sync(kFull, pv);
        const bool ex = act && pv;
        const uint32_t exm = active & pred;

        // ---- memory access validation (all executing lanes, before any effect)
        uint64_t va = 0;
        uint32_t bid = 0;
        if (op == LDG || op == STG) {
            const uint32_t w = 4u << ((mod & 3) > 2 ? 2 : (mod & 3));
            va = RD64(ra) + (uint64_t)(int64_t)(int32_t)imm;
            const uint32_t code_ = ex ? check_access(P, va, w, &bid) : 0u;
            const uint32_t mis = __ballot_sync(kFull, code_ == 1), unm = __ballot_sync(kFull, code_ == 2);
            if (mis | unm) { o.fault = mis ? 1 : 2; o.fault_pc = pcm; break; }
        }

        if (MODE == EMU_TRACE) {
            if ((step & 31) == lane)
                recbuf = make_uint4(k, pcm | (op << 16) | (groupmask_of(op, d0, d1, mod) << 24), active, pred);
            if ((step & 31) == 31) reinterpret_cast<uint4*>(rec_out)[step - 31 + lane] = recbuf;
        }

        const uint32_t bv = (mod & 0x80) ? imm : RD(rb);
        uint32_t next = pcm + 1;
        switch (op) {
            case NOP: break;
            case EXIT: if (ex) live = false; break;
            case BRA: if (ex) next = imm; break;
            case MOV: if (ex) WR(d0, bv); break;
            case S2R: {
                uint32_t v = 0;
                switch (imm) {
                    case 0: v = wic * 32 + lane; break;
                    case 1: v = cta; break;
                    case 2: v = in.block; break;
                    case 3: v = in.grid; break;
                    case 4: v = lane; break;
                    case 5: v = wic; break;
                }
                if (ex) WR(d0, v);
                break;
            }
            case IADD3: {
                const uint32_t a = RD(ra), c = RD(rc);
                const uint32_t x = (mod & 1) ? 0u - a : a, y = (mod & 2) ? 0u - bv : bv;
                const uint64_t s = (uint64_t)x + y + c;
                if (ex) {
                    WR(d0, (uint32_t)s);
                    const uint32_t p = d1 & 7;
                    if (p != 7) preds = (preds & ~(1u << p)) | ((uint32_t)((s >> 32) != 0) << p);
                }
                break;
            }
            case IMAD: if (ex) WR(d0, RD(ra) * bv + RD(rc)); break;
            case IMAD_WIDE: {
                const uint32_t a = RD(ra);
                const uint64_t prod = (mod & 1) ? (uint64_t)a * (uint64_t)bv
                                                : (uint64_t)((int64_t)(int32_t)a * (int64_t)(int32_t)bv);
                const uint64_t r = prod + RD64(rc);
                if (ex) { WR(d0, (uint32_t)r); WR(d0 + 1, (uint32_t)(r >> 32)); }
                break;
            }
            case SHF: {
                const uint32_t a = RD(ra), s = bv > 32 ? 32 : bv, m = mod & 3;
                uint32_t v;
                if (m == 0) v = s >= 32 ? 0u : a << s;
                else if (m == 1) v = s >= 32 ? 0u : a >> s;
                else v = (uint32_t)((int32_t)a >> (s >= 32 ? 31 : s));
                if (ex) WR(d0, v);
                break;
            }
            case LOP3: if (ex) WR(d0, dev_lop3(RD(ra), bv, RD(rc), ext & 0xFF)); break;
            case SEL: {
                const uint32_t p = rc & 7;
                const bool s = (((p == 7) ? 1u : ((preds >> p) & 1u)) ^ ((rc >> 3) & 1u)) != 0;
                if (ex) WR(d0, s ? RD(ra) : bv);
                break;
            }
            case ISETP: case FSETP: case DSETP: {
                bool v;
                const uint32_t c = mod & 7;
                if (op == ISETP) v = (mod & 8) ? dev_cmp_i<uint32_t>(RD(ra), bv, c) : dev_cmp_i<int32_t>((int32_t)RD(ra), (int32_t)bv, c);
                else if (op == FSETP) v = dev_cmp_f((double)u2f(RD(ra)), (double)u2f(RD(rb)), c);
                else v = dev_cmp_f(u2d(RD64(ra)), u2d(RD64(rb)), c);
                const uint32_t p = d0 & 7;
                if (ex && p != 7) preds = (preds & ~(1u << p)) | ((uint32_t)v << p);
                break;
            }
            case FADD: case FMUL: case FFMA: {
                const float x = u2f(RD(ra) ^ ((mod & 1) ? 0x80000000u : 0u));
                const float y = u2f(bv ^ ((mod & 2) ? 0x80000000u : 0u));
                const float z = u2f(RD(rc) ^ ((mod & 4) ? 0x80000000u : 0u));
                const float r = op == FADD ? __fadd_rn(x, y) : op == FMUL ? __fmul_rn(x, y) : __fmaf_rn(x, y, z);
                if (ex) WR(d0, fbits(r));
                break;
            }
            case FMNMX: if (ex) WR(d0, dev_fmnmx(RD(ra), bv, mod & 1)); break;
            case DADD: case DMUL: case DFMA: {
                const double x = u2d(RD64(ra) ^ ((mod & 1) ? 0x8000000000000000ull : 0ull));
                const double y = u2d(RD64(rb) ^ ((mod & 2) ? 0x8000000000000000ull : 0ull));
                const double z = u2d(RD64(rc) ^ ((mod & 4) ? 0x8000000000000000ull : 0ull));
                const double r = op == DADD ? __dadd_rn(x, y) : op == DMUL ? __dmul_rn(x, y) : __fma_rn(x, y, z);
                const uint64_t b = dbits(r);
                if (ex) { WR(d0, (uint32_t)b); WR(d0 + 1, (uint32_t)(b >> 32)); }
                break;
            }
            case LDG: {
                const uint32_t lw = (mod & 3) > 2 ? 2 : (mod & 3);
                if (ex) {
                    const fi_buffer B = P.buf[bid];
                    const bool zero = B.writer >= 0 && (uint32_t)B.writer >= k;
                    const uint8_t* src = img + (va - kVaBase);
                    if (lw == 0) {
                        WR(d0, zero ? 0u : __ldg(reinterpret_cast<const uint32_t*>(src)));
                    } else if (lw == 1) {
                        uint2 v = zero ? make_uint2(0, 0) : __ldg(reinterpret_cast<const uint2*>(src));
                        WR(d0, v.x); WR(d0 + 1, v.y);
                    } else {
                        uint4 v = zero ? make_uint4(0, 0, 0, 0) : __ldg(reinterpret_cast<const uint4*>(src));
                        WR(d0, v.x); WR(d0 + 1, v.y); WR(d0 + 2, v.z); WR(d0 + 3, v.w);
                    }
                }
                break;
            }
            case LDC: {
                const uint32_t w0 = imm >> 2;
                if (ex) {
                    WR(d0, w0 < in.cbank_len ? __ldg(&cb[w0]) : 0u);
                    if (mod & 1) WR(d0 + 1, w0 + 1 < in.cbank_len ? __ldg(&cb[w0 + 1]) : 0u);
                }
                break;
            }
            case STG: {
                const uint32_t lw = (mod & 3) > 2 ? 2 : (mod & 3), nw = 1u << lw;
                uint32_t v[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) v[i] = (uint32_t)i < nw ? RD(rb + i) : 0u;
                const uint32_t idx = __popc(exm & lt_mask) * nw;
                const uint32_t tot = __popc(exm) * nw;
                if (MODE == EMU_LEN) {
                    if (ex) {
                        uint8_t* dst = img_w + (va - kVaBase);
                        if (lw == 0) *reinterpret_cast<uint32_t*>(dst) = v[0];
                        else if (lw == 1) *reinterpret_cast<uint2*>(dst) = make_uint2(v[0], v[1]);
                        else *reinterpret_cast<uint4*>(dst) = make_uint4(v[0], v[1], v[2], v[3]);
                    }
                } else if (MODE == EMU_TRACE || step > hook.step) {
                    if (ex) {
                        for (uint32_t i = 0; i < nw; ++i) {
                            const uint32_t e = nst + idx + i;
                            if (MODE == EMU_TRACE || e < st_cap) {
                                fi_store s;
                                s.va = va + 4 * i; s.value = v[i]; s.step = step;
                                st_out[e] = s;
                            }
                        }
                    }
                }
                if (MODE != EMU_INJ || step > hook.step) nst += tot;
                break;
            }
            case I2F: if (ex) WR(d0, fbits((mod & 1) ? __uint2float_rn(RD(ra)) : __int2float_rn((int)RD(ra)))); break;
            case F2I: if (ex) WR(d0, dev_f2i(RD(ra))); break;
            case F2F_F64_F32: {
                const uint64_t b = dbits((double)u2f(RD(ra)));
                if (ex) { WR(d0, (uint32_t)b); WR(d0 + 1, (uint32_t)(b >> 32)); }
                break;
            }
            case F2F_F32_F64: if (ex) WR(d0, fbits(__double2float_rn(u2d(RD64(ra))))); break;
            case SHFL: {
                int64_t src;
                switch (mod & 3) {
                    case 0: src = bv & 31; break;
                    case 1: src = lane ^ (bv & 31); break;
                    case 2: src = (int64_t)lane + (int64_t)bv; if (src > 31) src = lane; break;
                    default: src = (int64_t)lane - (int64_t)bv; if (src < 0) src = lane; break;
                }
                __syncwarp();
                const uint32_t v = R[RROW(ra) * 32 + (uint32_t)src];
                __syncwarp();
                if (ex) WR(d0, v);
                break;
            }
            case IMNMX: {
                const uint32_t a = RD(ra);
                uint32_t v;
                if (mod & 8) v = (mod & 1) ? max(a, bv) : min(a, bv);
                else v = (uint32_t)((mod & 1) ? max((int32_t)a, (int32_t)bv) : min((int32_t)a, (int32_t)bv));
                if (ex) WR(d0, v);
                break;
            }
            default: break;
        }
        if (act) pc = next;

        if (MODE == EMU_INJ && step == hook.step) {
            // transient fault: corrupt one destination of this dynamic
            // instruction in one lane, after the instruction wrote it (C-7, C-8)
            o.fired = true;
            const bool lane_ok = (exm >> hook.lane) & 1u;
            if (pcm != hook.pc || !lane_ok) o.bad = true;
            if (lane == hook.lane) {
                if (hook.kind == 0) {
                    const uint32_t before = RD(hook.reg);
                    const uint32_t m = hook.bfm == FI_ZERO_VALUE ? before : hook.mask;
                    o.before = before; o.mask = m; o.after = before ^ m;
                    WR(hook.reg, o.after);
                } else {
                    const uint32_t p = hook.reg & 7;
                    const uint32_t before = (p == 7) ? 1u : ((preds >> p) & 1u);
                    uint32_t m = hook.mask, after;
                    if (hook.bfm == FI_FLIP_SINGLE_BIT || hook.bfm == FI_FLIP_TWO_BITS) after = before ^ 1u;
                    else if (hook.bfm == FI_RANDOM_VALUE) after = (m >> 31) & 1u;
                    else { m = before; after = 0u; }
                    o.before = before; o.mask = m; o.after = after;
                    if (p != 7) preds = (preds & ~(1u << p)) | (after << p);
                }
            }
        }
        ++step;
    }
#undef RROW
#undef RD
#undef WR
#undef RD64
    if (MODE == EMU_TRACE) {
        const uint32_t rem = step & 31;
        if (rem && lane < rem) reinterpret_cast<uint4*>(rec_out)[step - rem + lane] = recbuf;
    }
    o.steps = step;
    o.nstore = nst;
    if (MODE == EMU_INJ) {                            // broadcast the hook lane's values
        o.before = __shfl_sync(kFull, o.before, hook.lane);
        o.after = __shfl_sync(kFull, o.after, hook.lane);
        o.mask = __shfl_sync(kFull, o.mask, hook.lane);
    }
    return o;
}

}  // namespace fi
