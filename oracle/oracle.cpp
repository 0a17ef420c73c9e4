// oracle.cpp — CPU ORACLE (test infrastructure only; see oracle.h header).
//
// A plain serial interpreter of the mini-SASS program model plus
// the four steps of NVBitFI's method written as their definitions:
//   count    PAPER.md:78 §III-A, groups per Table II PAPER.md:94-104 (reading C-2)
//   select   PAPER.md:78 "random number n from the set 1..N" -> canonical
//            enumeration (C-3, C-4), Philox4x32-10 + Lemire (C-5)
//   inject   PAPER.md:78,138 one destination register of one dynamic instruction;
//            masks Table II PAPER.md:116-121 (C-5..C-8)
//   classify Table V PAPER.md:184-196 and PAPER.md:206 (C-9..C-12, C-14)
// No blocking, prefix sums, chunk tables or fused passes: per-lane loops,
// std::vector, std::map.  Compiled with -O2 -ffp-contract=off (no fast-math),
// so FADD/FMUL are never contracted and std::fma is the only fused op (C-13).
#include "oracle.h"

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstring>
#include <map>
#include <mutex>
#include <string>
#include <thread>
#include <vector>

namespace {

// ---------------------------------------------------------------------------
// opcode numbers of the input format; the oracle's own copy
// ---------------------------------------------------------------------------
enum Op {
    NOP = 0, EXIT, BRA, MOV, S2R, IADD3, IMAD, IMAD_WIDE, SHF, LOP3, SEL,
    ISETP, FSETP, DSETP, FADD, FMUL, FFMA, FMNMX, DADD, DMUL, DFMA,
    LDG, LDC, STG, I2F, F2I, F2F_F64_F32, F2F_F32_F64, SHFL, IMNMX, MUFU_RCP64, N_OPS
};
const int RZ = 127, PT = 7;
const uint64_t VA_BASE = 0x00007F0000000000ull;       // C-15
const uint32_t QNAN32 = 0x7FFFFFFFu;                  // C-13 canonical NaNs
const uint64_t QNAN64 = 0x7FFFFFFFFFFFFFFFull;

thread_local std::string g_err;

// ---------------------------------------------------------------------------
// Table II groups (reading C-2) and destination slots (reading C-6)
// ---------------------------------------------------------------------------
// Architectural destinations of one static instruction: GP registers (32-bit,
// ascending) and predicate registers.  RZ / PT writes are not destinations.
void dest_regs(const orc_insn& I, std::vector<int>& gp, std::vector<int>& pr) {
    gp.clear(); pr.clear();
    auto gpn = [&](int n) { if (I.d0 != RZ) for (int i = 0; i < n; ++i) gp.push_back(I.d0 + i); };
    switch (I.op) {
        case MOV: case S2R: case IMAD: case SHF: case LOP3: case SEL: case I2F: case F2I:
        case F2F_F32_F64: case SHFL: case IMNMX: case FADD: case FMUL: case FFMA: case FMNMX:
            gpn(1); break;
        case IADD3:
            gpn(1);
            if ((I.d1 & 7) != PT) pr.push_back(I.d1 & 7);   // predicate fields are 3 bits (§3.1)
            break;
        case IMAD_WIDE: case DADD: case DMUL: case DFMA: case F2F_F64_F32: case MUFU_RCP64:
            gpn(2); break;
        case LDG: gpn(1 << std::min(I.mod & 3, 2)); break;
        case LDC: gpn((I.mod & 1) ? 2 : 1); break;
        case ISETP: case FSETP: case DSETP:
            if ((I.d0 & 7) != PT) pr.push_back(I.d0 & 7);
            break;
        default: break;   // STG, BRA, EXIT, NOP: no destination
    }
}

// Group membership bits, Table II order.  Precedence (C-2): NODEST, PR, FP64,
// FP32, LD, OTHERS; GPPR = all - NODEST, GP = all - NODEST - PR.
uint32_t group_mask(const orc_insn& I) {
    std::vector<int> gp, pr;
    dest_regs(I, gp, pr);
    if (gp.empty() && pr.empty()) return 1u << ORC_G_NODEST;
    if (gp.empty()) return (1u << ORC_G_PR) | (1u << ORC_G_GPPR);
    int base;
    if (I.op == DADD || I.op == DMUL || I.op == DFMA) base = ORC_G_FP64;
    else if (I.op == FADD || I.op == FMUL || I.op == FFMA || I.op == FMNMX) base = ORC_G_FP32;
    else if (I.op == LDG || I.op == LDC) base = ORC_G_LD;
    else base = ORC_G_OTHERS;
    return (1u << base) | (1u << ORC_G_GPPR) | (1u << ORC_G_GP);
}

// Eligible destination slots for group g (C-6): GP registers ascending for the
// GP-type groups, predicates for G_PR, GP then predicates for G_GPPR.
void slots_for(const orc_insn& I, int g, std::vector<std::pair<int, int>>& out) {
    std::vector<int> gp, pr;
    dest_regs(I, gp, pr);
    out.clear();
    if (g == ORC_G_NODEST) return;
    if (g != ORC_G_PR) for (int r : gp) out.push_back({0, r});
    if (g == ORC_G_PR || g == ORC_G_GPPR) for (int p : pr) out.push_back({1, p});
}

// ---------------------------------------------------------------------------
// Philox4x32-10 (Salmon et al., Random123) and Lemire's unbiased range draw
// ---------------------------------------------------------------------------
void philox(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
    uint32_t c[4] = {ctr_in[0], ctr_in[1], ctr_in[2], ctr_in[3]};
    uint32_t k[2] = {key_in[0], key_in[1]};
    for (int r = 0; r < 10; ++r) {
        if (r > 0) { k[0] += 0x9E3779B9u; k[1] += 0xBB67AE85u; }
        uint64_t p0 = (uint64_t)0xD2511F53u * c[0];
        uint64_t p1 = (uint64_t)0xCD9E8D57u * c[2];
        uint32_t n0 = (uint32_t)(p1 >> 32) ^ c[1] ^ k[0];
        uint32_t n1 = (uint32_t)p1;
        uint32_t n2 = (uint32_t)(p0 >> 32) ^ c[3] ^ k[1];
        uint32_t n3 = (uint32_t)p0;
        c[0] = n0; c[1] = n1; c[2] = n2; c[3] = n3;
    }
    for (int i = 0; i < 4; ++i) out[i] = c[i];
}

// block a of replica j = Philox(ctr={j_lo, j_hi, a, 0x46490001},
// key={seed_lo, seed_hi}); x = w0 | w1<<32 from the block, u_dst/u_bit from
// block 0; s = hi64(x * N) accepted unless lo64(x * N) < (2^64 - N) mod N.
void draw(uint64_t seed, uint64_t j, uint64_t n, uint64_t& s, uint32_t& u_dst, uint32_t& u_bit, uint32_t& attempts) {
    uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
    uint32_t a = 0;
    for (;;) {
        uint32_t ctr[4] = {(uint32_t)j, (uint32_t)(j >> 32), a, 0x46490001u}, o[4];
        philox(ctr, key, o);
        if (a == 0) { u_dst = o[2]; u_bit = o[3]; }
        uint64_t x = (uint64_t)o[0] | ((uint64_t)o[1] << 32);
        unsigned __int128 m = (unsigned __int128)x * n;
        uint64_t lo = (uint64_t)m;
        uint64_t t = (0 - n) % n;             // (2^64 - n) mod n
        if (lo >= t) { s = (uint64_t)(m >> 64); attempts = a + 1; return; }
        ++a;
    }
}

// Table II bit-pattern masks with value = u/2^32 (C-5, C-8).  ZERO_VALUE's mask
// is the original register value, resolved at injection time (returns 0 here).
uint32_t mask_of(int bfm, uint32_t u) {
    switch (bfm) {
        case 0: return 1u << (uint32_t)(((uint64_t)32 * u) >> 32);              // 0x1 << (32 x value)
        case 1: return 3u << (uint32_t)(((uint64_t)31 * u) >> 32);              // 0x3 << (31 x value)
        case 2: return (uint32_t)(((uint64_t)0xFFFFFFFFu * u) >> 32);          // 0xffffffff x value
        default: return 0;                                                      // ZERO_VALUE
    }
}

// ---------------------------------------------------------------------------
// FP helpers (C-13): IEEE RN, no FTZ, canonical NaN results
// ---------------------------------------------------------------------------
inline float f32(uint32_t b) { float f; memcpy(&f, &b, 4); return f; }
inline uint32_t b32(float f) { uint32_t b; memcpy(&b, &f, 4); return std::isnan(f) ? QNAN32 : b; }
inline double f64(uint64_t b) { double d; memcpy(&d, &b, 8); return d; }
inline uint64_t b64(double d) { uint64_t b; memcpy(&b, &d, 8); return std::isnan(d) ? QNAN64 : b; }
inline uint32_t negf(uint32_t x, bool n) { return n ? x ^ 0x80000000u : x; }
inline uint64_t negd(uint64_t x, bool n) { return n ? x ^ 0x8000000000000000ull : x; }

// minNum / maxNum with -0 < +0 (C-13)
uint32_t fmnmx(uint32_t a, uint32_t b, bool is_max) {
    float x = f32(a), y = f32(b);
    if (std::isnan(x) && std::isnan(y)) return QNAN32;
    if (std::isnan(x)) return b;
    if (std::isnan(y)) return a;
    if (x == y) {                                  // equal values, maybe +0 / -0
        bool xneg = a >> 31;
        if (is_max) return xneg ? b : a;
        return xneg ? a : b;
    }
    if (is_max) return x > y ? a : b;
    return x < y ? a : b;
}

bool fcmp(double x, double y, int cmp) {        // ordered: false when NaN
    if (std::isnan(x) || std::isnan(y)) return false;
    switch (cmp) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
        default: return false;
    }
}
template <class T> bool icmp(T x, T y, int cmp) {
    switch (cmp) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
        default: return false;
    }
}

uint32_t f2i(uint32_t a) {                      // RZ, saturating, NaN -> 0
    float f = f32(a);
    if (std::isnan(f)) return 0;
    if (f >= 2147483648.0f) return 0x7FFFFFFFu;
    if (f < -2147483648.0f) return 0x80000000u;
    return (uint32_t)(int32_t)f;
}

uint32_t lop3(uint32_t a, uint32_t b, uint32_t c, uint32_t lut) {
    uint32_t r = 0;
    for (int i = 0; i < 8; ++i)
        if ((lut >> i) & 1) r |= ((i & 4) ? a : ~a) & ((i & 2) ? b : ~b) & ((i & 1) ? c : ~c);
    return r;
}

// ---------------------------------------------------------------------------
// Program, memory and one-warp interpreter (App. A.2 min-PC scheduling)
// ---------------------------------------------------------------------------
struct Prog {
    orc_program p;
    std::vector<uint32_t> gm;            // group mask per static instruction
    uint32_t n_warps = 0;
    bool sorted = false;                 // allocations in ascending, non-overlapping order
    bool single_instance() const { return p.n_inst == 1; }
};

// The allocation that contains byte offset `off`, or nullptr.  A binary search
// when the buffer table is sorted and non-overlapping (every generated program:
// the lookup is the same "which allocation holds this address" as a linear scan,
// which is kept for any other table); programs with thousands of SSA buffer
// versions (C3) made the linear scan the oracle's dominant cost.
const orc_buffer* find_buffer(const Prog& P, uint64_t off) {
    if (P.sorted) {
        uint32_t lo = 0, hi = P.p.n_buf;                 // first buffer with b.off > off
        while (lo < hi) {
            const uint32_t mid = (lo + hi) / 2;
            if (P.p.buf[mid].off <= off) lo = mid + 1; else hi = mid;
        }
        if (lo == 0) return nullptr;
        const orc_buffer& b = P.p.buf[lo - 1];
        return off < b.off + b.size ? &b : nullptr;
    }
    for (uint32_t i = 0; i < P.p.n_buf; ++i) {
        const orc_buffer& b = P.p.buf[i];
        if (off >= b.off && off < b.off + b.size) return &b;
    }
    return nullptr;
}

struct StoreW { uint64_t va; uint32_t value; uint64_t step; };   // one 32-bit word

// fault kinds (fi_inj.fault_kind): 0 none, 1 misaligned, 2 unmapped, 3 watchdog, 4 illegal pc
struct WarpResult { uint64_t steps = 0; int fault = 0; uint32_t fault_pc = 0; };

struct Hook {
    bool on = false;
    uint64_t step = 0; int lane = 0; int kind = 0; int reg = 0; int bfm = 0; uint32_t mask = 0; uint32_t pc = 0;
    bool fired = false, bad = false;
    uint32_t before = 0, after = 0, applied_mask = 0;
    // permanent / intermittent fault (rows f2/f3): every executed instance of
    // `perm_op` in lane `perm_lane` of this warp gets its destinations XOR-ed
    bool perm = false;
    uint32_t perm_op = 0, perm_lane = 0, perm_mask = 0, perm_q = 0, perm_rep = 0;
    uint64_t perm_seed = 0;
};

// The permanent-fault spec of one run (Table III [PAPER.md:128-134]).
struct PermSpec { uint32_t opcode, sm, lane, mask, q32, n_sm, rep; uint64_t seed; };

// Find the allocation containing [va, va+w).  C-15: valid iff aligned to the
// access width and fully inside one allocation.  Returns 0 ok, 1 misaligned, 2 unmapped.
int check_access(const Prog& P, uint64_t va, uint32_t w) {
    if (va % w) return 1;
    if (va < VA_BASE) return 2;
    uint64_t off = va - VA_BASE;
    const orc_buffer* b = find_buffer(P, off);
    return (b && off + w <= b->off + b->size) ? 0 : 2;
}

struct Warp {
    uint32_t R[32][128];
    uint8_t Pr[32];
    uint32_t pc[32];
    uint32_t live;
};

inline uint32_t rd(const Warp& W, int l, int r) { return r >= RZ ? 0u : W.R[l][r]; }
inline uint64_t rd2(const Warp& W, int l, int r) { return (uint64_t)rd(W, l, r) | ((uint64_t)rd(W, l, r + 1) << 32); }
inline void wr(Warp& W, int l, int r, uint32_t v) { if (r < RZ) W.R[l][r] = v; }
inline void wr2(Warp& W, int l, int r, uint64_t v) { wr(W, l, r, (uint32_t)v); wr(W, l, r + 1, (uint32_t)(v >> 32)); }
inline bool prd(const Warp& W, int l, int p) { return (p & 7) == PT ? true : ((W.Pr[l] >> (p & 7)) & 1); }
inline void pwr(Warp& W, int l, int p, bool v) {
    p &= 7;
    if (p == PT) return;
    W.Pr[l] = (uint8_t)((W.Pr[l] & ~(1u << p)) | ((v ? 1u : 0u) << p));
}

struct TraceSink { std::vector<orc_record>* rec = nullptr; };

// Interpret warp `wic` of CTA `cta` of instance k from its first instruction.
// Loads read `mem` (the memory state before the instance: stores are deferred to
// the end of the instance, C-14) and stores are appended to `stores` as 32-bit
// words in program order (step, lane ascending, word ascending).
WarpResult run_warp(const Prog& P, const std::vector<uint8_t>& mem, uint32_t k, uint32_t cta, uint32_t wic,
                    Hook* hook, uint64_t watchdog, std::vector<StoreW>* stores, TraceSink* trace,
                    uint64_t* counts8) {
    const orc_instance& in = P.p.inst[k];
    const orc_kernel& kn = P.p.kern[in.kernel];
    const orc_insn* code = P.p.code + kn.code_off;
    const uint32_t* gm = P.gm.data() + kn.code_off;
    Warp* Wp = new Warp;
    Warp& W = *Wp;
    memset(&W, 0, sizeof(W));
    uint32_t nlanes = std::min<uint32_t>(32, in.block - wic * 32);
    W.live = nlanes == 32 ? 0xFFFFFFFFu : ((1u << nlanes) - 1);
    WarpResult res;
    uint64_t step = 0;
    uint32_t vals[32][4];
    while (W.live) {
        uint32_t pcm = 0xFFFFFFFFu;
        for (int l = 0; l < 32; ++l) if ((W.live >> l) & 1) pcm = std::min(pcm, W.pc[l]);
        if (step >= watchdog) { res.fault = 3; res.fault_pc = pcm; break; }
        if (pcm >= kn.code_len) { res.fault = 4; res.fault_pc = pcm; break; }
        uint32_t active = 0;
        for (int l = 0; l < 32; ++l) if (((W.live >> l) & 1) && W.pc[l] == pcm) active |= 1u << l;
        const orc_insn& I = code[pcm];
        uint32_t pred = 0;
        for (int l = 0; l < 32; ++l) {
            bool v = prd(W, l, I.guard & 7) ^ ((I.guard >> 3) & 1);
            if (v) pred |= 1u << l;
        }
        uint32_t ex = active & pred;
        bool bimm = I.mod & 0x80;
        auto B = [&](int l) -> uint32_t { return bimm ? I.imm : rd(W, l, I.b); };

        // memory accesses: validate every executing lane first (C-9, C-15)
        if (I.op == LDG || I.op == STG) {
            uint32_t w = 4u << std::min(I.mod & 3, 2);
            int bad = 0;
            for (int l = 0; l < 32; ++l) if ((ex >> l) & 1) {
                uint64_t va = rd2(W, l, I.a) + (uint64_t)(int64_t)(int32_t)I.imm;
                int c = check_access(P, va, w);
                if (c == 1) bad = 1; else if (c == 2 && bad == 0) bad = 2;
            }
            if (bad) { res.fault = bad; res.fault_pc = pcm; break; }
        }
        if (trace && trace->rec) trace->rec->push_back({k, pcm | ((uint32_t)I.op << 16) | (gm[pcm] << 24), active, pred});
        if (counts8) {
            uint64_t c = (uint64_t)__builtin_popcount(ex);
            for (int g = 0; g < 8; ++g) if ((gm[pcm] >> g) & 1) counts8[g] += c;
        }

        // compute (all lanes read before any lane writes: matters for SHFL)
        for (int l = 0; l < 32; ++l) {
            if (!((ex >> l) & 1)) continue;
            uint32_t a = rd(W, l, I.a), b = B(l), c = rd(W, l, I.c);
            uint32_t* v = vals[l];
            switch (I.op) {
                case MOV: v[0] = b; break;
                case S2R: {
                    uint32_t sr[6] = {wic * 32 + (uint32_t)l, cta, in.block, in.grid, (uint32_t)l, wic};
                    v[0] = I.imm < 6 ? sr[I.imm] : 0; break;
                }
                case IADD3: {
                    uint32_t x = (I.mod & 1) ? 0u - a : a, y = (I.mod & 2) ? 0u - b : b;
                    uint64_t s = (uint64_t)x + y + c;
                    v[0] = (uint32_t)s; v[1] = (s >> 32) != 0; break;
                }
                case IMAD: v[0] = a * b + c; break;
                case IMAD_WIDE: {
                    uint64_t prod = (I.mod & 1) ? (uint64_t)a * (uint64_t)b
                                                : (uint64_t)((int64_t)(int32_t)a * (int64_t)(int32_t)b);
                    uint64_t r = prod + rd2(W, l, I.c);
                    v[0] = (uint32_t)r; v[1] = (uint32_t)(r >> 32); break;
                }
                case SHF: {
                    uint32_t s = std::min<uint32_t>(b, 32);
                    int mode = I.mod & 3;
                    if (mode == 0) v[0] = s >= 32 ? 0 : a << s;
                    else if (mode == 1) v[0] = s >= 32 ? 0 : a >> s;
                    else v[0] = s >= 32 ? (uint32_t)((int32_t)a >> 31) : (uint32_t)((int32_t)a >> s);
                    break;
                }
                case LOP3: v[0] = lop3(a, b, c, I.ext & 0xFF); break;
                case SEL: v[0] = (prd(W, l, I.c & 7) ^ ((I.c >> 3) & 1)) ? a : b; break;
                case ISETP: {
                    int cmp = I.mod & 7;
                    v[0] = (I.mod & 8) ? icmp<uint32_t>(a, b, cmp) : icmp<int32_t>((int32_t)a, (int32_t)b, cmp);
                    break;
                }
                case FSETP: v[0] = fcmp(f32(a), f32(b), I.mod & 7); break;
                case DSETP: v[0] = fcmp(f64(rd2(W, l, I.a)), f64(rd2(W, l, I.b)), I.mod & 7); break;
                case FADD: v[0] = b32(f32(negf(a, I.mod & 1)) + f32(negf(b, I.mod & 2))); break;
                case FMUL: v[0] = b32(f32(negf(a, I.mod & 1)) * f32(negf(b, I.mod & 2))); break;
                case FFMA: v[0] = b32(std::fmaf(f32(negf(a, I.mod & 1)), f32(negf(b, I.mod & 2)), f32(negf(c, I.mod & 4)))); break;
                case FMNMX: v[0] = fmnmx(a, b, I.mod & 1); break;
                case DADD: case DMUL: case DFMA: {
                    double x = f64(negd(rd2(W, l, I.a), I.mod & 1));
                    double y = f64(negd(rd2(W, l, I.b), I.mod & 2));
                    double z = f64(negd(rd2(W, l, I.c), I.mod & 4));
                    double r = I.op == DADD ? x + y : I.op == DMUL ? x * y : std::fma(x, y, z);
                    uint64_t rb = b64(r);
                    v[0] = (uint32_t)rb; v[1] = (uint32_t)(rb >> 32); break;
                }
                case LDG: {
                    uint32_t nw = 1u << std::min(I.mod & 3, 2);
                    uint64_t off = rd2(W, l, I.a) + (uint64_t)(int64_t)(int32_t)I.imm - VA_BASE;
                    for (uint32_t i = 0; i < nw; ++i) memcpy(&v[i], &mem[off + 4 * i], 4);
                    break;
                }
                case LDC: {
                    uint32_t nw = (I.mod & 1) ? 2 : 1, w0 = I.imm >> 2;
                    for (uint32_t i = 0; i < nw; ++i)
                        v[i] = (w0 + i < in.cbank_len) ? P.p.cbank[in.cbank_off + w0 + i] : 0u;
                    break;
                }
                case STG: break;
                case I2F: v[0] = b32((I.mod & 1) ? (float)a : (float)(int32_t)a); break;
                case F2I: v[0] = f2i(a); break;
                case F2F_F64_F32: {
                    uint64_t rb = b64((double)f32(a));
                    v[0] = (uint32_t)rb; v[1] = (uint32_t)(rb >> 32); break;
                }
                case F2F_F32_F64: v[0] = b32((float)f64(rd2(W, l, I.a))); break;
                case SHFL: {
                    int64_t src;
                    switch (I.mod & 3) {
                        case 0: src = b & 31; break;
                        case 1: src = l ^ (b & 31); break;
                        case 2: src = (int64_t)l + (int64_t)b; if (src > 31) src = l; break;
                        default: src = (int64_t)l - (int64_t)b; if (src < 0) src = l; break;
                    }
                    v[0] = rd(W, (int)src, I.a); break;
                }
                case MUFU_RCP64: {                              // 1/x in f64, round to nearest (§3.2)
                    uint64_t rb = b64(1.0 / f64(rd2(W, l, I.a)));
                    v[0] = (uint32_t)rb; v[1] = (uint32_t)(rb >> 32); break;
                }
                case IMNMX: {
                    bool mx = I.mod & 1;
                    if (I.mod & 8) v[0] = mx ? std::max(a, b) : std::min(a, b);
                    else v[0] = (uint32_t)(mx ? std::max((int32_t)a, (int32_t)b) : std::min((int32_t)a, (int32_t)b));
                    break;
                }
                default: break;
            }
        }
        // write back / control flow
        for (int l = 0; l < 32; ++l) {
            if (!((active >> l) & 1)) continue;
            bool e = (ex >> l) & 1;
            uint32_t* v = vals[l];
            uint32_t next = pcm + 1;
            if (e) switch (I.op) {
                case EXIT: W.live &= ~(1u << l); break;
                case BRA: next = I.imm; break;
                case MOV: case S2R: case IMAD: case SHF: case LOP3: case SEL: case I2F: case F2I:
                case F2F_F32_F64: case SHFL: case IMNMX: case FADD: case FMUL: case FFMA: case FMNMX:
                    wr(W, l, I.d0, v[0]); break;
                case IADD3: wr(W, l, I.d0, v[0]); pwr(W, l, I.d1, v[1]); break;
                case IMAD_WIDE: case DADD: case DMUL: case DFMA: case F2F_F64_F32: case MUFU_RCP64:
                    wr(W, l, I.d0, v[0]); wr(W, l, I.d0 + 1, v[1]); break;
                case LDG: { uint32_t nw = 1u << std::min(I.mod & 3, 2); for (uint32_t i = 0; i < nw; ++i) wr(W, l, I.d0 + i, v[i]); break; }
                case LDC: wr(W, l, I.d0, v[0]); if (I.mod & 1) wr(W, l, I.d0 + 1, v[1]); break;
                case ISETP: case FSETP: case DSETP: pwr(W, l, I.d0, v[0]); break;
                case STG: {
                    uint32_t nw = 1u << std::min(I.mod & 3, 2);
                    uint64_t va = rd2(W, l, I.a) + (uint64_t)(int64_t)(int32_t)I.imm;
                    for (uint32_t i = 0; i < nw; ++i) stores->push_back({va + 4 * i, rd(W, l, I.b + i), step});
                    break;
                }
                default: break;
            }
            W.pc[l] = next;
        }
        // transient fault hook: after the instruction writes its
        // destinations, corrupt one destination in one lane (C-7, C-8)
        if (hook && hook->on && step == hook->step) {
            hook->fired = true;
            int l = hook->lane;
            if (pcm != hook->pc || !((ex >> l) & 1)) hook->bad = true;
            if (hook->kind == 0) {
                uint32_t before = rd(W, l, hook->reg);
                uint32_t m = hook->bfm == 3 ? before : hook->mask;
                hook->before = before; hook->applied_mask = m; hook->after = before ^ m;
                wr(W, l, hook->reg, hook->after);
            } else {
                uint32_t before = prd(W, l, hook->reg) ? 1u : 0u, after;
                uint32_t m = hook->mask;
                if (hook->bfm == 0 || hook->bfm == 1) after = before ^ 1u;
                else if (hook->bfm == 2) after = (m >> 31) & 1u;
                else { m = before; after = 0; }
                hook->before = before; hook->applied_mask = m; hook->after = after;
                pwr(W, l, hook->reg, after != 0);
            }
        }
        // permanent fault: the same XOR mask on the destination
        // registers of every dynamic instance of the opcode in the faulty lane;
        // intermittent: only instances whose Philox draw is below q
        if (hook && hook->perm && I.op == hook->perm_op && ((ex >> hook->perm_lane) & 1)) {
            bool fire = true;
            if (hook->perm_q) {
                uint32_t wg = in.warp_begin + cta * ((in.block + 31) / 32) + wic;
                uint32_t ctr[4] = {wg, (uint32_t)step, hook->perm_rep, 0x46490002u};
                uint32_t key[2] = {(uint32_t)hook->perm_seed, (uint32_t)(hook->perm_seed >> 32)}, o[4];
                philox(ctr, key, o);
                fire = o[0] < hook->perm_q;
            }
            if (fire) {
                std::vector<int> gp, pr;
                dest_regs(I, gp, pr);
                int l = hook->perm_lane;
                for (int r : gp) wr(W, l, r, rd(W, l, r) ^ hook->perm_mask);
                if (hook->perm_mask & 1) for (int p : pr) pwr(W, l, p, !prd(W, l, p));
            }
        }
        ++step;
    }
    res.steps = step;
    delete Wp;
    return res;
}

void apply_stores(std::vector<uint8_t>& mem, const std::vector<StoreW>& st) {
    for (const StoreW& s : st) memcpy(&mem[s.va - VA_BASE], &s.value, 4);
}

template <class F> void parallel_for(uint32_t n, int n_threads, F f) {
    n_threads = std::max(1, std::min<int>(n_threads, (int)n));
    std::atomic<uint32_t> next{0};
    std::vector<std::thread> th;
    for (int t = 0; t < n_threads; ++t)
        th.emplace_back([&] { for (uint32_t i; (i = next.fetch_add(1)) < n;) f(i); });
    for (auto& t : th) t.join();
}

struct Golden {
    Prog P;
    std::vector<uint64_t> counts;        // [n_inst][8]
    std::vector<uint64_t> wcounts;       // [n_warps][8]
    std::vector<uint64_t> wlen;          // steps per warp
    std::vector<uint32_t> winst;         // instance of warp
    std::vector<uint8_t> final_mem;
    std::vector<orc_record> trace;
    std::vector<uint64_t> woff;          // record offset per warp (if trace)
    uint64_t n_rec = 0, n_gstores = 0;
    bool kept = false;
    std::string err;
};

bool prepare(Prog& P, const orc_program* p, std::string& err) {
    P.p = *p;
    P.gm.resize(p->n_code);
    for (uint32_t i = 0; i < p->n_code; ++i) P.gm[i] = group_mask(p->code[i]);
    uint32_t w = 0;
    for (uint32_t k = 0; k < p->n_inst; ++k) {
        const orc_instance& in = p->inst[k];
        if (in.warp_begin != w) { err = "instance warp_begin mismatch"; return false; }
        w += in.grid * ((in.block + 31) / 32);
        if (in.warp_end != w) { err = "instance warp_end mismatch"; return false; }
        if (in.kernel >= p->n_kern) { err = "bad kernel id"; return false; }
    }
    P.n_warps = w;
    P.sorted = true;
    for (uint32_t i = 1; i < p->n_buf && P.sorted; ++i)
        P.sorted = p->buf[i - 1].off + p->buf[i - 1].size <= p->buf[i].off;
    return true;
}

void warp_coords(const orc_instance& in, uint32_t w, uint32_t& cta, uint32_t& wic) {
    uint32_t wpc = (in.block + 31) / 32, lw = w - in.warp_begin;
    cta = lw / wpc; wic = lw % wpc;
}

// Run the whole program (all instances in launch order).  Each instance reads
// the memory state before it; stores are applied at its end in warp order, the
// faulty warp's last (C-14).  Used by the golden run and by full-mode injection.
struct FullRun {
    std::vector<uint8_t> mem;
    int fault = 0; uint32_t fault_pc = 0;
    int pdue = 0; uint32_t pdue_pc = 0;        // unchecked mode: first non-fatal fault (potential DUE)
    uint64_t n_faulty_stores = 0;
};

// `unchecked` (§8 row f4): the application does not check
// CUDA errors, so a memory fault or illegal instruction only ends the faulting
// warp (its earlier stores stand) and the run goes on; a hang (watchdog) is
// still detected by the monitor and ends the run.
void run_program(const Golden* G, const Prog& P, Hook* hook, uint32_t hook_warp, int n_threads, FullRun& out,
                 std::vector<uint64_t>* wlen_out, std::vector<uint64_t>* wcounts, bool keep_trace,
                 std::vector<std::vector<orc_record>>* wtraces, uint64_t* n_gstores, std::string* err,
                 bool unchecked = false, const PermSpec* perm = nullptr) {
    out.mem.assign(P.p.init_image, P.p.init_image + P.p.image_bytes);
    for (uint32_t k = 0; k < P.p.n_inst && !out.fault; ++k) {
        const orc_instance& in = P.p.inst[k];
        uint32_t nw = in.warp_end - in.warp_begin;
        std::vector<std::vector<StoreW>> st(nw);
        std::vector<WarpResult> rr(nw);
        auto body = [&](uint32_t i) {
            uint32_t w = in.warp_begin + i, cta, wic;
            warp_coords(in, w, cta, wic);
            uint64_t wd = G ? 10 * G->wlen[w] + 1024 : UINT64_MAX;      // C-10 watchdog
            TraceSink ts;
            std::vector<orc_record> tr;
            if (keep_trace) ts.rec = &tr;
            Hook ph;                                     // permanent fault: CTAs on the faulty SM (C-21)
            Hook* h = (hook && w == hook_warp) ? hook : nullptr;
            if (perm && cta % perm->n_sm == perm->sm) {
                ph.perm = true; ph.perm_op = perm->opcode; ph.perm_lane = perm->lane; ph.perm_mask = perm->mask;
                ph.perm_q = perm->q32; ph.perm_rep = perm->rep; ph.perm_seed = perm->seed;
                h = &ph;
            }
            rr[i] = run_warp(P, out.mem, k, cta, wic, h, wd, &st[i],
                             keep_trace ? &ts : nullptr, wcounts ? &(*wcounts)[8 * (size_t)w] : nullptr);
            if (wlen_out) (*wlen_out)[w] = rr[i].steps;
            if (keep_trace) (*wtraces)[w] = std::move(tr);
        };
        if (hook || perm) for (uint32_t i = 0; i < nw; ++i) body(i);   // replica-level parallelism instead
        else parallel_for(nw, n_threads, body);
        for (uint32_t i = 0; i < nw; ++i) {
            if (!rr[i].fault) continue;
            if (unchecked && rr[i].fault != 3) {
                if (!out.pdue) { out.pdue = rr[i].fault; out.pdue_pc = rr[i].fault_pc; }
                continue;
            }
            if (!out.fault) { out.fault = rr[i].fault; out.fault_pc = rr[i].fault_pc; }
        }
        if (out.fault) {
            if (err) *err = "fault in golden run at instance " + std::to_string(k) + " pc " + std::to_string(out.fault_pc);
            break;
        }
        uint32_t hw = hook ? hook_warp : UINT32_MAX;
        for (uint32_t i = 0; i < nw; ++i) {
            if (in.warp_begin + i == hw) continue;
            apply_stores(out.mem, st[i]);
            if (n_gstores) *n_gstores += st[i].size();
        }
        if (hw >= in.warp_begin && hw < in.warp_end) {
            apply_stores(out.mem, st[hw - in.warp_begin]);
            out.n_faulty_stores = st[hw - in.warp_begin].size();
        }
    }
}

bool output_differs(const Prog& P, const std::vector<uint8_t>& a, const std::vector<uint8_t>& b) {
    for (uint32_t i = 0; i < P.p.n_buf; ++i) {
        const orc_buffer& bf = P.p.buf[i];
        if (!(bf.flags & 1)) continue;
        if (memcmp(&a[bf.off], &b[bf.off], bf.size)) return true;
    }
    return false;
}

// C-12 secondary numeric classification (BASELINE.md §2 "rtol = 1e-6, atol = 0,
// NaN != number"): a faulty element f differs from the golden element g beyond
// rtol unless the bits are equal, or the buffer is a float buffer and both are
// finite with |f - g| <= rtol * |g| (IEEE double, round to nearest: this file is
// compiled with -ffp-contract=off).  u32 buffers: any difference.
enum { DT_U32 = 0, DT_F32 = 1, DT_F64 = 2 };
uint32_t buf_dtype_of(const orc_buffer& b) { return (b.flags >> 8) & 0xFF; }
bool elem_beyond_tol(uint32_t dtype, uint64_t fbits, uint64_t gbits, double rtol) {
    if (fbits == gbits) return false;
    double f, g;
    if (dtype == DT_F32) { f = (double)f32((uint32_t)fbits); g = (double)f32((uint32_t)gbits); }
    else if (dtype == DT_F64) { f = f64(fbits); g = f64(gbits); }
    else return true;
    if (!std::isfinite(f) || !std::isfinite(g)) return true;
    return !(std::fabs(f - g) <= rtol * std::fabs(g));
}

// Element by element over every output buffer: does the faulty image differ from
// the golden one beyond rtol somewhere?
bool output_beyond_tol(const Prog& P, const std::vector<uint8_t>& a, const std::vector<uint8_t>& b, double rtol) {
    for (uint32_t i = 0; i < P.p.n_buf; ++i) {
        const orc_buffer& bf = P.p.buf[i];
        if (!(bf.flags & 1)) continue;
        const uint32_t dt = buf_dtype_of(bf);
        const uint64_t w = dt == DT_F64 ? 8 : 4;
        for (uint64_t o = 0; o + w <= bf.size; o += w) {
            uint64_t x = 0, y = 0;
            memcpy(&x, &a[bf.off + o], w);
            memcpy(&y, &b[bf.off + o], w);
            if (elem_beyond_tol(dt, x, y, rtol)) return true;
        }
    }
    return false;
}

const orc_buffer* buffer_of(const Prog& P, uint64_t va) { return find_buffer(P, va - VA_BASE); }

bool is_output_addr(const Prog& P, uint64_t va) {
    const orc_buffer* b = find_buffer(P, va - VA_BASE);
    return b && (b->flags & 1);
}

}  // namespace

// ===========================================================================
// C API
// ===========================================================================
static std::string g_last_error;
extern "C" const char* orc_last_error(void) { return g_last_error.c_str(); }

extern "C" void* orc_golden_run(const orc_program* p, int n_threads, int keep_trace) {
    Golden* G = new Golden;
    if (!prepare(G->P, p, G->err)) { g_last_error = G->err; delete G; return nullptr; }
    const Prog& P = G->P;
    G->wlen.assign(P.n_warps, 0);
    G->wcounts.assign((size_t)P.n_warps * 8, 0);
    G->winst.resize(P.n_warps);
    for (uint32_t k = 0; k < P.p.n_inst; ++k)
        for (uint32_t w = P.p.inst[k].warp_begin; w < P.p.inst[k].warp_end; ++w) G->winst[w] = k;
    std::vector<std::vector<orc_record>> wtr;
    if (keep_trace) wtr.resize(P.n_warps);
    FullRun fr;
    std::string err;
    run_program(nullptr, P, nullptr, 0, n_threads, fr, &G->wlen, &G->wcounts, keep_trace, &wtr, &G->n_gstores, &err);
    if (fr.fault) { g_last_error = err; delete G; return nullptr; }
    G->final_mem = std::move(fr.mem);
    G->counts.assign((size_t)P.p.n_inst * 8, 0);
    for (uint32_t w = 0; w < P.n_warps; ++w) {
        for (int g = 0; g < 8; ++g) G->counts[8 * (size_t)G->winst[w] + g] += G->wcounts[8 * (size_t)w + g];
        G->n_rec += G->wlen[w];
    }
    if (keep_trace) {
        G->kept = true;
        G->woff.resize(P.n_warps + 1, 0);
        G->trace.reserve(G->n_rec);
        for (uint32_t w = 0; w < P.n_warps; ++w) {
            G->woff[w] = G->trace.size();
            G->trace.insert(G->trace.end(), wtr[w].begin(), wtr[w].end());
        }
        G->woff[P.n_warps] = G->trace.size();
    }
    return G;
}

extern "C" void orc_free(void* h) { delete (Golden*)h; }
extern "C" const char* orc_error(void* h) { return ((Golden*)h)->err.c_str(); }
extern "C" uint32_t orc_n_warps(void* h) { return ((Golden*)h)->P.n_warps; }
extern "C" uint64_t orc_n_records(void* h) { return ((Golden*)h)->n_rec; }
extern "C" uint64_t orc_n_golden_stores(void* h) { return ((Golden*)h)->n_gstores; }
extern "C" void orc_counts(void* h, uint64_t* out) { auto& v = ((Golden*)h)->counts; std::copy(v.begin(), v.end(), out); }
extern "C" void orc_warp_counts(void* h, uint64_t* out) { auto& v = ((Golden*)h)->wcounts; std::copy(v.begin(), v.end(), out); }
extern "C" void orc_warp_len(void* h, uint64_t* out) { auto& v = ((Golden*)h)->wlen; std::copy(v.begin(), v.end(), out); }
extern "C" void orc_final_image(void* h, uint8_t* out) { auto& v = ((Golden*)h)->final_mem; std::copy(v.begin(), v.end(), out); }
extern "C" int orc_trace(void* h, orc_record* out) {
    Golden* G = (Golden*)h;
    if (!G->kept) return 1;
    std::copy(G->trace.begin(), G->trace.end(), out);
    return 0;
}

extern "C" uint64_t orc_count_warps(const orc_program* p, uint32_t w0, uint32_t w1, int n_threads, uint64_t* counts8) {
    Prog P;
    std::string err;
    if (!prepare(P, p, err) || P.p.n_inst != 1) return 0;
    std::vector<uint8_t> mem(p->init_image, p->init_image + p->image_bytes);
    std::vector<uint64_t> wc((size_t)(w1 - w0) * 8, 0), wl(w1 - w0, 0);
    parallel_for(w1 - w0, n_threads, [&](uint32_t i) {
        uint32_t cta, wic;
        warp_coords(P.p.inst[0], w0 + i, cta, wic);
        std::vector<StoreW> st;
        WarpResult r = run_warp(P, mem, 0, cta, wic, nullptr, UINT64_MAX, &st, nullptr, &wc[8 * (size_t)i]);
        wl[i] = r.steps;
    });
    uint64_t n = 0;
    for (int g = 0; g < 8; ++g) counts8[g] = 0;
    for (uint32_t i = 0; i < w1 - w0; ++i) {
        n += wl[i];
        for (int g = 0; g < 8; ++g) counts8[g] += wc[8 * (size_t)i + g];
    }
    return n;
}

extern "C" void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) { philox(ctr, key, out); }
extern "C" void orc_draw(uint64_t seed, uint64_t j, uint64_t n_g, uint64_t* s, uint32_t* u_dst, uint32_t* u_bit, uint32_t* att) {
    draw(seed, j, n_g, *s, *u_dst, *u_bit, *att);
}
extern "C" uint32_t orc_mask(int bfm, uint32_t u) { return mask_of(bfm, u); }
extern "C" uint32_t orc_group_mask(const orc_insn* I) { return group_mask(*I); }
extern "C" uint32_t orc_dest_slots(const orc_insn* I, int g, uint8_t* kind, uint8_t* reg) {
    std::vector<std::pair<int, int>> s;
    slots_for(*I, g, s);
    for (size_t i = 0; i < s.size(); ++i) { kind[i] = (uint8_t)s[i].first; reg[i] = (uint8_t)s[i].second; }
    return (uint32_t)s.size();
}

// Selection: site s of group g is the s-th (0-based, C-4) counted
// lane-instruction of group g in canonical order (C-3): warps in trace order,
// dynamic order within a warp, lanes ascending within a record.  `out[i]` must
// already hold s, group, u_dst (and bfm/mask); this fills the location.
static int enumerate_sites_by_warp(Golden* G, uint32_t n, orc_site* out);

static int enumerate_sites(Golden* G, uint32_t n, orc_site* out) {
    const Prog& P = G->P;
    if (!G->kept) return enumerate_sites_by_warp(G, n, out);
    struct Want { uint64_t s; uint32_t idx; };
    std::vector<std::vector<Want>> per_g(8);
    for (uint32_t i = 0; i < n; ++i) per_g[out[i].group & 7].push_back({out[i].s, i});
    for (int g = 0; g < 8; ++g) {
        auto& v = per_g[g];
        if (v.empty()) continue;
        std::sort(v.begin(), v.end(), [](const Want& a, const Want& b) { return a.s < b.s; });
        uint64_t cum = 0;          // sites of group g before the current record
        size_t q = 0;
        std::vector<uint64_t> inst_before(P.p.n_inst + 1, 0);
        for (uint32_t k = 0; k < P.p.n_inst; ++k) inst_before[k + 1] = inst_before[k] + G->counts[8 * (size_t)k + g];
        for (uint32_t w = 0; w < P.n_warps && q < v.size(); ++w) {
            for (uint64_t r = G->woff[w]; r < G->woff[w + 1] && q < v.size(); ++r) {
                const orc_record& R = G->trace[r];
                if (!((R.insn >> (24 + g)) & 1)) continue;
                uint32_t ex = R.active & R.pred;
                uint64_t c = (uint64_t)__builtin_popcount(ex);
                while (q < v.size() && v[q].s < cum + c) {
                    uint64_t rank = v[q].s - cum;         // which counted lane, ascending
                    int lane = -1;
                    for (int l = 0, seen = 0; l < 32; ++l)
                        if ((ex >> l) & 1) { if ((uint64_t)seen == rank) { lane = l; break; } ++seen; }
                    orc_site& S = out[v[q].idx];
                    uint32_t k = R.instance;
                    const orc_instance& in = P.p.inst[k];
                    uint32_t cta, wic;
                    warp_coords(in, w, cta, wic);
                    S.instance = k; S.kernel_id = in.kernel; S.kernel_count = in.kernel_count;
                    S.warp = w; S.step = (uint32_t)(r - G->woff[w]); S.lane = (uint8_t)lane;
                    S.thread = cta * in.block + wic * 32 + (uint32_t)lane;
                    S.pc = R.insn & 0xFFFF;
                    S.instruction_count = v[q].s - inst_before[k];
                    const orc_insn& I = P.p.code[P.p.kern[in.kernel].code_off + S.pc];
                    std::vector<std::pair<int, int>> sl;
                    slots_for(I, g, sl);
                    if (sl.empty()) { G->err = "site without eligible destination"; return 4; }
                    S.n_elig = (uint8_t)sl.size();
                    S.slot = (uint8_t)(((uint64_t)sl.size() * S.u_dst) >> 32);   // floor(n x value), C-5
                    S.dst_kind = (uint8_t)sl[S.slot].first;
                    S.dst_reg = (uint8_t)sl[S.slot].second;
                    ++q;
                }
                cum += c;
            }
        }
        if (q != v.size()) { G->err = "s beyond the group's site count"; return 4; }
    }
    return 0;
}

// Selection without a kept trace (single-instance programs at full size, whose
// App. A.3 trace does not fit in host RAM): the same canonical order (C-3).  The
// warp holding site s is the first whose cumulative group-g count — warps in
// trace order, per-warp counts of the golden run — exceeds s; the rank inside
// it is found by re-interpreting that warp from the memory before the instance
// (the initial image of a single-instance program) and walking its records
// exactly as enumerate_sites walks the kept trace.
static int enumerate_sites_by_warp(Golden* G, uint32_t n, orc_site* out) {
    const Prog& P = G->P;
    if (!P.single_instance()) { G->err = "selection without a kept trace needs a single-instance program"; return 1; }
    std::vector<uint64_t> rank(n, 0);
    std::map<uint32_t, std::vector<uint32_t>> by_warp;      // warp -> indices into out
    for (int g = 0; g < 8; ++g) {
        std::vector<std::pair<uint64_t, uint32_t>> v;
        for (uint32_t i = 0; i < n; ++i) if ((out[i].group & 7) == g) v.push_back({out[i].s, i});
        if (v.empty()) continue;
        std::sort(v.begin(), v.end());
        uint64_t cum = 0;
        size_t q = 0;
        for (uint32_t w = 0; w < P.n_warps && q < v.size(); ++w) {
            uint64_t c = G->wcounts[8 * (size_t)w + g];
            while (q < v.size() && v[q].first < cum + c) {
                rank[v[q].second] = v[q].first - cum;
                by_warp[w].push_back(v[q].second);
                ++q;
            }
            cum += c;
        }
        if (q != v.size()) { G->err = "s beyond the group's site count"; return 4; }
    }
    std::vector<std::pair<uint32_t, std::vector<uint32_t>>> jobs(by_warp.begin(), by_warp.end());
    const std::vector<uint8_t> pre(P.p.init_image, P.p.init_image + P.p.image_bytes);
    const orc_instance& in = P.p.inst[0];
    std::atomic<int> status{0};
    parallel_for((uint32_t)jobs.size(), (int)std::max(1u, std::thread::hardware_concurrency()), [&](uint32_t jb) {
        uint32_t w = jobs[jb].first, cta, wic;
        warp_coords(in, w, cta, wic);
        std::vector<orc_record> tr;
        TraceSink ts;
        ts.rec = &tr;
        std::vector<StoreW> st;
        run_warp(P, pre, 0, cta, wic, nullptr, UINT64_MAX, &st, &ts, nullptr);
        for (uint32_t i : jobs[jb].second) {
            orc_site& S = out[i];
            const int g = S.group & 7;
            uint64_t seen = 0;
            bool found = false;
            for (size_t r = 0; r < tr.size() && !found; ++r) {
                if (!((tr[r].insn >> (24 + g)) & 1)) continue;
                uint32_t ex = tr[r].active & tr[r].pred;
                for (int l = 0; l < 32 && !found; ++l) {
                    if (!((ex >> l) & 1)) continue;
                    if (seen++ != rank[i]) continue;
                    S.instance = 0; S.kernel_id = in.kernel; S.kernel_count = in.kernel_count;
                    S.warp = w; S.step = (uint32_t)r; S.lane = (uint8_t)l;
                    S.thread = cta * in.block + wic * 32 + (uint32_t)l;
                    S.pc = tr[r].insn & 0xFFFF;
                    S.instruction_count = S.s;
                    const orc_insn& I = P.p.code[P.p.kern[in.kernel].code_off + S.pc];
                    std::vector<std::pair<int, int>> sl;
                    slots_for(I, g, sl);
                    if (sl.empty()) { status = 4; return; }
                    S.n_elig = (uint8_t)sl.size();
                    S.slot = (uint8_t)(((uint64_t)sl.size() * S.u_dst) >> 32);   // floor(n x value), C-5
                    S.dst_kind = (uint8_t)sl[S.slot].first;
                    S.dst_reg = (uint8_t)sl[S.slot].second;
                    found = true;
                }
            }
            if (!found) status = 4;
        }
    });
    if (status) { G->err = "warp re-run disagrees with the golden per-warp counts"; return 4; }
    return 0;
}

extern "C" int orc_select(void* h, uint64_t seed, const uint8_t* groups, uint32_t n_groups,
                          const uint8_t* bfms, uint32_t n_bfms, uint64_t j0, uint32_t n, orc_site* out) {
    Golden* G = (Golden*)h;
    const Prog& P = G->P;
    if (n_groups == 0 || n_bfms == 0) { G->err = "empty schedule"; return 1; }
    std::vector<uint64_t> total(8, 0);
    for (uint32_t k = 0; k < P.p.n_inst; ++k) for (int g = 0; g < 8; ++g) total[g] += G->counts[8 * (size_t)k + g];
    for (uint32_t i = 0; i < n; ++i) {
        uint64_t j = j0 + i;
        int g = groups[j % n_groups], b = bfms[(j / n_groups) % n_bfms];
        if (g == ORC_G_NODEST) { G->err = "G_NODEST is not injectable (C-16)"; return 3; }
        if (total[g] == 0) { G->err = "empty group"; return 2; }
        orc_site& S = out[i];
        memset(&S, 0, sizeof(S));
        uint32_t att;
        draw(seed, j, total[g], S.s, S.u_dst, S.u_bit, att);
        S.group = (uint8_t)g; S.bfm = (uint8_t)b;
        S.mask = mask_of(b, S.u_bit);
    }
    return enumerate_sites(G, n, out);
}

// Row f1, per-opcode profile ("counts for every opcode"): the plain
// sum of popc(active & pred) per (instance, opcode) over the trace.
extern "C" int orc_opcode_counts(void* h, uint64_t* out /*[n_inst][32]*/) {
    Golden* G = (Golden*)h;
    if (!G->kept) return 1;
    std::fill(out, out + (size_t)G->P.p.n_inst * 32, 0);
    for (const orc_record& R : G->trace)
        out[(size_t)R.instance * 32 + ((R.insn >> 16) & 31)] += (uint64_t)__builtin_popcount(R.active & R.pred);
    return 0;
}

// Row f1, approximate profiling: every instance is assumed to have
// the counts of the first instance of its static kernel.
static void approx_counts(const Golden* G, std::vector<uint64_t>& a) {
    const Prog& P = G->P;
    a.assign((size_t)P.p.n_inst * 8, 0);
    std::vector<int64_t> first(P.p.n_kern, -1);
    for (uint32_t k = 0; k < P.p.n_inst; ++k) {
        uint32_t kern = P.p.inst[k].kernel;
        if (first[kern] < 0) first[kern] = k;
        for (int g = 0; g < 8; ++g) a[8 * (size_t)k + g] = G->counts[8 * (size_t)first[kern] + g];
    }
}

extern "C" int orc_approx_counts(void* h, uint64_t* out) {
    std::vector<uint64_t> a;
    approx_counts((Golden*)h, a);
    std::copy(a.begin(), a.end(), out);
    return 0;
}

// Selection over an approximate profile: s is drawn over the approximate totals
// and read as (instance k, instruction_count) in launch order; the site is the
// instruction_count-th group-g site of instance k itself (C-3), or does not
// exist (C-17: flags = 1, "not injected").
extern "C" int orc_select_approx(void* h, uint64_t seed, const uint8_t* groups, uint32_t n_groups,
                                 const uint8_t* bfms, uint32_t n_bfms, uint64_t j0, uint32_t n, orc_site* out) {
    Golden* G = (Golden*)h;
    const Prog& P = G->P;
    if (!G->kept) { G->err = "selection needs keep_trace"; return 1; }
    if (n_groups == 0 || n_bfms == 0) { G->err = "empty schedule"; return 1; }
    std::vector<uint64_t> a;
    approx_counts(G, a);
    std::vector<uint64_t> total(8, 0);
    for (uint32_t k = 0; k < P.p.n_inst; ++k) for (int g = 0; g < 8; ++g) total[g] += a[8 * (size_t)k + g];
    for (uint32_t i = 0; i < n; ++i) {
        uint64_t j = j0 + i;
        int g = groups[j % n_groups], b = bfms[(j / n_groups) % n_bfms];
        if (g == ORC_G_NODEST) { G->err = "G_NODEST is not injectable (C-16)"; return 3; }
        if (total[g] == 0) { G->err = "empty group"; return 2; }
        orc_site& S = out[i];
        memset(&S, 0, sizeof(S));
        uint32_t att;
        draw(seed, j, total[g], S.s, S.u_dst, S.u_bit, att);
        S.group = (uint8_t)g; S.bfm = (uint8_t)b;
        S.mask = mask_of(b, S.u_bit);
        uint64_t cum = 0;
        uint32_t k = 0;
        for (k = 0; k < P.p.n_inst; ++k) {                // instance whose approximate range holds s
            if (S.s < cum + a[8 * (size_t)k + g]) break;
            cum += a[8 * (size_t)k + g];
        }
        const orc_instance& in = P.p.inst[k];
        S.instance = k; S.kernel_id = in.kernel; S.kernel_count = in.kernel_count;
        S.instruction_count = S.s - cum;
        uint64_t seen = 0;
        bool found = false;
        for (uint32_t w = in.warp_begin; w < in.warp_end && !found; ++w) {
            for (uint64_t r = G->woff[w]; r < G->woff[w + 1] && !found; ++r) {
                const orc_record& R = G->trace[r];
                if (!((R.insn >> (24 + g)) & 1)) continue;
                uint32_t ex = R.active & R.pred;
                for (int l = 0; l < 32 && !found; ++l) {
                    if (!((ex >> l) & 1)) continue;
                    if (seen == S.instruction_count) {
                        uint32_t cta, wic;
                        warp_coords(in, w, cta, wic);
                        S.warp = w; S.step = (uint32_t)(r - G->woff[w]); S.lane = (uint8_t)l;
                        S.thread = cta * in.block + wic * 32 + (uint32_t)l;
                        S.pc = R.insn & 0xFFFF;
                        const orc_insn& I = P.p.code[P.p.kern[in.kernel].code_off + S.pc];
                        std::vector<std::pair<int, int>> sl;
                        slots_for(I, g, sl);
                        S.n_elig = (uint8_t)sl.size();
                        S.slot = (uint8_t)(((uint64_t)sl.size() * S.u_dst) >> 32);
                        S.dst_kind = (uint8_t)sl[S.slot].first;
                        S.dst_reg = (uint8_t)sl[S.slot].second;
                        found = true;
                    }
                    ++seen;
                }
            }
        }
        if (!found) S.flags = 1;
    }
    return 0;
}

// Locate given indices s (u_dst = 0, FLIP_SINGLE_BIT with u_bit = 0): the
// enumeration alone, for the brute-force bijection pin.
extern "C" int orc_locate(void* h, int group, const uint64_t* s, uint32_t n, orc_site* out) {
    for (uint32_t i = 0; i < n; ++i) {
        memset(&out[i], 0, sizeof(orc_site));
        out[i].s = s[i]; out[i].group = (uint8_t)group; out[i].mask = 1;
    }
    return enumerate_sites((Golden*)h, n, out);
}

// Injection + classification.  FULL: the definition — re-run the whole program
// from its initial memory with the corruption, then compare every output
// buffer with the golden run bitwise (C-12), DUE taking precedence (Table V).
// WARP_LOCAL (single-instance programs): re-run only warp w, faulty and golden,
// and compare the final value of every address either run stored to (C-14).
// ORC_UNCHECKED in `mode` selects the potential-DUE semantics of row f4.
extern "C" int orc_inject(void* h, const orc_site* sites, uint32_t n, int mode, int n_threads, double rtol,
                          orc_inj* out) {
    Golden* G = (Golden*)h;
    const Prog& P = G->P;
    const bool unchecked = mode & ORC_UNCHECKED;
    mode &= ~ORC_UNCHECKED;
    if (mode == ORC_MODE_WARP_LOCAL && !P.single_instance()) mode = ORC_MODE_FULL;
    std::atomic<int> status{0};
    std::mutex mu;
    parallel_for(n, n_threads, [&](uint32_t i) {
        const orc_site& S = sites[i];
        orc_inj& R = out[i];
        memset(&R, 0, sizeof(R));
        if (S.flags & 1) { R.outcome = ORC_NOT_INJECTED; return; }      // C-17
        Hook hk;
        hk.on = true; hk.step = S.step; hk.lane = S.lane; hk.kind = S.dst_kind; hk.reg = S.dst_reg;
        hk.bfm = S.bfm; hk.mask = S.mask; hk.pc = S.pc;
        int fault = 0, pdue = 0; uint32_t fpc = 0; bool sdc = false, beyond = false;
        if (mode == ORC_MODE_FULL) {
            FullRun fr;
            run_program(G, P, &hk, S.warp, 1, fr, nullptr, nullptr, false, nullptr, nullptr, nullptr, unchecked);
            fault = fr.fault; fpc = fr.fault_pc;
            if (!fault && fr.pdue) { pdue = fr.pdue; fpc = fr.pdue_pc; }
            R.n_faulty_stores = (uint32_t)fr.n_faulty_stores;
            if (!fault) sdc = output_differs(P, fr.mem, G->final_mem);
            if (sdc && rtol > 0) beyond = output_beyond_tol(P, fr.mem, G->final_mem, rtol);
        } else {
            const orc_instance& in = P.p.inst[S.instance];
            uint32_t cta, wic;
            warp_coords(in, S.warp, cta, wic);
            std::vector<uint8_t> pre(P.p.init_image, P.p.init_image + P.p.image_bytes);
            std::vector<StoreW> fst, gst;
            WarpResult fr = run_warp(P, pre, S.instance, cta, wic, &hk, 10 * G->wlen[S.warp] + 1024, &fst, nullptr, nullptr);
            fault = fr.fault; fpc = fr.fault_pc;
            if (unchecked && fault && fault != 3) { pdue = fault; fault = 0; }   // the warp just stops (f4)
            R.n_faulty_stores = (uint32_t)fst.size();
            if (!fault) {
                run_warp(P, pre, S.instance, cta, wic, nullptr, UINT64_MAX, &gst, nullptr, nullptr);
                std::map<uint64_t, uint32_t> fin;                // faulty final value per address
                for (const StoreW& s : fst) fin[s.va] = s.value;
                for (const StoreW& s : gst)                       // golden-only: pre-instance value
                    if (!fin.count(s.va)) { uint32_t x; memcpy(&x, &pre[s.va - VA_BASE], 4); fin[s.va] = x; }
                for (auto& kv : fin) {
                    uint32_t g; memcpy(&g, &G->final_mem[kv.first - VA_BASE], 4);
                    if (g != kv.second && is_output_addr(P, kv.first)) { sdc = true; break; }
                }
                // rtol: each differing output element, its other words taken from
                // the faulty final state (fin) or, if untouched, the golden image
                if (sdc && rtol > 0) {
                    for (auto& kv : fin) {
                        const orc_buffer* b = buffer_of(P, kv.first);
                        if (!b || !(b->flags & 1)) continue;
                        const uint32_t dt = buf_dtype_of(*b);
                        const uint64_t w = dt == DT_F64 ? 8 : 4, e = kv.first - (kv.first - VA_BASE - b->off) % w;
                        uint64_t fe = 0, ge = 0;
                        for (uint64_t q = 0; q < w; q += 4) {
                            uint32_t gw, fw;
                            memcpy(&gw, &G->final_mem[e + q - VA_BASE], 4);
                            auto it = fin.find(e + q);
                            fw = it != fin.end() ? it->second : gw;
                            fe |= (uint64_t)fw << (8 * q);
                            ge |= (uint64_t)gw << (8 * q);
                        }
                        if (elem_beyond_tol(dt, fe, ge, rtol)) { beyond = true; break; }
                    }
                }
            }
        }
        if (!hk.fired || hk.bad) {
            std::lock_guard<std::mutex> lk(mu);
            G->err = "injection site not reached as selected (replica " + std::to_string(i) + ")";
            status = 4;
        }
        R.before = hk.before; R.after = hk.after; R.mask = hk.applied_mask;
        R.fault_kind = (uint8_t)(fault ? fault : pdue); R.fault_pc = fpc;
        R.flags = (uint8_t)((pdue ? ORC_POTENTIAL_DUE : 0) | (!fault && sdc && rtol > 0 && !beyond ? ORC_SDC_WITHIN_TOL : 0));
        R.outcome = fault ? ORC_DUE : (sdc ? ORC_SDC : ORC_MASKED);
    });
    return status;
}

// ---------------------------------------------------------------------------
// Single-instance helpers that need no whole-program golden run (full-size
// sampled parity and bounded CPU baselines).  Same definitions as above,
// restricted to one warp: the golden warp w and the faulty warp w are
// interpreted from the initial image (= the memory before the only instance).
// ---------------------------------------------------------------------------

// Rank of (step, lane) among the group-g sites of warp w in canonical order (C-3),
// and warp w's total group-g count.  Returns 0, or 1 if (step, lane) is not a site.
extern "C" int orc_warp_site_rank(const orc_program* p, uint32_t w, int g, uint32_t step, uint32_t lane,
                                  uint64_t* rank, uint64_t* total) {
    Prog P;
    std::string err;
    if (!prepare(P, p, err) || P.p.n_inst != 1 || w >= P.n_warps) return 2;
    std::vector<uint8_t> mem(p->init_image, p->init_image + p->image_bytes);
    std::vector<orc_record> tr;
    TraceSink ts;
    ts.rec = &tr;
    std::vector<StoreW> st;
    uint32_t cta, wic;
    warp_coords(P.p.inst[0], w, cta, wic);
    run_warp(P, mem, 0, cta, wic, nullptr, UINT64_MAX, &st, &ts, nullptr);
    uint64_t before = 0, tot = 0;
    bool hit = false;
    for (size_t r = 0; r < tr.size(); ++r) {
        if (!((tr[r].insn >> (24 + g)) & 1)) continue;
        uint32_t ex = tr[r].active & tr[r].pred;
        for (uint32_t l = 0; l < 32; ++l) {
            if (!((ex >> l) & 1)) continue;
            if (r == step && l == lane) { hit = true; before = tot; }
            ++tot;
        }
    }
    *rank = before;
    *total = tot;
    return hit ? 0 : 1;
}

// The inverse: the (step, lane, pc) of the rank-th group-g site of warp w
// (canonical order, C-3).  Returns 0, or 1 if rank >= warp w's group-g count.
extern "C" int orc_warp_site_at(const orc_program* p, uint32_t w, int g, uint64_t rank,
                                uint32_t* step, uint32_t* lane, uint32_t* pc) {
    Prog P;
    std::string err;
    if (!prepare(P, p, err) || P.p.n_inst != 1 || w >= P.n_warps) return 2;
    std::vector<uint8_t> mem(p->init_image, p->init_image + p->image_bytes);
    std::vector<orc_record> tr;
    TraceSink ts;
    ts.rec = &tr;
    std::vector<StoreW> st;
    uint32_t cta, wic;
    warp_coords(P.p.inst[0], w, cta, wic);
    run_warp(P, mem, 0, cta, wic, nullptr, UINT64_MAX, &st, &ts, nullptr);
    uint64_t seen = 0;
    for (size_t r = 0; r < tr.size(); ++r) {
        if (!((tr[r].insn >> (24 + g)) & 1)) continue;
        uint32_t ex = tr[r].active & tr[r].pred;
        for (uint32_t l = 0; l < 32; ++l) {
            if (!((ex >> l) & 1)) continue;
            if (seen == rank) { *step = (uint32_t)r; *lane = l; *pc = tr[r].insn & 0xFFFF; return 0; }
            ++seen;
        }
    }
    return 1;
}

// Warp-local injection without a whole-program golden run.  decided[i] = 0 when
// the outcome needs the golden value of a word written by ANOTHER warp (a wild
// faulty store into an output word outside warp w's golden stores) and no
// decided SDC word exists; otherwise the outcome is exact.
extern "C" int orc_inject_local(const orc_program* p, const orc_site* sites, uint32_t n, int n_threads,
                                orc_inj* out, uint8_t* decided) {
    Prog P;
    std::string err;
    if (!prepare(P, p, err) || P.p.n_inst != 1) return 2;
    const std::vector<uint8_t> pre(p->init_image, p->init_image + p->image_bytes);
    std::atomic<int> status{0};
    parallel_for(n, n_threads, [&](uint32_t i) {
        const orc_site& S = sites[i];
        orc_inj& R = out[i];
        memset(&R, 0, sizeof(R));
        uint32_t cta, wic;
        warp_coords(P.p.inst[0], S.warp, cta, wic);
        std::vector<StoreW> gst, fst;
        WarpResult gr = run_warp(P, pre, 0, cta, wic, nullptr, UINT64_MAX, &gst, nullptr, nullptr);
        Hook hk;
        hk.on = true; hk.step = S.step; hk.lane = S.lane; hk.kind = S.dst_kind; hk.reg = S.dst_reg;
        hk.bfm = S.bfm; hk.mask = S.mask; hk.pc = S.pc;
        WarpResult fr = run_warp(P, pre, 0, cta, wic, &hk, 10 * gr.steps + 1024, &fst, nullptr, nullptr);
        if (!hk.fired || hk.bad) status = 4;
        R.before = hk.before; R.after = hk.after; R.mask = hk.applied_mask;
        R.fault_kind = (uint8_t)fr.fault; R.fault_pc = fr.fault_pc;
        R.n_faulty_stores = (uint32_t)fst.size();
        decided[i] = 1;
        if (fr.fault) { R.outcome = ORC_DUE; return; }
        std::map<uint64_t, uint32_t> gold, fin;
        for (const StoreW& s : gst) gold[s.va] = s.value;
        for (const StoreW& s : fst) fin[s.va] = s.value;
        for (const StoreW& s : gst)
            if (!fin.count(s.va)) { uint32_t x; memcpy(&x, &pre[s.va - VA_BASE], 4); fin[s.va] = x; }
        bool sdc = false, unknown = false;
        for (auto& kv : fin) {
            if (!is_output_addr(P, kv.first)) continue;
            auto it = gold.find(kv.first);
            if (it == gold.end()) { unknown = true; continue; }
            if (it->second != kv.second) { sdc = true; break; }
        }
        R.outcome = sdc ? ORC_SDC : ORC_MASKED;
        if (!sdc && unknown) decided[i] = 0;
    });
    return status;
}

// Rows f2/f3: permanent / intermittent faults by the definition — the whole
// program re-run with the fault armed on every warp of every CTA mapped to the
// faulty SM (CTA c on SM c mod n_sm, reading C-21), outputs compared bitwise
// with the golden run (Table V), DUE taking precedence (C-9, C-10; f4 under
// ORC_UNCHECKED).
extern "C" int orc_inject_permanent(void* h, const orc_pfault* pf, uint32_t n, int mode, int n_threads, orc_inj* out) {
    Golden* G = (Golden*)h;
    const Prog& P = G->P;
    const bool unchecked = mode & ORC_UNCHECKED;
    parallel_for(n, n_threads, [&](uint32_t i) {
        orc_inj& R = out[i];
        memset(&R, 0, sizeof(R));
        PermSpec ps{pf[i].opcode, pf[i].sm, pf[i].lane, pf[i].mask, pf[i].q32, pf[i].n_sm ? pf[i].n_sm : 148, i,
                    pf[i].seed};
        FullRun fr;
        run_program(G, P, nullptr, 0, 1, fr, nullptr, nullptr, false, nullptr, nullptr, nullptr, unchecked, &ps);
        R.mask = pf[i].mask;
        if (fr.fault) { R.outcome = ORC_DUE; R.fault_kind = (uint8_t)fr.fault; R.fault_pc = fr.fault_pc; return; }
        R.flags = fr.pdue ? ORC_POTENTIAL_DUE : 0;
        R.fault_kind = (uint8_t)fr.pdue; R.fault_pc = fr.pdue_pc;
        R.outcome = output_differs(P, fr.mem, G->final_mem) ? ORC_SDC : ORC_MASKED;
    });
    return 0;
}

// The faulty final image of one permanent / intermittent fault replica `rep`
// (test pins of rows f2/f3).  Returns the fault kind (0 = none).
extern "C" int orc_permanent_image(void* h, const orc_pfault* pf, uint32_t rep, int mode, uint8_t* out_image) {
    Golden* G = (Golden*)h;
    PermSpec ps{pf->opcode, pf->sm, pf->lane, pf->mask, pf->q32, pf->n_sm ? pf->n_sm : 148, rep, pf->seed};
    FullRun fr;
    run_program(G, G->P, nullptr, 0, 1, fr, nullptr, nullptr, false, nullptr, nullptr, nullptr,
                (mode & ORC_UNCHECKED) != 0, &ps);
    std::copy(fr.mem.begin(), fr.mem.end(), out_image);
    return fr.fault ? fr.fault : fr.pdue;
}

// The faulty final image of one transient site by the definition (full mode:
// the whole program re-run with the corruption, PAPER.md:72 step (4), :78,
// :138) — for the multi-launch propagation pins.  Returns the fault kind
// (0 = none), or -1 if the site was not reached as selected.
extern "C" int orc_inject_image(void* h, const orc_site* site, int mode, uint8_t* out_image) {
    Golden* G = (Golden*)h;
    const orc_site& S = *site;
    Hook hk;
    hk.on = true; hk.step = S.step; hk.lane = S.lane; hk.kind = S.dst_kind; hk.reg = S.dst_reg;
    hk.bfm = S.bfm; hk.mask = S.mask; hk.pc = S.pc;
    FullRun fr;
    run_program(G, G->P, &hk, S.warp, 1, fr, nullptr, nullptr, false, nullptr, nullptr, nullptr,
                (mode & ORC_UNCHECKED) != 0);
    std::copy(fr.mem.begin(), fr.mem.end(), out_image);
    if (!hk.fired || hk.bad) return -1;
    return fr.fault ? fr.fault : fr.pdue;
}

// The profiler's count over a trace already in host RAM ("dynamic
// instruction counts ... Instructions that are not executed based on a predicate
// register are not included"): for every App. A.3 record, popc(active & pred)
// added to counts[instance][g] for each group g of its groupmask (Table II).  A
// plain loop per record; threads take contiguous record ranges and their
// partial sums are added at the end.  The CPU baseline of K1.
extern "C" int orc_scan_trace(const orc_record* rec, uint64_t n, uint32_t n_inst, int n_threads, uint64_t* counts) {
    n_threads = std::max(1, n_threads);
    std::vector<std::vector<uint64_t>> part(n_threads, std::vector<uint64_t>((size_t)n_inst * 8, 0));
    std::atomic<int> bad{0};
    std::vector<std::thread> th;
    for (int t = 0; t < n_threads; ++t)
        th.emplace_back([&, t] {
            const uint64_t r0 = n * (uint64_t)t / n_threads, r1 = n * (uint64_t)(t + 1) / n_threads;
            uint64_t* c = part[t].data();
            for (uint64_t r = r0; r < r1; ++r) {
                const orc_record& R = rec[r];
                if (R.instance >= n_inst) { bad = 1; return; }
                const uint64_t k = (uint64_t)__builtin_popcount(R.active & R.pred);
                const uint32_t gm = R.insn >> 24;
                for (int g = 0; g < 8; ++g)
                    if ((gm >> g) & 1) c[8 * (size_t)R.instance + g] += k;
            }
        });
    for (auto& x : th) x.join();
    std::fill(counts, counts + (size_t)n_inst * 8, 0);
    for (int t = 0; t < n_threads; ++t)
        for (size_t i = 0; i < (size_t)n_inst * 8; ++i) counts[i] += part[t][i];
    return bad ? 1 : 0;
}
