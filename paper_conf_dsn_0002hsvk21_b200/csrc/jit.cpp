// jit.cpp — the JIT-specialised emulator: per-program CUDA generated from the
// mini-SASS code and compiled by NVRTC for sm_100a (fi_jit_build), and K4 on it
// (fi_inject_jit).
//
// Why: the interpreter (emu.cuh) keeps the synthetic register file in shared
// memory and decodes every emulated instruction, ~26 SASS per emulated step on
// C2.  Here every static instruction becomes straight-line device code with the
// synthetic registers in real registers (R0..R{n_regs-1} are C++ locals with
// constant indices), so an FFMA is one predicated FFMA.  Semantics are those of
// DESIGN.md §3 and identical to emu.cuh's EMU_INJ mode step for step:
//   * min-pc scheduling with the same group-mode rule (a group of lanes sharing
//     pc runs alone until it branches divergently, exits or reaches parked lanes);
//   * a "block" (from any pc to the next BRA/EXIT or the end of the kernel code)
//     runs without per-step bookkeeping when it cannot reach parked lanes, the
//     watchdog or the injection site; otherwise instructions run one step at a
//     time through the same generated bodies (`S_i` labels);
//   * the site's corruption, store logging after the site, memory faults
//     (first faulting instruction in program order, C-9), watchdog (C-10), and
//     the restart from the golden checkpoint at or before the site.
// All generated control flow is warp-uniform (switch on the warp's pc, ballots);
// per-lane effects are predicated, so SHFL sees every lane's register.
#include <dlfcn.h>

#include <algorithm>
#include <chrono>
#include <cstdarg>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <atomic>
#include <bitset>
#include <cctype>
#include <mutex>
#include <thread>
#include <string>
#include <vector>

#include <cuda.h>
#include <cuda_runtime.h>

#include "../../include/fi.h"
#include "common.cuh"
#include "jit_k8.h"

namespace {

const char* const kPrelude =
#include "jit_prelude.inc"
    ;

// ---------------------------------------------------------------- generator
struct Src {
    std::string s;
    void operator()(const char* fmt, ...) __attribute__((format(printf, 2, 3))) {
        char buf[4096];
        va_list ap, ap2;
        va_start(ap, fmt);
        va_copy(ap2, ap);
        int n = std::vsnprintf(buf, sizeof buf, fmt, ap);
        va_end(ap);
        if (n > 0 && (size_t)n < sizeof buf) s.append(buf, (size_t)n);
        else if (n > 0) {                              // long lines (register kill lists)
            std::string big((size_t)n + 1, '\0');
            std::vsnprintf(&big[0], big.size(), fmt, ap2);
            s.append(big.data(), (size_t)n);
        }
        va_end(ap2);
    }
};

constexpr int kJbcSlots = 4;                        // JBC_SLOTS of jit_prelude.cuh
constexpr uint32_t kJitSliceLen = 0x100;            // internal modes bit: golden pass 1 = control slice
// loop prefetch distance in iterations (C2, K4 / golden pass 2: 1 -> 6.37 / 14.8 ms,
// 2 -> 6.62 / 15.1, 3 -> 6.62 / 15.1, none -> 6.86 / 20.1; profiles/r02/k4_prefetch_distance.log)
constexpr uint32_t kPrefetchIters = 1;
constexpr uint32_t kTmplRecs = 128;
constexpr uint32_t kJctxBytes = 3712;                 // JCTX_BYTES of jit_prelude.cuh                   // golden trace pass: record template per warp (records)

struct Gen {
    uint32_t NR;                                      // register rows (fi_program.n_regs)
    std::string R(uint32_t j) const { return j < NR ? "R" + std::to_string(j) : std::string("0u"); }
    std::string R64(uint32_t j) const { return "jpair(" + R(j) + ", " + R(j + 1) + ")"; }
    bool W(uint32_t j) const { return j < NR; }
    static std::string guard(uint32_t g) {
        if (g == 7) return "true";
        const uint32_t gs = g & 7, neg = (g >> 3) & 1;
        if (gs == 7) return neg ? "false" : "true";
        char b[96];
        std::snprintf(b, sizeof b, neg ? "(!Q%u)" : "Q%u", gs);
        return b;
    }
    std::string bv(const fi_insn& I) const {
        if (I.mod & 0x80) {
            char b[32];
            std::snprintf(b, sizeof b, "0x%08Xu", I.imm);
            return b;
        }
        return R(I.b);
    }
    static std::string hex(uint32_t v) {
        char b[32];
        std::snprintf(b, sizeof b, "0x%08Xu", v);
        return b;
    }
    // writes of n consecutive registers from d0 under `ex` (values v0..)
    void wr(Src& o, uint32_t d0, const char* const* vals, uint32_t n) const {
        if (d0 == fi::kRZ) return;
        for (uint32_t q = 0; q < n; ++q)
            if (W(d0 + q)) o("if (ex) R%u = %s; ", d0 + q, vals[q]);
    }

    // a plain instruction (emu.cuh exec_plain): `ex` is declared
    void plain(Src& o, const fi_insn& I) const {
        using namespace fi;
        const uint32_t op = I.op, mod = I.mod;
        const std::string a = R(I.a), c = R(I.c), b = bv(I);
        switch (op) {
            case FFMA: {
                // sm_100 FFMA returns the canonical 0x7FFFFFFF for every NaN (C-13 as is;
                // emu.cuh's batched FFMA path relies on the same, pinned by parity tests)
                o("{ const float x = ju2f(%s ^ %s), y = ju2f(%s ^ %s), z = ju2f(%s ^ %s); "
                  "const u32 v = __float_as_uint(__fmaf_rn(x, y, z)); ",
                  a.c_str(), hex((mod & 1u) << 31).c_str(), b.c_str(), hex((mod & 2u) << 30).c_str(), c.c_str(),
                  hex((mod & 4u) << 29).c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case MOV: { o("{ const u32 v = %s; ", b.c_str()); const char* v[] = {"v"}; wr(o, I.d0, v, 1); o("}\n"); return; }
            case S2R: {
                const char* e = "0u";
                switch (I.imm) {
                    case 0: e = "wic * 32u + lane"; break;
                    case 1: e = "cta"; break;
                    case 2: e = "JIN_(block)"; break;
                    case 3: e = "JIN_(grid)"; break;
                    case 4: e = "lane"; break;
                    case 5: e = "wic"; break;
                }
                const char* v[] = {e};
                o("{ ");
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case IADD3: {
                const uint32_t pb = I.d1 & 7;
                o("{ const u32 a_ = %s, c_ = %s, b_ = %s; const u32 x = %s, y = %s; const u64 s_ = (u64)x + y + c_; "
                  "const u32 v = (u32)s_; ",
                  a.c_str(), c.c_str(), b.c_str(), (mod & 1) ? "0u - a_" : "a_", (mod & 2) ? "0u - b_" : "b_");
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                if (pb != 7) o("if (ex) Q%u = (s_ >> 32) != 0ull; ", pb);
                o("}\n");
                return;
            }
            case IMAD: {
                o("{ const u32 v = %s * %s + %s; ", a.c_str(), b.c_str(), c.c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case IMAD_WIDE: {
                o("{ const u32 a_ = %s, b_ = %s; const u64 p_ = %s; const u64 r_ = p_ + %s; "
                  "const u32 v0 = (u32)r_, v1 = (u32)(r_ >> 32); ",
                  a.c_str(), b.c_str(),
                  (mod & 1) ? "(u64)a_ * (u64)b_" : "(u64)((i64)(i32)a_ * (i64)(i32)b_)", R64(I.c).c_str());
                const char* v[] = {"v0", "v1"};
                wr(o, I.d0, v, 2);
                o("}\n");
                return;
            }
            case SHF: {
                o("{ const u32 v = jshf(%s, %s, %uu); ", a.c_str(), b.c_str(), mod & 3u);
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case LOP3: {
                o("{ const u32 v = jlop3<%uu>(%s, %s, %s); ", I.ext & 0xFFu, a.c_str(), b.c_str(), c.c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case SEL: {
                const uint32_t pb = I.c & 0xF, p = pb & 7;
                std::string cond = p == 7 ? "true" : ("Q" + std::to_string(p));
                o("{ const bool s_ = %s%s; const u32 v = s_ ? %s : %s; ", (pb >> 3) & 1u ? "!" : "", cond.c_str(),
                  a.c_str(), b.c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case ISETP: case FSETP: case DSETP: {
                const uint32_t pb = I.d0 & 7, cc = mod & 7;
                if (op == ISETP)
                    o("{ const bool v = %s(%s, %s, %uu); ", (mod & 8) ? "jcmp_u" : "jcmp_s",
                      (mod & 8) ? a.c_str() : ("(i32)" + a).c_str(), (mod & 8) ? b.c_str() : ("(i32)" + b).c_str(), cc);
                else if (op == FSETP)
                    o("{ const bool v = jcmp_f((double)ju2f(%s), (double)ju2f(%s), %uu); ", a.c_str(), R(I.b).c_str(), cc);
                else
                    o("{ const bool v = jcmp_f(ju2d(%s), ju2d(%s), %uu); ", R64(I.a).c_str(), R64(I.b).c_str(), cc);
                if (pb != 7) o("if (ex) Q%u = v; ", pb);
                o("}\n");
                return;
            }
            case FADD: case FMUL: {
                o("{ const float x = ju2f(%s ^ %s), y = ju2f(%s ^ %s); const u32 v = jfbits(%s(x, y)); ", a.c_str(),
                  hex((mod & 1u) << 31).c_str(), b.c_str(), hex((mod & 2u) << 30).c_str(),
                  op == FADD ? "__fadd_rn" : "__fmul_rn");
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case FMNMX: {
                o("{ const u32 v = jfmnmx(%s, %s, %s); ", a.c_str(), b.c_str(), (mod & 1) ? "true" : "false");
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case DADD: case DMUL: case DFMA: {
                o("{ const double x = ju2d(%s ^ %s), y = ju2d(%s ^ %s), z = ju2d(%s ^ %s); ", R64(I.a).c_str(),
                  (mod & 1) ? "0x8000000000000000ull" : "0ull", R64(I.b).c_str(),
                  (mod & 2) ? "0x8000000000000000ull" : "0ull", R64(I.c).c_str(),
                  (mod & 4) ? "0x8000000000000000ull" : "0ull");
                o("const u64 r_ = jdbits(%s); const u32 v0 = (u32)r_, v1 = (u32)(r_ >> 32); ",
                  op == DADD ? "__dadd_rn(x, y)" : op == DMUL ? "__dmul_rn(x, y)" : "__fma_rn(x, y, z)");
                (void)0;
                const char* v[] = {"v0", "v1"};
                wr(o, I.d0, v, 2);
                o("}\n");
                return;
            }
            case LDC: {
                const uint32_t w0 = I.imm >> 2;
                o("{ const u32 v0 = %uu < cbank_len ? __ldg(&cb[%uu]) : 0u; ", w0, w0);
                if (mod & 1) {
                    o("const u32 v1 = %uu < cbank_len ? __ldg(&cb[%uu]) : 0u; ", w0 + 1, w0 + 1);
                    const char* v[] = {"v0", "v1"};
                    wr(o, I.d0, v, 2);
                } else {
                    const char* v[] = {"v0"};
                    wr(o, I.d0, v, 1);
                }
                o("}\n");
                return;
            }
            case I2F: {
                o("{ const u32 v = jfbits(%s); ", (mod & 1) ? ("__uint2float_rn(" + a + ")").c_str()
                                                            : ("__int2float_rn((int)" + a + ")").c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case F2I: { o("{ const u32 v = jf2i(%s); ", a.c_str()); const char* v[] = {"v"}; wr(o, I.d0, v, 1); o("}\n"); return; }
            case F2F_F64_F32: {
                o("{ const u64 r_ = jdbits((double)ju2f(%s)); const u32 v0 = (u32)r_, v1 = (u32)(r_ >> 32); ", a.c_str());
                const char* v[] = {"v0", "v1"};
                wr(o, I.d0, v, 2);
                o("}\n");
                return;
            }
            case F2F_F32_F64: {
                o("{ const u32 v = jfbits(__double2float_rn(ju2d(%s))); ", R64(I.a).c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case SHFL: {
                o("{ const u32 src_ = jshfl_src(lane, %s, %uu); const u32 v = __shfl_sync(JFULL, %s, src_); ", b.c_str(),
                  mod & 3u, a.c_str());
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            case MUFU_RCP64: {
                o("{ const u64 r_ = jdbits(__drcp_rn(ju2d(%s))); const u32 v0 = (u32)r_, v1 = (u32)(r_ >> 32); ",
                  R64(I.a).c_str());
                const char* v[] = {"v0", "v1"};
                wr(o, I.d0, v, 2);
                o("}\n");
                return;
            }
            case IMNMX: {
                if (mod & 8)
                    o("{ const u32 a_ = %s, b_ = %s; const u32 v = %s; ", a.c_str(), b.c_str(),
                      (mod & 1) ? "max(a_, b_)" : "min(a_, b_)");
                else
                    o("{ const i32 a_ = (i32)%s, b_ = (i32)%s; const u32 v = (u32)%s; ", a.c_str(), b.c_str(),
                      (mod & 1) ? "max(a_, b_)" : "min(a_, b_)");
                const char* v[] = {"v"};
                wr(o, I.d0, v, 1);
                o("}\n");
                return;
            }
            default: o("/* nop */\n"); return;
        }
    }

    // LDG / STG.  `stepx` = this instruction's step.
    uint32_t mode = 0;                               // JM_INJ / JM_LEN / JM_TRACE of jit_prelude.cuh
    std::vector<uint8_t> sl;                         // JM_LEN as the control slice: in-slice flag per pc (else empty)
    bool skip(const fi_insn& I, uint32_t pc) const { return !sl.empty() && !sl[pc] && I.op != fi::BRA && I.op != fi::EXIT; }
    // buffer-cache entry (JBufCache slot) of each address register of the kernel being generated
    std::vector<int> slot_of = std::vector<int>(256, 0);
    int slot(const fi_insn& I) const { return slot_of[I.a & 0xFF]; }
    // trace record of the instruction at pc (App. A.3): written only in JM_TRACE
    // Block code writes the records of a whole block when it leaves it (flush_recs);
    // here only a guarded instruction's predicate mask is kept for that.
    void rec(Src& o, const fi_insn& I, uint32_t pc, const char* stepx, const char* pv) const {
        (void)stepx;
        if (mode != 2 || I.guard == 7) return;
        o("gb_%u = __ballot_sync(JFULL, %s); ", pc, pv);
    }
    // the trace records of block steps [pcm, E] (App. A.3), lanes striding over them:
    // {instance, trace-insn word, active mask, guard-predicate mask}; call before the
    // step counter moves past the block
    void flush_recs(Src& o, const fi_insn* code, uint32_t L, uint32_t E, uint32_t tmpl_L = ~0u) const {
        if (mode != 2) return;
        if (tmpl_L != ~0u) {
            // the full-warp copy of the templated self-loop (JFW_ = 1 there), entered at
            // its leader, every guard true for all lanes: the records are the warp's
            // template with only the position changing — one bulk (TMA) store of the
            // template from shared memory, issued by lane 0
            o("   if (JFW_ && pcm == %uu", tmpl_L);
            std::string all;
            for (uint32_t q = tmpl_L; q <= E; ++q)
                if (code[q].guard != 7) all += (all.empty() ? "" : " & ") + std::string("gb_") + std::to_string(q);
            if (!all.empty()) o(" && (%s) == JFULL", all.c_str());
            o(") { if (jelect()) jbulk_st_p(&rec_out[step], jtm_, %uu, JPOL_);\n"
              "     if (JPCC_) { const u32 o_ = (JPRB_ + step) & 1023u; if (o_ + %uu < 1024u) { "
              "JPADD_; } else { JPFLUSH_; jprof_tmpl_cross(&jx->prof, lane, "
              "1024u - o_); } } } else\n", (E + 1 - tmpl_L) * 16, E + 1 - tmpl_L);
        }
        o("   { const u32 n_ = %uu - pcm; for (u32 jb_ = 0u; jb_ < n_; jb_ += 32u) { const u32 j_ = jb_ + lane; "
          "const bool v_ = j_ < n_; const u32 p_ = pcm + j_; u32 pr_ = JFULL; ",
          E + 1);
        for (uint32_t q = L; q <= E; ++q)
            if (code[q].guard != 7) o("if (p_ == %uu) pr_ = gb_%u; ", q, q);
        // streaming stores (evict-first): the 16-B records are written once and read by
        // other kernels, so they must not push the image lines the loads reuse out of L2
        o("const u32 w_ = v_ ? __ldg(&ins[p_]) : 0u; if (v_) __stcs(&rec_out[step + j_], make_uint4(k, w_, amask, pr_));\n"
          "     if (jx->prof.cc) { JPFLUSH_; jprof_round(&jx->prof, lane, jx->prof.rb + step + jb_, v_, __popc(amask & pr_), w_ >> 24); } } }\n");
    }
    void mem(Src& o, const fi_insn& I, uint32_t pc, const char* stepx) const {
        using namespace fi;
        const uint32_t lw = (I.mod & 3) > 2 ? 2 : (I.mod & 3), nw = 1u << lw;
        if (skip(I, pc)) {                             // sliced length pass: count the stored words only
            if (I.op == STG)
                o("{ const bool pv = %s; const u32 exm_ = amask & __ballot_sync(JFULL, pv); nst += __popc(exm_) * %uu; }\n",
                  guard(I.guard).c_str(), nw);
            return;
        }
        o("{ const bool pv = %s; const bool ex = inA && pv; ", guard(I.guard).c_str());
        rec(o, I, pc, stepx, "pv");
        o("const u64 va = %s + (u64)(i64)(i32)%s; ", R64(I.a).c_str(), hex(I.imm).c_str());
        if (I.op == LDG) {
            o("uint4 v_; const u32 c_ = jldg<%uu, %d>(A, jimg, bc, va, k, ex, v_%s); ", lw, slot(I),
              mode == 3 ? ", &PG" : "");
            o("if (__ballot_sync(JFULL, c_ != 0u)) { fault = __ballot_sync(JFULL, c_ == 1u) ? 1u : 2u; fault_pc = %uu; "
              "step = %s; goto finish; } ", pc, stepx);
            if (mode == 3) o("if (ex) jpage_c<%uu, %d>(A, bc, PG, va, v_); ", nw, slot(I));
            const char* v[] = {"v_.x", "v_.y", "v_.z", "v_.w"};
            wr(o, I.d0, v, nw);
            o("}\n");
        } else {
            o("const u32 exm_ = amask & __ballot_sync(JFULL, pv); bool z_ = false; "
              "const u32 c_ = ex ? jcheck<%d>(A, bc, va, %uu, k, &z_%s) : 0u; ", slot(I), 4u << lw,
              mode == 3 ? ", &PG" : "");
            o("if (__ballot_sync(JFULL, c_ != 0u)) { fault = __ballot_sync(JFULL, c_ == 1u) ? 1u : 2u; fault_pc = %uu; "
              "step = %s; goto finish; } ", pc, stepx);
            if (mode == 1) {                           // golden pass 1: into the image
                o("if (ex) { u8* d_ = img_w + (va - JVA_BASE); ");
                if (lw == 0) o("*reinterpret_cast<u32*>(d_) = %s; ", R(I.b).c_str());
                else if (lw == 1) o("*reinterpret_cast<uint2*>(d_) = make_uint2(%s, %s); ", R(I.b).c_str(), R(I.b + 1).c_str());
                else
                    o("*reinterpret_cast<uint4*>(d_) = make_uint4(%s, %s, %s, %s); ", R(I.b).c_str(), R(I.b + 1).c_str(),
                      R(I.b + 2).c_str(), R(I.b + 3).c_str());
                o("} nst += __popc(exm_) * %uu; }\n", nw);
                return;
            }
            if (mode == 2) {                           // golden pass 2: the stores into the image as well
                o("if (ex && img_w) { u8* d_ = img_w + (va - JVA_BASE); ");
                if (lw == 0) o("*reinterpret_cast<u32*>(d_) = %s; ", R(I.b).c_str());
                else if (lw == 1) o("*reinterpret_cast<uint2*>(d_) = make_uint2(%s, %s); ", R(I.b).c_str(), R(I.b + 1).c_str());
                else
                    o("*reinterpret_cast<uint4*>(d_) = make_uint4(%s, %s, %s, %s); ", R(I.b).c_str(), R(I.b + 1).c_str(),
                      R(I.b + 2).c_str(), R(I.b + 3).c_str());
                o("} ");
            }
            o("const u32 sst_ = %s; if (%s) { if (ex) { const u32 idx_ = __popc(exm_ & lt_mask) * %uu; ",
              stepx, (mode == 2 || mode == 3) ? "true" : "sst_ > hstep", nw);
            for (uint32_t q = 0; q < nw; ++q) {
                if (mode == 2)
                    o("{ jfi_store e_; e_.va = va + %uu; e_.value = %s; e_.step = sst_; st_out[nst + idx_ + %uu] = e_; } ",
                      4 * q, R(I.b + q).c_str(), q);
                else
                    o("if (nst + idx_ + %uu < st_cap) { jfi_store e_; e_.va = va + %uu; e_.value = %s; e_.step = sst_; "
                      "st_out[nst + idx_ + %uu] = e_; } ",
                      q, 4 * q, R(I.b + q).c_str(), q);
            }
            o("} nst += __popc(exm_) * %uu; } }\n", nw);
        }
    }

    // m consecutive independent LDGs (block mode): all address checks first, one
    // fault ballot (the first faulting load in program order wins, C-9), then all
    // loads in flight together, then the register writes in program order.
    void ldg_batch(Src& o, const fi_insn* code, uint32_t i0, uint32_t m,
                   const std::vector<std::string>& stride = {}) const {
        o(" { // LDG batch %u..%u\n", i0, i0 + m - 1);
        for (uint32_t j = 0; j < m; ++j) {
            const fi_insn& I = code[i0 + j];
            o("  const bool pv%u = %s; const bool ex%u = inA && pv%u; const u64 va%u = %s + (u64)(i64)(i32)%s; "
              "bool z%u = false; u32 c%u = 0u;\n",
              j, guard(I.guard).c_str(), j, j, j, R64(I.a).c_str(), hex(I.imm).c_str(), j, j);
        }
        // fast path: every executing lane hits its buffer cache (no table lookups, no
        // cache updates); otherwise the full checks in program order
        // (bitwise, not short-circuit: every test is evaluated, no branches)
        // A load off the same address register, guard and width as an earlier one of
        // the batch, at a positive offset delta that is a multiple of the width, only
        // adds `lo32(va_first) - lo + delta < size16` to the first's check (same buffer,
        // same high word, same alignment, same writer-rule flag)
        o("  if (__ballot_sync(JFULL, !(true");
        for (uint32_t j = 0; j < m; ++j) {
            const fi_insn& I = code[i0 + j];
            const uint32_t lw = (I.mod & 3) > 2 ? 2 : (I.mod & 3);
            uint32_t lead = j;
            for (uint32_t q = 0; q < j && lead == j; ++q) {
                const fi_insn& Q = code[i0 + q];
                const uint32_t qw = (Q.mod & 3) > 2 ? 2 : (Q.mod & 3);
                const int64_t d = (int64_t)(int32_t)I.imm - (int64_t)(int32_t)Q.imm;
                if (Q.a == I.a && Q.guard == I.guard && qw == lw && slot(Q) == slot(I) && d > 0 && d < 4096 &&
                    d % (4 << lw) == 0)
                    lead = q;
            }
            if (lead != j) {
                o(" & (!ex%u | jhit_more<%d>(bc, va%u, %uu, &z%u))", j, slot(I), lead,
                  (uint32_t)((int64_t)(int32_t)I.imm - (int64_t)(int32_t)code[i0 + lead].imm), j);
            } else {
                o(" & (!ex%u | jhit<%d>(bc, va%u, %uu, &z%u))", j, slot(I), j, 4u << lw, j);
            }
        }
        o("))) {\n");
        for (uint32_t j = 0; j < m; ++j) {
            const fi_insn& I = code[i0 + j];
            const uint32_t lw = (I.mod & 3) > 2 ? 2 : (I.mod & 3);
            o("   c%u = ex%u ? jcheck<%d>(A, bc, va%u, %uu, k, &z%u%s) : 0u;\n", j, j, slot(I), j, 4u << lw, j,
              mode == 3 ? ", &PG" : "");
        }
        // (a fault needs a lane that missed its cache: the fault ballots are on the slow path only)
        o("   if (__ballot_sync(JFULL, 0u");
        for (uint32_t j = 0; j < m; ++j) o(" | c%u", j);
        o(")) {\n");
        for (uint32_t j = 0; j < m; ++j)
            o("    if (__ballot_sync(JFULL, c%u != 0u)) { fault = __ballot_sync(JFULL, c%u == 1u) ? 1u : 2u; "
              "fault_pc = %uu; step = step + (%uu - pcm); goto finish; }\n",
              j, j, i0 + j, i0 + j);
        o("   }\n  }\n");
        for (uint32_t j = 0; j < m; ++j) {
            char sx[64], pvn[16];
            std::snprintf(sx, sizeof sx, "step + (%uu - pcm)", i0 + j);
            std::snprintf(pvn, sizeof pvn, "pv%u", j);
            if (mode == 2) { o("  "); rec(o, code[i0 + j], i0 + j, sx, pvn); o("\n"); }
        }
        // loads straight into the destination registers (predicated, program order)
        for (uint32_t j = 0; j < m; ++j) {
            const fi_insn& I = code[i0 + j];
            const uint32_t lw = (I.mod & 3) > 2 ? 2 : (I.mod & 3), nw = 1u << lw;
            // (a word the writer rule zeroes is read from a zero line: one unconditional load)
            o("  if (ex%u) { uint4 v_ = make_uint4(0u, 0u, 0u, 0u); "
              "const u8* p_ = z%u ? reinterpret_cast<const u8*>(jzero16) : jimg + (va%u - JVA_BASE); ",
              j, j, j);
            if (lw == 0) o("v_.x = jld32(p_); ");
            else if (lw == 1) o("const uint2 t_ = jld64(p_); v_.x = t_.x; v_.y = t_.y; ");
            else o("v_ = jld128(p_); ");
            if (mode == 3) o("jpage_c<%uu, %d>(A, bc, PG, va%u, v_); ", nw, slot(I), j);
            if (I.d0 != fi::kRZ)
                for (uint32_t q = 0; q < nw; ++q)
                    if (W(I.d0 + q)) o("R%u = v_.%c; ", I.d0 + q, "xyzw"[q]);
            o("}\n");
        }
        // the lines of a loop-carried pointer (address + loop-invariant stride)
        // kPrefetchIters iterations ahead into L1 while this one computes; a hint only
        // (no architectural effect), issued only for addresses inside a cached buffer
        // (one per address pair: the batch's other loads off the same pointer are
        // usually in the same lines)
        for (uint32_t j = 0; j < m && j < stride.size(); ++j) {
            bool first = !stride[j].empty();
            for (uint32_t q = 0; q < j && first; ++q) first = code[i0 + q].a != code[i0 + j].a;
            if (first) {
                o("  if (ex%u) jprefetch<%d>(jimg, bc, va%u + %uull * (%s));\n", j, slot(code[i0 + j]), j, kPrefetchIters,
                  stride[j].c_str());
            }
        }
        o(" }\n");
    }
};

// consecutive LDGs from i0 that may be batched: none crosses a leader (a jump
// target) and none's address pair is written by an earlier LDG of the batch
static uint32_t ldg_batch_len(const fi_insn* code, uint32_t n, uint32_t i0, const std::vector<uint8_t>& leader) {
    using namespace fi;
    uint32_t m = 0;
    for (uint32_t j = i0; j < n && code[j].op == LDG && m < 8 && (j == i0 || !leader[j]); ++j) {
        bool hazard = false;
        for (uint32_t q = i0; q < j && !hazard; ++q) {
            const Dests d = dests_of(code[q].op, code[q].d0, code[q].d1, code[q].mod);
            for (uint32_t x = 0; x < 2; ++x) {
                const uint32_t a = code[j].a + x;
                if (code[j].a != kRZ && a >= d.gp_base && a < d.gp_base + d.n_gp) hazard = true;
            }
        }
        if (hazard) break;
        ++m;
    }
    return m;
}

// Per load of the LDG batch at i0 (length m) inside the self-looping block
// [L, E] (code[E] = BRA to L): the change of its address over one iteration as
// a C++ expression of the current registers, or "" if not a plain pointer walk.
// The address pair (a, a+1) must be written in the block by exactly one
// unguarded IMAD.WIDE d = a * b + (a, a+1) whose a/b operands the block never
// writes (so the stride is loop-invariant and readable at the batch).
static std::vector<std::string> batch_strides(const Gen& G, const fi_insn* code, uint32_t L, uint32_t E, uint32_t i0,
                                              uint32_t m) {
    using namespace fi;
    std::vector<std::string> st(m);
    auto writes = [&](uint32_t q, uint32_t r) {
        const Dests d = dests_of(code[q].op, code[q].d0, code[q].d1, code[q].mod);
        return r >= d.gp_base && r < d.gp_base + d.n_gp;
    };
    for (uint32_t j = 0; j < m; ++j) {
        const uint32_t a = code[i0 + j].a;
        if (a == kRZ || a + 1 >= G.NR) continue;
        int w = -1, nw = 0;
        for (uint32_t q = L; q <= E; ++q) {
            if (q >= i0 && q < i0 + m) continue;
            if (writes(q, a) || writes(q, a + 1)) { w = (int)q; ++nw; }
        }
        if (nw != 1) continue;
        const fi_insn& W = code[w];
        if (W.op != IMAD_WIDE || W.guard != 7 || W.d0 != a || W.c != a) continue;
        bool inv = true;
        for (uint32_t q = L; q <= E && inv; ++q) {
            if (W.a != kRZ && writes(q, W.a)) inv = false;
            if (!(W.mod & 0x80) && W.b != kRZ && writes(q, W.b)) inv = false;
        }
        if (!inv) continue;
        const std::string x = G.R(W.a), y = G.bv(W);
        st[j] = (W.mod & 1) ? "(u64)" + x + " * (u64)" + y : "(u64)((i64)(i32)" + x + " * (i64)(i32)" + y + ")";
    }
    return st;
}

// The control slice of one static kernel (golden pass 1 as a length pass): the
// instructions whose results can reach a BRA / EXIT / STG guard predicate — the
// only things that decide the per-warp step count (min-pc scheduling, A.2) and
// the stored-word count.  Flow-insensitive over registers: an instruction is in
// the slice if it writes a GP register or predicate some slice instruction (or a
// root guard) reads; reads are over-approximated like the liveness below (operand
// fields a, a+1, c, c+1, b..b+3 unless b is an immediate; the guard; SEL's
// predicate).  Everything else (FFMAs feeding only stores, loads feeding only
// them) is skipped by the sliced pass: it cannot change the pc sequence or an
// active / guard mask.
std::vector<uint8_t> control_slice(const fi_insn* code, uint32_t n) {
    using namespace fi;
    std::vector<uint8_t> in(n, 0);
    std::bitset<256> nr;
    uint32_t np = 0;                                  // needed predicates (bits 0..6)
    auto need_srcs = [&](const fi_insn& I) {
        if ((I.guard & 7) != 7) np |= 1u << (I.guard & 7);
        if (I.op == SEL && (I.c & 7) != 7) np |= 1u << (I.c & 7);
        if (I.op == NOP || I.op == EXIT || I.op == BRA || I.op == S2R || I.op == LDC) return;
        for (uint32_t r : {(uint32_t)I.a, I.a + 1u, (uint32_t)I.c, I.c + 1u}) if (r < kRZ) nr.set(r);
        if (!(I.mod & 0x80)) for (uint32_t q = 0; q < 4; ++q) if (I.b + q < kRZ) nr.set(I.b + q);
    };
    for (uint32_t i = 0; i < n; ++i)
        if ((code[i].op == BRA || code[i].op == EXIT || code[i].op == STG) && (code[i].guard & 7) != 7)
            np |= 1u << (code[i].guard & 7);
    for (bool ch = true; ch;) {
        ch = false;
        for (uint32_t i = 0; i < n; ++i) {
            if (in[i]) continue;
            const fi_insn& I = code[i];
            if (I.op == BRA || I.op == EXIT || I.op == STG || I.op == NOP) continue;
            const Dests d = dests_of(I.op, I.d0, I.d1, I.mod);
            bool hit = d.has_pr && ((np >> d.pr) & 1u);
            for (uint32_t q = 0; q < d.n_gp && !hit; ++q) hit = d.gp_base + q < 256 && nr[d.gp_base + q];
            if (!hit) continue;
            in[i] = 1;
            need_srcs(I);
            ch = true;
        }
    }
    return in;
}

// Generate the device function of one static kernel (EMU_INJ mode).
// Generate the device function of one static kernel in mode `mode` (JM_INJ,
// JM_LEN, JM_TRACE); `blen`/leader tables are emitted once (with_tables).
// kern_* arguments kept in the warp's JCtx (shared memory) instead of registers
const char* const kCtxNames[] = {"hstep", "hpc", "hlane", "hkind", "hreg", "hbfm", "hmask", "k", "cta", "wic",
                                 "watchdog", "ck", "ck_interval", "st_out", "st_cap", "Rs", "dec", "ins",
                                 "img_w", "rec_out", "pgp"};
// warp state that block code rarely touches (store count, fault, the site's values):
// per lane in the context (JCtx arrays), not in registers
const char* const kCtxLaneNames[] = {"nst", "fault", "fault_pc", "before", "after", "msk", "fired", "bad"};

void gen_kernel(Src& o, const Gen& G0, uint32_t kid, const fi_insn* code, uint32_t n, uint32_t mode, bool with_tables,
                bool slice_len = false) {
    using namespace fi;
    Gen G = G0;
    G.mode = mode;
    if (mode == 1 && slice_len) {
        G.sl = control_slice(code, n);
        o("__device__ const u8 kslice_%u[%u] = {", kid, n);
        for (uint32_t i = 0; i < n; ++i) o("%u%s", G.sl[i], i + 1 < n ? "," : "");
        o("};\n");
    }
    // one cache entry per address register, in order of first use (wrapping beyond JBC_SLOTS)
    int nslots = 0;                                   // entries this kernel uses (the others stay empty)
    {
        std::vector<int> seen(256, -1);
        int next = 0;
        for (uint32_t i = 0; i < n; ++i) {
            if (code[i].op != LDG && code[i].op != STG) continue;
            const uint32_t a = code[i].a & 0xFF;
            if (seen[a] < 0) seen[a] = next++ % kJbcSlots;
            G.slot_of[a] = seen[a];
        }
        nslots = std::min(next, kJbcSlots);
    }
    const uint32_t NR = G.NR;
    static const char* const mname[] = {"inj", "len", "trace", "page"};
    // block length from each pc: to the next BRA/EXIT inclusive, or the code end
    std::vector<uint32_t> blen(n);
    for (int64_t i = (int64_t)n - 1; i >= 0; --i) {
        const uint32_t op = code[i].op;
        blen[i] = (op == BRA || op == EXIT || i + 1 == (int64_t)n) ? 1u : blen[i + 1] + 1u;
    }
    // leaders: pc 0, branch targets, and the pc after every BRA / EXIT.  Blocks
    // are entered only at leaders (few merge points keep the block code
    // straight-line for the compiler); any other pc runs in step mode
    // (jinterp_inj) until a leader is reached.
    std::vector<uint8_t> leader(n + 1, 0);
    leader[0] = 1;
    for (uint32_t i = 0; i < n; ++i) {
        if (code[i].op == BRA && code[i].imm < n) leader[code[i].imm] = 1;
        if ((code[i].op == BRA || code[i].op == EXIT) && i + 1 < n) leader[i + 1] = 1;
    }
    // ---- per-thread register liveness (every mode but the trace pass, whose checkpoints
    // copy the whole register file).  The dispatch loop reaches step mode, which spills
    // every register, from every block exit, and a lane-predicated write `if (ex) R = v`
    // keeps the old value of the lanes that do not execute: to the compiler every
    // synthetic register is live everywhere.  `kills(keep)` zeroes, on the entries and
    // exits of the block code, the registers no lane can read again there: the active
    // lanes go to the path's targets, the parked ones wait at pcs >= npc >= the block's
    // end (the `fits` rule), so keep = live_in(targets) | live_from[end].  The values
    // are unobservable (outcomes come from stores; the site's before/after from the
    // instruction that writes them); SHFL sources are never zeroed (SHFL reads parked
    // and exited lanes).  Reads are over-approximated (operand fields and every register
    // the instruction's own code mentions); only an unguarded `if (ex) R = v` kills.
    typedef std::bitset<256> RSet;
    std::vector<RSet> lin(n + 1), lfrom(n + 2);     // live-in per pc; lfrom[e] = union of lin[q], q >= e
    RSet shfl;
    const bool use_kill = mode != 2;
    if (use_kill) {
        std::vector<RSet> rd(n), kl(n);
        for (uint32_t i = 0; i < n; ++i) {
            const fi_insn& I = code[i];
            auto add = [&](uint32_t j) { if (j < NR && j < 256) rd[i].set(j); };
            if (I.op != NOP && I.op != EXIT && I.op != BRA && I.op != S2R && I.op != LDC) {
                add(I.a); add(I.a + 1u); add(I.c); add(I.c + 1u);
                if (!(I.mod & 0x80)) for (uint32_t q = 0; q < 4; ++q) add(I.b + q);
            }
            if (I.op == BRA || I.op == EXIT) continue;
            Src t;
            if (I.op == LDG || I.op == STG) G.mem(t, I, i, "step");
            else if (!G.skip(I, i)) { t("{ const bool ex = true; "); G.plain(t, I); t("}"); }
            const std::string& s = t.s;
            const bool uncond = G.guard(I.guard) == "true";
            for (size_t p = 0; p < s.size(); ++p) {
                if (s[p] != 'R' || (p > 0 && (std::isalnum((unsigned char)s[p - 1]) || s[p - 1] == '_'))) continue;
                size_t q = p + 1;
                if (q >= s.size() || !std::isdigit((unsigned char)s[q])) continue;
                uint32_t v = 0;
                while (q < s.size() && std::isdigit((unsigned char)s[q])) v = v * 10 + (uint32_t)(s[q++] - '0');
                if (q < s.size() && (std::isalnum((unsigned char)s[q]) || s[q] == '_')) continue;
                const bool w = s.compare(q, 3, " = ") == 0 && (q + 3 >= s.size() || s[q + 3] != '=');
                if (!w) add(v);
                else if (uncond && p >= 8 && s.compare(p - 8, 8, "if (ex) ") == 0 && v < 256) kl[i].set(v);
            }
            if (I.op == SHFL) shfl |= rd[i];
        }
        for (bool ch = true; ch;) {
            ch = false;
            for (int64_t i = (int64_t)n - 1; i >= 0; --i) {
                RSet out = lin[i + 1];
                if (code[i].op == BRA && code[i].imm < n) out |= lin[code[i].imm];
                const RSet in = rd[i] | (out & ~kl[i]);
                if (in != lin[i]) { lin[i] = in; ch = true; }
            }
        }
        for (int64_t e = (int64_t)n; e >= 0; --e) lfrom[e] = lin[e] | lfrom[e + 1];
    }
    auto kills = [&](const RSet& keep) -> std::string {
        std::string s;
        if (!use_kill) return s;
        for (uint32_t j = 0; j < NR && j < 256; ++j)
            if (!keep[j] && !shfl[j]) s += "R" + std::to_string(j) + " = 0u; ";
        return s;
    };
    auto entry_kills = [&](uint32_t L) { return kills(lin[L] | lfrom[std::min(n, L + blen[L])]); };
    // per pc: the block length if pc is a leader, else 0 (step mode's exit test)
    if (with_tables) {
        o("__device__ const unsigned short kblen_%u[%u] = {", kid, n);
        for (uint32_t i = 0; i < n; ++i)
            o("%u%s", leader[i] ? std::min<uint32_t>(blen[i], 0xFFFF) : 0u, i + 1 < n ? "," : "");
        o("};\n");
    }
    // (inlined into its one entry kernel: as a separate function ptxas re-loaded the global
    // memory descriptor into uniform registers before every image load, and spilled more;
    // K4 6.29 -> 6.18 ms, golden pass 2 14.6 -> 14.2 ms on C2, profiles/r02/s6/k4_inline_ab.log)
    o("__device__ __forceinline__ void kern_%u_%s(const JArgs& A_, const u32 hstep_p, const u32 hpc_p, const u32 hlane_p, "
      "const u32 hkind_p, const u32 hreg_p, const u32 hbfm_p, const u32 hmask_p, const u32 k_p, const u32 cta_p, "
      "const u32 wic_p, const u32 watchdog_p, u32* __restrict__ ck_p, const u32 ck_interval_p, "
      "jfi_store* __restrict__ st_out_p, const u32 st_cap_p, JOut& out_p, u32* __restrict__ Rs_p, "
      "const uint4* __restrict__ dec_p, const u32* __restrict__ ins_p, u8* __restrict__ img_w_p, "
      "uint4* __restrict__ rec_out_p, const JPage* __restrict__ pgp_p) {\n", kid, mname[mode]);
    // The arguments go to this warp's context in shared memory and are read where
    // they are used (mostly cold paths): held in registers they would compete with
    // the synthetic registers across the block code.
    o("extern __shared__ u32 jsmem[];\nJCtx* const jx = reinterpret_cast<JCtx*>(jsmem + %uu + (threadIdx.x >> 5) * "
      "(JCTX_BYTES / 4u));\n", 4u * (NR + 1) * 32u);
    o("if ((threadIdx.x & 31u) == 0u) { jx->hstep = hstep_p; jx->hpc = hpc_p; jx->hlane = hlane_p; jx->hkind = hkind_p; "
      "jx->hreg = hreg_p; jx->hbfm = hbfm_p; jx->hmask = hmask_p; jx->k = k_p; jx->cta = cta_p; jx->wic = wic_p; "
      "jx->watchdog = watchdog_p; jx->ck = ck_p; jx->ck_interval = ck_interval_p; jx->st_out = st_out_p; "
      "jx->st_cap = st_cap_p; jx->out = &out_p; jx->Rs = Rs_p; jx->dec = dec_p; jx->ins = ins_p; jx->img_w = img_w_p; "
      "jx->rec_out = rec_out_p; jx->pgp = pgp_p; }\n__syncwarp();\n");
    for (const char* nm : kCtxNames) o("#define %s (jx->%s)\n", nm, nm);
    for (const char* nm : kCtxLaneNames) o("#define %s (jx->%s_[threadIdx.x & 31u])\n", nm, nm);
    o("#define out (*jx->out)\n");
    o("(void)img_w; (void)rec_out; (void)ins;\n");
    if (mode == 3) o("const JPage PG = *pgp;               // the replica slot's pages (K8)\n");
    // the image base in a register; the other kernel arguments are read where they
    // are used (cold paths), so they do not hold registers across the block code
    o("const JArgs& A = A_; const u8* __restrict__ const jimg = A_.img;\n");
    o("const u32 lane = threadIdx.x & 31u, lt_mask = (1u << lane) - 1u;\n");
    // the instance's fields are read where they are used (S2R, LDC: cold block code):
    // cached in registers they would be live across every block of the dispatch loop
    o("#define JIN_(f) (__ldg(&A.inst[k].f))\n#define cbank_len JIN_(cbank_len)\n#define cb (A.cbank + JIN_(cbank_off))\n"
      "(void)lt_mask;\n");
    for (uint32_t j = 0; j < NR; ++j) o("u32 R%u;%s", j, (j % 16 == 15) ? "\n" : " ");
    o("\nconst u32 nl_ = JIN_(block) - wic * 32u; bool live = lane < (nl_ > 32u ? 32u : nl_);\n");
    o("u32 pc = 0u, step = 0u; bool Q0 = false, Q1 = false, Q2 = false, Q3 = false, Q4 = false, Q5 = false, "
      "Q6 = false;\n");
    o("if (%s) {\n  u32 c_ = hstep / ck_interval;\n"
      "  while (c_ > 0u && __ldg(&ck[(u64)c_ * %uu + %uu]) > hstep) --c_;   // the last checkpoint at or before the site\n"
      "  const u32* __restrict__ src = ck + (u64)c_ * %uu;\n",
      mode == 0 ? "ck" : "false", (NR + 4) * 32, (NR + 3) * 32, (NR + 4) * 32);
    for (uint32_t j = 0; j < NR; ++j) o("  R%u = __ldg(&src[%uu + lane]);\n", j, j * 32);
    o("  pc = __ldg(&src[%uu + lane]); const u32 pw_ = __ldg(&src[%uu + lane]); live = __ldg(&src[%uu + lane]) != 0u; "
      "step = __ldg(&src[%uu + lane]); out_p.start = step;\n  Q0 = pw_ & 1u; Q1 = (pw_ >> 1) & 1u; Q2 = (pw_ >> 2) & 1u; Q3 = (pw_ >> 3) & 1u; "
      "Q4 = (pw_ >> 4) & 1u; Q5 = (pw_ >> 5) & 1u; Q6 = (pw_ >> 6) & 1u;\n} else {\n",
      NR * 32, NR * 32 + 32, NR * 32 + 64, NR * 32 + 96);
    for (uint32_t j = 0; j < NR; ++j) o("R%u = 0u;%s", j, (j % 16 == 15) ? "\n" : " ");
    o("\n}\n");
    o("u32 livem = __ballot_sync(JFULL, live);\nbool conv = false; u32 upc = 0u, amask = 0u, npc = 0xFFFFFFFFu;\n"
      "jx->nst_[lane] = 0u; jx->fault_[lane] = 0u; jx->fault_pc_[lane] = 0u; jx->before_[lane] = 0u; "
      "jx->after_[lane] = 0u; jx->msk_[lane] = 0u; jx->fired_[lane] = 0u; jx->bad_[lane] = 0u;\n"
      "JBufCache bc; uint4 recbuf = make_uint4(0u, 0u, 0u, 0u); (void)recbuf;\n"
      "if (jx->bck == k%s) {                 // this warp's cache from its previous job of the same instance\n"
      "#pragma unroll\n for (int s_ = 0; s_ < %d; ++s_) { bc.lo[s_] = jx->bc_[s_ * 4][lane]; "
      "bc.sz[s_] = jx->bc_[s_ * 4 + 1][lane]; %s"
      "bc.z[s_] = (jx->bcz_[lane] >> s_) & 1u; } }\n"
      "// golden trace pass: the last step was a BRA / EXIT; next checkpoint and its threshold step\n"
      "u32 brk = 1u, ckn = 0u, ckx = %s; (void)brk; (void)ckn; (void)ckx;\nu32 lexm_ = 0u; (void)lexm_;\n"
      "// blocks run only within [step, lim): lim = the watchdog, or the injection step while it is pending,\n"
      "// or the next checkpoint step (golden trace pass)\n"
      "u32 lim = %s;\n", mode == 3 ? " && jx->bckp == (u32)(size_t)PG.ptab" : "", nslots,
      mode == 3 ? "bc.b[s_] = jx->bc_[s_ * 4 + 2][lane]; bc.pb[s_] = jx->bc_[s_ * 4 + 3][lane]; " : "",
      mode == 2 ? "ck ? 0u : 0xFFFFFFFFu" : "0xFFFFFFFFu",
      mode == 0 ? "(hstep >= step && hstep < watchdog) ? hstep : watchdog" : "watchdog");
    if (mode == 2)
        o("bool tmpl_ = false; (void)tmpl_;\nuint4* const jtm_ = reinterpret_cast<uint4*>(jsmem + %uu + (threadIdx.x >> 5) * "
          "%uu); (void)jtm_;   // the warp's record template (after the 4 JCtx)\n",
          4u * (NR + 1) * 32u + 4u * (kJctxBytes / 4u), kTmplRecs * 4u);
    o("for (;;) {\n if (!livem) break;\n u32 pcm, active;\n"
      " if (conv) { pcm = upc; active = amask; }\n"
      " else { pcm = __reduce_min_sync(JFULL, live ? pc : 0xFFFFFFFFu); active = __ballot_sync(JFULL, live && pc == pcm);\n"
      "   npc = active == livem ? 0xFFFFFFFFu : __reduce_min_sync(JFULL, (live && pc != pcm) ? pc : 0xFFFFFFFFu);\n"
      "   conv = true; upc = pcm; amask = active; }\n"
      " const bool inA = (amask >> lane) & 1u;\n");
    if (mode == 2) {
        // golden checkpoints (emu.cuh): the state before the first step at or past
        // each multiple of ck_interval that follows a BRA / EXIT — every arrival here
        // from block code is such a step, so blocks never stop at a multiple
        o(" if (brk && step >= ckx) {\n  for (; ckn <= step / ck_interval; ++ckn) {\n"
          "   u32* dst_ = ck + (u64)ckn * %uu;\n", (NR + 4) * 32);
        for (uint32_t j = 0; j < NR; ++j) o("   __stcs(&dst_[%uu + lane], R%u);%s", j * 32, j, (j % 8 == 7) ? "\n" : "");
        o("\n   dst_[%uu + lane] = live ? (inA ? upc : pc) : 0u;\n"
          "   dst_[%uu + lane] = (u32)Q0 | ((u32)Q1 << 1) | ((u32)Q2 << 2) | ((u32)Q3 << 3) | ((u32)Q4 << 4) | "
          "((u32)Q5 << 5) | ((u32)Q6 << 6);\n   dst_[%uu + lane] = live ? 1u : 0u;\n   dst_[%uu + lane] = step;\n  }\n"
          "  ckx = ckn * ck_interval;\n }\n",
          NR * 32, NR * 32 + 32, NR * 32 + 64, NR * 32 + 96);
    }
    o(" if (step >= watchdog) { fault = 3u; fault_pc = pcm; break; }\n"
      " if (pcm >= %uu) { fault = 4u; fault_pc = pcm; break; }\n",
      n);
    if (mode == 2)                                    // guard masks of this block's predicated steps (flush_recs)
        for (uint32_t q = 0; q < n; ++q)
            if (code[q].guard != 7) o("u32 gb_%u = 0u; (void)gb_%u;\n", q, q);
    // dispatch: a whole block when it fits, else one step
    o(" switch (pcm) {\n");
    for (uint32_t i = 0; i < n; ++i)
        if (leader[i])
            o("  case %u: if (%uu <= npc && step + %uu <= lim) { %sgoto B%u; } goto S_any;\n", i, i + blen[i], blen[i],
              entry_kills(i).c_str(), i);
    o("  default: goto S_any;\n }\n");
    // ---- block code (fallthrough from a leader to the block's BRA / EXIT)
    char stepx[64];
    auto run_start = [&](uint32_t E) {               // first pc of the straight-line run ending at E
        uint32_t q = E;
        while (q > 0 && code[q - 1].op != BRA && code[q - 1].op != EXIT) --q;
        return q;
    };
    auto flush_end = [&]() { G.flush_recs(o, code, run_start(n - 1), n - 1); };
    uint32_t batch_end = 0;                           // LDGs [.., batch_end) already emitted as a batch
    uint32_t tmpl_L = ~0u;                            // the self-loop whose records come from a template
    uint32_t loop_L = ~0u;                            // leader of the self-loop being emitted
    bool loop_dup = false;                            // ... emitted twice (full-warp copy + general)
    std::string loop_saved;                           // the output before that loop's body
    for (uint32_t i = 0; i < n; ++i) {
        const fi_insn& I = code[i];
        std::snprintf(stepx, sizeof stepx, "step + (%uu - pcm)", i);
        if (leader[i]) o(" B%u:\n", i);
        // a block whose BRA jumps back to its own leader is emitted as a structured
        // inner loop: the uniform-taken back edge that fits is its `continue`, so the
        // loop has one header and the compiler keeps loop-carried registers in place
        // (chaining through the label made a multi-entry loop: the allocator gave the
        // accumulators different homes at the top and the bottom and copied them on
        // every iteration)
        //   The loop body is emitted twice when no other pc inside it is a leader: a copy
        // for a full warp (all 32 lanes in amask, constant over the loop since its only
        // exit is the BRA), where `inA` is the constant true and every lane-predicated
        // write becomes an unconditional one — predicated accumulators and loads made the
        // allocator keep two homes per loop-carried register and copy between them on
        // every iteration — and the general copy.
        if (leader[i] && code[i + blen[i] - 1].op == BRA && code[i + blen[i] - 1].imm == i && blen[i] > 1) {
            loop_L = i;
            loop_dup = true;
            for (uint32_t q = i + 1; q < i + blen[i]; ++q) loop_dup = loop_dup && !leader[q];
            if (loop_dup && mode == 2 && tmpl_L == ~0u && blen[i] <= kTmplRecs) tmpl_L = i;
            if (loop_dup) {
                loop_saved = std::move(o.s);
                o.s.clear();
            } else {
                o(" for (;;) {  // self-loop %u..%u\n", i, i + blen[i] - 1);
            }
        }
        if (i < batch_end) {
            if (i + 1 == n) {
                flush_end();
                o(" { %sstep += %uu - pcm; upc = %uu; if (upc >= npc) { conv = false; if (inA) pc = upc; } continue; }\n",
                  kills(RSet()).c_str(), n, n);
            }
            continue;
        }
        if (I.op == LDG && G.sl.empty()) {
            const uint32_t m = ldg_batch_len(code, n, i, leader);
            if (m >= 2) {
                // the block holding the batch: from its leader L to its BRA / EXIT E
                uint32_t L = i;
                while (L > 0 && !leader[L]) --L;
                const uint32_t E = L + blen[L] - 1;
                const bool self_loop = code[E].op == BRA && code[E].imm == L;
                G.ldg_batch(o, code, i, m, self_loop ? batch_strides(G, code, L, E, i, m) : std::vector<std::string>());
                batch_end = i + m;
                if (i + m == n) {
                    flush_end();
                    o(" { %sstep += %uu - pcm; upc = %uu; if (upc >= npc) { conv = false; if (inA) pc = upc; } continue; }\n",
                      kills(RSet()).c_str(), n, n);
                }
                continue;
            }
        }
        if (I.op == BRA) {
            // block chaining: a uniform branch to a block that fits goes straight to
            // its code (the loop-top checks it skips cannot fire: see `fits`)
            auto chain = [&](uint32_t L) -> std::string {
                if (L >= n || !leader[L]) return "";
                char b[256];
                std::snprintf(b, sizeof b, "if (%uu <= npc && step + %uu <= lim%s) { pcm = %uu; ", L + blen[L], blen[L],
                              mode == 2 ? " && step < ckx" : "", L);
                return b + entry_kills(L) + "goto B" + std::to_string(L) + "; } ";
            };
            o(" { const bool pv = %s; %s", G.guard(I.guard).c_str(), mode == 2 ? "brk = 1u; " : "");
            G.rec(o, I, i, stepx, "pv");
            G.flush_recs(o, code, run_start(i), i, loop_L == I.imm && loop_L == tmpl_L ? tmpl_L : ~0u);
            const RSet keep_ft = use_kill ? lfrom[i + 1] : RSet();
            const RSet keep_tk = use_kill ? (I.imm < n ? lin[I.imm] : RSet()) | lfrom[i + 1] : RSet();
            if (loop_L == I.imm && i + 1 == loop_L + blen[loop_L]) {
                // the self-loop's back edge (uniform taken, next iteration fits), else its exit
                const uint32_t L = loop_L;
                o("lexm_ = amask & __ballot_sync(JFULL, pv); step += %uu - pcm;\n"
                  "   if (lexm_ == amask && %uu <= npc && step + %uu <= lim%s) { pcm = %uu; %s@@BACK@@ } }\n"
                  "   break;\n",
                  i + 1, L + blen[L], blen[L], mode == 2 ? " && step < ckx" : "", L, entry_kills(L).c_str());
                auto back = [](std::string b, const std::string& with) {
                    const size_t at = b.rfind("@@BACK@@");
                    return b.replace(at, 8, with);
                };
                if (loop_dup) {
                    std::string body = std::move(o.s);
                    o.s = std::move(loop_saved);
                    o(" if (amask == JFULL) { const bool inA = true; (void)inA;\n");
                    if (L == tmpl_L)                  // the warp's record template of this block (once per job)
                        // (every lane waits for its own bulk groups: the copies are issued by an
                        // elected lane)
                        o(" if (!tmpl_) { jbulk_wait_read(); __syncwarp();\n"
                          "   for (u32 j_ = lane; j_ < %uu; j_ += 32u) jtm_[j_] = make_uint4(k, __ldg(&ins[%uu + j_]), JFULL, JFULL);\n"
                          "   jfence_async(); __syncwarp(); tmpl_ = true; if (jx->prof.cc) jprof_tcnt(&jx->prof, lane, %uu, jtm_); }\n",
                          i + 1 - L, L, i + 1 - L);
                    // the full-warp copy unrolled twice: ptxas gives half of the loop-carried
                    // registers alternating homes, copied back on every back edge of a
                    // one-iteration loop; with two iterations per trip the homes swap roles
                    // (the template loop's profile state, constant over the loop, read once)
                    if (L == tmpl_L)
                        o(" const bool jpc_ = jx->prof.cc != nullptr; const u32 jrb_ = (u32)jx->prof.rb; (void)jpc_; (void)jrb_;\n"
                          " const u32 jtc_ = lane < 8u ? jx->prof.tcnt_[lane] : 0u; u32 jpa_ = 0u; (void)jtc_; (void)jpa_;\n"
                          " const u64 jpol_ = jpolicy_ef(); (void)jpol_;\n#undef JPOL_\n#define JPOL_ jpol_\n"
                          "#undef JPCC_\n#define JPCC_ jpc_\n#undef JPRB_\n#define JPRB_ jrb_\n"
                          "#undef JPADD_\n#define JPADD_ (jpa_ += jtc_)\n"
                          "#undef JPFLUSH_\n#define JPFLUSH_ { if (lane < 8u) jx->prof.pcnt_[lane] += jpa_; jpa_ = 0u; }\n");
                    o("#undef JFW_\n#define JFW_ 1\n for (;;) {  // self-loop %u..%u, full warp, two iterations per trip\n {\n",
                      L, i);
                    o.s += back(body, "goto U" + std::to_string(L) + "_;");
                    o(" }\n U%u_: ;\n {\n", L);
                    o.s += back(body, "continue;");
                    o(" }\n }\n#undef JFW_\n#define JFW_ 0\n");
                    if (L == tmpl_L)   // (the loop is left only through its breaks: flush the register count there)
                        o(" JPFLUSH_;\n#undef JPCC_\n#define JPCC_ (jx->prof.cc != nullptr)\n#undef JPRB_\n#define JPRB_ ((u32)jx->prof.rb)\n"
                          "#undef JPADD_\n#define JPADD_ { if (lane < 8u) jx->prof.pcnt_[lane] += jx->prof.tcnt_[lane]; }\n"
                          "#undef JPFLUSH_\n#define JPFLUSH_ {}\n#undef JPOL_\n#define JPOL_ jpolicy_ef()\n");
                    o(" } else {\n for (;;) {  // self-loop %u..%u\n", L, i);
                    o.s += back(body, "continue;");
                    o(" } }\n");
                } else {
                    o.s = back(std::move(o.s), "continue;");
                    o(" }\n");
                }
                o(" { const u32 exm_ = lexm_;\n");
                loop_L = ~0u;
            } else {
                o("const u32 exm_ = amask & __ballot_sync(JFULL, pv); step += %uu - pcm;\n", i + 1);
            }
            o("   if (exm_ == 0u) { %s%supc = %uu; } else if (exm_ == amask) { %s%supc = %uu; }\n"
              "   else { %sconv = false; if (inA) pc = ((exm_ >> lane) & 1u) ? %uu : %uu; }\n"
              "   if (conv && (amask == 0u || upc >= npc)) { conv = false; if ((amask >> lane) & 1u) pc = upc; }\n"
              "   continue; }\n",
              chain(i + 1).c_str(), kills(keep_ft).c_str(), i + 1, chain(I.imm).c_str(),
              kills(keep_tk).c_str(), I.imm, kills(keep_tk).c_str(), I.imm, i + 1);
        } else if (I.op == EXIT) {
            o(" { const bool pv = %s; %s", G.guard(I.guard).c_str(), mode == 2 ? "brk = 1u; " : "");
            G.rec(o, I, i, stepx, "pv");
            G.flush_recs(o, code, run_start(i), i);
            o("const u32 exm_ = amask & __ballot_sync(JFULL, pv); step += %uu - pcm;\n"
              "   if (inA && pv) live = false; livem &= ~exm_; amask &= ~exm_; upc = %uu; %s\n"
              "   if (conv && (amask == 0u || upc >= npc)) { conv = false; if ((amask >> lane) & 1u) pc = upc; }\n"
              "   continue; }\n",
              i + 1, i + 1, kills(use_kill ? lfrom[i + 1] : RSet()).c_str());
        } else {
            if (I.op == LDG || I.op == STG) {
                G.mem(o, I, i, stepx);
            } else if (!G.skip(I, i)) {
                o(" { const bool pv = %s; const bool ex = inA && pv; (void)pv; ", G.guard(I.guard).c_str());
                G.rec(o, I, i, stepx, "pv");
                G.plain(o, I);
                o(" }\n");
            }
            if (i + 1 == n) {
                flush_end();
                o(" { %sstep += %uu - pcm; upc = %uu; if (upc >= npc) { conv = false; if (inA) pc = upc; } continue; }\n",
                  kills(RSet()).c_str(), n, n);
            }
        }
    }
    // ---- step mode: registers to the warp's shared-memory file, interpreter, back
    // (the per-lane context names are member names of JState / JOut too: spelled out below)
    for (const char* nm : kCtxLaneNames) o("#undef %s\n", nm);
    o(" S_any: {\n");
    for (uint32_t j = 0; j < NR; ++j) o("  Rs[%uu + lane] = R%u;%s", j * 32, j, (j % 8 == 7) ? "\n" : "");
    o("\n  JState st_; st_.pc = pc; st_.live = live; st_.step = step; st_.livem = livem; st_.conv = conv; "
      "st_.upc = upc; st_.amask = amask; st_.npc = npc; st_.nst = jx->nst_[lane]; st_.fault = jx->fault_[lane]; "
      "st_.fault_pc = jx->fault_pc_[lane]; st_.before = jx->before_[lane]; st_.after = jx->after_[lane]; "
      "st_.msk = jx->msk_[lane]; st_.fired = jx->fired_[lane]; st_.bad = jx->bad_[lane]; st_.lim = lim;\n"
      "  st_.preds = (u32)Q0 | ((u32)Q1 << 1) | ((u32)Q2 << 2) | ((u32)Q3 << 3) | ((u32)Q4 << 4) | ((u32)Q5 << 5) | "
      "((u32)Q6 << 6); st_.recbuf = recbuf; st_.brk = brk; st_.ckn = ckn;\n"
      "  __syncwarp();\n"
      "  JBufCache bcs_;                     // (step mode's own cache: bc's address never escapes, so it stays in registers)\n"
      "  const u32 done_ = jinterp<%u>(A, st_, bcs_, Rs, dec, kblen_%u, %uu, k, cta, wic, watchdog, hstep, hpc, hlane, "
      "hkind, hreg, hbfm, hmask, st_out, st_cap, %uu, img_w, rec_out, ck, ck_interval, ins, pgp, %s, %s);\n"
      "  __syncwarp();\n",
      mode, kid, n, NR, G.sl.empty() ? "(const u8*)0" : ("kslice_" + std::to_string(kid)).c_str(),
      mode == 2 ? "&jx->prof" : "(JProf*)0");
    for (uint32_t j = 0; j < NR; ++j) o("  R%u = Rs[%uu + lane];%s", j, j * 32, (j % 8 == 7) ? "\n" : "");
    o("\n  pc = st_.pc; live = st_.live; step = st_.step; livem = st_.livem; conv = st_.conv; upc = st_.upc; "
      "amask = st_.amask; npc = st_.npc; jx->nst_[lane] = st_.nst; jx->fault_[lane] = st_.fault; "
      "jx->fault_pc_[lane] = st_.fault_pc; jx->before_[lane] = st_.before; jx->after_[lane] = st_.after; "
      "jx->msk_[lane] = st_.msk; jx->fired_[lane] = st_.fired; jx->bad_[lane] = st_.bad; lim = st_.lim; "
      "recbuf = st_.recbuf; brk = st_.brk; ckn = st_.ckn; if (ck) ckx = ckn * ck_interval;\n"
      "  Q0 = st_.preds & 1u; Q1 = (st_.preds >> 1) & 1u; Q2 = (st_.preds >> 2) & 1u; Q3 = (st_.preds >> 3) & 1u; "
      "Q4 = (st_.preds >> 4) & 1u; Q5 = (st_.preds >> 5) & 1u; Q6 = (st_.preds >> 6) & 1u;\n"
      "  if (done_) goto finish;\n  continue;\n }\n}\n");
    o("finish:\n");
    // (only the entries this kernel uses, and the K8 page fields only in PAGE mode:
    // whatever the block code never reads would otherwise hold registers across it)
    o(" {                                 // the buffer cache for this warp's next job\n"
      "#pragma unroll\n  for (int s_ = 0; s_ < %d; ++s_) { jx->bc_[s_ * 4][lane] = bc.lo[s_]; "
      "jx->bc_[s_ * 4 + 1][lane] = bc.sz[s_]; %s}\n"
      "#pragma unroll\n  for (int s_ = %d; s_ < JBC_SLOTS; ++s_) jx->bc_[s_ * 4 + 1][lane] = 0u;\n"
      "  u32 z_ = 0u;\n#pragma unroll\n  for (int s_ = 0; s_ < %d; ++s_) z_ |= (u32)bc.z[s_] << s_;\n"
      "  jx->bcz_[lane] = z_; __syncwarp(); if (lane == 0u) { jx->bck = k; %s} __syncwarp(); }\n",
      nslots,
      mode == 3 ? "jx->bc_[s_ * 4 + 2][lane] = bc.b[s_]; jx->bc_[s_ * 4 + 3][lane] = bc.pb[s_]; " : "", nslots, nslots,
      mode == 3 ? "jx->bckp = (u32)(size_t)PG.ptab; " : "");
    if (mode == 2) o(" jbulk_wait(); __syncwarp();     // the template stores are complete (each lane's own groups)\n");
    if (mode == 2)                                    // checkpoints the warp never reached: absent
        o(" if (ck) for (; ckn < (step + ck_interval - 1u) / ck_interval; ++ckn) {\n"
          "   for (u32 r_ = 0u; r_ < %uu; ++r_) ck[(u64)ckn * %uu + r_ * 32u + lane] = 0u;\n"
          "   ck[(u64)ckn * %uu + %uu + lane] = 0xFFFFFFFFu; }\n",
          NR + 3, (NR + 4) * 32, (NR + 4) * 32, (NR + 3) * 32);
    o("#undef out\n");
    o(" { JOut& out_ = *jx->out; out_.steps = step; out_.fault = jx->fault_[lane]; out_.fault_pc = jx->fault_pc_[lane]; "
      "out_.nstore = jx->nst_[lane];\n"
      " out_.before = __shfl_sync(JFULL, jx->before_[lane], hlane); out_.after = __shfl_sync(JFULL, jx->after_[lane], hlane);\n"
      " out_.mask = __shfl_sync(JFULL, jx->msk_[lane], hlane); out_.fired = jx->fired_[lane]; out_.bad = jx->bad_[lane]; }\n}\n");
    for (const char* nm : kCtxNames) o("#undef %s\n", nm);
    o("#undef JIN_\n#undef cbank_len\n#undef cb\n\n");
}

// The module source of static kernel `only` (its device functions, and entry kernels
// that serve only it), or of every kernel (only < 0: fi_jit_source's combined view).
std::string generate(const fi_insn* code, const fi_kernel* kern, uint32_t n_kern, uint32_t n_regs, uint32_t modes,
                     int only = -1) {
    const bool slice_len = modes & kJitSliceLen;    // golden pass 1 as the control slice (fi_jit_build decides)
    // resident 128-thread CTAs per SM the register budget targets (3: <= 168 registers)
    const uint32_t min_blocks = 3;
    Src o;
    o.s += kPrelude;
    Gen G{n_regs};
    auto mine = [&](uint32_t k) { return only < 0 || (uint32_t)only == k; };
    for (uint32_t k = 0; k < n_kern; ++k) {
        if (!mine(k)) continue;
        bool tables = true;
        if (modes & FI_JIT_INJECT) { gen_kernel(o, G, k, code + kern[k].code_off, kern[k].code_len, 0, tables); tables = false; }
        if (modes & FI_JIT_GOLDEN) {
            gen_kernel(o, G, k, code + kern[k].code_off, kern[k].code_len, 1, tables, slice_len);
            gen_kernel(o, G, k, code + kern[k].code_off, kern[k].code_len, 2, false);
            tables = false;
        }
        if (modes & FI_JIT_PAGE) gen_kernel(o, G, k, code + kern[k].code_off, kern[k].code_len, 3, tables);
    }
    const uint32_t rs = (n_regs + 1) * 32, zrow = n_regs * 32, ckw = (n_regs + 4) * 32;
    if (modes & FI_JIT_INJECT) {
    // K4 on the generated kernels: persistent warps over the LPT-ordered replicas
    // (same scheduling and outputs as inject.cu's k_inject)
    o("extern \"C\" __global__ void __launch_bounds__(128, %u) k_inject_jit(", min_blocks);
    o("const JArgs A, const u64* __restrict__ warp_off, "
      "const jfi_site* __restrict__ sites, const u32 n, jfi_inj* __restrict__ out, jfi_store* __restrict__ log, "
      "const u32 cap, const u32* ckpt, const u64* __restrict__ ck_off, const u32 ck_interval, "
      "const u32* __restrict__ order, u32* counter, u32* status, u32* smq, const u32 nsm, const u32 dealt) {\n"
      " extern __shared__ u32 jsmem[];\n"
      " const u32 lane = threadIdx.x & 31u;\n"
      " u32* Rs = jsmem + (threadIdx.x >> 5) * %uu;\n"
      " Rs[%uu + lane] = 0u;                     // the zero row (RZ, indices >= n_regs)\n"
      " { JCtx* jx0_ = reinterpret_cast<JCtx*>(jsmem + %uu + (threadIdx.x >> 5) * (JCTX_BYTES / 4u)); "
          "if ((threadIdx.x & 31u) == 0u) jx0_->bck = 0xFFFFFFFFu; __syncwarp(); }\n"
      " const u32 sm_ = jsmid();\n"
      " for (;;) {\n  const u32 p = jnext_job(counter, smq, sm_, nsm, dealt, n, lane);\n"
      "  if (p >= n) return;\n  const u32 i = order[p]; const jfi_site S = sites[i];\n"
      "  if (S.flags & 1u) { if (%s && lane == 0u) { jfi_inj r; r.before = r.after = r.mask = r.fault_pc = 0u; "
      "r.fault_kind = 0; r.outcome = 3; r.overflow = 0; r.flags = 0; r.n_faulty_stores = 0u; out[i] = r; } continue; }\n"
      "  const jfi_instance in = A.inst[S.instance]; const u32 wpc = (in.block + 31u) / 32u, lw = S.warp - in.warp_begin;\n"
      "  if (%s) continue;                       // another module's replica\n"
      "  const u64 L = warp_off[S.warp + 1] - warp_off[S.warp]; const u64 wd = 10ull * L + 1024ull;\n"
      "  const u32 watchdog = wd > 0xFFFFFFFFull ? 0xFFFFFFFFu : (u32)wd;\n"
      "  u32* ck = ckpt ? (u32*)ckpt + ck_off[S.warp] * %uull : (u32*)0;\n"
      "  JOut o; o.start = 0u;\n  switch (in.kernel) {\n",
      rs, zrow, 4 * rs, only <= 0 ? "true" : "false",
      only < 0 ? "false" : ("in.kernel != " + std::to_string(only) + "u").c_str(), ckw);
    for (uint32_t k = 0; k < n_kern; ++k)
        if (mine(k)) o("   case %u: kern_%u_inj(A, S.step, S.pc, S.lane, S.dst_kind, S.dst_reg, S.bfm, S.mask, S.instance, lw / wpc, "
          "lw %% wpc, watchdog, ck, ck ? ck_interval : 0u, log + (u64)i * cap, cap, o, Rs, A.dec + %uu, A.ins + %uu, "
          "(u8*)0, (uint4*)0, (const JPage*)0); break;\n",
          k, k, kern[k].code_off, kern[k].code_off);
    o("   default: o.steps = 0; o.fired = false; o.bad = true; o.fault = 0; o.fault_pc = 0; o.nstore = 0; "
      "o.before = o.after = o.mask = 0; break;\n  }\n"
      "  if (lane == 0u) {\n   jfi_inj r; r.before = o.before; r.after = o.after; r.mask = o.mask; r.fault_pc = o.fault_pc;\n"
      "   r.fault_kind = (u8)o.fault; r.outcome = 0; r.overflow = o.nstore > cap; r.flags = 0; r.n_faulty_stores = o.nstore;\n"
      "   out[i] = r;\n   if (!o.fired || o.bad) atomicOr(status, 1u << 6);\n"
      "   atomicAdd((unsigned long long*)(counter + 2), (unsigned long long)(o.steps - o.start));\n  }\n  __syncwarp();\n }\n}\n");
    }
    if (modes & FI_JIT_PAGE) {
        // K8's re-execution of instance t (propagate8.cu k8_exec) on the generated kernels
        o("extern \"C\" __global__ void __launch_bounds__(128, %u) k8_exec_jit(const JArgs A, const JK8 K, const u32 t) {\n"
          " extern __shared__ u32 jsmem[];\n const u32 lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;\n"
          " u32* Rs = jsmem + wib * %uu;\n Rs[%uu + lane] = 0u;\n"
          " { JCtx* jx0_ = reinterpret_cast<JCtx*>(jsmem + %uu + (threadIdx.x >> 5) * (JCTX_BYTES / 4u)); if ((threadIdx.x & 31u) == 0u) jx0_->bck = 0xFFFFFFFFu; __syncwarp(); }\n"
          " jfi_store* scr = K.scratch + (u64)(blockIdx.x * 4u + wib) * K.log_cap;\n"
          " const jfi_instance in = A.inst[t];\n const u32 nw = in.warp_end - in.warp_begin, wpc = (in.block + 31u) / 32u;\n"
          " const u64 items = (u64)(*K.n_active) * nw;\n const bool unchecked = K.flags & 1u;\n"
          " u64 nsteps_ = 0ull;                       // this warp's emulated steps, one atomic at its end\n"
          " for (;;) {\n  u32 it = 0u; if (lane == 0u) it = atomicAdd(K.work, 1u); it = __shfl_sync(JFULL, it, 0);\n"
          "  if (it >= items) { if (lane == 0u && nsteps_) atomicAdd(K.steps, (unsigned long long)nsteps_); return; }\n"
          "  const u32 s = K.active[it / nw], lw = it %% nw, w = in.warp_begin + lw;\n"
          "  if (K.slot[s].overflow) continue;\n"
          "  const u64 L = K.warp_off[w + 1] - K.warp_off[w]; const u64 wd = 10ull * L + 1024ull;\n"
          "  const u32 watchdog = wd > 0xFFFFFFFFull ? 0xFFFFFFFFu : (u32)wd;\n"
          "  JPage pg; pg.ptab = K.ptab + (u64)s * K.total_pages; pg.pool = K.pool; pg.page_base = K.page_base; "
          "pg.last_ref = K.last_ref; pg.dropped = K.dropped + (u64)s * K.dwords; pg.bcount = K.bcount + (u64)s * K.n_buf; "
          "pg.inexact = &K.slot[s].inexact; pg.t = t;\n"
          "  JOut o; o.start = 0u;\n  switch (in.kernel) {\n",
          min_blocks, rs, zrow, 4 * rs);
        for (uint32_t k = 0; k < n_kern; ++k)
            if (mine(k)) o("   case %u: kern_%u_page(A, 0xFFFFFFFFu, 0u, 0u, 0u, 0u, 0u, 0u, t, lw / wpc, lw %% wpc, watchdog, (u32*)0, "
              "0u, scr, K.log_cap, o, Rs, A.dec + %uu, A.ins + %uu, (u8*)0, (uint4*)0, &pg); break;\n",
              k, k, kern[k].code_off, kern[k].code_off);
        o("   default: o.steps = 0; o.fault = 4; o.fault_pc = 0; o.nstore = 0; break;\n  }\n"
          "  nsteps_ += o.steps - o.start;\n"
          "  if (o.fault) {\n   if (lane == 0u) {\n"
          "    const unsigned long long key = ((unsigned long long)t << 43) | ((unsigned long long)lw << 19) | "
          "((unsigned long long)o.fault << 16) | (o.fault_pc & 0xFFFFu);\n"
          "    if (!(unchecked && o.fault != 3u)) atomicMin(&K.slot[s].fault_key, key); "
          "else atomicMin(&K.slot[s].pdue_key, key);\n   }\n"
          "   if (!(unchecked && o.fault != 3u)) continue;\n  }\n"
          "  if (o.nstore > K.log_cap) { if (lane == 0u) jk8_err(K, s, 8); continue; }\n"
          "  jk8_updates(A, K, s, lw, scr, o.nstore, K.gst + K.gst_off[w], K.gst_off[w + 1] - K.gst_off[w], (i64)t);\n"
          " }\n}\n");
    }
    if (modes & FI_JIT_GOLDEN) {
        // golden pass 1 (one launch per instance k, golden.cu k_golden_len) and pass 2
        // (every warp in one launch, golden.cu k_golden_trace) on the generated kernels
        o("extern \"C\" __global__ void __launch_bounds__(128, %u) k_golden_len_jit(const JArgs A, const u32 k, "
          "u8* img_w, u64* warp_len, u64* warp_nst, u32* status) {\n"
          " extern __shared__ u32 jsmem[];\n const u32 lane = threadIdx.x & 31u;\n"
          " u32* Rs = jsmem + (threadIdx.x >> 5) * %uu;\n Rs[%uu + lane] = 0u;\n"
          " { JCtx* jx0_ = reinterpret_cast<JCtx*>(jsmem + %uu + (threadIdx.x >> 5) * (JCTX_BYTES / 4u)); if ((threadIdx.x & 31u) == 0u) jx0_->bck = 0xFFFFFFFFu; __syncwarp(); }\n"
          " const jfi_instance in = A.inst[k];\n const u32 lw = blockIdx.x * 4u + (threadIdx.x >> 5);\n"
          " if (lw >= in.warp_end - in.warp_begin) return;\n const u32 wpc = (in.block + 31u) / 32u;\n"
          " JOut o;\n switch (in.kernel) {\n",
          min_blocks, rs, zrow, 4 * rs);
        for (uint32_t k = 0; k < n_kern; ++k)
            if (mine(k)) o("  case %u: kern_%u_len(A, 0xFFFFFFFFu, 0u, 0u, 0u, 0u, 0u, 0u, k, lw / wpc, lw %% wpc, 0xFFFFFFFFu, (u32*)0, "
              "0u, (jfi_store*)0, 0u, o, Rs, A.dec + %uu, A.ins + %uu, img_w, (uint4*)0, (const JPage*)0); break;\n",
              k, k, kern[k].code_off, kern[k].code_off);
        o("  default: o.steps = 0; o.fault = 9; o.nstore = 0; break;\n }\n"
          " if (lane == 0u) { warp_len[in.warp_begin + lw] = o.steps; warp_nst[in.warp_begin + lw] = o.nstore; "
          "if (o.fault) atomicOr(status, 1u << 4); }\n}\n");
        // (one launch per instance k, like pass 1: each module serves its own kernel's instances)
        o("extern \"C\" __global__ void __launch_bounds__(128, %u) k_golden_trace_jit(const JArgs A, const u32 k, "
          "const u64* __restrict__ warp_off, const u64* __restrict__ gst_off, uint4* rec, jfi_store* gst, u32* ckpt, "
          "const u64* __restrict__ ck_off, const u32 ck_interval, u32* status, u8* img_w_all, const u32 w_lo, const u32 w_hi, "
          "const u32 own_lo, const u32 own_hi, u32* pcc, unsigned long long* pic) {\n"
          " extern __shared__ u32 jsmem[];\n const u32 lane = threadIdx.x & 31u;\n"
          " u32* Rs = jsmem + (threadIdx.x >> 5) * %uu;\n Rs[%uu + lane] = 0u;\n"
          " JCtx* const jx0_ = reinterpret_cast<JCtx*>(jsmem + %uu + (threadIdx.x >> 5) * (JCTX_BYTES / 4u));\n"
          " if (lane == 0u) jx0_->bck = 0xFFFFFFFFu;\n __syncwarp();\n"
          " const jfi_instance in = A.inst[k];\n const u32 lw = blockIdx.x * 4u + (threadIdx.x >> 5);\n"
          " if (lw >= in.warp_end - in.warp_begin) return;\n const u32 w = in.warp_begin + lw, wpc = (in.block + 31u) / 32u;\n"
          " if (w < w_lo || w >= w_hi) return;            // another rank's warp (owner-computes golden run)\n"
          " u8* img_w = (w >= own_lo && w < own_hi) ? img_w_all : (u8*)0;   // image stores: the owner only\n"
          " const u64 r0 = warp_off[w], g0 = gst_off[w];\n"
          " if (lane == 0u) { jx0_->prof.cc = pcc; jx0_->prof.rb = r0; }\n"
          " if (lane < 8u) { jx0_->prof.pch_[lane] = (u32)(r0 >> 10); jx0_->prof.pcnt_[lane] = 0u; jx0_->prof.ptot_[lane] = 0ull; }\n"
          " __syncwarp();\n"
          " u32* ck = ckpt ? ckpt + ck_off[w] * %uull : (u32*)0;\n"
          " JOut o;\n switch (in.kernel) {\n",
          min_blocks, rs, zrow, 4 * rs, ckw);
        for (uint32_t k = 0; k < n_kern; ++k)
            if (mine(k)) o("  case %u: kern_%u_trace(A, 0xFFFFFFFFu, 0u, 0u, 0u, 0u, 0u, 0u, k, lw / wpc, lw %% wpc, 0xFFFFFFFFu, ck, "
              "ck ? ck_interval : 0u, gst + g0, 0xFFFFFFFFu, o, Rs, A.dec + %uu, A.ins + %uu, img_w, rec + r0, "
              "(const JPage*)0); break;\n",
              k, k, kern[k].code_off, kern[k].code_off);
        o("  default: o.steps = 0; o.fault = 9; o.nstore = 0; break;\n }\n"
          " if (lane == 0u && (o.fault || o.steps != warp_off[w + 1] - r0 || o.nstore != gst_off[w + 1] - g0)) "
          "atomicOr(status, 1u << 4);\n"
          " if (pcc && lane < 8u) {            // the fused profile: the last chunk's counts, the warp's totals\n"
          "  jprof_next(&jx0_->prof, lane);\n"
          "  if (jx0_->prof.ptot_[lane]) atomicAdd(&pic[(u64)k * 8u + lane], (unsigned long long)jx0_->prof.ptot_[lane]); }\n}\n");
    }
    return o.s;
}

// ---------------------------------------------------------------- NVRTC + driver
typedef int (*nvrtcCreateProgram_t)(void**, const char*, const char*, int, const char* const*, const char* const*);
typedef int (*nvrtcCompileProgram_t)(void*, int, const char* const*);
typedef int (*nvrtcGetSize_t)(void*, size_t*);
typedef int (*nvrtcGetData_t)(void*, char*);
typedef int (*nvrtcDestroyProgram_t)(void**);

struct Nvrtc {
    void* h = nullptr;
    nvrtcCreateProgram_t create = nullptr;
    nvrtcCompileProgram_t compile = nullptr;
    nvrtcGetSize_t log_size = nullptr, cubin_size = nullptr;
    nvrtcGetData_t log = nullptr, cubin = nullptr;
    nvrtcDestroyProgram_t destroy = nullptr;
    bool ok = false;
};

Nvrtc& nvrtc() {
    static Nvrtc N;
    static std::once_flag once;
    std::call_once(once, [] {
        const char* cands[] = {"libnvrtc.so.12", "/usr/local/cuda/lib64/libnvrtc.so.12", "libnvrtc.so"};
        for (const char* c : cands)
            if ((N.h = dlopen(c, RTLD_NOW | RTLD_LOCAL))) break;
        if (!N.h) return;
        N.create = (nvrtcCreateProgram_t)dlsym(N.h, "nvrtcCreateProgram");
        N.compile = (nvrtcCompileProgram_t)dlsym(N.h, "nvrtcCompileProgram");
        N.log_size = (nvrtcGetSize_t)dlsym(N.h, "nvrtcGetProgramLogSize");
        N.log = (nvrtcGetData_t)dlsym(N.h, "nvrtcGetProgramLog");
        N.cubin_size = (nvrtcGetSize_t)dlsym(N.h, "nvrtcGetCUBINSize");
        N.cubin = (nvrtcGetData_t)dlsym(N.h, "nvrtcGetCUBIN");
        N.destroy = (nvrtcDestroyProgram_t)dlsym(N.h, "nvrtcDestroyProgram");
        N.ok = N.create && N.compile && N.log_size && N.log && N.cubin_size && N.cubin && N.destroy;
    });
    return N;
}

typedef CUresult (*cuModuleLoadData_t)(CUmodule*, const void*);
typedef CUresult (*cuModuleGetFunction_t)(CUfunction*, CUmodule, const char*);
typedef CUresult (*cuModuleUnload_t)(CUmodule);
typedef CUresult (*cuLaunchKernel_t)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                                     CUstream, void**, void**);
typedef CUresult (*cuOccupancy_t)(int*, CUfunction, int, size_t);
typedef CUresult (*cuFuncSetAttribute_t)(CUfunction, CUfunction_attribute, int);

struct Drv {
    cuModuleLoadData_t load = nullptr;
    cuModuleGetFunction_t get = nullptr;
    cuModuleUnload_t unload = nullptr;
    cuLaunchKernel_t launch = nullptr;
    cuOccupancy_t occ = nullptr;
    cuFuncSetAttribute_t set_attr = nullptr;
    bool ok = false;
};

Drv& drv() {
    static Drv D;
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        cudaGetDriverEntryPoint("cuModuleLoadData", (void**)&D.load, cudaEnableDefault, &q);
        cudaGetDriverEntryPoint("cuModuleGetFunction", (void**)&D.get, cudaEnableDefault, &q);
        cudaGetDriverEntryPoint("cuModuleUnload", (void**)&D.unload, cudaEnableDefault, &q);
        cudaGetDriverEntryPoint("cuLaunchKernel", (void**)&D.launch, cudaEnableDefault, &q);
        cudaGetDriverEntryPoint("cuOccupancyMaxActiveBlocksPerMultiprocessor", (void**)&D.occ, cudaEnableDefault, &q);
        cudaGetDriverEntryPoint("cuFuncSetAttribute", (void**)&D.set_attr, cudaEnableDefault, &q);
        D.ok = D.load && D.get && D.unload && D.launch && D.occ && D.set_attr;
    });
    return D;
}

thread_local std::string g_jit_log;

}  // namespace

// step mode's shared-memory register files: 4 warps x (n_regs + 1) rows x 32 lanes
// + 4 warps' JCtx (JCTX_BYTES of jit_prelude.cuh)
static size_t jit_smem(uint32_t n_regs) { return (size_t)4 * (n_regs + 1) * 128 + 4 * kJctxBytes; }
// ... + the golden trace pass's 4 record templates (16 B per record)
static size_t jit_smem_trace(uint32_t n_regs) { return jit_smem(n_regs) + (size_t)4 * kTmplRecs * 16; }

// one CUmodule per static kernel (compiled in parallel: ptxas time grows faster
// than linearly with the size of one program), each with the entry kernels of
// its own kernel
struct fi_jit_mod {
    CUmodule mod = nullptr;
    CUfunction inject = nullptr, glen = nullptr, gtrace = nullptr, k8exec = nullptr;
};
struct fi_jit {
    size_t smem = 0, smem_trace = 0;
    uint32_t modes = 0;
    std::vector<fi_jit_mod> m;                        // [static kernel]
    uint32_t n_regs = 0, n_code = 0;
    bool len_sliced = false;                          // golden pass 1 generated as the control slice
    double compile_s = 0;
    size_t src_bytes = 0, cubin_bytes = 0;
};

namespace fi {
size_t aux_dec_offset(const fi_program* p);
size_t aux_ins_offset(const fi_program* p);
void launch_lpt_order(const fi_program* p, const fi_site* sites, const uint64_t* warp_off, uint32_t ck_interval,
                      uint32_t n, uint32_t* order, uint32_t* counter, cudaStream_t s);
}

extern "C" const char* fi_jit_log(void) { return g_jit_log.c_str(); }

extern "C" size_t fi_jit_source(const fi_insn* code_host, uint32_t n_code, const fi_kernel* kern_host, uint32_t n_kern,
                                uint32_t n_regs, uint32_t modes, char* buf, size_t buf_bytes) {
    if (!code_host || !kern_host || !n_kern || n_regs == 0 || n_regs > fi::kRZ || !(modes & 7) ||
        (modes & ~(7u | kJitSliceLen)))
        return 0;
    for (uint32_t k = 0; k < n_kern; ++k)
        if ((uint64_t)kern_host[k].code_off + kern_host[k].code_len > n_code) return 0;
    const std::string s = generate(code_host, kern_host, n_kern, n_regs, modes);
    if (buf && buf_bytes) {
        const size_t m = std::min(buf_bytes - 1, s.size());
        std::memcpy(buf, s.data(), m);
        buf[m] = 0;
    }
    return s.size() + 1;
}

namespace {
fi_status compile_cubin(const fi_insn* code, const fi_kernel* kern, uint32_t n_kern, uint32_t n_regs, uint32_t modes,
                        std::string& src, std::vector<char>& cubin, int only = -1) {
    Nvrtc& N = nvrtc();
    if (!N.ok) { g_jit_log = "libnvrtc.so.12 not found"; return FI_E_CUDA; }
    src = generate(code, kern, n_kern, n_regs, modes, only);
    // FI_JIT_DUMP=<p> (profiling aid): the module's source and cubin are written to
    // <p>[_k<kernel>].cu / .cubin, and the program is NAMED by that path, so the line
    // table of the -lineinfo cubin points at a file that exists (ncu --import-source)
    std::string dump;
    if (const char* d = std::getenv("FI_JIT_DUMP"))
        dump = std::string(d) + (only > 0 ? "_k" + std::to_string(only) : std::string());
    if (!dump.empty())
        if (FILE* f = std::fopen((dump + ".cu").c_str(), "wb")) { std::fwrite(src.data(), 1, src.size(), f); std::fclose(f); }
    const std::string pname = dump.empty() ? std::string("fi_jit.cu") : dump + ".cu";
    void* prog = nullptr;
    if (N.create(&prog, src.c_str(), pname.c_str(), 0, nullptr, nullptr)) { g_jit_log = "nvrtcCreateProgram failed"; return FI_E_CUDA; }
    // --fmad=false: FMUL + FADD are never contracted (C-13); fixed, not configurable
    const std::vector<const char*> opts = {"--gpu-architecture=sm_100a", "--std=c++17", "--fmad=false", "-lineinfo"};
    const int rc = N.compile(prog, (int)opts.size(), opts.data());
    size_t ls = 0;
    N.log_size(prog, &ls);
    std::string lg(ls, '\0');
    if (ls) N.log(prog, &lg[0]);
    g_jit_log = lg;
    if (rc) { N.destroy(&prog); return FI_E_PROGRAM; }
    size_t cs = 0;
    N.cubin_size(prog, &cs);
    cubin.resize(cs);
    N.cubin(prog, cubin.data());
    N.destroy(&prog);
    if (!dump.empty())
        if (FILE* f = std::fopen((dump + ".cubin").c_str(), "wb")) { std::fwrite(cubin.data(), 1, cubin.size(), f); std::fclose(f); }
    return FI_OK;
}

bool valid_kernels(const fi_kernel* kern, uint32_t n_kern, uint32_t n_code) {
    for (uint32_t k = 0; k < n_kern; ++k)
        if ((uint64_t)kern[k].code_off + kern[k].code_len > n_code) return false;
    return true;
}

// every static kernel's module, NVRTC programs compiled by a pool of threads
fi_status compile_all(const fi_insn* code, const fi_kernel* kern, uint32_t n_kern, uint32_t n_regs, uint32_t modes,
                      std::vector<std::vector<char>>& cubins, size_t& src_bytes) {
    cubins.assign(n_kern, {});
    std::vector<fi_status> st(n_kern, FI_OK);
    std::vector<std::string> logs(n_kern);
    std::vector<size_t> sb(n_kern, 0);
    std::atomic<uint32_t> next{0};
    auto work = [&] {
        for (uint32_t k; (k = next.fetch_add(1)) < n_kern;) {
            std::string src;
            st[k] = compile_cubin(code, kern, n_kern, n_regs, modes, src, cubins[k], (int)k);
            logs[k] = g_jit_log;                      // (thread_local: carried back to the caller)
            sb[k] = src.size();
        }
    };
    uint32_t nt = std::max(1u, std::min<uint32_t>(n_kern, std::thread::hardware_concurrency()));
    if (const char* e = std::getenv("FI_JIT_THREADS")) nt = std::max(1, std::atoi(e));
    std::vector<std::thread> pool;
    for (uint32_t t = 1; t < nt; ++t) pool.emplace_back(work);
    work();
    for (auto& t : pool) t.join();
    src_bytes = 0;
    for (uint32_t k = 0; k < n_kern; ++k) {
        src_bytes += sb[k];
        if (st[k]) { g_jit_log = "static kernel " + std::to_string(k) + ": " + logs[k]; return st[k]; }
    }
    g_jit_log = logs.empty() ? std::string() : logs[0];
    return FI_OK;
}
}  // namespace

extern "C" fi_status fi_jit_compile_check(const fi_insn* code_host, uint32_t n_code, const fi_kernel* kern_host,
                                          uint32_t n_kern, uint32_t n_regs, uint32_t modes, size_t* cubin_bytes) {
    if (!code_host || !kern_host || !n_kern || n_regs == 0 || n_regs > fi::kRZ || !(modes & 7) ||
        (modes & ~(7u | kJitSliceLen)))
        return FI_E_ARG;
    if (!valid_kernels(kern_host, n_kern, n_code)) return FI_E_ARG;
    std::vector<std::vector<char>> cubins;
    size_t sb = 0;
    fi_status e = compile_all(code_host, kern_host, n_kern, n_regs, modes, cubins, sb);
    if (cubin_bytes) {
        *cubin_bytes = 0;
        for (auto& c : cubins) *cubin_bytes += c.size();
    }
    return e;
}

extern "C" fi_status fi_jit_build(const fi_program* p, const fi_kernel* kern_host, uint32_t modes, fi_jit** out) {
    if (!p || !kern_host || !out || !p->code_host || !p->n_kern || p->n_regs == 0 || p->n_regs > fi::kRZ || !modes ||
        modes > 7)
        return FI_E_ARG;
    if (!valid_kernels(kern_host, p->n_kern, p->n_code)) return FI_E_ARG;
    *out = nullptr;
    Drv& D = drv();
    if (!D.ok) { g_jit_log = "CUDA driver entry points unavailable"; return FI_E_CUDA; }
    const auto t0 = std::chrono::steady_clock::now();
    fi_status e0 = fi::cuda_status(cudaFree(0));       // bind the device's primary context to this thread
    if (e0) return e0;
    // golden pass 1 as the control slice when its loads cannot see another launch's
    // stores: a single-launch program, or no load in any kernel's slice (the sliced
    // pass writes no image; pass 2 does, launch by launch)
    bool slice = p->n_inst == 1;
    if (!slice && p->inst_host) {
        slice = true;
        for (uint32_t k = 0; k < p->n_kern && slice; ++k) {
            const fi_insn* c = p->code_host + kern_host[k].code_off;
            const std::vector<uint8_t> sl = control_slice(c, kern_host[k].code_len);
            for (uint32_t i = 0; i < kern_host[k].code_len && slice; ++i) slice = !(sl[i] && c[i].op == fi::LDG);
        }
    }
    const uint32_t gen_modes = modes | ((slice && (modes & FI_JIT_GOLDEN)) ? kJitSliceLen : 0u);
    std::vector<std::vector<char>> cubins;
    size_t src_bytes = 0;
    fi_status e = compile_all(p->code_host, kern_host, p->n_kern, p->n_regs, gen_modes, cubins, src_bytes);
    if (e) return e;
    fi_jit* j = new fi_jit();
    j->smem = jit_smem(p->n_regs);
    j->smem_trace = jit_smem_trace(p->n_regs);
    j->m.resize(p->n_kern);
    bool ok = true;
    size_t cubin_bytes = 0;
    for (uint32_t k = 0; k < p->n_kern && ok; ++k) {
        fi_jit_mod& M = j->m[k];
        cubin_bytes += cubins[k].size();
        ok = D.load(&M.mod, cubins[k].data()) == CUDA_SUCCESS;
        auto get = [&](CUfunction* f, const char* name, size_t smem) {
            ok = ok && D.get(f, M.mod, name) == CUDA_SUCCESS &&
                 D.set_attr(*f, CU_FUNC_ATTRIBUTE_MAX_DYNAMIC_SHARED_SIZE_BYTES, (int)smem) == CUDA_SUCCESS;
        };
        if (modes & FI_JIT_INJECT) get(&M.inject, "k_inject_jit", j->smem);
        if (modes & FI_JIT_GOLDEN) {
            get(&M.glen, "k_golden_len_jit", j->smem);
            get(&M.gtrace, "k_golden_trace_jit", j->smem_trace);
        }
        if (modes & FI_JIT_PAGE) get(&M.k8exec, "k8_exec_jit", j->smem);
    }
    if (!ok) {
        g_jit_log += "\ncuModuleLoadData / cuModuleGetFunction / cuFuncSetAttribute failed";
        for (auto& M : j->m) if (M.mod) D.unload(M.mod);
        delete j;
        return FI_E_CUDA;
    }
    j->modes = modes;
    j->len_sliced = (gen_modes & kJitSliceLen) != 0;
    j->n_regs = p->n_regs;
    j->n_code = p->n_code;
    j->src_bytes = src_bytes;
    j->cubin_bytes = cubin_bytes;
    j->compile_s = std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count();
    *out = j;
    return FI_OK;
}

extern "C" double fi_jit_compile_seconds(const fi_jit* j) { return j ? j->compile_s : 0.0; }
extern "C" int fi_jit_len_sliced(const fi_jit* j) { return j && j->len_sliced ? 1 : 0; }

extern "C" void fi_jit_free(fi_jit* j) {
    if (!j) return;
    for (auto& M : j->m) if (M.mod) drv().unload(M.mod);
    delete j;
}

namespace {
struct JArgsHost {                                   // = JArgs of jit_prelude.cuh
    const uint8_t* img;
    const uint32_t* gran;
    const fi_buffer* buf;
    const fi_instance* inst;
    const uint32_t* cbank;
    const uint4* dec;
    const uint32_t* ins;
    uint64_t image_bytes;
    uint32_t n_inst;
};

JArgsHost jargs(const fi_program* p, const uint8_t* image) {
    const char* aux = reinterpret_cast<const char*>(p->aux);
    return JArgsHost{image,
                     reinterpret_cast<const uint32_t*>(aux),   // granule map at aux offset 0
                     p->buf, p->inst, p->cbank,
                     reinterpret_cast<const uint4*>(aux + fi::aux_dec_offset(p)),
                     reinterpret_cast<const uint32_t*>(aux + fi::aux_ins_offset(p)),
                     p->image_bytes, p->n_inst};
}

fi_status launch(CUfunction f, uint32_t grid, size_t smem, cudaStream_t s, void** args) {
    const CUresult r = drv().launch(f, grid, 1, 1, 128, 1, 1, (unsigned)smem, (CUstream)s, args, nullptr);
    if (r != CUDA_SUCCESS) {
        g_jit_log = "cuLaunchKernel failed: " + std::to_string((int)r);
        return FI_E_CUDA;
    }
    return fi::launch_status();
}
}  // namespace

extern "C" fi_status fi_inject_jit(const fi_jit* j, const fi_program* p, const uint8_t* image, const fi_trace* t,
                                   const fi_site* sites, uint32_t n, fi_inj* out, fi_store* log, uint32_t log_cap,
                                   void* ws, size_t ws_bytes, uint32_t* dev_status, void* stream) {
    if (!j || !p || !image || !t || !sites || !out || !dev_status || (log_cap && !log) || !p->aux) return FI_E_ARG;
    if (!(j->modes & FI_JIT_INJECT) || j->n_regs != p->n_regs || j->n_code != p->n_code) return FI_E_ARG;
    if (t->ckpt && (!t->ckpt_off || !t->ckpt_interval)) return FI_E_ARG;
    if (n == 0) return FI_OK;
    if (!ws || ws_bytes < fi_inject_workspace(n)) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    uint32_t* counter = reinterpret_cast<uint32_t*>(ws);
    uint32_t* order = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + 256);
    const uint32_t ck_iv = t->ckpt ? t->ckpt_interval : 0;
    fi::launch_lpt_order(p, sites, t->warp_off, ck_iv, n, order, counter, s);
    fi_status e = fi::launch_status();
    if (e) return e;
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    JArgsHost A = jargs(p, image);
    const uint64_t* warp_off = t->warp_off;
    const uint32_t* ckpt = t->ckpt;
    const uint64_t* ck_off = t->ckpt_off;
    // the per-SM deal counters (jnext_job): after the order, 256-B aligned
    uint32_t* smq = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + 256 + (((size_t)n * 4 + 255) & ~(size_t)255));
    uint32_t nsm = (uint32_t)std::min(std::max(sms, 1), 256), dealt = 0;
    void* args[] = {&A, (void*)&warp_off, (void*)&sites, &n, &out, &log, &log_cap, (void*)&ckpt, (void*)&ck_off,
                    (void*)&ck_iv, &order, &counter, &dev_status, &smq, &nsm, &dealt};
    // each static kernel's module takes its own replicas off the LPT queue (k_lpt_order
    // reset the queue counter; it is reset again before every later module).  The
    // first `dealt` positions — the longest replicas, one per resident warp — are dealt
    // to the SMs in snake order (every SM gets an equal share of the long ones whatever
    // the hardware's CTA placement), the rest come off the shared queue; the grid is
    // the whole persistent grid, so every SM has warps to take its share.
    for (size_t k = 0; k < j->m.size(); ++k) {
        if (k) {
            e = fi::cuda_status(cudaMemsetAsync(counter, 0, 4, s));
            if (e) return e;
        }
        e = fi::cuda_status(cudaMemsetAsync(smq, 0, (size_t)nsm * 4, s));
        if (e) return e;
        drv().occ(&per, j->m[k].inject, 128, j->smem);
        const uint32_t grid = (uint32_t)std::max(1, sms * std::max(1, per));
        dealt = (uint32_t)std::min<uint64_t>(n, (uint64_t)grid * 4);
        e = launch(j->m[k].inject, grid, j->smem, s, args);
        if (e) return e;
    }
    return FI_OK;
}

namespace fi {
// propagate8.cu's k8 loop: k8_exec of instance t on the JIT module (K = JK8 layout, jit_k8.h)
fi_status jit_k8_exec(const fi_jit* j, const fi_program* p, const uint8_t* image, const JK8Host& K, uint32_t t,
                      uint32_t max_grid, cudaStream_t s) {
    if (!j || !(j->modes & FI_JIT_PAGE) || j->n_regs != p->n_regs || j->n_code != p->n_code) return FI_E_ARG;
    if (!p->inst_host || t >= p->n_inst || p->inst_host[t].kernel >= j->m.size()) return FI_E_ARG;
    CUfunction f = j->m[p->inst_host[t].kernel].k8exec;
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    drv().occ(&per, f, 128, j->smem);
    const uint32_t grid = std::max<uint32_t>(1, std::min<uint32_t>((uint32_t)std::max(1, sms * std::max(1, per)), max_grid));
    JArgsHost A = jargs(p, image);
    JK8Host KK = K;
    uint32_t tt = t;
    void* args[] = {&A, &KK, &tt};
    return launch(f, grid, j->smem, s, args);
}
}  // namespace fi

extern "C" fi_status fi_golden_lengths_jit(const fi_jit* j, const fi_program* p, uint8_t* image, uint64_t* warp_len,
                                           uint64_t* warp_nstore, uint32_t* dev_status, void* stream) {
    if (!j || !p || !image || !warp_len || !warp_nstore || !dev_status || !p->inst_host || !p->aux) return FI_E_ARG;
    if (!(j->modes & FI_JIT_GOLDEN) || j->n_regs != p->n_regs || j->n_code != p->n_code) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    JArgsHost A = jargs(p, image);
    for (uint32_t k = 0; k < p->n_inst; ++k) {
        const uint32_t nw = p->inst_host[k].warp_end - p->inst_host[k].warp_begin;
        if (!nw) continue;
        uint32_t kk = k;
        void* args[] = {&A, &kk, &image, &warp_len, &warp_nstore, &dev_status};
        if (p->inst_host[k].kernel >= j->m.size()) return FI_E_ARG;
        fi_status e = launch(j->m[p->inst_host[k].kernel].glen, (nw + 3) / 4, j->smem, s, args);
        if (e) return e;
    }
    return FI_OK;
}

extern "C" fi_status fi_golden_trace_jit(const fi_jit* j, const fi_program* p, uint8_t* image, const fi_trace* t,
                                         uint32_t* dev_status, void* stream) {
    return fi_golden_trace_jit_range(j, p, image, t, 0, p ? p->n_warps : 0, 0, p ? p->n_warps : 0, nullptr, nullptr,
                                     dev_status, stream);
}

extern "C" fi_status fi_golden_trace_jit_range(const fi_jit* j, const fi_program* p, uint8_t* image, const fi_trace* t,
                                               uint32_t w_lo, uint32_t w_hi, uint32_t own_lo, uint32_t own_hi,
                                               uint64_t* inst_counts, uint32_t* chunk_counts,
                                               uint32_t* dev_status, void* stream) {
    if (!inst_counts != !chunk_counts) return FI_E_ARG;
    if (!j || !p || !image || !t || !t->warp_off || !t->gstore_off || !t->rec || !dev_status || !p->aux) return FI_E_ARG;
    if (!(j->modes & FI_JIT_GOLDEN) || j->n_regs != p->n_regs || j->n_code != p->n_code) return FI_E_ARG;
    if (t->ckpt && (!t->ckpt_off || !t->ckpt_interval)) return FI_E_ARG;
    if (!p->n_warps) return FI_OK;
    if (!p->inst_host) return FI_E_ARG;
    JArgsHost A = jargs(p, image);
    uint32_t iv = t->ckpt ? t->ckpt_interval : 0;
    const uint64_t* woff = t->warp_off;
    const uint64_t* goff = t->gstore_off;
    const uint64_t* ckoff = t->ckpt_off;
    fi_record* rec = t->rec;
    fi_store* gst = t->gstore;
    uint32_t* ck = t->ckpt;
    for (uint32_t k = 0; k < p->n_inst; ++k) {        // one launch per instance, on its kernel's module
        const uint32_t nw = p->inst_host[k].warp_end - p->inst_host[k].warp_begin;
        if (!nw) continue;
        if (p->inst_host[k].kernel >= j->m.size()) return FI_E_ARG;
        uint32_t kk = k;
        if (p->inst_host[k].warp_end <= w_lo || p->inst_host[k].warp_begin >= w_hi) continue;   // no warp of this rank
        void* args[] = {&A, &kk, (void*)&woff, (void*)&goff, &rec, &gst, &ck, (void*)&ckoff, &iv, &dev_status, &image,
                        &w_lo, &w_hi, &own_lo, &own_hi, &chunk_counts, &inst_counts};
        fi_status e = launch(j->m[p->inst_host[k].kernel].gtrace, (nw + 3) / 4, j->smem_trace, (cudaStream_t)stream, args);
        if (e) return e;
    }
    return FI_OK;
}
