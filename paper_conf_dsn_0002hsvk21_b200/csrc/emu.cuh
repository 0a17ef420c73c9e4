// emu.cuh — warp-per-warp mini-SASS emulator, sm_100a.
//
// One CUDA warp emulates one synthetic warp: CUDA lane λ is synthetic lane λ,
// so per-lane state (pc, live, predicates) lives in registers and warp-level
// decisions (min-PC scheduling, active / pred masks) are single REDUX / VOTE
// instructions.  The 32-bit register file is a [n_regs+1][32] u32 array in
// shared memory (row n_regs is all zeros and serves RZ and any index >= n_regs),
// so every register access is one bank-conflict-free LDS/STS.
//
// Hot-loop design:
//  * instructions are pre-decoded once per program (fi_program_prepare) into
//    16 B with register operands already turned into shared-memory byte offsets,
//    plus a per-instruction "run length": how many straight-line instructions
//    (no branch, exit or global memory access) start there;
//  * while every live lane sits at the same pc (no divergence — the common case)
//    the warp executes whole straight-line runs without per-step scheduling,
//    watchdog or control-flow bookkeeping, prefetching the next decoded
//    instruction; only while lanes are split does it use REDUX.MIN + VOTE per step;
//  * FFMA (the dominant opcode of GEMM-like kernels) has its own fast path;
//  * each lane caches its last two buffers' bounds, so most LDG/STG skip the
//    granule-table lookup;
//  * the golden trace pass stores register-file checkpoints: checkpoint c is the
//    warp state before the first step s >= c*interval that follows a BRA or EXIT
//    (or s = 0), its step s stored with it (absent: 0xFFFFFFFF), so no engine
//    has to stop a straight-line block at a multiple of the interval; an
//    injection replica restarts from the last checkpoint whose step is at or
//    before its site instead of re-executing the whole prefix (the prefix is
//    identical to the golden run by construction).
//
// Memory follows DESIGN.md §3.5: loads of instance k read the golden final
// image where the buffer's writer < k and zero where writer >= k (equivalent to
// the state before k under SSA), so neither the golden passes nor injection
// replicas ever snapshot memory.
//
// Modes:
//   EMU_LEN    golden pass 1: stores go to the image; count steps and stored words
//   EMU_TRACE  golden pass 2: trace records (App. A.3), golden store log, checkpoints
//   EMU_INJ    injection replica: corrupt one destination after
//              the site's instruction; log stores after the site; faults end the run
#pragma once
#include "common.cuh"
#include "sem.cuh"

namespace fi {

constexpr uint32_t kFull = 0xFFFFFFFFu;
constexpr int kLdgBatch = 4;          // independent LDGs issued together
enum EmuMode { EMU_LEN = 0, EMU_TRACE = 1, EMU_INJ = 2, EMU_PROP = 3, EMU_PAGE = 4 };

// ---- prepared program data (fi_program.aux) --------------------------------
// per instance: the buffers its constant bank points into (count, then ids;
// count > kInstBufs = "unknown", never skipped by K7)
constexpr uint32_t kInstBufs = 15;

struct AuxLayout { size_t gran, dec, fdec, fbl, ins, run, ib, total; };
constexpr uint32_t kFfmaBatch = 8;                   // independent simple FFMAs emulated together
__host__ __device__ inline size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }
__host__ __device__ inline AuxLayout aux_layout(uint64_t image_bytes, uint32_t n_code, uint32_t n_inst) {
    AuxLayout L;
    L.gran = 0;
    L.dec = align256(((image_bytes + 255) >> 8) * sizeof(uint32_t));
    L.fdec = L.dec + align256((size_t)n_code * 16);
    L.fbl = L.fdec + align256(((size_t)n_code + kFfmaBatch) * 16);   // padded: batches load 8 entries
    L.ins = L.fbl + align256((size_t)n_code);
    L.run = L.ins + align256((size_t)n_code * 4);
    L.ib = L.run + align256((size_t)n_code * 4);
    L.total = L.ib + align256((size_t)n_inst * (kInstBufs + 1) * 4);
    return L;
}

// "plain" = may run inside a straight-line run: no control flow, no global memory
__host__ __device__ inline bool is_plain(uint32_t op) { return op != BRA && op != EXIT && op != LDG && op != STG; }

// decoded instruction (uint4):
//   x = op | guard << 8 | mod << 16 | pb << 24     pb: IADD3 carry pred, *SETP dest pred, LOP3 lut, SEL pred
//   y = ra | rb << 16                               smem byte offsets (row*128), RZ / >= n_regs -> zero row
//   z = rc | rd << 16                               rd = 0xFFFF when the write is discarded
//   w = imm
// simple-FFMA entry (fdec, uint4): x, y, z = byte offsets of the a, b, c operand
// rows, w = destination row offset; fbl (u8) = batch length: the longest run
// (<= kFfmaBatch) of simple FFMAs from here in which no FFMA reads or writes a
// register written by an earlier one (so all reads may go first).
__host__ __device__ inline uint4 decode_insn(const fi_insn& I, uint32_t zr) {
    auto row = [&](uint32_t r) -> uint32_t { return (r < zr ? r : zr) * 128u; };
    uint32_t pb = 0;
    if (I.op == IADD3) pb = I.d1 & 7;
    else if (I.op == ISETP || I.op == FSETP || I.op == DSETP) pb = I.d0 & 7;
    else if (I.op == LOP3) pb = I.ext & 0xFF;
    else if (I.op == SEL) pb = I.c & 0xF;
    uint4 d;
    d.x = (uint32_t)I.op | ((uint32_t)I.guard << 8) | ((uint32_t)I.mod << 16) | (pb << 24);
    d.y = row(I.a) | (row(I.b) << 16);
    d.z = row(I.c) | ((I.d0 < zr ? I.d0 * 128u : 0xFFFFu) << 16);
    d.w = I.imm;
    return d;
}

struct EmuProg {
    const uint4* dec;          // decoded code
    const uint4* fdec;         // simple-FFMA operand offsets
    const uint8_t* fbl;        // simple-FFMA independent batch length
    const uint32_t* ins;       // trace insn word per static instruction: pc | op<<16 | groupmask<<24
    const uint32_t* run;       // straight-line run length starting at each static instruction
    const fi_kernel* kern;
    const fi_instance* inst;
    const uint32_t* cbank;
    const fi_buffer* buf;
    const uint32_t* gran;
    const uint32_t* ib;        // per-instance referenced buffers [n_inst][kInstBufs+1]
    uint64_t image_bytes;
    uint32_t n_regs;
    uint32_t n_inst;
};

inline EmuProg make_emu_prog(const fi_program* p) {
    const AuxLayout L = aux_layout(p->image_bytes, p->n_code, p->n_inst);
    const char* a = reinterpret_cast<const char*>(p->aux);
    return EmuProg{reinterpret_cast<const uint4*>(a + L.dec), reinterpret_cast<const uint4*>(a + L.fdec),
                   reinterpret_cast<const uint8_t*>(a + L.fbl), reinterpret_cast<const uint32_t*>(a + L.ins),
                   reinterpret_cast<const uint32_t*>(a + L.run), p->kern, p->inst, p->cbank, p->buf,
                   reinterpret_cast<const uint32_t*>(a + L.gran), reinterpret_cast<const uint32_t*>(a + L.ib),
                   p->image_bytes, p->n_regs, p->n_inst};
}

// checkpoint = (n_regs + 3) rows of 32 words: registers, then pc, predicates, live
// rows: n_regs registers, pc, predicates, live, step (all lanes hold the step)
__host__ __device__ inline size_t ckpt_bytes(uint32_t n_regs) { return (size_t)(n_regs + 4) * 128; }

struct HookIn {
    uint32_t step, lane, kind, reg, bfm, mask, pc;   // transient site (EMU_INJ)
    // permanent / intermittent fault (EMU_PROP, rows f2/f3): every executed dynamic
    // instance of perm_op in lane perm_lane has its destinations XOR-ed with
    // perm_mask; intermittent: only when Philox(warp, step, rep) < perm_q
    bool perm_on;
    uint32_t perm_op, perm_lane, perm_mask, perm_q, perm_rep, perm_warp;
    uint64_t perm_seed;
};

struct EmuOut {
    uint32_t steps = 0, fault = 0, fault_pc = 0, nstore = 0;
    uint32_t start = 0;                              // EMU_INJ: the step it restarted at (checkpoint)
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

// the §3.2 opcode semantics: ONE copy, shared with the JIT (sem.cuh)
using fisem::u2f;
using fisem::fbits;
using fisem::u2d;
using fisem::dbits;
using fisem::RegFile;
using fisem::LaneCtx;
using fisem::exec_plain;
using fisem::guard_of;

// Image data loads bypass L1 allocation: the small L1 left next to the register
// files must keep the decoded code, granule map and buffer table resident.
__device__ __forceinline__ uint32_t ld_img32(const uint8_t* p) {
    uint32_t r;
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
    return r;
}
__device__ __forceinline__ uint2 ld_img64(const uint8_t* p) {
    uint2 r;
    asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
}
__device__ __forceinline__ uint4 ld_img128(const uint8_t* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// Per-lane two-entry cache of buffer bounds (image offsets) for memory checks.
struct BufCache {
    uint64_t lo0 = 1, hi0 = 0, lo1 = 1, hi1 = 0;   // empty ranges
    bool z0 = false, z1 = false;                   // writer rule: reads of this buffer return 0
};

// 0 ok, 1 misaligned, 2 unmapped (C-15).  On success *zero = writer rule flag for instance k.
__device__ __forceinline__ uint32_t check_access(const EmuProg& P, BufCache& C, uint64_t va, uint32_t w, uint32_t k,
                                                 bool* zero) {
    if (va & (w - 1)) return 1;
    const uint64_t off = va - kVaBase;
    // (off < hi first: an address just below the VA base wraps off + w around)
    if (off >= C.lo0 && off < C.hi0 && off + w <= C.hi0) { *zero = C.z0; return 0; }
    if (off >= C.lo1 && off < C.hi1 && off + w <= C.hi1) { *zero = C.z1; return 0; }
    if (va < kVaBase || off >= P.image_bytes) return 2;
    const uint32_t b = __ldg(&P.gran[off >> 8]);
    if (b == kNoBuf) return 2;
    const uint64_t lo = __ldg(&P.buf[b].off), hi = lo + __ldg(&P.buf[b].size);
    if (off + w > hi) return 2;
    const int32_t wr = __ldg(&P.buf[b].writer);
    C.lo1 = C.lo0; C.hi1 = C.hi0; C.z1 = C.z0;
    C.lo0 = lo; C.hi0 = hi; C.z0 = wr >= 0 && (uint32_t)wr >= k;
    *zero = C.z0;
    return 0;
}

// Register-file access: Rb = this lane's column as a byte pointer, offsets are row*128.

// Faulty-memory overlay of one replica during downstream propagation (K7): an
// open-addressing table of 32-bit words {va_lo, va_hi, value, used}; a word
// present here holds the replica's current value, any other word has its
// golden value (DESIGN.md §3.5 writer rule).
struct Overlay {
    uint4* tab;
    uint32_t mask;                                   // capacity - 1 (power of two)
    uint32_t gen;                                    // this replica's generation tag (slots are reused)
};
__device__ __forceinline__ uint32_t ov_hash(uint64_t va) {
    return (uint32_t)(((va >> 2) * 0x9E3779B97F4A7C15ull) >> 32);
}
// Entries of older generations (earlier replicas of the same slot) count as
// empty: ov_put inserts at the first slot of the probe chain not tagged with the
// current generation, so a live entry is never behind such a slot.
__device__ __forceinline__ bool ov_find(const Overlay& o, uint64_t va, uint32_t& v) {
    uint32_t h = ov_hash(va) & o.mask;
    for (uint32_t probes = 0; probes <= o.mask; ++probes) {
        const uint4 e = __ldcg(&o.tab[h]);
        if (e.w != o.gen) return false;
        if (e.x == (uint32_t)va && e.y == (uint32_t)(va >> 32)) { v = e.z; return true; }
        h = (h + 1) & o.mask;
    }
    return false;
}

// Faulty memory of one replica slot in batched propagation (K8): copy-on-write
// 4 KB pages per buffer (page p of buffer b = page_base[b] + offset/4096);
// ptab[p] = pool page holding the replica's words, or >= kPageClaim when the
// replica's word is the golden state.  A load from a buffer whose pages were
// dropped after its last golden reference (a wild load) marks the slot inexact.
constexpr uint32_t kPageWords = 1024;
constexpr uint32_t kPageNone = 0xFFFFFFFFu, kPageClaim = 0xFFFFFFFEu;
struct PageView {
    const uint32_t* ptab;
    const uint32_t* pool;
    const uint32_t* page_base;
    const uint32_t* last_ref;
    const uint32_t* dropped;     // bit per buffer
    uint32_t* inexact;
    uint32_t t;
};
__device__ __forceinline__ void page_find(const EmuProg& P, const PageView& V, uint64_t va, uint32_t& v) {
    const uint64_t off = va - kVaBase;
    const uint32_t b = __ldg(&P.gran[off >> 8]);
    const uint64_t rel = off - __ldg(&P.buf[b].off);
    const uint32_t e = V.ptab[__ldg(&V.page_base[b]) + (uint32_t)(rel >> 12)];
    if (e < kPageClaim) v = __ldcg(&V.pool[(size_t)e * kPageWords + ((rel >> 2) & (kPageWords - 1))]);
    else if (__ldg(&V.last_ref[b]) < V.t && ((V.dropped[b >> 5] >> (b & 31)) & 1u)) *V.inexact = 1u;
}

template <int MODE>
__device__ __forceinline__ EmuOut emulate(const EmuProg P, uint8_t* img_w, const uint8_t* img,
                                          uint32_t k, uint32_t cta, uint32_t wic, uint32_t* __restrict__ R,
                                          uint32_t watchdog, fi_record* __restrict__ rec_out,
                                          fi_store* __restrict__ st_out, uint32_t st_cap, HookIn hook,
                                          uint32_t* __restrict__ ck, uint32_t ck_interval,
                                          Overlay ov = Overlay{nullptr, 0}, PageView pg = PageView{}) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t lt_mask = (1u << lane) - 1u;
    const fi_instance in = P.inst[k];
    const fi_kernel kn = P.kern[in.kernel];
    const uint4* __restrict__ dec = P.dec + kn.code_off;
    const uint32_t* __restrict__ ins = P.ins + kn.code_off;
    const uint32_t* __restrict__ runl = P.run + kn.code_off;
    const uint32_t zr = P.n_regs;
    const uint32_t ckw = (zr + 4) * 32;              // words per checkpoint
    const RegFile F{reinterpret_cast<char*>(R + lane), R, zr * 128};
    const LaneCtx LC{lane, cta, wic, in.block, in.grid, in.cbank_len, P.cbank + in.cbank_off};
    const bool use_ck = ck != nullptr && ck_interval != 0;
    // permanent / intermittent hook (row f2/f3): every step is inspected, so the
    // straight-line fast paths are off while it is armed
    const bool perm = (MODE == EMU_PROP || MODE == EMU_PAGE) && hook.perm_on;

    uint32_t nl = in.block - wic * 32;
    bool live = lane < (nl > 32 ? 32u : nl);
    uint32_t pc = 0, preds = 0, step = 0;
    EmuOut o;
    if (MODE == EMU_INJ && use_ck) {
        // restart from the last golden checkpoint at or before the site
        uint32_t c = hook.step / ck_interval;
        while (c > 0 && __ldg(&ck[(size_t)c * ckw + (zr + 3) * 32]) > hook.step) --c;
        const uint32_t* src = ck + (size_t)c * ckw;
        for (uint32_t r = 0; r < zr; ++r) R[r * 32 + lane] = __ldg(&src[r * 32 + lane]);
        R[zr * 32 + lane] = 0u;
        pc = __ldg(&src[zr * 32 + lane]);
        preds = __ldg(&src[zr * 32 + 32 + lane]);
        live = __ldg(&src[zr * 32 + 64 + lane]) != 0u;
        step = __ldg(&src[(zr + 3) * 32 + lane]);
        o.start = step;
    } else {
        for (uint32_t r = 0; r <= zr; ++r) R[r * 32 + lane] = 0u;
    }
    uint32_t livem = __ballot_sync(kFull, live);
    // Group mode (`conv`): the lanes of `amask` share pc `upc` and every other live
    // lane is parked at a pc >= npc > upc, so by the min-pc rule (§3.3) the group
    // keeps running alone, with no per-step scheduling, until it branches
    // divergently, exits, or reaches npc (where parked lanes rejoin).
    bool conv = false;
    uint32_t upc = 0, amask = 0, npc = 0xFFFFFFFFu;
    uint32_t nst = 0;
    bool brk = true;                                 // the last step was a BRA / EXIT (or none yet)
    uint32_t ckn = 0;                                // EMU_TRACE: next checkpoint to write
    uint4 recbuf = make_uint4(0, 0, 0, 0);
    BufCache bc;
    __syncwarp();

    for (;;) {
        if (!livem) break;
        uint32_t pcm, active;
        if (conv) {
            pcm = upc;
            active = amask;
        } else {
            pcm = __reduce_min_sync(kFull, live ? pc : 0xFFFFFFFFu);
            active = __ballot_sync(kFull, live && pc == pcm);
            npc = active == livem ? 0xFFFFFFFFu : __reduce_min_sync(kFull, (live && pc != pcm) ? pc : 0xFFFFFFFFu);
            conv = true; upc = pcm; amask = active;
        }
        const bool inA = (amask >> lane) & 1u;
        if (MODE == EMU_TRACE && use_ck && brk && step >= ckn * ck_interval) {
            // checkpoints ckn .. step/interval: this state (one per multiple passed)
            for (; ckn <= step / ck_interval; ++ckn) {
                uint32_t* dst = ck + (size_t)ckn * ckw;
                for (uint32_t r = 0; r < zr; ++r) dst[r * 32 + lane] = R[r * 32 + lane];
                dst[zr * 32 + lane] = live ? (inA ? upc : pc) : 0u;
                dst[zr * 32 + 32 + lane] = preds;
                dst[zr * 32 + 64 + lane] = live ? 1u : 0u;
                dst[(zr + 3) * 32 + lane] = step;
            }
        }
        brk = false;
        if (step >= watchdog) { o.fault = 3; o.fault_pc = pcm; break; }
        if (pcm >= kn.code_len) { o.fault = 4; o.fault_pc = pcm; break; }

        if (conv && !perm) {
            // ---- straight-line run: no scheduling / control bookkeeping per step
            const uint32_t rw = __ldg(&runl[pcm]);
            uint32_t run = rw & 0xFFFF, lr = (rw >> 16) & 0xFF, fr = rw >> 24;
            uint32_t lim = min(watchdog - step, npc - pcm);   // stop where parked lanes rejoin
            if (MODE == EMU_INJ && hook.step >= step) lim = min(lim, hook.step - step);
            run = min(run, lim);
            lr = min(min(lr, lim), (uint32_t)kLdgBatch);
            fr = min(fr, lim);
            if (fr) {
                // ---- simple-FFMA run (unguarded, unmodified FFMAs), emulated in
                //      batches of independent FFMAs: all operand reads, then the FMAs,
                //      then the writes.  No NaN canonicalisation is needed here: sm_100
                //      FFMA returns 0x7FFFFFFF for every NaN result (C-13 holds as is;
                //      pinned by the special-value parity tests).
                const uint4* fq = P.fdec + kn.code_off + pcm;
                const uint8_t* fl = P.fbl + kn.code_off + pcm;
                uint32_t sb = step;
                for (uint32_t left = fr; left;) {
                    const uint32_t nb = min((uint32_t)__ldg(fl), left);
                    uint4 e[kFfmaBatch];
#pragma unroll
                    for (uint32_t b = 0; b < kFfmaBatch; ++b) e[b] = __ldg(fq + b);
                    float x[kFfmaBatch], y[kFfmaBatch], z[kFfmaBatch];
                    if (nb == kFfmaBatch) {                   // full batch: no per-FFMA predication
#pragma unroll
                        for (uint32_t b = 0; b < kFfmaBatch; ++b) {
                            x[b] = u2f(F.rd(e[b].x));
                            y[b] = u2f(F.rd(e[b].y));
                            z[b] = u2f(F.rd(e[b].z));
                        }
                        if (inA) {
#pragma unroll
                            for (uint32_t b = 0; b < kFfmaBatch; ++b)
                                *reinterpret_cast<float*>(F.Rb + e[b].w) = __fmaf_rn(x[b], y[b], z[b]);
                        }
                    } else {
#pragma unroll
                        for (uint32_t b = 0; b < kFfmaBatch; ++b) {
                            if (b < nb) {
                                x[b] = u2f(F.rd(e[b].x));
                                y[b] = u2f(F.rd(e[b].y));
                                z[b] = u2f(F.rd(e[b].z));
                            }
                        }
#pragma unroll
                        for (uint32_t b = 0; b < kFfmaBatch; ++b) {
                            if (b < nb && inA)
                                *reinterpret_cast<float*>(F.Rb + e[b].w) = __fmaf_rn(x[b], y[b], z[b]);
                        }
                    }
                    if (MODE == EMU_TRACE) {
                        for (uint32_t b = 0; b < nb; ++b) {
                            const uint32_t s = sb + b;
                            if ((s & 31) == lane) recbuf = make_uint4(k, __ldg(&ins[pcm + (s - step)]), amask, kFull);
                            if ((s & 31) == 31) __stcs(&reinterpret_cast<uint4*>(rec_out)[s - 31 + lane], recbuf);
                        }
                    }
                    fq += nb;
                    fl += nb;
                    sb += nb;
                    left -= nb;
                }
                step += fr;
                upc = pcm + fr;
                if (upc >= npc) { conv = false; if (inA) pc = upc; }
                continue;
            }
            if (lr >= 2) {
                // ---- LDG batch: independent loads in flight together
                uint4 vals[kLdgBatch];
                uint32_t dsts[kLdgBatch], lws[kLdgBatch], preds_b[kLdgBatch];
                bool exs[kLdgBatch];
                int first_bad = -1;
                uint32_t bad_kind = 0;
#pragma unroll
                for (int b = 0; b < kLdgBatch; ++b) {
                    exs[b] = false;
                    vals[b] = make_uint4(0, 0, 0, 0);
                    if ((uint32_t)b < lr) {
                        const uint4 D = __ldg(&dec[pcm + b]);
                        const uint32_t guard = (D.x >> 8) & 0xFF, mod = (D.x >> 16) & 0xFF;
                        const bool pv = guard == 7 ? true : guard_of(guard, preds);
                        preds_b[b] = guard == 7 ? kFull : __ballot_sync(kFull, pv);
                        const bool ex = inA && pv;
                        const uint32_t lw = (mod & 3) > 2 ? 2 : (mod & 3);
                        const uint64_t va = F.rd64(D.y & 0xFFFF) + (uint64_t)(int64_t)(int32_t)D.w;
                        bool zero = false;
                        const uint32_t c = ex ? check_access(P, bc, va, 4u << lw, k, &zero) : 0u;
                        const uint32_t bm = __ballot_sync(kFull, c != 0);
                        if (bm && first_bad < 0) {
                            first_bad = b;
                            bad_kind = __ballot_sync(kFull, c == 1) ? 1 : 2;
                        }
                        const uint8_t* src = img + (va - kVaBase);
                        if (ex && !c && !zero) {
                            if (lw == 0) vals[b].x = ld_img32(src);
                            else if (lw == 1) { const uint2 t = ld_img64(src); vals[b].x = t.x; vals[b].y = t.y; }
                            else vals[b] = ld_img128(src);
                        }
                        if (MODE == EMU_PROP && ex && !c) {  // the replica's overlay wins
                            uint32_t* vw = &vals[b].x;
                            for (uint32_t q = 0; q < (1u << lw); ++q) ov_find(ov, va + 4 * q, vw[q]);
                        }
                        if (MODE == EMU_PAGE && ex && !c) {  // the replica's pages win
                            uint32_t* vw = &vals[b].x;
                            for (uint32_t q = 0; q < (1u << lw); ++q) page_find(P, pg, va + 4 * q, vw[q]);
                        }
                        exs[b] = ex;
                        dsts[b] = D.z >> 16;
                        lws[b] = lw;
                    }
                }
                if (first_bad >= 0) {                 // the first faulting load in program order (C-9)
                    o.fault = bad_kind;
                    o.fault_pc = pcm + first_bad;
                    step += first_bad;
                    break;
                }
#pragma unroll
                for (int b = 0; b < kLdgBatch; ++b) {
                    if ((uint32_t)b < lr) {
                        if (exs[b]) {
                            F.wr(dsts[b], vals[b].x);
                            if (lws[b] >= 1) F.wr(dsts[b] + 128, vals[b].y);
                            if (lws[b] >= 2) { F.wr(dsts[b] + 256, vals[b].z); F.wr(dsts[b] + 384, vals[b].w); }
                        }
                        if (MODE == EMU_TRACE) {
                            const uint32_t s = step + b;
                            if ((s & 31) == lane) recbuf = make_uint4(k, __ldg(&ins[pcm + b]), amask, preds_b[b]);
                            if ((s & 31) == 31) __stcs(&reinterpret_cast<uint4*>(rec_out)[s - 31 + lane], recbuf);
                        }
                    }
                }
                step += lr;
                upc = pcm + lr;
                if (upc >= npc) { conv = false; if (inA) pc = upc; }
                continue;
            }
            if (run) {
                uint4 Dn = __ldg(&dec[pcm]);
                for (uint32_t j = 0; j < run; ++j) {
                    const uint4 D = Dn;
                    Dn = __ldg(&dec[pcm + min(j + 1, run - 1)]);
                    const uint32_t guard = (D.x >> 8) & 0xFF;
                    bool pv = true;
                    uint32_t pred = kFull;
                    if (guard != 7) {
                        pv = guard_of(guard, preds);
                        pred = __ballot_sync(kFull, pv);
                    }
                    if (MODE == EMU_TRACE) {
                        const uint32_t s = step + j;
                        if ((s & 31) == lane) recbuf = make_uint4(k, __ldg(&ins[pcm + j]), amask, pred);
                        if ((s & 31) == 31) __stcs(&reinterpret_cast<uint4*>(rec_out)[s - 31 + lane], recbuf);
                    }
                    exec_plain(F, LC, D, inA && pv, preds);
                }
                step += run;
                upc = pcm + run;
                if (upc >= npc) { conv = false; if (inA) pc = upc; }
                continue;
            }
        }

        // ---- one general step (branch, exit, memory, divergent lanes, the site)
        const uint4 D = __ldg(&dec[pcm]);
        const uint32_t op = D.x & 0xFF, guard = (D.x >> 8) & 0xFF, mod = (D.x >> 16) & 0xFF;
        const uint32_t ia = D.y & 0xFFFF, ib = D.y >> 16, id = D.z >> 16;
        const uint32_t imm = D.w;
        const bool act = (active >> lane) & 1u;
        const bool pv = guard == 7 ? true : guard_of(guard, preds);
        const uint32_t pred = guard == 7 ? kFull : __ballot_sync(kFull, pv);
        const bool ex = act && pv;
        const uint32_t exm = active & pred;

        if (MODE == EMU_TRACE) {
            if ((step & 31) == lane) recbuf = make_uint4(k, __ldg(&ins[pcm]), active, pred);
            if ((step & 31) == 31) __stcs(&reinterpret_cast<uint4*>(rec_out)[step - 31 + lane], recbuf);
        }

        uint32_t taken = 0;                           // lanes that branch
        brk = op == EXIT || op == BRA;
        if (op == EXIT) {
            if (ex) live = false;
            livem &= ~exm;
            amask &= ~exm;
        } else if (op == BRA) {
            taken = exm;
        } else if (op == LDG || op == STG) {
            const uint32_t lw = (mod & 3) > 2 ? 2 : (mod & 3), nw = 1u << lw, w = 4u << lw;
            const uint64_t va = F.rd64(ia) + (uint64_t)(int64_t)(int32_t)imm;
            bool zero = false;
            const uint32_t code_ = ex ? check_access(P, bc, va, w, k, &zero) : 0u;
            const uint32_t bad = __ballot_sync(kFull, code_ != 0);
            if (bad) {                                // memory fault: DUE (C-9); the step has no effect
                o.fault = __ballot_sync(kFull, code_ == 1) ? 1 : 2;
                o.fault_pc = pcm;
                break;
            }
            if (op == LDG) {
                if (ex) {
                    const uint8_t* src = img + (va - kVaBase);
                    uint4 v = make_uint4(0, 0, 0, 0);
                    if (!zero) {
                        if (lw == 0) v.x = ld_img32(src);
                        else if (lw == 1) { const uint2 t = ld_img64(src); v.x = t.x; v.y = t.y; }
                        else v = ld_img128(src);
                    }
                    if (MODE == EMU_PROP) {                   // the replica's overlay wins
                        uint32_t* vw = &v.x;
                        for (uint32_t q = 0; q < nw; ++q) ov_find(ov, va + 4 * q, vw[q]);
                    }
                    if (MODE == EMU_PAGE) {                   // the replica's pages win
                        uint32_t* vw = &v.x;
                        for (uint32_t q = 0; q < nw; ++q) page_find(P, pg, va + 4 * q, vw[q]);
                    }
                    F.wr(id, v.x);
                    if (lw >= 1) F.wr(id + 128, v.y);
                    if (lw >= 2) { F.wr(id + 256, v.z); F.wr(id + 384, v.w); }
                }
            } else {
                uint32_t v[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) v[i] = (uint32_t)i < nw ? F.rd(min(ib + 128u * i, F.zb)) : 0u;
                const uint32_t idx = __popc(exm & lt_mask) * nw;
                const uint32_t tot = __popc(exm) * nw;
                if (MODE == EMU_LEN) {
                    if (ex) {
                        uint8_t* dst = img_w + (va - kVaBase);
                        if (lw == 0) *reinterpret_cast<uint32_t*>(dst) = v[0];
                        else if (lw == 1) *reinterpret_cast<uint2*>(dst) = make_uint2(v[0], v[1]);
                        else *reinterpret_cast<uint4*>(dst) = make_uint4(v[0], v[1], v[2], v[3]);
                    }
                } else if (MODE == EMU_TRACE || MODE == EMU_PROP || MODE == EMU_PAGE || step > hook.step) {
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
            }
        } else {
            exec_plain(F, LC, D, ex, preds);
        }

        // control flow: advance / branch, tracking convergence
        if (taken == 0) upc = pcm + 1;              // (always in group mode here: active = amask)
        else if (taken == active) upc = imm;
        else {
            conv = false;
            if (act) pc = ((taken >> lane) & 1u) ? imm : pcm + 1;
        }
        if (conv && (amask == 0 || upc >= npc)) {     // group exited / reached parked lanes
            conv = false;
            if ((amask >> lane) & 1u) pc = upc;
        }

        if (perm && op == hook.perm_op && lane == hook.perm_lane && ex) {
            // permanent fault: same XOR mask on the destination
            // registers of every dynamic instance; intermittent: a
            // random subset of them (reading C-21 / C-22)
            bool fire = true;
            if (hook.perm_q) {
                const uint4 r = philox4x32_10(make_uint4(hook.perm_warp, step, hook.perm_rep, 0x46490002u),
                                              make_uint2((uint32_t)hook.perm_seed, (uint32_t)(hook.perm_seed >> 32)));
                fire = r.x < hook.perm_q;
            }
            if (fire) {
                const Dests dd = dests_of(op, id == 0xFFFFu ? kRZ : id / 128, D.x >> 24, mod);
                for (uint32_t q = 0; q < dd.n_gp; ++q) F.wr(id + 128 * q, F.rd(id + 128 * q) ^ hook.perm_mask);
                if (dd.has_pr && (hook.perm_mask & 1u)) preds ^= 1u << dd.pr;
            }
        }
        if (MODE == EMU_INJ && step == hook.step) {
            // transient fault: corrupt one destination of this dynamic
            // instruction in one lane, after the instruction wrote it (C-7, C-8)
            o.fired = true;
            if (pcm != hook.pc || !((exm >> hook.lane) & 1u)) o.bad = true;
            if (lane == hook.lane) {
                if (hook.kind == 0) {
                    const uint32_t ri = min(hook.reg, zr) * 128;
                    const uint32_t before = F.rd(ri);
                    const uint32_t m = hook.bfm == FI_ZERO_VALUE ? before : hook.mask;
                    o.before = before; o.mask = m; o.after = before ^ m;
                    F.wr(ri, o.after);
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
    if (MODE == EMU_TRACE) {
        const uint32_t rem = step & 31;
        if (rem && lane < rem) __stcs(&reinterpret_cast<uint4*>(rec_out)[step - rem + lane], recbuf);
        if (use_ck)                                   // checkpoints the warp never reached: absent (zero rows, step ~0)
            for (; ckn < (step + ck_interval - 1) / ck_interval; ++ckn) {
                for (uint32_t r = 0; r < zr + 3; ++r) ck[(size_t)ckn * ckw + r * 32 + lane] = 0u;
                ck[(size_t)ckn * ckw + (zr + 3) * 32 + lane] = ~0u;
            }
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
