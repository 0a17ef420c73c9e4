// jit_prelude.cuh — device helpers of the JIT-specialised emulator (jit.cpp).
//
// This header is embedded as text into libfi.so and prepended to the CUDA
// source jit.cpp generates per program, which NVRTC compiles for sm_100a.  It is
// self-contained (NVRTC sees no system headers).  The semantics are DESIGN.md
// §3 — the same as emu.cuh's interpreter, which the generated code must match
// bit for bit (both are checked against the CPU oracle by the parity tests).
typedef unsigned char u8;
typedef unsigned int u32;
typedef int i32;
typedef unsigned long long u64;
typedef long long i64;

#define JFULL 0xFFFFFFFFu
#define JQNAN32 0x7FFFFFFFu
#define JQNAN64 0x7FFFFFFFFFFFFFFFull
#define JVA_BASE 0x00007F0000000000ull
#define JNOBUF 0xFFFFFFFFu

// layouts identical to include/fi.h
struct jfi_instance { u32 kernel, kernel_count, grid, block, cbank_off, cbank_len, warp_begin, warp_end; };
struct jfi_buffer { u64 off, size; i32 writer; u32 flags; };
struct jfi_store { u64 va; u32 value, step; };
struct jfi_site {
    u64 s, instruction_count;
    u32 instance, kernel_id, kernel_count, warp, step, thread;
    u32 pc, u_dst, u_bit, mask;
    u8 lane, group, bfm, slot, dst_kind, dst_reg, n_elig, flags;
};
struct jfi_inj {
    u32 before, after, mask, fault_pc;
    u8 fault_kind, outcome, overflow, flags;
    u32 n_faulty_stores;
};

struct JArgs {
    const u8* img;               // golden final image
    const u32* gran;             // buffer id per 256-B granule
    const jfi_buffer* buf;
    const jfi_instance* inst;
    const u32* cbank;
    const uint4* dec;            // pre-decoded code (fi_program_prepare), for step mode
    const u32* ins;              // trace insn word per static instruction (pc | op << 16 | groups << 24)
    u64 image_bytes;
    u32 n_inst;
};

struct JOut {
    u32 steps, fault, fault_pc, nstore, before, after, mask;
    u32 start;                                       // K4: the step it restarted at (its checkpoint's)
    bool fired, bad;
};
// a generated kern_*'s arguments, per warp in shared memory after the 4 warps'
// step-mode register files (jit.cpp kCtxNames, jit_smem)
struct JPage;
// golden pass 2's fused profile: K1's counts (profile.cu) taken
// while the records are written.  Lane g < 8 keeps group g: pch_ = the chunk of the
// warp's NEXT record, pcnt_ = its count so far; a finished chunk's count is added
// to chunk_counts (atomics: a chunk can span two warps) and to the warp's total,
// which goes to inst_counts at the end
struct JProf {
    u32* cc;                                         // chunk_counts [C][8], zeroed by the caller; 0 = off
    u64 rb;                                          // the warp's first global record
    u32 pch_[8], pcnt_[8], tcnt_[8];                 // per group: chunk, its count, one template pass's count
    u64 ptot_[8];                                    // per group: the warp's finished chunks' total
    u32 tmask_[4][8];                                // [word][group]: template record 32*word + bit has the group
};
struct JCtx {
    u32 hstep, hpc, hlane, hkind, hreg, hbfm, hmask, k, cta, wic, watchdog, ck_interval, st_cap;
    u32* ck; jfi_store* st_out; JOut* out; u32* Rs; const uint4* dec; const u32* ins; u8* img_w; uint4* rec_out;
    const JPage* pgp;
    // per lane: warp state block code rarely touches (jit.cpp kCtxLaneNames)
    u32 nst_[32], fault_[32], fault_pc_[32], before_[32], after_[32], msk_[32], fired_[32], bad_[32];
    // the lane's buffer cache (JBufCache) carried from one job of this CUDA warp to
    // the next inside a launch: valid while the instance is bck (the writer rule of
    // an entry depends on the instance); set invalid by every entry kernel
    u32 bck;
    u32 bckp;                                        // PAGE mode: ... and the slot (its page table's low word)
    u32 bc_[16][32];                                 // [slot * 4 + {lo, sz, b, pb}][lane]
    u32 bcz_[32];                                    // bit slot: the entry's writer-rule flag
    JProf prof;                                      // golden pass 2 only
};
#define JCTX_BYTES 3712u
// golden trace pass: bulk (TMA) stores of a warp's record template from shared
// memory (jit.cpp flush_recs), evict-first in L2 like the per-lane __stcs records;
// one elected lane issues them; every lane waits for its own groups before the
// template is rewritten and before the warp's job ends
#define JFW_ 0
// golden pass 2's fused profile: is it on, and the warp's first global record
// (jit.cpp flush_recs; the template loop reads both once)
#define JPCC_ (jx->prof.cc != nullptr)
#define JPRB_ ((u32)jx->prof.rb)
// the template pass's count update, and the flush of a count kept in a register
// (the full-warp template loop keeps it there; elsewhere it goes straight to smem)
#define JPADD_ { if (lane < 8u) jx->prof.pcnt_[lane] += jx->prof.tcnt_[lane]; }
#define JPFLUSH_ {}
#define JPOL_ jpolicy_ef()
__device__ __forceinline__ bool jelect() {
    u32 p;
    asm volatile("{\n\t.reg .pred e;\n\telect.sync _|e, 0xFFFFFFFF;\n\tselp.u32 %0, 1, 0, e;\n\t}" : "=r"(p));
    return p != 0u;
}
__device__ __forceinline__ u64 jpolicy_ef() {
    u64 pol;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
    return pol;
}
__device__ __forceinline__ void jbulk_st_p(uint4* g, const uint4* s, u32 bytes, u64 pol) {
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;\n\t"
                 "cp.async.bulk.commit_group;" :: "l"(g), "r"((u32)__cvta_generic_to_shared(s)), "r"(bytes), "l"(pol)
                 : "memory");
}
__device__ __forceinline__ void jbulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void jbulk_wait() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }
__device__ __forceinline__ void jfence_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// ---- the fused profile (JProf): per record, popc(active & pred) thread-level
// instructions to every group of its trace-insn word's group byte (K1's rule)
__device__ __forceinline__ void jprof_next(JProf* P, u32 g) {         // lane g < 8: its chunk is complete
    const u32 v = P->pcnt_[g];
    if (v) atomicAdd(&P->cc[(u64)P->pch_[g] * 8u + g], v);
    P->ptot_[g] += v;
    P->pcnt_[g] = 0u;
    P->pch_[g] += 1u;
}
// up to 32 consecutive records from global record rb0 (the warp's next): lane j's
// is rb0 + j, valid for a prefix of the lanes, cnt threads, group byte gm
__device__ __noinline__ void jprof_round(JProf* P, u32 lane, u64 rb0, bool v, u32 cnt, u32 gm) {
    const u32 b = 1024u - (u32)(rb0 & 1023u);                         // lanes >= b: the next chunk
    const u32 nv = __popc(__ballot_sync(JFULL, v));
    u32 lo = 0u, hi = 0u;
#pragma unroll
    for (u32 g = 0; g < 8u; ++g) {
        const u32 x = (v && ((gm >> g) & 1u)) ? cnt : 0u;
        const u32 s0 = __reduce_add_sync(JFULL, lane < b ? x : 0u);
        const u32 s1 = b < 32u ? __reduce_add_sync(JFULL, lane < b ? 0u : x) : 0u;
        if (lane == g) { lo = s0; hi = s1; }
    }
    if (lane < 8u) {
        P->pcnt_[lane] += lo;
        if (nv >= b) { jprof_next(P, lane); P->pcnt_[lane] = hi; }
    }
}
// the record template's per-group count and membership masks (full warp, every
// guard true: 32 threads per record)
__device__ __forceinline__ void jprof_tcnt(JProf* P, u32 lane, u32 n, const uint4* tm) {
    u32 t = 0u;
    for (u32 j = 0; j < 128u; j += 32u) {
        const u32 i = j + lane;
        const u32 gm = i < n ? tm[i].y >> 24 : 0u;
#pragma unroll
        for (u32 g = 0; g < 8u; ++g) {
            const u32 m = __ballot_sync(JFULL, (gm >> g) & 1u);
            if (lane == g) { t += 32u * __popc(m); P->tmask_[j >> 5][g] = m; }
        }
    }
    if (lane < 8u) P->tcnt_[lane] = t;
}
// a template pass whose first o records end the current chunk
__device__ __noinline__ void jprof_tmpl_cross(JProf* P, u32 lane, u32 o) {
    if (lane < 8u) {
        u32 pre = 0u;
#pragma unroll
        for (u32 w = 0; w < 4u; ++w) {
            const u32 lo = w * 32u;
            const u32 m = o >= lo + 32u ? 0xFFFFFFFFu : (o > lo ? (1u << (o - lo)) - 1u : 0u);
            pre += __popc(P->tmask_[w][lane] & m);
        }
        pre *= 32u;
        P->pcnt_[lane] += pre;
        jprof_next(P, lane);
        P->pcnt_[lane] = P->tcnt_[lane] - pre;
    }
}
// a step-mode record (the same for every lane): record index r
__device__ __forceinline__ void jprof_one(JProf* P, u32 lane, u64 r, u32 cnt, u32 gm) {
    if (lane < 8u) {
        if ((gm >> lane) & 1u) P->pcnt_[lane] += cnt;
        if ((r & 1023u) == 1023u) jprof_next(P, lane);
    }
}
static_assert(sizeof(JCtx) <= JCTX_BYTES, "JCtx fits its smem slot");

// The §3.2 opcode semantics come from sem.cuh (embedded ahead of this file): ONE
// copy shared with the interpreter (emu.cuh).  The generated code spells them:
__device__ __forceinline__ float ju2f(u32 x) { return fisem::u2f(x); }
__device__ __forceinline__ u32 jfbits(float f) { return fisem::fbits(f); }
__device__ __forceinline__ double ju2d(u64 x) { return fisem::u2d(x); }
__device__ __forceinline__ u64 jdbits(double d) { return fisem::dbits(d); }
__device__ __forceinline__ u64 jpair(u32 lo, u32 hi) { return fisem::pair(lo, hi); }
__device__ __forceinline__ u32 jfmnmx(u32 a, u32 b, bool mx) { return fisem::fmnmx(a, b, mx); }
__device__ __forceinline__ bool jcmp_f(double x, double y, u32 c) { return fisem::cmp_f(x, y, c); }
__device__ __forceinline__ bool jcmp_s(i32 x, i32 y, u32 c) { return fisem::cmp_s(x, y, c); }
__device__ __forceinline__ bool jcmp_u(u32 x, u32 y, u32 c) { return fisem::cmp_u(x, y, c); }
__device__ __forceinline__ u32 jf2i(u32 a) { return fisem::f2i(a); }
template <u32 LUT>
__device__ __forceinline__ u32 jlop3(u32 a, u32 b, u32 c) { return fisem::lop3(a, b, c, LUT); }
__device__ __forceinline__ u32 jshf(u32 a, u32 bv, u32 m) { return fisem::shf(a, bv, m); }
__device__ __forceinline__ u32 jshfl_src(u32 lane, u32 bv, u32 m) { return fisem::shfl_src(lane, bv, m); }

// image loads: read-only path, allocating in L1 (a CTA's warps share lines in the
// golden passes; the loop prefetch puts the next iteration's lines there) — 3-5 %
// faster than .L1::no_allocate for K4 and golden pass 2 on C2
__device__ __forceinline__ u32 jld32(const u8* p) {
    u32 r;
    asm volatile("ld.global.nc.u32 %0, [%1];" : "=r"(r) : "l"(p));
    return r;
}
__device__ __forceinline__ uint2 jld64(const u8* p) {
    uint2 r;
    asm volatile("ld.global.nc.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
}
__device__ __forceinline__ uint4 jld128(const u8* p) {
    uint4 r;
    asm volatile("ld.global.nc.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// K4's job queue (the whole warp calls it, the same result in every lane): LPT
// positions [0, dealt) are dealt to the SMs in snake order — round r of SM s is
// position r*nsm + (r odd ? nsm-1-s : s) — and taken by that SM's warps through its
// own counter; then [dealt, n) off the shared counter; then the warp steals the
// rounds left in the other SMs' deals (an SM the hardware gave no warps), the lanes
// looking at 32 SMs' counters at a time.  Every position is handed out exactly once:
// each (SM, round) by one atomicAdd result.  Returns a position >= n when nothing is
// left.
__device__ __forceinline__ u32 jsmid() { u32 r; asm volatile("mov.u32 %0, %%smid;" : "=r"(r)); return r; }
__device__ __forceinline__ u32 jdeal_pos(u32 r, u32 s, u32 nsm) { return r * nsm + ((r & 1u) ? nsm - 1u - s : s); }
__device__ __noinline__ u32 jnext_job(u32* counter, u32* smq, u32 sm, u32 nsm, u32 dealt, u32 n, u32 lane) {
    u32 p = n;
    if (lane == 0u) {
        if (sm < nsm) {
            const u32 q = jdeal_pos(atomicAdd(&smq[sm], 1u), sm, nsm);
            if (q < dealt) p = q;
        }
        if (p >= n) {
            const u32 g = dealt + atomicAdd(counter, 1u);
            if (g < n) p = g;
        }
    }
    p = __shfl_sync(0xFFFFFFFFu, p, 0);
    if (p < n) return p;
    for (u32 s0 = 0; s0 < nsm; s0 += 32u) {
        const u32 s = s0 + lane;
        u32 m = __ballot_sync(0xFFFFFFFFu, s < nsm && jdeal_pos(*(volatile u32*)&smq[s], s, nsm) < dealt);
        while (m) {
            const u32 t = s0 + (u32)__ffs(m) - 1u;
            m &= m - 1u;
            u32 q = dealt;
            if (lane == 0u) q = jdeal_pos(atomicAdd(&smq[t], 1u), t, nsm);
            q = __shfl_sync(0xFFFFFFFFu, q, 0);
            if (q < dealt) return q;
        }
    }
    return n;
}

// per-lane cache of buffer bounds, JBC_SLOTS entries, 32-bit: image offset `lo`
// and the size floored to 16 B (`sz`; 0 = empty entry).  The generator gives each
// memory instruction a fixed entry (slot) by its address register, so a loop that
// walks several buffers through different pointers keeps one entry per pointer;
// the step-mode interpreter uses entry 0 of its own cache.  Only buffers with
// lo % 16 == 0 and lo + size <= 2^31 are cached (others always take jcheck's
// full path), so for an aligned address va = JVA_BASE + off: off is in the entry
// iff hi32(va) == hi32(JVA_BASE) and (u32)(lo32(va) - lo) < sz — an offset below
// lo wraps to >= 2^31 > sz, and d < sz with d, sz multiples of the access width w
// gives d + w <= sz <= size.  A miss is never wrong, only slower.
static_assert((JVA_BASE & 0xFFFFFFFFull) == 0, "the cache tests the low word of va only");
#define JVA_HI ((u32)(JVA_BASE >> 32))
#define JBC_SLOTS 4
struct JBufCache {
    u32 lo[JBC_SLOTS], sz[JBC_SLOTS];
    bool z[JBC_SLOTS];
    u32 b[JBC_SLOTS], pb[JBC_SLOTS];   // buffer ids and their first page index (K8 page tables; 0 elsewhere)
    __device__ __forceinline__ JBufCache() {
#pragma unroll
        for (int i = 0; i < JBC_SLOTS; ++i) { lo[i] = 0; sz[i] = 0; z[i] = false; b[i] = 0; pb[i] = 0; }
    }
};

// cache-only check against entry S: true iff the access is aligned and inside the
// buffer cached there (then *zero is that buffer's writer-rule flag); no state change
template <int S>
__device__ __forceinline__ bool jhit(const JBufCache& C, u64 va, u32 w, bool* zero) {
    const u32 vlo = (u32)va;
    *zero = C.z[S];
    return ((u32)(va >> 32) == JVA_HI) & ((vlo & (w - 1)) == 0) & (vlo - C.lo[S] < C.sz[S]);
}
// the same check for va_first + delta, given jhit(va_first) (jit.cpp ldg_batch)
template <int S>
__device__ __forceinline__ bool jhit_more(const JBufCache& C, u64 va_first, u32 delta, bool* zero) {
    *zero = C.z[S];
    return (u32)va_first - C.lo[S] + delta < C.sz[S];
}
__device__ const uint4 jzero16[1] = {{0u, 0u, 0u, 0u}};   // the zero line of writer-rule loads
// L1 prefetch of an address inside the buffer cached in entry S (else nothing)
template <int S>
__device__ __forceinline__ void jprefetch(const u8* __restrict__ img, const JBufCache& C, u64 va) {
    const u32 vlo = (u32)va;
    if (((u32)(va >> 32) == JVA_HI) & (vlo - C.lo[S] < C.sz[S]))
        asm volatile("prefetch.global.L1 [%0];" ::"l"(img + (va - JVA_BASE)));
}

// the replica slot's view of memory during instance t (K8, PAGE mode)
struct JPage {
    const u32* ptab;             // the slot's page table
    const u32* pool; const u32* page_base; const u32* last_ref; const u32* dropped;
    const u32* bcount;           // the slot's page count per buffer (constant during a launch)
    u32* inexact; u32 t;
};
#define JPB_NONE 0xFFFFFFFFu     // cache entry's page base when the slot holds no page of the buffer
// 0 ok, 1 misaligned, 2 unmapped (C-15); *zero = writer rule for instance k.
// A miss refills entry S.
template <int S>
__device__ __forceinline__ u32 jcheck(const JArgs& A, JBufCache& C, u64 va, u32 w, u32 k, bool* zero,
                                      const JPage* pg = nullptr) {
    if (va & (w - 1)) return 1;
    if (jhit<S>(C, va, w, zero)) return 0;
    const u64 off = va - JVA_BASE;
    if (va < JVA_BASE || off >= A.image_bytes) return 2;
    const u32 b = __ldg(&A.gran[off >> 8]);
    if (b == JNOBUF) return 2;
    const u64 lo = __ldg(&A.buf[b].off), size = __ldg(&A.buf[b].size);
    if (off + w > lo + size) return 2;
    const i32 wr = __ldg(&A.buf[b].writer);
    const bool z = wr >= 0 && (u32)wr >= k;
    *zero = z;
    if ((lo & 15u) == 0 && lo + size <= 0x80000000ull && size >= 16) {
        C.lo[S] = (u32)lo; C.sz[S] = (u32)size & ~15u; C.z[S] = z; C.b[S] = b;
        // PAGE mode: JPB_NONE when the slot has no page of the buffer and no page of it was
        // dropped past its last reference — the golden words stand, jpage_c skips the
        // page-table load
        C.pb[S] = 0u;
        if (pg) {
            const bool dropped = __ldg(&pg->last_ref[b]) < pg->t && ((pg->dropped[b >> 5] >> (b & 31)) & 1u);
            C.pb[S] = (pg->bcount[b] == 0u && !dropped) ? JPB_NONE : __ldg(&pg->page_base[b]);
        }
    }
    return 0;
}

// one LDG of 1/2/4 words for this lane; returns the fault code (0 ok)
template <u32 LW, int S>
__device__ __forceinline__ u32 jldg(const JArgs& A, const u8* __restrict__ img, JBufCache& C, u64 va, u32 k, bool ex,
                                    uint4& v, const JPage* pg = nullptr) {
    bool zero = false;
    const u32 c = ex ? jcheck<S>(A, C, va, 4u << LW, k, &zero, pg) : 0u;
    v = make_uint4(0, 0, 0, 0);
    if (ex && !c && !zero) {
        const u8* src = img + (va - JVA_BASE);
        if (LW == 0) v.x = jld32(src);
        else if (LW == 1) { const uint2 t = jld64(src); v.x = t.x; v.y = t.y; }
        else v = jld128(src);
    }
    return c;
}

// ---------------------------------------------------------------------------
// Step-at-a-time mode of the JIT module.  Whenever a block cannot run (entry
// off a leader, divergent groups, the injection step, the watchdog's last
// steps) the generated code spills its registers to the warp's shared-memory
// register file ([n_regs+1][32] words, row n_regs all zero) and this
// interpreter runs single steps from the pre-decoded code (fi_program_prepare's
// layout, emu.cuh) until the warp reaches a leader whose block fits again, ends
// or faults.  Same semantics as emu.cuh's general step.
struct JState {
    u32 pc, live, step, livem, conv, upc, amask, npc, nst, fault, fault_pc, before, after, msk, fired, bad, lim, preds;
    u32 brk, ckn;                                    // last step was BRA / EXIT; next golden checkpoint (JM_TRACE)
    uint4 recbuf;                                    // golden trace pass: this lane's record of the 32-step window
};
#define JM_INJ 0                                     // injection replica (K4): hook, stores after the site logged
#define JM_LEN 1                                     // golden pass 1: steps / stores counted (+ image stores unless sliced)
#define JM_TRACE 2                                   // golden pass 2: trace records, store log, checkpoints, image stores

__device__ __forceinline__ bool jguard(u32 guard, u32 preds) { return fisem::guard_of(guard, preds); }
typedef fisem::RegFile JRegs;                        // this lane's column of the smem register file

// ---------------------------------------------------------------------------
// K8 (propagate8.cu) on the JIT module: re-execution of instance t for every
// active replica slot over its copy-on-write pages.  Layouts mirror
// propagate8.cu's Slot and the K8Args fields k8_exec uses.
#define JM_PAGE 3
#define JPAGE_WORDS 1024u
#define JPAGE_CLAIM 0xFFFFFFFEu
struct JSlot {
    u32 rep, k0, alive, outcome;
    u32 npages, inexact, overflow, pend_n;
    u32 for_n, pdue, perm, pad1;
    unsigned long long fault_key, pdue_key;
};
struct JK8 {
    const u64* warp_off; const u64* gst_off; const jfi_store* gst;
    JSlot* slot;
    const u32* ptab; u32 total_pages;
    const u32* pool; const u32* page_base; const u32* last_ref; const u32* dropped; u32 dwords;
    jfi_store* pend; u32 pend_cap;
    jfi_store* forn; u32 foreign_cap;
    const u32* active; const u32* n_active; u32* work;
    jfi_store* scratch; u32 log_cap;
    u32 flags; u32* status;
    unsigned long long* steps;                      // emulated warp-steps of the re-executed warps (summed)
    const u32* bcount; u32 n_buf;                   // [slot][buffer] page counts
};

// The replica's words of an aligned access of NW words (one 4 KB page): its page
// if it has one, else the golden value already in v.  A load from a buffer whose
// pages were dropped after its last golden reference marks the slot inexact.
template <u32 NW>
__device__ __forceinline__ void jpage(const JArgs& A, const JPage& G, u64 va, uint4& v) {
    const u64 off = va - JVA_BASE;
    const u32 b = __ldg(&A.gran[off >> 8]);
    const u64 rel = off - __ldg(&A.buf[b].off);
    const u32 e = G.ptab[__ldg(&G.page_base[b]) + (u32)(rel >> 12)];
    if (e < JPAGE_CLAIM) {
        const u32* src = G.pool + (u64)e * JPAGE_WORDS + ((rel >> 2) & (JPAGE_WORDS - 1));
        if (NW == 1) v.x = __ldcg(src);
        else if (NW == 2) { const uint2 t = __ldcg(reinterpret_cast<const uint2*>(src)); v.x = t.x; v.y = t.y; }
        else v = __ldcg(reinterpret_cast<const uint4*>(src));
    } else if (__ldg(&G.last_ref[b]) < G.t && ((G.dropped[b >> 5] >> (b & 31)) & 1u)) {
        *G.inexact = 1u;
    }
}
// the same through entry S of the lane's buffer cache when it holds the access
// (one page-table load), else jpage's full lookup
template <u32 NW, int S>
__device__ __forceinline__ void jpage_c(const JArgs& A, const JBufCache& C, const JPage& G, u64 va, uint4& v) {
    const u32 rel = (u32)va - C.lo[S];
    if (!(rel < C.sz[S])) { jpage<NW>(A, G, va, v); return; }
    if (C.pb[S] == JPB_NONE) return;                 // no page of this buffer in the slot
    const u32 b = C.b[S];
    const u32 e = G.ptab[C.pb[S] + (rel >> 12)];
    if (e < JPAGE_CLAIM) {
        const u32* src = G.pool + (u64)e * JPAGE_WORDS + ((rel >> 2) & (JPAGE_WORDS - 1));
        if (NW == 1) v.x = __ldcg(src);
        else if (NW == 2) { const uint2 t = __ldcg(reinterpret_cast<const uint2*>(src)); v.x = t.x; v.y = t.y; }
        else v = __ldcg(reinterpret_cast<const uint4*>(src));
    } else if (__ldg(&G.last_ref[b]) < G.t && ((G.dropped[b >> 5] >> (b & 31)) & 1u)) {
        *G.inexact = 1u;
    }
}
__device__ __forceinline__ void jpage_n(const JArgs& A, const JPage& G, u64 va, u32 nw, uint4& v) {
    if (nw == 1) jpage<1>(A, G, va, v);
    else if (nw == 2) jpage<2>(A, G, va, v);
    else jpage<4>(A, G, va, v);
}


// Step mode (emu.cuh's general step; MODE = JM_INJ / JM_LEN / JM_TRACE).  Returns
// 1 when the warp is done (finished or faulted), 0 when it stands at a leader
// whose block fits.  `ck` (JM_TRACE): the warp's checkpoint destination, or 0.
template <int MODE>
__device__ __noinline__ u32 jinterp(const JArgs& A, JState& S, JBufCache& bc, u32* R, const uint4* __restrict__ dec,
                                    const unsigned short* __restrict__ blen, const u32 code_len, const u32 k,
                                    const u32 cta, const u32 wic, const u32 watchdog, const u32 hstep, const u32 hpc,
                                    const u32 hlane, const u32 hkind, const u32 hreg, const u32 hbfm,
                                    const u32 hmask, jfi_store* __restrict__ st_out, const u32 st_cap,
                                    const u32 zr, u8* __restrict__ img_w, uint4* __restrict__ rec_out,
                                    u32* __restrict__ ck, const u32 ck_interval, const u32* __restrict__ ins,
                                    const JPage* __restrict__ pg, const u8* __restrict__ slice, JProf* prof) {
    // slice (JM_LEN as the control slice, jit.cpp): 0 = the instruction cannot
    // affect control flow or the store counts — only BRA / EXIT and STG counting
    // run for it (no loads, no image stores)
    const u32 lane = threadIdx.x & 31, lt_mask = (1u << lane) - 1u;
    const JRegs F{reinterpret_cast<char*>(R + lane), R, zr * 128};
    const jfi_instance in = A.inst[k];
    const u32* cb = A.cbank + in.cbank_off;
    bool live = S.live != 0, conv = S.conv != 0;
    u32 pc = S.pc, step = S.step, livem = S.livem, upc = S.upc, amask = S.amask, npc = S.npc, nst = S.nst;
    u32 preds = S.preds, lim = S.lim, brk = S.brk, ckn = S.ckn;
    uint4 recbuf = S.recbuf;
    u32 done = 0;
    for (;;) {
        if (!livem) { done = 1; break; }
        u32 pcm, active;
        if (conv) { pcm = upc; active = amask; }
        else {
            pcm = __reduce_min_sync(JFULL, live ? pc : 0xFFFFFFFFu);
            active = __ballot_sync(JFULL, live && pc == pcm);
            npc = active == livem ? 0xFFFFFFFFu : __reduce_min_sync(JFULL, (live && pc != pcm) ? pc : 0xFFFFFFFFu);
            conv = true; upc = pcm; amask = active;
        }
        if (MODE == JM_TRACE && ck && brk && step >= ckn * ck_interval) {
            // golden checkpoints ckn .. step/interval (emu.cuh): the state before the
            // first step at or past the multiple that follows a BRA / EXIT
            const bool inA = (amask >> lane) & 1u;
            for (; ckn <= step / ck_interval; ++ckn) {
                u32* dst = ck + (u64)ckn * (zr + 4) * 32;
                for (u32 r = 0; r < zr; ++r) dst[r * 32 + lane] = R[r * 32 + lane];
                dst[zr * 32 + lane] = live ? (inA ? upc : pc) : 0u;
                dst[zr * 32 + 32 + lane] = preds;
                dst[zr * 32 + 64 + lane] = live ? 1u : 0u;
                dst[zr * 32 + 96 + lane] = step;
            }
        }
        if (step >= watchdog) { S.fault = 3; S.fault_pc = pcm; done = 1; break; }
        if (pcm >= code_len) { S.fault = 4; S.fault_pc = pcm; done = 1; break; }
        const u32 bl = blen[pcm];                     // 0 unless pcm is a leader
        if (bl && pcm + bl <= npc && step + bl <= lim) break;      // the generated block runs from here
        const uint4 D = __ldg(&dec[pcm]);
        const u32 op = D.x & 0xFF, guard = (D.x >> 8) & 0xFF, mod = (D.x >> 16) & 0xFF;
        const u32 ia = D.y & 0xFFFF, ib = D.y >> 16, id = D.z >> 16, imm = D.w;
        const bool act = (active >> lane) & 1u;
        const bool pv = guard == 7 ? true : jguard(guard, preds);
        const u32 pred = guard == 7 ? JFULL : __ballot_sync(JFULL, pv);
        const bool ex = act && pv;
        const u32 exm = active & pred;
        if (MODE == JM_TRACE) {                       // one trace record per step (App. A.3)
            const u32 w = __ldg(&ins[pcm]);
            if (lane == 0) __stcs(&rec_out[step], make_uint4(k, w, active, pred));
            if (prof->cc) jprof_one(prof, lane, prof->rb + step, __popc(active & pred), w >> 24);
        }
        u32 taken = 0;
        brk = op == 1 || op == 2;
        if (MODE == JM_LEN && slice && !slice[pcm] && op != 1 && op != 2) {
            if (op == 23) nst += __popc(exm) * (1u << ((mod & 3) > 2 ? 2 : (mod & 3)));
        } else if (op == 1) {                         // EXIT
            if (ex) live = false;
            livem &= ~exm;
            amask &= ~exm;
        } else if (op == 2) {                         // BRA
            taken = exm;
        } else if (op == 21 || op == 23) {            // LDG / STG
            const u32 lw = (mod & 3) > 2 ? 2 : (mod & 3), nw = 1u << lw, w = 4u << lw;
            const u64 va = F.rd64(ia) + (u64)(i64)(i32)imm;
            bool zero = false;
            const u32 c = ex ? jcheck<0>(A, bc, va, w, k, &zero, MODE == JM_PAGE ? pg : nullptr) : 0u;
            if (__ballot_sync(JFULL, c != 0u)) {      // memory fault: DUE (C-9); the step has no effect
                S.fault = __ballot_sync(JFULL, c == 1u) ? 1u : 2u;
                S.fault_pc = pcm;
                done = 1;
                break;
            }
            if (op == 21) {
                if (ex) {
                    uint4 v = make_uint4(0, 0, 0, 0);
                    if (!zero) {
                        const u8* src = A.img + (va - JVA_BASE);
                        if (lw == 0) v.x = jld32(src);
                        else if (lw == 1) { const uint2 t = jld64(src); v.x = t.x; v.y = t.y; }
                        else v = jld128(src);
                    }
                    if (MODE == JM_PAGE) {            // the replica's pages win
                        if (nw == 1) jpage_c<1, 0>(A, bc, *pg, va, v);
                        else if (nw == 2) jpage_c<2, 0>(A, bc, *pg, va, v);
                        else jpage_c<4, 0>(A, bc, *pg, va, v);
                    }
                    F.wr(id, v.x);
                    if (lw >= 1) F.wr(id + 128, v.y);
                    if (lw >= 2) { F.wr(id + 256, v.z); F.wr(id + 384, v.w); }
                }
            } else {
                u32 v[4];
#pragma unroll
                for (int i = 0; i < 4; ++i) v[i] = (u32)i < nw ? F.rd(min(ib + 128u * i, F.zb)) : 0u;
                if (MODE == JM_TRACE && img_w && ex) {   // golden pass 2: stores go to the image too
                    u8* dst = img_w + (va - JVA_BASE);
                    if (lw == 0) *reinterpret_cast<u32*>(dst) = v[0];
                    else if (lw == 1) *reinterpret_cast<uint2*>(dst) = make_uint2(v[0], v[1]);
                    else *reinterpret_cast<uint4*>(dst) = make_uint4(v[0], v[1], v[2], v[3]);
                }
                if (MODE == JM_LEN) {                 // golden pass 1: stores go to the image
                    if (ex) {
                        u8* dst = img_w + (va - JVA_BASE);
                        if (lw == 0) *reinterpret_cast<u32*>(dst) = v[0];
                        else if (lw == 1) *reinterpret_cast<uint2*>(dst) = make_uint2(v[0], v[1]);
                        else *reinterpret_cast<uint4*>(dst) = make_uint4(v[0], v[1], v[2], v[3]);
                    }
                    nst += __popc(exm) * nw;
                } else if (MODE == JM_TRACE || MODE == JM_PAGE || step > hstep) {   // store logs
                    if (ex) {
                        const u32 idx = __popc(exm & lt_mask) * nw;
                        for (u32 i = 0; i < nw; ++i) {
                            const u32 e = nst + idx + i;
                            if (MODE == JM_TRACE || e < st_cap) {
                                jfi_store s_; s_.va = va + 4 * i; s_.value = v[i]; s_.step = step; st_out[e] = s_;
                            }
                        }
                    }
                    nst += __popc(exm) * nw;
                }
            }
        } else {
            fisem::exec_plain(F, fisem::LaneCtx{lane, cta, wic, in.block, in.grid, in.cbank_len, cb}, D, ex, preds);
        }
        if (taken == 0) upc = pcm + 1;
        else if (taken == active) upc = imm;
        else { conv = false; if (act) pc = ((taken >> lane) & 1u) ? imm : pcm + 1; }
        if (conv && (amask == 0 || upc >= npc)) { conv = false; if ((amask >> lane) & 1u) pc = upc; }
        if (MODE == JM_INJ && step == hstep) {        // the transient fault (C-7, C-8)
            S.fired = 1;
            if (pcm != hpc || !((exm >> hlane) & 1u)) S.bad = 1;
            if (lane == hlane) {
                if (hkind == 0) {
                    const u32 ri = min(hreg, zr) * 128;
                    const u32 b = F.rd(ri);
                    const u32 m = hbfm == 3 ? b : hmask;
                    S.before = b; S.msk = m; S.after = b ^ m;
                    F.wr(ri, S.after);
                } else {
                    const u32 p = hreg & 7;
                    const u32 b = (p == 7) ? 1u : ((preds >> p) & 1u);
                    u32 m = hmask, a;
                    if (hbfm == 0 || hbfm == 1) a = b ^ 1u;
                    else if (hbfm == 2) a = (m >> 31) & 1u;
                    else { m = b; a = 0u; }
                    S.before = b; S.msk = m; S.after = a;
                    if (p != 7) preds = (preds & ~(1u << p)) | (a << p);
                }
            }
        }
        ++step;
        if (MODE == JM_INJ && step > hstep) lim = watchdog;
    }
    S.pc = pc; S.live = live; S.step = step; S.livem = livem; S.conv = conv; S.upc = upc; S.amask = amask;
    S.npc = npc; S.nst = nst; S.preds = preds; S.lim = lim; S.recbuf = recbuf; S.brk = brk; S.ckn = ckn;
    return done;
}

__device__ __forceinline__ u32 jk8_page_of(const JArgs& A, const JK8& K, u64 va, u32& b, u32& word) {
    const u64 off = va - JVA_BASE;
    b = __ldg(&A.gran[off >> 8]);
    const u64 rel = off - __ldg(&A.buf[b].off);
    word = (u32)(rel >> 2) & (JPAGE_WORDS - 1);
    return __ldg(&K.page_base[b]) + (u32)(rel >> 12);
}
// golden value of word va after instance t (t = -1: initial image)
__device__ __forceinline__ u32 jk8_gstate(const JArgs& A, u64 va, i64 t) {
    const i32 wr = __ldg(&A.buf[__ldg(&A.gran[(va - JVA_BASE) >> 8])].writer);
    return (wr >= 0 && (i64)wr > t) ? 0u : __ldg(reinterpret_cast<const u32*>(A.img + (va - JVA_BASE)));
}
__device__ __forceinline__ u32 jk8_cur(const JArgs& A, const JK8& K, u32 s, u64 va, i64 t) {
    u32 b, w;
    const u32 p = jk8_page_of(A, K, va, b, w);
    const u32 e = K.ptab[(u64)s * K.total_pages + p];
    if (e < JPAGE_CLAIM) return __ldcg(&K.pool[(u64)e * JPAGE_WORDS + w]);
    return jk8_gstate(A, va, t - 1);
}
__device__ __forceinline__ bool jk8_no_change(const JArgs& A, const JK8& K, u32 s, u64 va, u32 v, i64 t) {
    u32 b, w;
    const u32 p = jk8_page_of(A, K, va, b, w);
    return K.ptab[(u64)s * K.total_pages + p] == 0xFFFFFFFFu && v == jk8_gstate(A, va, t);
}
__device__ __forceinline__ void jk8_err(const JK8& K, u32 s, u32 code) {
    K.slot[s].overflow = 1;
    atomicOr(K.status, 1u << code);
}
// propagate8.cu warp_updates8 with mark_foreign = true (a re-executed warp):
// F deduplicated (last write wins) and G \ F with the replica's old values, appended
// to the slot's pending list; F entries outside G are also "foreign" (C-14)
__device__ void jk8_updates(const JArgs& A, const JK8& K, u32 s, u32 w_idx, const jfi_store* F, u64 nF,
                            const jfi_store* G, u64 nG, i64 t) {
    const u32 lane = threadIdx.x & 31;
    jfi_store* pend = K.pend + (u64)s * K.pend_cap;
    bool same = nF == nG;
    for (u64 b = 0; b < nF && same; b += 32) {
        const u64 j = b + lane;
        same = __all_sync(JFULL, j >= nF || F[j].va == G[j].va);
    }
    if (same) {
        for (u64 b = 0; b < nF; b += 32) {
            const u64 j = b + lane;
            jfi_store f; f.va = 0; f.value = 0; f.step = 0;
            bool keep = false;
            if (j < nF) {
                f = F[j];
                f.step = w_idx;
                keep = !jk8_no_change(A, K, s, f.va, f.value, t);
            }
            const u32 m = __ballot_sync(JFULL, keep);
            u32 base = 0;
            if (lane == 0 && m) base = atomicAdd(&K.slot[s].pend_n, (u32)__popc(m));
            base = __shfl_sync(JFULL, base, 0);
            if (keep) {
                const u32 pos = base + __popc(m & ((1u << lane) - 1));
                if (pos < K.pend_cap) pend[pos] = f;
                else jk8_err(K, s, 8);
            }
        }
        return;
    }
    for (u64 b = 0; b < nF; b += 32) {
        const u64 j = b + lane;
        bool keep = false, foreign = false;
        jfi_store f; f.va = 0; f.value = 0; f.step = 0;
        if (j < nF) {
            f = F[j];
            keep = true;
            for (u64 q = j + 1; q < nF && keep; ++q) keep = F[q].va != f.va;
            if (keep) {
                foreign = true;
                for (u64 q = 0; q < nG && foreign; ++q) foreign = G[q].va != f.va;
            }
            if (keep && !foreign && jk8_no_change(A, K, s, f.va, f.value, t)) keep = false;
        }
        const u32 m = __ballot_sync(JFULL, keep);
        u32 base = 0;
        if (lane == 0 && m) base = atomicAdd(&K.slot[s].pend_n, (u32)__popc(m));
        base = __shfl_sync(JFULL, base, 0);
        if (keep) {
            const u32 pos = base + __popc(m & ((1u << lane) - 1));
            f.step = w_idx | (foreign ? 0x80000000u : 0u);
            if (pos < K.pend_cap) pend[pos] = f;
            else jk8_err(K, s, 8);
            if (foreign) {
                const u32 fp = atomicAdd(&K.slot[s].for_n, 1u);
                if (fp < K.foreign_cap) K.forn[(u64)s * K.foreign_cap + fp] = f;
                else jk8_err(K, s, 8);
            }
        }
    }
    for (u64 b = 0; b < nG; b += 32) {
        const u64 j = b + lane;
        bool keep = false;
        jfi_store g; g.va = 0; g.value = 0; g.step = 0;
        if (j < nG) {
            const u64 va = G[j].va;
            bool inF = false;
            for (u64 q = 0; q < nF && !inF; ++q) inF = F[q].va == va;
            if (!inF) {
                g.va = va;
                g.value = jk8_cur(A, K, s, va, t);
                g.step = w_idx;
                keep = !jk8_no_change(A, K, s, va, g.value, t);
            }
        }
        const u32 m = __ballot_sync(JFULL, keep);
        u32 base = 0;
        if (lane == 0 && m) base = atomicAdd(&K.slot[s].pend_n, (u32)__popc(m));
        base = __shfl_sync(JFULL, base, 0);
        if (keep) {
            const u32 pos = base + __popc(m & ((1u << lane) - 1));
            if (pos < K.pend_cap) pend[pos] = g;
            else jk8_err(K, s, 8);
        }
    }
}
