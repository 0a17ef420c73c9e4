// propagate8.cu — K8: batched, instance-major outcome propagation for long
// multi-instance programs (C3-class: thousands of launches).
//
// Same definition as K7 (PAPER.md:72 step (4), :206; readings C-12, C-14, C-19):
// after the faulty warp's instance k0, every later instance that references a
// buffer holding a corrupted word is re-executed against the replica's faulty
// memory and the run is classified on the whole program's outputs.  K7 walks one
// replica's later launches on one CUDA warp; K8 keeps a batch of replicas in
// lockstep over the launches and re-executes instance t for every affected
// replica at once — (replica, warp) pairs spread over the whole GPU.
//
// Faulty memory of a replica slot: copy-on-write 4 KB pages per buffer in a
// shared pool (ptab[slot][page], page = page_base[buffer] + offset / 4 KB); every
// word without a page has its golden value (DESIGN.md §3.5 writer rule).
// Per instance t (host loop, all stream-ordered):
//   activate  slots with k0 < t whose pages touch a buffer t references
//   exec      one CUDA warp per (active slot, warp of t): emulate over the pages,
//             diff the stores with the warp's golden store log -> updates
//             (a faulty store at an address the golden warp does not store is
//             "foreign": the only kind two warps can share, C-14 order decides)
//   k0        slots whose faulty warp ran in t: K4's store log -> updates
//   mark/alloc/apply  end-of-instance visibility (C-14): pages claimed, taken from
//             the pool and filled with the golden state after t, updates written
//             (foreign ones last, the highest warp index winning)
//   gc        pages equal to the golden state are returned (a replica without
//             pages is Masked); buffers past their last reference lose their pages
//             (a later wild load from one marks the replica inexact -> 0xFF)
// then SDC iff a page of an output buffer differs from the golden final image.
#include <algorithm>
#include <vector>

#include "emu.cuh"
#include "jit_k8.h"

namespace fi {
size_t golden_smem(uint32_t n_regs);
namespace {

constexpr int kWPB8 = 4;
constexpr uint32_t kForeignCap = 256;
constexpr uint32_t kNoRep = 0xFFFFFFFFu;

struct Slot {
    uint32_t rep, k0, alive, outcome;
    uint32_t npages, inexact, overflow, pend_n;
    uint32_t for_n, pdue, perm, pad1;                // perm: permanent / intermittent fault (rows f2/f3)
    unsigned long long fault_key;                    // (t << 43 | w << 19 | kind << 16 | pc), min = first
    unsigned long long pdue_key;
};

struct K8Args {
    EmuProg P;
    const uint8_t* img;
    const uint64_t* warp_off; const uint64_t* gst_off; const fi_store* gst;
    const fi_site* sites; fi_inj* inj; const fi_store* log; uint32_t log_cap;
    Slot* slot; uint32_t B;
    uint32_t* ptab; uint32_t total_pages;
    uint32_t* bcount;                                // [B][n_buf]
    uint32_t* dropped; uint32_t dwords;              // [B][dwords]
    uint32_t* pool; uint32_t* free_stack; int* free_top; uint32_t pool_pages;
    const uint32_t* page_base; const uint32_t* last_ref; uint32_t n_buf;
    fi_store* pend; uint32_t pend_cap;               // [B][pend_cap]
    fi_store* forn;                                  // [B][kForeignCap]
    uint32_t* active; uint32_t* n_active; uint32_t* work;
    uint2* need; uint32_t* n_need; uint32_t need_cap;
    fi_store* scratch;                               // [resident warps][log_cap]
    const uint32_t* dying; const uint32_t* dying_off;   // CSR over instances
    uint32_t flags; uint32_t* status; uint64_t* hist;
    const fi_pfault* pf; const uint64_t* opw;        // permanent mode (else null)
    const uint32_t* kop;                             // per static kernel: bit op set iff the kernel has opcode op
    double rtol;                                     // > 0: C-12 secondary numeric classification
};

__device__ __forceinline__ uint32_t buf_of(const EmuProg& P, uint64_t va) { return __ldg(&P.gran[(va - kVaBase) >> 8]); }
__device__ __forceinline__ uint32_t gword(const uint8_t* img, uint64_t va) {
    return __ldg(reinterpret_cast<const uint32_t*>(img + (va - kVaBase)));
}
// golden value of word va after instance t (t = -1: initial image)
__device__ __forceinline__ uint32_t gstate(const EmuProg& P, const uint8_t* img, uint64_t va, int64_t t) {
    const int32_t wr = __ldg(&P.buf[buf_of(P, va)].writer);
    return (wr >= 0 && (int64_t)wr > t) ? 0u : gword(img, va);
}
__device__ __forceinline__ uint32_t page_of(const K8Args& A, uint64_t va, uint32_t& b, uint32_t& word) {
    const uint64_t off = va - kVaBase;
    b = __ldg(&A.P.gran[off >> 8]);
    const uint64_t rel = off - __ldg(&A.P.buf[b].off);
    word = (uint32_t)(rel >> 2) & (kPageWords - 1);
    return __ldg(&A.page_base[b]) + (uint32_t)(rel >> 12);
}
// replica's value of word va before instance t's stores (its page, else golden after t-1)
__device__ __forceinline__ uint32_t cur_value(const K8Args& A, uint32_t s, uint64_t va, int64_t t) {
    uint32_t b, w;
    const uint32_t p = page_of(A, va, b, w);
    const uint32_t e = A.ptab[(size_t)s * A.total_pages + p];
    if (e < kPageClaim) return __ldcg(&A.pool[(size_t)e * kPageWords + w]);
    return gstate(A.P, A.img, va, t - 1);
}

// Does pool page e differ from the golden state after t of page p (buffer b)?  All
// words of a page belong to one buffer, so the writer rule is uniform; words past
// the buffer's end are 0.  One warp, 16-B loads.
__device__ __forceinline__ bool page_differs(const K8Args& A, uint32_t e, uint32_t b, uint32_t p, int64_t t) {
    const uint32_t lane = threadIdx.x & 31;
    const int32_t wr = __ldg(&A.P.buf[b].writer);
    const bool zero = wr >= 0 && (int64_t)wr > t;
    const uint64_t boff = __ldg(&A.P.buf[b].off), bsz = __ldg(&A.P.buf[b].size);
    const uint64_t rel0 = (uint64_t)(p - __ldg(&A.page_base[b])) << 12;
    const uint4* pg = reinterpret_cast<const uint4*>(A.pool + (size_t)e * kPageWords);
    bool d = false;
#pragma unroll 4
    for (uint32_t q = lane; q < kPageWords / 4; q += 32) {
        const uint64_t rel = rel0 + 16ull * q;
        const uint4 v = __ldcg(&pg[q]);
        uint4 g = make_uint4(0, 0, 0, 0);
        if (!zero && rel < bsz) g = __ldg(reinterpret_cast<const uint4*>(A.img + boff + rel));
        d |= (v.x != g.x) | (v.y != g.y) | (v.z != g.z) | (v.w != g.w);
    }
    return __any_sync(kFull, d);
}

__device__ __forceinline__ void set_err(const K8Args& A, uint32_t s, uint32_t code) {
    A.slot[s].overflow = 1;
    FI_DEV_ERR(A.status, code);
}

// An update that leaves a word without a page at its golden value after t changes
// nothing (k8_foreign accounts for the dropped entry through the golden log).
__device__ __forceinline__ bool no_change(const K8Args& A, uint32_t s, uint64_t va, uint32_t v, int64_t t) {
    uint32_t b, w;
    const uint32_t p = page_of(A, va, b, w);
    return A.ptab[(size_t)s * A.total_pages + p] == kPageNone && v == gstate(A.P, A.img, va, t);
}

// Updates of one warp (F = its stores in program order, G = its golden stores):
// F deduplicated (last write wins) and G \ F with the replica's old values.
// Appended to the slot's pending list; F entries outside G are also "foreign".
__device__ void warp_updates8(const K8Args& A, uint32_t s, uint32_t w_idx, const fi_store* F, uint64_t nF,
                              const fi_store* G, uint64_t nG, int64_t t, bool mark_foreign) {
    const uint32_t lane = threadIdx.x & 31;
    fi_store* pend = A.pend + (size_t)s * A.pend_cap;
    // fast path: the faulty warp stored exactly the golden addresses in the golden
    // order (a golden warp stores each word once), so the updates are F itself
    bool same = nF == nG;
    for (uint64_t b = 0; b < nF && same; b += 32) {
        const uint64_t j = b + lane;
        same = __all_sync(kFull, j >= nF || F[j].va == G[j].va);
    }
    if (same) {
        for (uint64_t b = 0; b < nF; b += 32) {
            const uint64_t j = b + lane;
            fi_store f{};
            bool keep = false;
            if (j < nF) {
                f = F[j];
                f.step = w_idx;
                keep = !no_change(A, s, f.va, f.value, t);
            }
            const uint32_t m = __ballot_sync(kFull, keep);
            uint32_t base = 0;
            if (lane == 0 && m) base = atomicAdd(&A.slot[s].pend_n, (uint32_t)__popc(m));
            base = __shfl_sync(kFull, base, 0);
            if (keep) {
                const uint32_t pos = base + __popc(m & ((1u << lane) - 1));
                if (pos < A.pend_cap) pend[(size_t)pos] = f;
                else set_err(A, s, FI_E_CAPACITY);
            }
        }
        return;
    }
    for (uint64_t b = 0; b < nF; b += 32) {
        const uint64_t j = b + lane;
        bool keep = false, foreign = false;
        fi_store f{};
        if (j < nF) {
            f = F[j];
            keep = true;
            for (uint64_t q = j + 1; q < nF && keep; ++q) keep = F[q].va != f.va;
            if (keep && mark_foreign) {
                foreign = true;
                for (uint64_t q = 0; q < nG && foreign; ++q) foreign = G[q].va != f.va;
            }
            if (keep && !foreign && no_change(A, s, f.va, f.value, t)) keep = false;
        }
        const uint32_t m = __ballot_sync(kFull, keep);
        uint32_t base = 0;
        if (lane == 0 && m) base = atomicAdd(&A.slot[s].pend_n, (uint32_t)__popc(m));
        base = __shfl_sync(kFull, base, 0);
        if (keep) {
            const uint32_t pos = base + __popc(m & ((1u << lane) - 1));
            f.step = w_idx | (foreign ? 0x80000000u : 0u);
            if (pos < A.pend_cap) pend[(size_t)pos] = f;
            else set_err(A, s, FI_E_CAPACITY);
            if (foreign) {
                const uint32_t fp = atomicAdd(&A.slot[s].for_n, 1u);
                if (fp < kForeignCap) A.forn[(size_t)s * kForeignCap + fp] = f;
                else set_err(A, s, FI_E_CAPACITY);
            }
        }
    }
    for (uint64_t b = 0; b < nG; b += 32) {
        const uint64_t j = b + lane;
        bool keep = false;
        fi_store g{};
        if (j < nG) {
            const uint64_t va = G[j].va;
            bool inF = false;
            for (uint64_t q = 0; q < nF && !inF; ++q) inF = F[q].va == va;
            if (!inF) {
                g.va = va;
                g.value = cur_value(A, s, va, t);
                g.step = w_idx;
                keep = !no_change(A, s, va, g.value, t);
            }
        }
        const uint32_t m = __ballot_sync(kFull, keep);
        uint32_t base = 0;
        if (lane == 0 && m) base = atomicAdd(&A.slot[s].pend_n, (uint32_t)__popc(m));
        base = __shfl_sync(kFull, base, 0);
        if (keep) {
            const uint32_t pos = base + __popc(m & ((1u << lane) - 1));
            if (pos < A.pend_cap) pend[(size_t)pos] = g;
            else set_err(A, s, FI_E_CAPACITY);
        }
    }
}

// ---- batch setup: slot state from K4's results
__global__ void k8_setup(K8Args A, const uint32_t* reps, uint32_t nb) {
    const uint32_t s = blockIdx.x * blockDim.x + threadIdx.x;
    if (s >= A.B) return;
    Slot z{};
    z.rep = kNoRep;
    z.fault_key = ~0ull;
    z.pdue_key = ~0ull;
    if (s < nb && A.pf) {                            // permanent: armed from the first launch
        z.rep = reps[s];
        z.alive = 1;
        z.outcome = FI_MASKED;
        z.perm = 1;
    } else if (s < nb) {
        const uint32_t i = reps[s];
        const fi_site S = A.sites[i];
        const fi_inj R = A.inj[i];
        const bool unchecked = A.flags & FI_UNCHECKED;
        z.rep = i;
        z.k0 = S.instance;
        z.alive = 1;
        z.outcome = FI_MASKED;
        if (S.flags & FI_SITE_NOT_INJECTED) { z.alive = 0; z.outcome = FI_NOT_INJECTED; }
        else if (R.overflow) { z.alive = 0; z.outcome = 0xFF; z.overflow = 1; }
        else if (R.fault_kind && !(unchecked && R.fault_kind != 3)) { z.alive = 0; z.outcome = FI_DUE; }
        else if (R.fault_kind) z.pdue = 1;
    }
    A.slot[s] = z;
}

__global__ void k8_free_init(uint32_t* free_stack, int* free_top, uint32_t n) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) free_stack[i] = i;
    if (i == 0) *free_top = (int)n;
}

// ---- which slots re-execute instance t (one block)
__global__ void __launch_bounds__(1024) k8_activate(K8Args A, uint32_t t) {
    __shared__ uint32_t cnt;
    if (threadIdx.x == 0) cnt = 0;
    __syncthreads();
    const uint32_t* ib = A.P.ib + (size_t)t * (kInstBufs + 1);
    const uint32_t nref = __ldg(&ib[0]);
    for (uint32_t s = threadIdx.x; s < A.B; s += blockDim.x) {
        Slot& z = A.slot[s];
        z.pend_n = 0;
        z.for_n = 0;
        bool act = false;
        if (z.alive && (z.perm || z.k0 < t) && !z.overflow) {
            if (nref > kInstBufs) act = true;
            else
                for (uint32_t q = 0; q < nref && !act; ++q)
                    act = A.bcount[(size_t)s * A.n_buf + __ldg(&ib[1 + q])] != 0;
            if (z.perm && !act) {                    // the faulty SM runs the opcode in t
                const fi_pfault F = A.pf[z.rep];
                const fi_instance in = A.P.inst[t];
                const uint32_t nsm = F.n_sm ? F.n_sm : 148u;
                act = F.sm < nsm && F.sm < in.grid && ((__ldg(&A.kop[in.kernel]) >> (F.opcode & 31)) & 1u);
            }
        }
        if (act) A.active[atomicAdd(&cnt, 1u)] = s;
    }
    __syncthreads();
    if (threadIdx.x == 0) { *A.n_active = cnt; *A.work = 0; *A.n_need = 0; }
}

// ---- re-execute instance t for every active slot: one CUDA warp per (slot, warp)
__global__ void __launch_bounds__(kWPB8 * 32) k8_exec(K8Args A, uint32_t t) {
    extern __shared__ uint32_t smem[];
    const uint32_t wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t gw = blockIdx.x * kWPB8 + wib;
    uint32_t* R = smem + wib * (A.P.n_regs + 1) * 32;
    fi_store* scr = A.scratch + (size_t)gw * A.log_cap;
    const fi_instance in = A.P.inst[t];
    const uint32_t nw = in.warp_end - in.warp_begin, wpc = (in.block + 31) / 32;
    const uint64_t items = (uint64_t)(*A.n_active) * nw;
    const bool unchecked = A.flags & FI_UNCHECKED;
    for (;;) {
        uint32_t it = 0;
        if (lane == 0) it = atomicAdd(A.work, 1u);
        it = __shfl_sync(kFull, it, 0);
        if (it >= items) return;
        const uint32_t s = A.active[it / nw], lw = it % nw, w = in.warp_begin + lw;
        if (A.slot[s].overflow) continue;
        const uint64_t L = A.warp_off[w + 1] - A.warp_off[w];
        const uint64_t wd = 10 * L + 1024;                                                   // C-10
        const uint32_t watchdog = wd > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)wd;
        PageView pv{A.ptab + (size_t)s * A.total_pages, A.pool, A.page_base, A.last_ref,
                    A.dropped + (size_t)s * A.dwords, &A.slot[s].inexact, t};
        HookIn h{};
        if (A.pf) {                                   // CTAs on the faulty SM (C-21)
            const fi_pfault F = A.pf[A.slot[s].rep];
            const uint32_t nsm = F.n_sm ? F.n_sm : 148u;
            if ((lw / wpc) % nsm == F.sm) {
                h.perm_on = true; h.perm_op = F.opcode; h.perm_lane = F.lane; h.perm_mask = F.mask;
                h.perm_q = F.q32; h.perm_rep = A.slot[s].rep; h.perm_warp = w; h.perm_seed = F.seed;
            }
        }
        const EmuOut o = emulate<EMU_PAGE>(A.P, nullptr, A.img, t, lw / wpc, lw % wpc, R, watchdog, nullptr, scr,
                                           A.log_cap, h, nullptr, 0, Overlay{nullptr, 0}, pv);
        if (o.fault) {
            if (lane == 0) {
                const unsigned long long key = ((unsigned long long)t << 43) | ((unsigned long long)lw << 19) |
                                               ((unsigned long long)o.fault << 16) | (o.fault_pc & 0xFFFFu);
                if (!(unchecked && o.fault != 3)) atomicMin(&A.slot[s].fault_key, key);
                else atomicMin(&A.slot[s].pdue_key, key);
            }
            if (!(unchecked && o.fault != 3)) continue;     // DUE: its updates no longer matter
        }
        if (o.nstore > A.log_cap) {
            if (lane == 0) set_err(A, s, FI_E_CAPACITY);
            continue;
        }
        warp_updates8(A, s, lw, scr, o.nstore, A.gst + A.gst_off[w], A.gst_off[w + 1] - A.gst_off[w], t, true);
    }
}

// ---- slots whose faulty warp ran in instance t: K4's store log -> updates
__global__ void __launch_bounds__(kWPB8 * 32) k8_k0(K8Args A, uint32_t t) {
    const uint32_t s = blockIdx.x * kWPB8 + (threadIdx.x >> 5);
    if (s >= A.B) return;
    const Slot z = A.slot[s];
    if (!z.alive || z.perm || z.k0 != t || z.overflow) return;
    const fi_site S = A.sites[z.rep];
    const fi_inj Rj = A.inj[z.rep];
    const fi_store* G = A.gst + A.gst_off[S.warp];
    const uint64_t nGall = A.gst_off[S.warp + 1] - A.gst_off[S.warp];
    const uint32_t lane = threadIdx.x & 31;
    uint64_t gs = nGall;
    for (uint64_t b = 0; b < nGall; b += 32) {          // golden stores after the site
        const bool after = b + lane < nGall && G[b + lane].step > S.step;
        const uint32_t m = __ballot_sync(kFull, after);
        if (m) { gs = b + __ffs(m) - 1; break; }
    }
    warp_updates8(A, s, S.warp - A.P.inst[t].warp_begin, A.log + (uint64_t)z.rep * A.log_cap, Rj.n_faulty_stores,
                  G + gs, nGall - gs, t, false);
}

// ---- end of instance: claim pages for every pending update
__global__ void k8_mark(K8Args A) {
    const uint32_t s = blockIdx.y;
    const uint32_t n = min(A.slot[s].pend_n, A.pend_cap);
    const fi_store* pend = A.pend + (size_t)s * A.pend_cap;
    uint32_t* pt = A.ptab + (size_t)s * A.total_pages;
    for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
        uint32_t b, w;
        const uint32_t p = page_of(A, pend[j].va, b, w);
        if (pt[p] == kPageNone && atomicCAS(&pt[p], kPageNone, kPageClaim) == kPageNone) {
            const uint32_t q = atomicAdd(A.n_need, 1u);
            if (q < A.need_cap) A.need[q] = make_uint2(s, p);
            else set_err(A, s, FI_E_CAPACITY);
        }
    }
}

// ---- take pool pages for the claimed ones, filled with the golden state after t
__global__ void __launch_bounds__(256) k8_alloc(K8Args A, uint32_t t) {
    const uint32_t nn = min(*A.n_need, A.need_cap);
    for (uint32_t q = blockIdx.x; q < nn; q += gridDim.x) {
        const uint2 e = A.need[q];
        const uint32_t s = e.x, p = e.y;
        __shared__ int pg;
        __shared__ uint32_t sb;
        if (threadIdx.x == 0) {
            pg = atomicSub(A.free_top, 1) - 1;
            // buffer of page p: largest b with page_base[b] <= p
            uint32_t lo = 0, hi = A.n_buf;
            while (hi - lo > 1) {
                const uint32_t mid = (lo + hi) / 2;
                if (__ldg(&A.page_base[mid]) <= p) lo = mid; else hi = mid;
            }
            sb = lo;
        }
        __syncthreads();
        if (pg < 0) {
            if (threadIdx.x == 0) set_err(A, s, FI_E_CAPACITY);
            __syncthreads();
            continue;
        }
        const uint32_t page = A.free_stack[pg];
        const uint32_t b = sb;
        const uint64_t boff = __ldg(&A.P.buf[b].off), bsz = __ldg(&A.P.buf[b].size);
        const uint64_t rel0 = (uint64_t)(p - __ldg(&A.page_base[b])) << 12;
        const int32_t wr = __ldg(&A.P.buf[b].writer);
        const bool zero = wr >= 0 && (int64_t)wr > (int64_t)t;            // writer rule, golden after t
        uint4* dst = reinterpret_cast<uint4*>(A.pool + (size_t)page * kPageWords);
        for (uint32_t q = threadIdx.x; q < kPageWords / 4; q += blockDim.x) {
            const uint64_t rel = rel0 + 16ull * q;
            uint4 g = make_uint4(0, 0, 0, 0);
            if (!zero && rel < bsz) g = __ldg(reinterpret_cast<const uint4*>(A.img + boff + rel));
            dst[q] = g;
        }
        __syncthreads();
        if (threadIdx.x == 0) {
            __threadfence();
            A.ptab[(size_t)s * A.total_pages + p] = page;
            atomicAdd(&A.bcount[(size_t)s * A.n_buf + b], 1u);
            atomicAdd(&A.slot[s].npages, 1u);
        }
        __syncthreads();
    }
}

// ---- write the updates (non-foreign ones touch distinct words across warps)
__global__ void k8_apply(K8Args A) {
    const uint32_t s = blockIdx.y;
    const uint32_t n = min(A.slot[s].pend_n, A.pend_cap);
    const fi_store* pend = A.pend + (size_t)s * A.pend_cap;
    const uint32_t* pt = A.ptab + (size_t)s * A.total_pages;
    for (uint32_t j = blockIdx.x * blockDim.x + threadIdx.x; j < n; j += gridDim.x * blockDim.x) {
        const fi_store f = pend[j];
        if (f.step & 0x80000000u) continue;
        uint32_t b, w;
        const uint32_t p = page_of(A, f.va, b, w);
        const uint32_t e = pt[p];
        if (e < kPageClaim) A.pool[(size_t)e * kPageWords + w] = f.value;
    }
}

// ---- foreign updates: among all updates of the word — the pending ones and the
//      golden warp's (which may have been dropped as a no-op) — the one from the
//      highest warp index wins (C-14)
__global__ void __launch_bounds__(32) k8_foreign(K8Args A, uint32_t t) {
    const uint32_t s = blockIdx.x, lane = threadIdx.x;
    const uint32_t nf = min(A.slot[s].for_n, kForeignCap);
    if (!nf) return;
    const uint32_t n = min(A.slot[s].pend_n, A.pend_cap);
    const fi_store* pend = A.pend + (size_t)s * A.pend_cap;
    const uint32_t* pt = A.ptab + (size_t)s * A.total_pages;
    const fi_instance in = A.P.inst[t];
    const uint64_t g0 = A.gst_off[in.warp_begin], g1 = A.gst_off[in.warp_end];
    for (uint32_t q = 0; q < nf; ++q) {
        const fi_store f = A.forn[(size_t)s * kForeignCap + q];
        uint32_t mx = 0;
        for (uint32_t j = lane; j < n; j += 32)
            if (pend[j].va == f.va) mx = max(mx, (pend[j].step & 0x7FFFFFFFu) + 1);
        for (uint64_t j = g0 + lane; j < g1; j += 32)
            if (A.gst[j].va == f.va) {                 // golden writer of the word: its warp
                uint32_t lo = in.warp_begin, hi = in.warp_end;
                while (hi - lo > 1) {
                    const uint32_t mid = (lo + hi) / 2;
                    if (A.gst_off[mid] <= j) lo = mid; else hi = mid;
                }
                mx = max(mx, lo - in.warp_begin + 1);
            }
        mx = __reduce_max_sync(kFull, mx);
        if (lane == 0 && mx == (f.step & 0x7FFFFFFFu) + 1) {
            uint32_t b, w;
            const uint32_t p = page_of(A, f.va, b, w);
            const uint32_t e = pt[p];
            if (e < kPageClaim) A.pool[(size_t)e * kPageWords + w] = f.value;
        }
        __syncwarp();
    }
}

// ---- return pages equal to the golden state (buffers t writes) and the pages of
//      buffers past their last reference; a slot without pages is Masked.  One
//      warp per page.
__global__ void __launch_bounds__(1024) k8_gc(K8Args A, uint32_t t) {
    const uint32_t s = blockIdx.x;
    Slot& z = A.slot[s];
    if (!z.alive || z.k0 > t) return;
    const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5, nwb = blockDim.x >> 5;
    uint32_t* pt = A.ptab + (size_t)s * A.total_pages;
    const uint32_t* ib = A.P.ib + (size_t)t * (kInstBufs + 1);
    const uint32_t nref = __ldg(&ib[0]) > kInstBufs ? 0u : __ldg(&ib[0]);
    const uint32_t d0 = __ldg(&A.dying_off[t]), d1 = __ldg(&A.dying_off[t + 1]);
    for (uint32_t q = 0; q < nref + (d1 - d0); ++q) {
        const bool dying = q >= nref;
        const uint32_t b = dying ? __ldg(&A.dying[d0 + q - nref]) : __ldg(&ib[1 + q]);
        if (!dying && __ldg(&A.P.buf[b].writer) != (int32_t)t) continue;   // unchanged by t's golden stores
        if (A.bcount[(size_t)s * A.n_buf + b] == 0) continue;
        const uint32_t pb = __ldg(&A.page_base[b]), pe = __ldg(&A.page_base[b + 1]);
        for (uint32_t p = pb + wib; p < pe; p += nwb) {
            const uint32_t e = pt[p];
            if (e >= kPageClaim) continue;
            const bool diff = page_differs(A, e, b, p, t);
            if (lane == 0 && (dying || !diff)) {
                pt[p] = kPageNone;
                A.free_stack[atomicAdd(A.free_top, 1)] = e;
                atomicSub(&A.bcount[(size_t)s * A.n_buf + b], 1u);
                atomicSub(&z.npages, 1u);
                if (dying && diff) atomicOr(&A.dropped[(size_t)s * A.dwords + (b >> 5)], 1u << (b & 31));
            }
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        if (z.fault_key != ~0ull) z.alive = 0;                       // DUE (C-9, C-10): nothing left to decide
        else if (z.npages == 0 && !z.perm) z.alive = 0;              // golden state again: Masked from here on
    }
}

// ---- outcome of every slot of the batch
__global__ void __launch_bounds__(256) k8_final(K8Args A) {
    const uint32_t s = blockIdx.x;
    Slot& z = A.slot[s];
    if (z.rep == kNoRep) return;
    __shared__ uint32_t sdc, beyond;
    if (threadIdx.x == 0) { sdc = 0; beyond = 0; }
    __syncthreads();
    const bool tol = A.rtol > 0.0 && !z.perm;
    uint32_t outcome = z.outcome;
    if (z.overflow || z.inexact) outcome = 0xFF;
    else if (z.fault_key != ~0ull) outcome = FI_DUE;
    else if (outcome == FI_MASKED) {
        // the dense compare of the replica's remaining output pages with the golden
        // final image; with rtol > 0 every differing ELEMENT (buffer dtype; an f64's
        // two words lie in one page) is also checked against rtol (C-12)
        const uint32_t* pt = A.ptab + (size_t)s * A.total_pages;
        for (uint32_t b = 0; b < A.n_buf; ++b) {
            const uint32_t bf = __ldg(&A.P.buf[b].flags);
            if (!(bf & 1u) || A.bcount[(size_t)s * A.n_buf + b] == 0) continue;
            const uint32_t dt = buf_dtype(bf);
            const uint32_t pb = __ldg(&A.page_base[b]), pe = __ldg(&A.page_base[b + 1]);
            const uint64_t boff = __ldg(&A.P.buf[b].off), bsz = __ldg(&A.P.buf[b].size);
            for (uint32_t p = pb; p < pe; ++p) {
                const uint32_t e = pt[p];
                if (e >= kPageClaim) continue;
                const uint64_t rel0 = (uint64_t)(p - pb) << 12;
                const uint32_t* pw = A.pool + (size_t)e * kPageWords;
                for (uint32_t w = threadIdx.x; w < kPageWords; w += blockDim.x) {
                    const uint64_t rel = rel0 + 4ull * w;
                    if (rel >= bsz) continue;
                    const uint64_t va = kVaBase + boff + rel;
                    const uint32_t v = __ldcg(&pw[w]), g = gword(A.img, va);
                    if (v == g) continue;
                    sdc = 1;
                    if (!tol) continue;
                    bool bt;
                    if (dt != 2) {
                        bt = beyond_tol(dt, v, g, A.rtol);
                    } else {
                        const uint32_t w0 = w & ~1u;
                        const uint64_t lo = va - 4ull * (w - w0);
                        bt = beyond_tol(2, (uint64_t)__ldcg(&pw[w0]) | ((uint64_t)__ldcg(&pw[w0 + 1]) << 32),
                                        (uint64_t)gword(A.img, lo) | ((uint64_t)gword(A.img, lo + 4) << 32), A.rtol);
                    }
                    if (bt) beyond = 1;
                }
            }
        }
        __syncthreads();
        outcome = sdc ? FI_SDC : FI_MASKED;
    }
    const bool within = tol && outcome == FI_SDC && !beyond;
    if (threadIdx.x == 0) {
        fi_inj& r = A.inj[z.rep];
        if (z.perm) { r = fi_inj{}; r.mask = A.pf[z.rep].mask; }
        const bool pdue = z.pdue || z.pdue_key != ~0ull;
        if (!r.fault_kind) {                                         // first downstream fault, run order
            const unsigned long long key = z.fault_key != ~0ull ? z.fault_key : z.pdue_key;
            if (key != ~0ull) { r.fault_kind = (uint8_t)((key >> 16) & 7u); r.fault_pc = (uint32_t)(key & 0xFFFFu); }
        }
        r.outcome = (uint8_t)outcome;
        r.flags = ((pdue && outcome != FI_DUE && outcome != FI_NOT_INJECTED && outcome != 0xFF) ? FI_POTENTIAL_DUE : 0u) |
                  (within ? FI_SDC_WITHIN_TOL : 0u);
        if (outcome == 0xFF) {
            r.flags = (z.overflow ? FI_UNCLASSIFIED_CAPACITY : 0u) | (z.inexact ? FI_UNCLASSIFIED_WILD : 0u);
            if (z.overflow) FI_DEV_ERR(A.status, FI_E_CAPACITY);
        }
        else if (z.perm)                                             // opcode-weighted outcomes
            atomicAdd((unsigned long long*)&A.hist[outcome],
                      (unsigned long long)(A.opw ? A.opw[A.pf[z.rep].opcode & (FI_NOPS - 1)] : 1ull));
        else if (outcome != FI_NOT_INJECTED) {
            const fi_site S = A.sites[z.rep];
            atomicAdd((unsigned long long*)&A.hist[((uint32_t)S.group * 4 + S.bfm) * 3 + outcome], 1ull);
        }
    }
}

}  // namespace
}  // namespace fi

using namespace fi;

namespace {
struct K8Layout { size_t steps, slot, ptab, bcount, dropped, pool, fstack, ftop, pend, forn, active, nact, work, need, nneed,
                  scratch, page_base, last_ref, dying_off, dying, reps, kop, total; };
K8Layout k8_layout(uint64_t image_bytes, uint32_t n_buf, uint32_t n_inst, uint32_t n, uint32_t B, uint32_t pool_pages,
                   uint32_t pend_cap, uint32_t log_cap, uint32_t scratch_warps) {
    const uint64_t tp = image_bytes / 4096 + n_buf + 1;          // >= sum of per-buffer pages
    const uint32_t dw = (n_buf + 31) / 32;
    K8Layout L;
    size_t o = 0;
    auto take = [&](size_t bytes) { const size_t r = o; o += align256(bytes); return r; };
    L.steps = take(8);                               // offset 0: emulated warp-steps of the JIT re-execution (fi.h)
    L.slot = take((size_t)B * sizeof(Slot));
    L.ptab = take((size_t)B * tp * 4);
    L.bcount = take((size_t)B * n_buf * 4);
    L.dropped = take((size_t)B * dw * 4);
    L.pool = take((size_t)pool_pages * 4096);
    L.fstack = take((size_t)pool_pages * 4);
    L.ftop = take(8);
    L.pend = take((size_t)B * pend_cap * sizeof(fi_store));
    L.forn = take((size_t)B * kForeignCap * sizeof(fi_store));
    L.active = take((size_t)B * 4);
    L.nact = take(4);
    L.work = take(4);
    L.need = take((size_t)pool_pages * 8);
    L.nneed = take(4);
    L.scratch = take((size_t)scratch_warps * log_cap * sizeof(fi_store));
    L.page_base = take(((size_t)n_buf + 1) * 4);
    L.last_ref = take((size_t)n_buf * 4);
    L.dying_off = take(((size_t)n_inst + 1) * 4);
    L.dying = take((size_t)n_buf * 4);
    L.reps = take((size_t)n * 4);
    L.kop = take(4096);
    L.total = o;
    return L;
}
uint32_t k8_scratch_warps() {
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return (uint32_t)std::max(sms, 1) * 16 * kWPB8;               // >= resident warps of k8_exec
}
}  // namespace

extern "C" size_t fi_classify_batched_workspace(const fi_program* p, uint32_t n, uint32_t log_cap, uint32_t batch,
                                                uint32_t pool_pages, uint32_t pend_cap) {
    if (!p || !batch || !pool_pages || !pend_cap) return 0;
    return k8_layout(p->image_bytes, p->n_buf, p->n_inst, n, batch, pool_pages, pend_cap, log_cap,
                     k8_scratch_warps()).total;
}

static fi_status k8_run(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                        const fi_pfault* pf, const uint64_t* opw, uint32_t n, fi_inj* out, const fi_store* log,
                        uint32_t log_cap, uint64_t* hist, uint32_t flags, double rtol, uint64_t* hist_tol,
                        uint32_t batch, uint32_t pool_pages,
                        uint32_t pend_cap, void* ws, size_t ws_bytes, uint32_t* dev_status, void* stream,
                        const fi_jit* jit = nullptr) {
    if (jit && pf) return FI_E_ARG;                  // the JIT engine serves transient faults
    if (!p || !image || !t || (!sites && !pf) || !out || !hist || !dev_status || !p->aux || !p->inst_host ||
        !p->code_host)
        return FI_E_ARG;
    if (n == 0) return FI_OK;
    if (!batch || !pool_pages || !pend_cap) return FI_E_ARG;
    const uint32_t sw = k8_scratch_warps();
    const K8Layout L = k8_layout(p->image_bytes, p->n_buf, p->n_inst, n, batch, pool_pages, pend_cap, log_cap, sw);
    if (!ws || ws_bytes < L.total) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    fi_status e;
    // ---- host-side tables: per-buffer page numbering, last reference, dying lists
    std::vector<fi_buffer> bufs(p->n_buf);
    std::vector<uint32_t> ib((size_t)p->n_inst * (kInstBufs + 1));
    std::vector<fi_site> hs(sites ? n : 0);
    const AuxLayout AL = aux_layout(p->image_bytes, p->n_code, p->n_inst);
    if ((e = cuda_status(cudaMemcpyAsync(bufs.data(), p->buf, bufs.size() * sizeof(fi_buffer), cudaMemcpyDeviceToHost, s))) ||
        (e = cuda_status(cudaMemcpyAsync(ib.data(), reinterpret_cast<const char*>(p->aux) + AL.ib, ib.size() * 4,
                                         cudaMemcpyDeviceToHost, s))) ||
        (sites && (e = cuda_status(cudaMemcpyAsync(hs.data(), sites, (size_t)n * sizeof(fi_site),
                                                   cudaMemcpyDeviceToHost, s)))) ||
        (e = cuda_status(cudaStreamSynchronize(s))))
        return e;
    std::vector<uint32_t> page_base(p->n_buf + 1, 0), last_ref(p->n_buf, 0);
    for (uint32_t b = 0; b < p->n_buf; ++b) page_base[b + 1] = page_base[b] + (uint32_t)((bufs[b].size + 4095) / 4096);
    bool unknown = false;
    for (uint32_t k = 0; k < p->n_inst; ++k) {
        const uint32_t c = ib[(size_t)k * (kInstBufs + 1)];
        if (c > kInstBufs) { unknown = true; continue; }
        for (uint32_t q = 0; q < c; ++q) {
            const uint32_t b = ib[(size_t)k * (kInstBufs + 1) + 1 + q];
            last_ref[b] = std::max(last_ref[b], k);
        }
    }
    std::vector<uint32_t> dying_off(p->n_inst + 1, 0), dying;
    {
        std::vector<std::vector<uint32_t>> per(p->n_inst);
        for (uint32_t b = 0; b < p->n_buf; ++b) {
            if (unknown || (bufs[b].flags & 1u)) { last_ref[b] = p->n_inst; continue; }   // never dropped
            per[last_ref[b]].push_back(b);
        }
        for (uint32_t k = 0; k < p->n_inst; ++k) {
            dying_off[k + 1] = dying_off[k] + (uint32_t)per[k].size();
            dying.insert(dying.end(), per[k].begin(), per[k].end());
        }
    }
    // replicas in order of their faulty instance, batched
    std::vector<uint32_t> order(n);
    for (uint32_t i = 0; i < n; ++i) order[i] = i;
    if (sites)
        std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return hs[a].instance < hs[b].instance; });
    // per static kernel: which opcodes it contains (permanent faults arm only where the opcode runs)
    if (p->n_kern > 1024) return FI_E_ARG;
    std::vector<uint32_t> kop(std::max<uint32_t>(p->n_kern, 1), 0);
    {
        std::vector<fi_kernel> kh(p->n_kern);
        if (p->n_kern &&
            (e = cuda_status(cudaMemcpy(kh.data(), p->kern, kh.size() * sizeof(fi_kernel), cudaMemcpyDeviceToHost))))
            return e;
        for (uint32_t k = 0; k < p->n_kern; ++k)
            for (uint32_t q = 0; q < kh[k].code_len; ++q) kop[k] |= 1u << (p->code_host[kh[k].code_off + q].op & 31);
    }

    char* w = reinterpret_cast<char*>(ws);
    K8Args A;
    A.P = make_emu_prog(p);
    A.img = image; A.warp_off = t->warp_off; A.gst_off = t->gstore_off; A.gst = t->gstore;
    A.sites = sites; A.inj = out; A.log = log; A.log_cap = log_cap;
    A.slot = reinterpret_cast<Slot*>(w + L.slot); A.B = batch;
    A.ptab = reinterpret_cast<uint32_t*>(w + L.ptab); A.total_pages = page_base[p->n_buf];
    A.bcount = reinterpret_cast<uint32_t*>(w + L.bcount);
    A.dropped = reinterpret_cast<uint32_t*>(w + L.dropped); A.dwords = (p->n_buf + 31) / 32;
    A.pool = reinterpret_cast<uint32_t*>(w + L.pool);
    A.free_stack = reinterpret_cast<uint32_t*>(w + L.fstack); A.free_top = reinterpret_cast<int*>(w + L.ftop);
    A.pool_pages = pool_pages;
    A.page_base = reinterpret_cast<uint32_t*>(w + L.page_base);
    A.last_ref = reinterpret_cast<uint32_t*>(w + L.last_ref); A.n_buf = p->n_buf;
    A.pend = reinterpret_cast<fi_store*>(w + L.pend); A.pend_cap = pend_cap;
    A.forn = reinterpret_cast<fi_store*>(w + L.forn);
    A.active = reinterpret_cast<uint32_t*>(w + L.active); A.n_active = reinterpret_cast<uint32_t*>(w + L.nact);
    A.work = reinterpret_cast<uint32_t*>(w + L.work);
    A.need = reinterpret_cast<uint2*>(w + L.need); A.n_need = reinterpret_cast<uint32_t*>(w + L.nneed);
    A.need_cap = pool_pages;
    A.scratch = reinterpret_cast<fi_store*>(w + L.scratch);
    A.dying_off = reinterpret_cast<uint32_t*>(w + L.dying_off);
    A.dying = reinterpret_cast<uint32_t*>(w + L.dying);
    A.flags = flags; A.status = dev_status; A.hist = hist;
    A.pf = pf; A.opw = opw;
    A.kop = reinterpret_cast<uint32_t*>(w + L.kop);
    A.rtol = rtol;
    uint32_t* d_reps = reinterpret_cast<uint32_t*>(w + L.reps);
    if ((e = cuda_status(cudaMemcpyAsync(const_cast<uint32_t*>(A.page_base), page_base.data(), page_base.size() * 4, cudaMemcpyHostToDevice, s))) ||
        (e = cuda_status(cudaMemcpyAsync(const_cast<uint32_t*>(A.last_ref), last_ref.data(), last_ref.size() * 4, cudaMemcpyHostToDevice, s))) ||
        (e = cuda_status(cudaMemcpyAsync(const_cast<uint32_t*>(A.dying_off), dying_off.data(), dying_off.size() * 4, cudaMemcpyHostToDevice, s))) ||
        (!dying.empty() &&
         (e = cuda_status(cudaMemcpyAsync(const_cast<uint32_t*>(A.dying), dying.data(), dying.size() * 4, cudaMemcpyHostToDevice, s)))) ||
        (e = cuda_status(cudaMemcpyAsync(const_cast<uint32_t*>(A.kop), kop.data(), kop.size() * 4,
                                         cudaMemcpyHostToDevice, s))) ||
        (e = cuda_status(cudaMemcpyAsync(d_reps, order.data(), (size_t)n * 4, cudaMemcpyHostToDevice, s))))
        return e;

    const size_t smem = golden_smem(p->n_regs);
    if ((e = cuda_status(cudaFuncSetAttribute((const void*)k8_exec, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem))))
        return e;
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k8_exec, kWPB8 * 32, smem);
    const uint32_t exec_grid = std::min<uint32_t>((uint32_t)std::max(1, sms * std::max(1, per)), sw / kWPB8);
    const uint32_t fix_grid = (uint32_t)std::max(1, sms * 4);
    JK8Host JK{A.warp_off, A.gst_off, A.gst, A.slot, A.ptab, A.total_pages, A.pool, A.page_base, A.last_ref,
               A.dropped, A.dwords, A.pend, A.pend_cap, A.forn, kForeignCap, A.active, A.n_active, A.work,
               A.scratch, A.log_cap, A.flags, A.status, reinterpret_cast<unsigned long long*>(w + L.steps),
               A.bcount, A.n_buf};
    if ((e = cuda_status(cudaMemsetAsync(w + L.steps, 0, 8, s)))) return e;

    for (uint32_t b0 = 0; b0 < n; b0 += batch) {
        const uint32_t nb = std::min(batch, n - b0);
        const uint32_t kmin = sites ? hs[order[b0]].instance : 0u;
        if ((e = cuda_status(cudaMemsetAsync(A.ptab, 0xFF, (size_t)batch * A.total_pages * 4, s))) ||
            (e = cuda_status(cudaMemsetAsync(A.bcount, 0, (size_t)batch * p->n_buf * 4, s))) ||
            (e = cuda_status(cudaMemsetAsync(A.dropped, 0, (size_t)batch * A.dwords * 4, s))))
            return e;
        k8_free_init<<<(pool_pages + 255) / 256, 256, 0, s>>>(A.free_stack, A.free_top, pool_pages);
        k8_setup<<<(batch + 127) / 128, 128, 0, s>>>(A, d_reps + b0, nb);
        if ((e = launch_status())) return e;
        for (uint32_t tt = kmin; tt < p->n_inst; ++tt) {
            k8_activate<<<1, 1024, 0, s>>>(A, tt);
            if (tt > kmin || pf) {
                if (jit) {
                    if ((e = jit_k8_exec(jit, p, image, JK, tt, sw / kWPB8, s))) return e;
                } else {
                    k8_exec<<<exec_grid, kWPB8 * 32, smem, s>>>(A, tt);
                }
            }
            k8_k0<<<(batch + kWPB8 - 1) / kWPB8, kWPB8 * 32, 0, s>>>(A, tt);
            k8_mark<<<dim3(std::max<uint32_t>(1, fix_grid / batch + 1), batch), 256, 0, s>>>(A);
            k8_alloc<<<fix_grid, 256, 0, s>>>(A, tt);
            k8_apply<<<dim3(std::max<uint32_t>(1, fix_grid / batch + 1), batch), 256, 0, s>>>(A);
            k8_foreign<<<batch, 32, 0, s>>>(A, tt);
            k8_gc<<<batch, 1024, 0, s>>>(A, tt);
            if ((e = launch_status())) return e;
        }
        k8_final<<<batch, 256, 0, s>>>(A);
        if ((e = launch_status())) return e;
    }
    if (rtol > 0.0 && sites) return launch_hist_tol(sites, out, n, hist_tol, s);
    return FI_OK;
}

extern "C" fi_status fi_classify_batched(const fi_program* p, const uint8_t* image, const fi_trace* t,
                                         const fi_site* sites, uint32_t n, fi_inj* out, const fi_store* log,
                                         uint32_t log_cap, uint64_t* hist, uint32_t flags, double rtol,
                                         uint64_t* hist_tol, uint32_t batch, uint32_t pool_pages, uint32_t pend_cap,
                                         void* ws, size_t ws_bytes, uint32_t* dev_status, void* stream) {
    if (!sites || !(rtol >= 0.0)) return FI_E_ARG;
    return k8_run(p, image, t, sites, nullptr, nullptr, n, out, log, log_cap, hist, flags, rtol, hist_tol, batch,
                  pool_pages, pend_cap, ws, ws_bytes, dev_status, stream);
}

extern "C" fi_status fi_classify_batched_jit(const fi_jit* j, const fi_program* p, const uint8_t* image,
                                             const fi_trace* t, const fi_site* sites, uint32_t n, fi_inj* out,
                                             const fi_store* log, uint32_t log_cap, uint64_t* hist, uint32_t flags,
                                             double rtol, uint64_t* hist_tol, uint32_t batch, uint32_t pool_pages,
                                             uint32_t pend_cap, void* ws, size_t ws_bytes, uint32_t* dev_status,
                                             void* stream) {
    if (!sites || !j || !(rtol >= 0.0)) return FI_E_ARG;
    return k8_run(p, image, t, sites, nullptr, nullptr, n, out, log, log_cap, hist, flags, rtol, hist_tol, batch,
                  pool_pages, pend_cap, ws, ws_bytes, dev_status, stream, j);
}

extern "C" fi_status fi_inject_permanent_batched(const fi_program* p, const uint8_t* image, const fi_trace* t,
                                                 const fi_pfault* faults, uint32_t n, const uint64_t* op_weights,
                                                 fi_inj* out, uint32_t log_cap, uint64_t* hist, uint32_t flags,
                                                 uint32_t batch, uint32_t pool_pages, uint32_t pend_cap, void* ws,
                                                 size_t ws_bytes, uint32_t* dev_status, void* stream) {
    if (!faults) return FI_E_ARG;
    return k8_run(p, image, t, nullptr, faults, op_weights, n, out, nullptr, log_cap, hist, flags, 0.0, nullptr,
                  batch, pool_pages, pend_cap, ws, ws_bytes, dev_status, stream);
}
