// propagate.cu — K7: outcome of an injected run of a MULTI-instance program.
//
// PAPER.md:72 step (4) / :206 compares the whole program's outputs with the
// golden run, so a corrupted intermediate buffer matters only through the later
// kernels that read it.  Per replica (one CUDA warp, persistent over replicas):
//   1. the faulty warp's result in its instance k (from K4's store log and the
//      golden store log, C-14) is turned into updates of a per-replica
//      faulty-memory overlay D (word -> current value; every word not in D has
//      its golden value);
//   2. for every later instance k' in launch order: if none of D's buffers is
//      referenced by k' (its constant bank's pointers, prepared in aux), k' runs
//      exactly as in the golden run and is skipped; otherwise every warp of k' is
//      re-executed by the emulator (EMU_PROP: loads see D), and its stores —
//      against its golden store log — become updates, applied at the end of k'
//      (C-14 visibility);
//   3. DUE if a re-executed warp faults or hangs (C-9, C-10; under FI_UNCHECKED
//      only hangs), else SDC iff some output word of D differs from the golden
//      final image (C-12), else Masked.  D empty of differences => Masked early.
// Exact given the program model: a warp that reads no word of D executes as in
// the golden run, and SSA buffers (§3.5) make the golden state before any
// instance a function of the final image.
#include <algorithm>

#include "emu.cuh"

namespace fi {
size_t golden_smem(uint32_t n_regs);
namespace {

constexpr int kWPB = 4;
constexpr uint32_t kDirtyBufs = 32;                  // tracked dirty buffer ids (more -> never skip)

struct PropArgs {
    EmuProg P;
    const uint8_t* img;
    const uint64_t* warp_off; const uint64_t* gst_off; const fi_store* gst;
    const fi_site* sites; fi_inj* inj; uint32_t n; uint32_t n_inst;
    fi_store* log; uint32_t cap;                     // per replica K4 log (reused for re-executed warps)
    const uint32_t* order; uint32_t* counter;
    uint4* ov; uint32_t ov_cap;                      // per warp-slot overlay
    fi_store* pend; uint32_t pend_cap;               // per warp-slot pending updates
    uint32_t* dbuf;                                  // per warp-slot: [count, ids...]
    uint32_t* ov_list; uint32_t list_cap;            // per warp-slot: slots in use (for scans)
    uint64_t* hist; uint32_t flags; uint32_t* status;
    const fi_pfault* pf;                             // permanent / intermittent faults (rows f2/f3), else null
    const uint64_t* opw;                             // opcode weights [FI_NOPS] or null
    double rtol;                                     // > 0: C-12 secondary numeric classification
};

__device__ __forceinline__ uint32_t buf_id(const EmuProg& P, uint64_t va) { return __ldg(&P.gran[(va - kVaBase) >> 8]); }
__device__ __forceinline__ uint32_t gword(const uint8_t* img, uint64_t va) {
    return __ldg(reinterpret_cast<const uint32_t*>(img + (va - kVaBase)));
}
// golden value of word va after instance t (t = -1: the initial image)
__device__ __forceinline__ uint32_t gstate(const EmuProg& P, const uint8_t* img, uint64_t va, int64_t t) {
    const int32_t wr = __ldg(&P.buf[buf_id(P, va)].writer);
    return (wr >= 0 && (int64_t)wr > t) ? 0u : gword(img, va);
}

// insert or update va -> v in the overlay (generation-tagged slots, so no clearing
// between replicas); returns false when full.  Called by one lane at a time.
__device__ bool ov_put(uint4* tab, uint32_t mask, uint32_t gen, uint64_t va, uint32_t v, uint32_t* list,
                       uint32_t* list_n, uint32_t list_cap) {
    uint32_t h = ov_hash(va) & mask;
    for (uint32_t p = 0; p <= mask; ++p) {
        uint4 e = __ldcg(&tab[h]);
        if (e.w != gen) {
            if (*list_n >= list_cap) return false;
            tab[h] = make_uint4((uint32_t)va, (uint32_t)(va >> 32), v, gen);
            list[(*list_n)++] = h;
            return true;
        }
        if (e.x == (uint32_t)va && e.y == (uint32_t)(va >> 32)) {
            tab[h].z = v;
            return true;
        }
        h = (h + 1) & mask;
    }
    return false;
}

// current faulty value of word va before instance t (overlay, else golden)
__device__ __forceinline__ uint32_t cur_value(const PropArgs& A, const Overlay& ov, uint64_t va, int64_t t) {
    uint32_t v;
    if (ov_find(ov, va, v)) return v;
    return gstate(A.P, A.img, va, t - 1);
}

// Updates of one warp's execution in instance t: faulty stores F (program order,
// last write wins) and golden stores G of the same warp that F does not repeat
// (their words keep the value they had before t).  Appended to the pending list.
// Returns false on pending overflow.
__device__ bool warp_updates(const PropArgs& A, const Overlay& ov, const fi_store* F, uint64_t nF, const fi_store* G,
                             uint64_t nG, int64_t t, fi_store* pend, uint32_t& np) {
    const uint32_t lane = threadIdx.x & 31;
    for (uint64_t b = 0; b < nF; b += 32) {
        const uint64_t j = b + lane;
        bool keep = false;
        fi_store f{};
        if (j < nF) {
            f = F[j];
            keep = true;
            for (uint64_t q = j + 1; q < nF && keep; ++q) keep = F[q].va != f.va;
        }
        const uint32_t m = __ballot_sync(kFull, keep);
        const uint32_t pos = np + __popc(m & ((1u << lane) - 1));
        if (keep && pos < A.pend_cap) pend[pos] = f;
        np += __popc(m);
    }
    for (uint64_t b = 0; b < nG; b += 32) {
        const uint64_t j = b + lane;
        bool keep = false;
        fi_store gnew{};
        if (j < nG) {
            const uint64_t va = G[j].va;
            bool inF = false;
            for (uint64_t q = 0; q < nF && !inF; ++q) inF = F[q].va == va;
            if (!inF) {
                keep = true;
                gnew.va = va;
                gnew.value = cur_value(A, ov, va, t);
            }
        }
        const uint32_t m = __ballot_sync(kFull, keep);
        const uint32_t pos = np + __popc(m & ((1u << lane) - 1));
        if (keep && pos < A.pend_cap) pend[pos] = gnew;
        np += __popc(m);
    }
    return np <= A.pend_cap;
}

__global__ void __launch_bounds__(kWPB * 32) k_propagate(const PropArgs A) {
    extern __shared__ uint32_t smem[];
    const uint32_t wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t slot = blockIdx.x * kWPB + wib;
    uint4* tab = A.ov + (size_t)slot * A.ov_cap;
    fi_store* pend = A.pend + (size_t)slot * A.pend_cap;
    uint32_t* dbuf = A.dbuf + (size_t)slot * (kDirtyBufs + 1);
    uint32_t* list = A.ov_list + (size_t)slot * (A.list_cap + 1);
    Overlay ov{tab, A.ov_cap - 1, 0};
    uint32_t* R = smem + wib * (A.P.n_regs + 1) * 32;
    const uint32_t* ibl = nullptr;
    for (;;) {
        uint32_t p = 0;
        if (lane == 0) p = atomicAdd(A.counter, 1u);
        p = __shfl_sync(kFull, p, 0);
        if (p >= A.n) return;
        const uint32_t i = A.order[p];
        const uint32_t gen = p + 1;
        ov.gen = gen;
        const bool permanent = A.pf != nullptr;
        const fi_site S = permanent ? fi_site{} : A.sites[i];
        const fi_inj Rj = permanent ? fi_inj{} : A.inj[i];
        const fi_pfault PF = permanent ? A.pf[i] : fi_pfault{};
        const uint32_t nsm = PF.n_sm ? PF.n_sm : 148u;      // CTA c runs on SM c mod n_sm (C-21)
        uint32_t outcome = FI_MASKED, fkind = 0, fpc = 0;
        bool pdue = false, overflow = false, within = false;
        const bool unchecked = A.flags & FI_UNCHECKED;
        if (S.flags & FI_SITE_NOT_INJECTED) {
            outcome = FI_NOT_INJECTED;
        } else if (Rj.overflow) {
            outcome = 0xFF;
        } else if (Rj.fault_kind && !(unchecked && Rj.fault_kind != 3)) {
            outcome = FI_DUE;
        } else {
            pdue = Rj.fault_kind != 0;
            uint32_t ndb = 0, nlist = 0;
            bool db_over = false;
            uint32_t np = 0;
            bool ok = true;
            int64_t t = -1;
            if (!permanent) {
                // ---- 1. the faulty warp's instance
                const fi_store* G = A.gst + A.gst_off[S.warp];
                const uint64_t nGall = A.gst_off[S.warp + 1] - A.gst_off[S.warp];
                uint64_t gs = 0;
                for (uint64_t b = 0; b < nGall; b += 32) {
                    const bool after = b + lane < nGall && G[b + lane].step > S.step;
                    const uint32_t m = __ballot_sync(kFull, after);
                    if (m) { gs = b + __ffs(m) - 1; break; }
                    gs = min(b + 32, nGall);
                }
                ok = warp_updates(A, ov, A.log + (uint64_t)i * A.cap, Rj.n_faulty_stores, G + gs, nGall - gs,
                                  S.instance, pend, np);
                t = S.instance;
            }
            bool done = false;
            while (!done) {
                // ---- apply the pending updates of instance t (end-of-instance visibility)
                if (!ok) { overflow = true; break; }
                for (uint32_t u = 0; u < np && !overflow; ++u) {
                    if (lane == 0) {
                        const fi_store f = pend[u];
                        if (!ov_put(tab, ov.mask, gen, f.va, f.value, list + 1, &nlist, A.list_cap)) overflow = true;
                        if (f.value != gstate(A.P, A.img, f.va, t)) {
                            const uint32_t bid = buf_id(A.P, f.va);
                            bool have = false;
                            for (uint32_t q = 0; q < ndb; ++q) have |= dbuf[1 + q] == bid;
                            if (!have) { if (ndb < kDirtyBufs) dbuf[1 + ndb++] = bid; else db_over = true; }
                        }
                    }
                    overflow = __shfl_sync(kFull, overflow, 0);
                }
                __syncwarp();
                ndb = __shfl_sync(kFull, ndb, 0);
                nlist = __shfl_sync(kFull, nlist, 0);
                db_over = __shfl_sync(kFull, db_over, 0);
                if (overflow) break;
                // ---- any difference left?  (D empty of differences => Masked from here on)
                bool diff = false;
                for (uint32_t b = 0; b < nlist && !diff; b += 32) {
                    bool d = false;
                    if (b + lane < nlist) {
                        const uint4 e = __ldcg(&tab[list[1 + b + lane]]);
                        const uint64_t va = (uint64_t)e.x | ((uint64_t)e.y << 32);
                        d = e.z != gstate(A.P, A.img, va, t);
                    }
                    diff = __any_sync(kFull, d);
                }
                if (!diff && !permanent) break;              // a permanent fault keeps firing later
                // ---- next instance that references a dirty buffer (or, for a
                //      permanent fault, runs the opcode on the faulty SM)
                int64_t nk = t + 1;
                bool all = false;
                for (; nk < (int64_t)A.n_inst; ++nk) {
                    all = true;
                    if (db_over) break;
                    ibl = A.P.ib + (size_t)nk * (kInstBufs + 1);
                    const uint32_t cnt = __ldg(&ibl[0]);
                    if (cnt > kInstBufs) break;                       // unknown references: run it
                    bool hit = false;
                    for (uint32_t q = lane; q < cnt * kDirtyBufs && !hit; q += 32) {
                        const uint32_t a = q / kDirtyBufs, d = q % kDirtyBufs;
                        hit = d < ndb && __ldg(&ibl[1 + a]) == dbuf[1 + d];
                    }
                    if (__any_sync(kFull, hit)) break;
                    all = false;
                    if (permanent) {
                        const fi_instance ink = A.P.inst[nk];
                        if (PF.sm >= nsm || PF.sm >= ink.grid) continue;              // no CTA of nk runs on the faulty SM
                        const fi_kernel kn = A.P.kern[ink.kernel];
                        bool has = false;
                        for (uint32_t q = lane; q < kn.code_len && !has; q += 32)
                            has = (__ldg(&A.P.dec[kn.code_off + q].x) & 0xFF) == PF.opcode;
                        if (__any_sync(kFull, has)) break;
                    }
                }
                if (nk >= (int64_t)A.n_inst) break;
                // ---- re-execute the warps of instance nk against the overlay: all of
                //      them when it may read dirty words, else the faulty SM's
                t = nk;
                const fi_instance in = A.P.inst[t];
                const uint32_t wpc = (in.block + 31) / 32;
                np = 0;
                for (uint32_t w = in.warp_begin; w < in.warp_end && ok; ++w) {
                    const uint32_t lw = w - in.warp_begin;
                    const bool hooked = permanent && (lw / wpc) % nsm == PF.sm;
                    if (!all && !hooked) continue;
                    const uint64_t L = A.warp_off[w + 1] - A.warp_off[w];
                    const uint64_t wd = 10 * L + 1024;
                    const uint32_t watchdog = wd > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)wd;
                    HookIn h{};
                    if (hooked) {
                        h.perm_on = true; h.perm_op = PF.opcode; h.perm_lane = PF.lane; h.perm_mask = PF.mask;
                        h.perm_q = PF.q32; h.perm_rep = i; h.perm_warp = w; h.perm_seed = PF.seed;
                    }
                    fi_store* flog = A.log + (uint64_t)i * A.cap;
                    const EmuOut o = emulate<EMU_PROP>(A.P, nullptr, A.img, (uint32_t)t, lw / wpc, lw % wpc, R,
                                                       watchdog, nullptr, flog, A.cap, h, nullptr, 0, ov);
                    if (o.fault && !fkind) { fkind = o.fault; fpc = o.fault_pc; }
                    if (o.fault && !(unchecked && o.fault != 3)) {
                        outcome = FI_DUE; fkind = o.fault; fpc = o.fault_pc; done = true; break;
                    }
                    if (o.fault) pdue = true;
                    if (o.nstore > A.cap) { overflow = true; done = true; break; }
                    ok = warp_updates(A, ov, flog, o.nstore, A.gst + A.gst_off[w], A.gst_off[w + 1] - A.gst_off[w],
                                      t, pend, np);
                }
                if (outcome == FI_DUE || overflow) break;
            }
            if (overflow) outcome = 0xFF;
            else if (outcome != FI_DUE) {
                // ---- SDC iff an output word of D differs from the golden final image;
                //      with rtol > 0 also: does some differing output ELEMENT (an f64's
                //      other word from D, else golden) differ beyond rtol (C-12)?
                const bool tol = A.rtol > 0.0 && !permanent;
                bool sdc = false, beyond = false;
                for (uint32_t b = 0; b < nlist && (!sdc || (tol && !beyond)); b += 32) {
                    bool d = false, bt = false;
                    if (b + lane < nlist) {
                        const uint4 e = __ldcg(&tab[list[1 + b + lane]]);
                        const uint64_t va = (uint64_t)e.x | ((uint64_t)e.y << 32);
                        const uint32_t bf = __ldg(&A.P.buf[buf_id(A.P, va)].flags);
                        d = (bf & 1u) && e.z != gword(A.img, va);
                        if (d && tol) {
                            const uint32_t dt = buf_dtype(bf);
                            if (dt != 2) {
                                bt = beyond_tol(dt, e.z, gword(A.img, va), A.rtol);
                            } else {
                                const uint64_t lo = va & ~7ull;
                                uint32_t f0 = gword(A.img, lo), f1 = gword(A.img, lo + 4);
                                ov_find(ov, lo, f0);
                                ov_find(ov, lo + 4, f1);
                                bt = beyond_tol(2, (uint64_t)f0 | ((uint64_t)f1 << 32),
                                                (uint64_t)gword(A.img, lo) | ((uint64_t)gword(A.img, lo + 4) << 32),
                                                A.rtol);
                            }
                        }
                    }
                    sdc |= __any_sync(kFull, d);
                    beyond |= __any_sync(kFull, bt);
                }
                within = tol && sdc && !beyond;
                outcome = sdc ? FI_SDC : FI_MASKED;
            }
        }
        if (lane == 0) {
            if (permanent) {
                fi_inj r = {};
                r.mask = PF.mask;
                r.fault_kind = (uint8_t)fkind;
                r.fault_pc = fpc;
                A.inj[i] = r;
            } else if (!Rj.fault_kind && fkind) {        // first downstream fault, run order
                A.inj[i].fault_kind = (uint8_t)fkind;
                A.inj[i].fault_pc = fpc;
            }
            A.inj[i].outcome = (uint8_t)outcome;
            A.inj[i].flags = ((pdue && outcome != FI_DUE && outcome != FI_NOT_INJECTED) ? FI_POTENTIAL_DUE : 0u) |
                             (within ? FI_SDC_WITHIN_TOL : 0u);
            if (outcome == 0xFF) FI_DEV_ERR(A.status, FI_E_CAPACITY);
            else if (permanent)                     // opcode-weighted outcomes
                atomicAdd((unsigned long long*)&A.hist[outcome],
                          (unsigned long long)(A.opw ? A.opw[PF.opcode & (FI_NOPS - 1)] : 1ull));
            else if (outcome != FI_NOT_INJECTED)
                atomicAdd((unsigned long long*)&A.hist[((uint32_t)S.group * 4 + S.bfm) * 3 + outcome], 1ull);
        }
        __syncwarp();
    }
}

}  // namespace

// Per replica slot: overlay of a power-of-two capacity (load <= 1/2 for
// ov_words differing words; a transient fault's words are bounded by its log),
// the pending-update list of one instance.
void propagate_caps(uint32_t log_cap, uint32_t ov_words, uint32_t& ov_cap, uint32_t& pend_cap) {
    const uint64_t words = std::max<uint64_t>({(uint64_t)log_cap, 4096ull, (uint64_t)ov_words});
    uint64_t c = 1;
    while (c < (ov_words ? 2 : 4) * words) c <<= 1;
    ov_cap = (uint32_t)std::min<uint64_t>(c, 1ull << 31);
    pend_cap = (uint32_t)std::min<uint64_t>(ov_words ? words + 2ull * log_cap : 2 * words, 0xFFFFFFFFull);
}

size_t propagate_slot_bytes(uint32_t ov_cap, uint32_t pend_cap) {
    return (size_t)ov_cap * 16 + (size_t)pend_cap * 16 + (kDirtyBufs + 1) * 4 + ((size_t)ov_cap + 1) * 4;
}

fi_status launch_propagate(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                           uint32_t n, fi_inj* out, const fi_store* log, uint32_t log_cap, uint64_t* hist,
                           uint32_t flags, void* ws, size_t ws_bytes, const uint32_t* order, uint32_t* counter,
                           uint32_t* dev_status, cudaStream_t s, const fi_pfault* pf, const uint64_t* opw,
                           uint32_t ov_words, double rtol) {
    const size_t smem = golden_smem(p->n_regs);
    fi_status e = cuda_status(cudaFuncSetAttribute((const void*)k_propagate, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (e) return e;
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_propagate, kWPB * 32, smem);
    uint32_t ov_cap, pend_cap;
    propagate_caps(log_cap, ov_words, ov_cap, pend_cap);
    const size_t sb = propagate_slot_bytes(ov_cap, pend_cap);
    uint64_t slots = std::min<uint64_t>((uint64_t)std::max(1, sms * std::max(1, per)) * kWPB, ((uint64_t)n + kWPB - 1) / kWPB * kWPB);
    slots = std::min<uint64_t>(slots, ws_bytes / sb / kWPB * kWPB);
    if (slots == 0) return FI_E_ARG;
    char* b = reinterpret_cast<char*>(ws);
    PropArgs A;
    A.P = make_emu_prog(p);
    A.img = image; A.warp_off = t->warp_off; A.gst_off = t->gstore_off; A.gst = t->gstore;
    A.sites = sites; A.inj = out; A.n = n; A.n_inst = p->n_inst;
    A.log = const_cast<fi_store*>(log); A.cap = log_cap;
    A.order = order; A.counter = counter;
    A.ov = reinterpret_cast<uint4*>(b); b += (size_t)slots * ov_cap * 16;
    A.ov_cap = ov_cap;
    A.pend = reinterpret_cast<fi_store*>(b); b += (size_t)slots * pend_cap * 16;
    A.pend_cap = pend_cap;
    A.dbuf = reinterpret_cast<uint32_t*>(b); b += (size_t)slots * (kDirtyBufs + 1) * 4;
    A.ov_list = reinterpret_cast<uint32_t*>(b);
    A.list_cap = ov_cap;
    A.hist = hist; A.flags = flags; A.status = dev_status;
    A.pf = pf; A.opw = opw;
    A.rtol = rtol;
    // generation tags restart at 1 for every call: clear the overlay tables once
    if ((e = cuda_status(cudaMemsetAsync(A.ov, 0, (size_t)slots * ov_cap * 16, s)))) return e;
    k_propagate<<<(unsigned)(slots / kWPB), kWPB * 32, smem, s>>>(A);
    return launch_status();
}

__global__ void k_iota_p(uint32_t* order, uint32_t n, uint32_t* counter) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) order[i] = i;
    if (i == 0) *counter = 0;
}

}  // namespace fi

using namespace fi;

extern "C" size_t fi_inject_permanent_workspace(uint32_t n, uint32_t log_cap, uint32_t ov_words,
                                                uint32_t max_slots) {
    uint32_t ov_cap, pend_cap;
    propagate_caps(log_cap, ov_words, ov_cap, pend_cap);
    const size_t sb = propagate_slot_bytes(ov_cap, pend_cap);
    uint64_t slots = std::min<uint64_t>(((uint64_t)n + 3) / 4 * 4, 148ull * 16);
    if (max_slots) slots = std::min<uint64_t>(slots, ((uint64_t)std::max<uint32_t>(max_slots, 4) + 3) / 4 * 4);
    return 256 + align256((size_t)n * 4) + slots * sb;
}

extern "C" fi_status fi_inject_permanent(const fi_program* p, const uint8_t* image, const fi_trace* t,
                                         const fi_pfault* faults, uint32_t n, const uint64_t* op_weights, fi_inj* out,
                                         fi_store* log, uint32_t log_cap, uint32_t ov_words, uint64_t* hist,
                                         uint32_t flags, void* ws, size_t ws_bytes, uint32_t* dev_status,
                                         void* stream) {
    if (!p || !image || !t || !faults || !out || !log || !hist || !dev_status || !p->aux) return FI_E_ARG;
    if (n == 0) return FI_OK;
    if (!ws || ws_bytes < fi_inject_permanent_workspace(n, log_cap, ov_words, 4)) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    uint32_t* counter = reinterpret_cast<uint32_t*>(ws);
    uint32_t* order = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + 256);
    const size_t head = 256 + align256((size_t)n * 4);
    k_iota_p<<<(n + 255) / 256, 256, 0, s>>>(order, n, counter);
    fi_status e = launch_status();
    if (e) return e;
    return launch_propagate(p, image, t, nullptr, n, out, log, log_cap, hist, flags,
                            reinterpret_cast<char*>(ws) + head, ws_bytes - head, order, counter, dev_status, s,
                            faults, op_weights, ov_words, 0.0);
}
