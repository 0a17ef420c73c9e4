// inject.cu — K4 injection replicas and K5 outcome classification.
//
// K4 ("When that instruction is reached, the injection code will
// corrupt the destination register of the instruction based on the bit-pattern
// selection value"; :138 "corrupting a single destination register of a single
// dynamic instruction"): one CUDA warp per replica re-executes the site's
// synthetic warp from its first instruction over the golden final image (the
// NVBitFI analog of instrumenting only the target dynamic kernel);
// stores after the site go to the replica's log slot.
//
// K5 (Table V [PAPER.md:184-196], [PAPER.md:206]): DUE if the replica crashed
// (memory fault) or hung (watchdog) — C-9, C-10; otherwise the warp's final
// contribution to memory is compared with the golden run (C-12, C-14):
//   D = { a in F : last faulty value(a) != golden(a) }
//     U { a in G_suffix \ F : value before the instance(a) != golden(a) }
// where F is the faulty store log after the site and G_suffix the golden
// warp's stores after the site (stores up to the site are identical in both).
// SDC iff D hits an output buffer, else Masked.
#include <algorithm>

#include "emu.cuh"

namespace fi {
size_t golden_smem(uint32_t n_regs);
namespace {

constexpr int kWPB = 4;

constexpr int kBuckets = 1024;

// Longest-expected-first replica order (LPT scheduling): counting sort, one CTA,
// of the steps each replica must emulate after its restart point.  The golden
// remaining length is the estimate, except for a replica whose corrupted
// register is a loop-control operand (read by an ISETP whose predicate guards a
// backward BRA of the same static kernel): its loop may run longer than the
// golden one, so it goes first (estimate 2x its warp length).  Order only:
// results do not depend on it.
constexpr uint32_t kLptMaxKern = 256;
__global__ void __launch_bounds__(1024)
k_lpt_order(const fi_site* __restrict__ sites, const uint64_t* __restrict__ warp_off, uint32_t ck_interval,
            uint32_t n, uint32_t* __restrict__ order, uint32_t* __restrict__ counter, const fi_insn* __restrict__ code,
            const fi_kernel* __restrict__ kern, uint32_t n_kern) {
    __shared__ uint32_t hist[kBuckets];
    __shared__ uint32_t s_max;
    __shared__ uint32_t ctl[kLptMaxKern][4];         // per static kernel: loop-control registers (bit mask)
    const bool use_ctl = code && kern && n_kern <= kLptMaxKern;
    auto cost = [&](uint32_t i) -> uint64_t {
        const fi_site S = sites[i];
        if (S.flags & FI_SITE_NOT_INJECTED) return 0;
        const uint64_t L = warp_off[S.warp + 1] - warp_off[S.warp];
        if (use_ctl && S.dst_kind == 0 && S.kernel_id < n_kern && S.dst_reg < 128 &&
            ((ctl[S.kernel_id][S.dst_reg >> 5] >> (S.dst_reg & 31)) & 1u))
            return 2 * L;
        const uint64_t start = ck_interval ? (uint64_t)(S.step / ck_interval) * ck_interval : 0;
        return L > start ? L - start : 0;
    };
    for (uint32_t b = threadIdx.x; b < kBuckets; b += blockDim.x) hist[b] = 0;
    if (threadIdx.x == 0) { s_max = 0; *counter = 0; *reinterpret_cast<unsigned long long*>(counter + 2) = 0; }
    if (use_ctl) {
        for (uint32_t q = threadIdx.x; q < n_kern * 4; q += blockDim.x) ctl[q >> 2][q & 3] = 0;
        __syncthreads();
        // one warp per static kernel: each lane takes ISETPs, then scans for a backward
        // BRA guarded by the ISETP's predicate
        const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
        for (uint32_t k = w; k < n_kern; k += blockDim.x >> 5) {
            const fi_kernel K = kern[k];
            for (uint32_t pc = lane; pc < K.code_len; pc += 32) {
                const fi_insn I = code[K.code_off + pc];
                if (I.op != ISETP || (I.d0 & 7) == kPT) continue;
                bool loop = false;
                for (uint32_t q = 0; q < K.code_len && !loop; ++q) {
                    const fi_insn B = code[K.code_off + q];
                    loop = B.op == BRA && (B.guard & 7) == (I.d0 & 7) && B.imm <= q;
                }
                if (!loop) continue;
                if (I.a < 128) atomicOr(&ctl[k][I.a >> 5], 1u << (I.a & 31));
                if (!(I.mod & 0x80) && I.b < 128) atomicOr(&ctl[k][I.b >> 5], 1u << (I.b & 31));
            }
        }
    }
    __syncthreads();
    uint32_t mx = 0;
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) mx = max(mx, (uint32_t)min(cost(i), (uint64_t)0xFFFFFFFFu));
    atomicMax(&s_max, mx);
    __syncthreads();
    const uint32_t shift = max(0, 32 - __clz(s_max) - 10);
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
        const uint32_t b = kBuckets - 1 - min((uint32_t)(min(cost(i), (uint64_t)0xFFFFFFFFu) >> shift), (uint32_t)kBuckets - 1);
        atomicAdd(&hist[b], 1u);
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        uint32_t run = 0;
        for (int b = 0; b < kBuckets; ++b) { const uint32_t c = hist[b]; hist[b] = run; run += c; }
    }
    __syncthreads();
    for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) {
        const uint32_t b = kBuckets - 1 - min((uint32_t)(min(cost(i), (uint64_t)0xFFFFFFFFu) >> shift), (uint32_t)kBuckets - 1);
        order[atomicAdd(&hist[b], 1u)] = i;
    }
}

__global__ void __launch_bounds__(kWPB * 32)
k_inject(EmuProg P, const uint8_t* img, const uint64_t* __restrict__ warp_off, const fi_site* __restrict__ sites,
         uint32_t n, fi_inj* __restrict__ out, fi_store* __restrict__ log, uint32_t cap, uint32_t* ckpt,
         const uint64_t* __restrict__ ck_off, uint32_t ck_interval, const uint32_t* __restrict__ order,
         uint32_t* counter, uint32_t* status) {
    extern __shared__ uint32_t smem[];
    const uint32_t wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
    for (;;) {                                        // persistent warp: take the next replica
    uint32_t p = 0;
    if (lane == 0) p = atomicAdd(counter, 1u);
    p = __shfl_sync(kFull, p, 0);
    if (p >= n) return;
    const uint32_t i = order[p];
    const fi_site S = sites[i];
    if (S.flags & FI_SITE_NOT_INJECTED) {             // row f1 / C-17: nothing to inject
        if (lane == 0) {
            fi_inj r = {};
            r.outcome = FI_NOT_INJECTED;
            out[i] = r;
        }
        continue;
    }
    const fi_instance in = P.inst[S.instance];
    const uint32_t wpc = (in.block + 31) / 32, lw = S.warp - in.warp_begin;
    const uint64_t L = warp_off[S.warp + 1] - warp_off[S.warp];
    const uint64_t wd = 10 * L + 1024;                                                   // C-10
    const uint32_t watchdog = wd > 0xFFFFFFFFull ? 0xFFFFFFFFu : (uint32_t)wd;
    uint32_t* R = smem + wib * (P.n_regs + 1) * 32;
    const HookIn h{S.step, S.lane, S.dst_kind, S.dst_reg, S.bfm, S.mask, S.pc};
    uint32_t* ck = ckpt ? ckpt + ck_off[S.warp] * (ckpt_bytes(P.n_regs) / 4) : nullptr;
    const EmuOut o = emulate<EMU_INJ>(P, nullptr, img, S.instance, lw / wpc, lw % wpc, R, watchdog, nullptr,
                                      log + (uint64_t)i * cap, cap, h, ck, ckpt ? ck_interval : 0);
    if (lane == 0) {
        fi_inj r;
        r.before = o.before; r.after = o.after; r.mask = o.mask; r.fault_pc = o.fault_pc;
        r.fault_kind = (uint8_t)o.fault; r.outcome = 0; r.overflow = o.nstore > cap; r.flags = 0;
        r.n_faulty_stores = o.nstore;
        out[i] = r;
        if (!o.fired || o.bad) FI_DEV_ERR(status, FI_E_SITE);
        atomicAdd(reinterpret_cast<unsigned long long*>(counter + 2), (unsigned long long)(o.steps - o.start));
    }
    __syncwarp();
    }
}

struct ClsArgs {
    const fi_buffer* buf; const uint32_t* gran; const uint8_t* img;
    const fi_store* gstore; const uint64_t* gstore_off;
    const fi_site* sites; fi_inj* inj; uint32_t n;
    const fi_store* log; uint32_t cap;
    uint64_t* hist; uint32_t flags; uint32_t* status;
    double rtol;
};

__device__ __forceinline__ uint32_t buf_of(const ClsArgs& A, uint64_t va) {
    return __ldg(&A.gran[(va - kVaBase) >> 8]);
}
__device__ __forceinline__ bool is_output(const ClsArgs& A, uint64_t va) {
    const uint32_t b = buf_of(A, va);
    return b != kNoBuf && (__ldg(&A.buf[b].flags) & 1u);
}
__device__ __forceinline__ uint32_t golden_word(const ClsArgs& A, uint64_t va) {
    return __ldg(reinterpret_cast<const uint32_t*>(A.img + (va - kVaBase)));
}
// value of word va before instance k (DESIGN.md §3.5 writer rule)
__device__ __forceinline__ uint32_t pre_word(const ClsArgs& A, uint64_t va, uint32_t k) {
    const uint32_t b = buf_of(A, va);
    const int32_t wr = __ldg(&A.buf[b].writer);
    return (wr >= 0 && (uint32_t)wr >= k) ? 0u : golden_word(A, va);
}

constexpr int kClsWarps = 4;
constexpr uint8_t kSlow = 0xFE;                      // k_classify -> k_classify_slow hand-off outcome

// a 16-B log entry through the read-only path (both logs are read-only here)
__device__ __forceinline__ fi_store ld_store_nc(const fi_store* p) {
    const uint4 w = __ldg(reinterpret_cast<const uint4*>(p));
    fi_store s;
    static_assert(sizeof(fi_store) == 16, "fi_store is 16 B");
    memcpy(&s, &w, 16);
    return s;
}

__global__ void __launch_bounds__(kClsWarps * 32) k_classify(const ClsArgs A) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t i = blockIdx.x * kClsWarps + (threadIdx.x >> 5);
    if (i >= A.n) return;
    const fi_site S = A.sites[i];
    const fi_inj R = A.inj[i];
    uint32_t outcome;
    // f4: under FI_UNCHECKED only a hang is fatal; other faults just ended the warp
    const bool pdue = (A.flags & FI_UNCHECKED) && R.fault_kind && R.fault_kind != 3;
    if (S.flags & FI_SITE_NOT_INJECTED) {
        if (lane == 0) { A.inj[i].outcome = FI_NOT_INJECTED; A.inj[i].flags = 0; }
        return;
    }
    if (R.fault_kind && !pdue) {
        outcome = FI_DUE;
    } else if (R.overflow) {
        outcome = 0xFF;
    } else {
        const fi_store* G = A.gstore + A.gstore_off[S.warp];
        const uint64_t nGall = A.gstore_off[S.warp + 1] - A.gstore_off[S.warp];
        // first golden entry after the site (entries are in step order)
        uint64_t gs = 0;
        for (uint64_t b = 0; b < nGall; b += 32) {
            const bool after = b + lane < nGall && G[b + lane].step > S.step;
            const uint32_t m = __ballot_sync(kFull, after);
            if (m) { gs = b + __ffs(m) - 1; break; }
            gs = min(b + 32, nGall);
        }
        const fi_store* Gs = G + gs;
        const uint64_t nG = nGall - gs, nF = R.n_faulty_stores;
        const fi_store* F = A.log + (uint64_t)i * A.cap;
        // fast path: same store addresses in the same order; golden words are stored
        // once per warp, so then the golden value of F[j] is Gs[j].
        // One pass over both logs, 4 entries per lane in flight: address equality
        // and "an output word differs" together (the latter decides only if every
        // address matched)
        bool same_addr = nF == nG, vdiff = false;
        for (uint64_t b = 0; same_addr && b < nF; b += 128) {
            fi_store f[4], g[4];
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const uint64_t j = b + u * 32 + lane;
                if (j < nF) { f[u] = ld_store_nc(F + j); g[u] = ld_store_nc(Gs + j); }
            }
            bool d = false, v = false;
#pragma unroll
            for (int u = 0; u < 4; ++u) {
                const uint64_t j = b + u * 32 + lane;
                if (j < nF) {
                    d |= f[u].va != g[u].va;
                    v |= f[u].va == g[u].va && f[u].value != g[u].value && is_output(A, f[u].va);
                }
            }
            same_addr = !__any_sync(kFull, d);
            vdiff |= v;
        }
        // different store addresses: k_classify_slow decides (outcome kSlow meanwhile)
        outcome = !same_addr ? kSlow : __any_sync(kFull, vdiff) ? FI_SDC : FI_MASKED;
    }
    if (lane == 0) {
        A.inj[i].outcome = (uint8_t)outcome;
        A.inj[i].flags = pdue ? FI_POTENTIAL_DUE : 0;
        if (outcome == 0xFF) FI_DEV_ERR(A.status, FI_E_CAPACITY);
        else if (outcome != kSlow) atomicAdd((unsigned long long*)&A.hist[((uint32_t)S.group * 4 + S.bfm) * 3 + outcome], 1ull);
    }
}

// first golden store-log entry of warp w after step `step` (entries are in step order)
__device__ uint64_t golden_suffix(const ClsArgs& A, uint32_t w, uint32_t step, uint32_t lane) {
    const fi_store* G = A.gstore + A.gstore_off[w];
    const uint64_t nGall = A.gstore_off[w + 1] - A.gstore_off[w];
    uint64_t gs = 0;
    for (uint64_t b = 0; b < nGall; b += 32) {
        const uint32_t m = __ballot_sync(kFull, b + lane < nGall && G[b + lane].step > step);
        if (m) { gs = b + __ffs(m) - 1; break; }
        gs = min(b + 32, nGall);
    }
    return gs;
}

// K5's general case (faulty and golden store sequences differ in addresses), one
// CTA per such replica (persistent over the replicas k_classify marked kSlow):
//   SDC <=> some output word's final faulty value differs from its golden final value
//   (a) a faulty store that is the last faulty write to its address and differs, or
//   (b) a golden store after the site the faulty run never wrote, whose value before
//       the instance differs from the golden final value (C-12).
// The pairwise "any later write to the same address" / "any faulty write to this
// address" tests run over 256-entry smem tiles of the faulty log (broadcast reads).
constexpr int kSlowThreads = 256;
__global__ void __launch_bounds__(kSlowThreads) k_classify_slow(const ClsArgs A) {
    __shared__ uint64_t tva[kSlowThreads];
    __shared__ uint64_t s_gs;
    const uint32_t t = threadIdx.x, lane = t & 31;
    for (uint32_t i = blockIdx.x; i < A.n; i += gridDim.x) {
        if (A.inj[i].outcome != kSlow) continue;
        const fi_site S = A.sites[i];
        const fi_inj R = A.inj[i];
        const bool pdue = (A.flags & FI_UNCHECKED) && R.fault_kind && R.fault_kind != 3;
        if (t < 32) { const uint64_t gs = golden_suffix(A, S.warp, S.step, lane); if (t == 0) s_gs = gs; }
        __syncthreads();
        const uint64_t gs = s_gs;
        const fi_store* Gs = A.gstore + A.gstore_off[S.warp] + gs;
        const uint64_t nG = A.gstore_off[S.warp + 1] - A.gstore_off[S.warp] - gs, nF = R.n_faulty_stores;
        const fi_store* F = A.log + (uint64_t)i * A.cap;
        bool sdc = false;
        for (uint64_t jb = 0; jb < nF && !sdc; jb += kSlowThreads) {           // (a)
            const uint64_t j = jb + t;
            const bool have = j < nF;
            const fi_store f = have ? F[j] : fi_store{0, 0, 0};
            bool last = have;
            for (uint64_t qb = jb; qb < nF; qb += kSlowThreads) {
                __syncthreads();
                if (qb + t < nF) tva[t] = F[qb + t].va;
                __syncthreads();
                const uint32_t qn = (uint32_t)(nF - qb < (uint64_t)kSlowThreads ? nF - qb : (uint64_t)kSlowThreads);
                for (uint32_t q = 0; q < qn; ++q) last &= !(qb + q > j && tva[q] == f.va);
            }
            sdc = __syncthreads_or(last && is_output(A, f.va) && f.value != golden_word(A, f.va));
        }
        for (uint64_t jb = 0; jb < nG && !sdc; jb += kSlowThreads) {           // (b)
            const uint64_t j = jb + t;
            const bool have = j < nG;
            const uint64_t va = have ? Gs[j].va : 0;
            bool inF = false;
            for (uint64_t qb = 0; qb < nF; qb += kSlowThreads) {
                __syncthreads();
                if (qb + t < nF) tva[t] = F[qb + t].va;
                __syncthreads();
                const uint32_t qn = (uint32_t)(nF - qb < (uint64_t)kSlowThreads ? nF - qb : (uint64_t)kSlowThreads);
                for (uint32_t q = 0; q < qn; ++q) inF |= tva[q] == va;
            }
            sdc = __syncthreads_or(have && !inF && is_output(A, va) && pre_word(A, va, S.instance) != golden_word(A, va));
        }
        if (t == 0) {
            const uint32_t outcome = sdc ? FI_SDC : FI_MASKED;
            A.inj[i].outcome = (uint8_t)outcome;
            A.inj[i].flags = pdue ? FI_POTENTIAL_DUE : 0;
            atomicAdd((unsigned long long*)&A.hist[((uint32_t)S.group * 4 + S.bfm) * 3 + outcome], 1ull);
        }
        __syncthreads();
    }
}

// C-12 secondary numeric classification of a single-instance replica that K5
// found SDC (one CTA per replica, persistent): every output word whose final
// faulty value differs from the golden one — (a) the last faulty write to an
// address, (b) a golden store after the site the faulty run never repeated,
// whose faulty value is the word before the instance — is checked as part of its
// ELEMENT (the buffer's dtype; an f64 element's other word takes its own faulty
// final value by the same rules).  FI_SDC_WITHIN_TOL iff no element differs
// beyond rtol.  Plain serial scans: this mode is off the graded path.
__device__ uint32_t faulty_final(const ClsArgs& A, const fi_store* F, uint64_t nF, const fi_store* Gs, uint64_t nG,
                                 uint64_t va, uint32_t k) {
    for (uint64_t q = nF; q-- > 0;)
        if (F[q].va == va) return F[q].value;
    for (uint64_t q = 0; q < nG; ++q)
        if (Gs[q].va == va) return pre_word(A, va, k);
    return golden_word(A, va);
}
__device__ bool elem_beyond(const ClsArgs& A, const fi_store* F, uint64_t nF, const fi_store* Gs, uint64_t nG,
                            uint64_t va, uint32_t fv, uint32_t k) {
    const uint32_t dt = buf_dtype(__ldg(&A.buf[buf_of(A, va)].flags));
    if (dt != 2) return beyond_tol(dt, fv, golden_word(A, va), A.rtol);
    const uint64_t lo = va & ~7ull, hi = lo + 4;
    const uint32_t flo = va == lo ? fv : faulty_final(A, F, nF, Gs, nG, lo, k);
    const uint32_t fhi = va == hi ? fv : faulty_final(A, F, nF, Gs, nG, hi, k);
    const uint64_t f = (uint64_t)flo | ((uint64_t)fhi << 32);
    const uint64_t g = (uint64_t)golden_word(A, lo) | ((uint64_t)golden_word(A, hi) << 32);
    return beyond_tol(2, f, g, A.rtol);
}

__global__ void __launch_bounds__(kSlowThreads) k_classify_tol(const ClsArgs A) {
    __shared__ uint64_t s_gs;
    const uint32_t t = threadIdx.x, lane = t & 31;
    for (uint32_t i = blockIdx.x; i < A.n; i += gridDim.x) {
        if (A.inj[i].outcome != FI_SDC) continue;
        const fi_site S = A.sites[i];
        const fi_inj R = A.inj[i];
        if (t < 32) { const uint64_t gs = golden_suffix(A, S.warp, S.step, lane); if (t == 0) s_gs = gs; }
        __syncthreads();
        const fi_store* Gs = A.gstore + A.gstore_off[S.warp] + s_gs;
        const uint64_t nG = A.gstore_off[S.warp + 1] - A.gstore_off[S.warp] - s_gs, nF = R.n_faulty_stores;
        const fi_store* F = A.log + (uint64_t)i * A.cap;
        bool beyond = false;
        for (uint64_t j = t; j < nF && !beyond; j += kSlowThreads) {                // (a)
            const fi_store f = F[j];
            if (!is_output(A, f.va) || f.value == golden_word(A, f.va)) continue;
            bool last = true;
            for (uint64_t q = j + 1; q < nF && last; ++q) last = F[q].va != f.va;
            if (last) beyond = elem_beyond(A, F, nF, Gs, nG, f.va, f.value, S.instance);
        }
        for (uint64_t j = t; j < nG && !beyond; j += kSlowThreads) {                // (b)
            const uint64_t va = Gs[j].va;
            if (!is_output(A, va)) continue;
            const uint32_t pv = pre_word(A, va, S.instance);
            if (pv == golden_word(A, va)) continue;
            bool inF = false;
            for (uint64_t q = 0; q < nF && !inF; ++q) inF = F[q].va == va;
            if (!inF) beyond = elem_beyond(A, F, nF, Gs, nG, va, pv, S.instance);
        }
        beyond = __syncthreads_or(beyond);
        if (t == 0 && !beyond) A.inj[i].flags |= FI_SDC_WITHIN_TOL;
        __syncthreads();
    }
}

__global__ void k_hist_tol(const fi_site* sites, const fi_inj* inj, uint32_t n, uint64_t* hist_tol) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    uint32_t o = inj[i].outcome;
    if (o == FI_SDC && (inj[i].flags & FI_SDC_WITHIN_TOL)) o = FI_MASKED;
    if (o > FI_DUE) return;                          // not injected (C-17) / unclassified
    const fi_site S = sites[i];
    atomicAdd((unsigned long long*)&hist_tol[((uint32_t)S.group * 4 + S.bfm) * 3 + o], 1ull);
}

}  // namespace

fi_status launch_hist_tol(const fi_site* sites, const fi_inj* inj, uint32_t n, uint64_t* hist_tol, cudaStream_t s) {
    if (!hist_tol || !n) return FI_OK;
    k_hist_tol<<<(n + 255) / 256, 256, 0, s>>>(sites, inj, n, hist_tol);
    return launch_status();
}

void launch_lpt_order(const fi_program* p, const fi_site* sites, const uint64_t* warp_off, uint32_t ck_interval,
                      uint32_t n, uint32_t* order, uint32_t* counter, cudaStream_t s) {
    k_lpt_order<<<1, 1024, 0, s>>>(sites, warp_off, ck_interval, n, order, counter, p->code, p->kern, p->n_kern);
}
}  // namespace fi

using namespace fi;

// [0, 256): queue counter and the emulated-step count; then the LPT order (u32 per
// replica); then the JIT engine's per-SM deal counters (u32 per SM, up to 256 SMs)
extern "C" size_t fi_inject_workspace(uint32_t n) { return 256 + (((size_t)n * 4 + 255) & ~(size_t)255) + 1024; }

extern "C" fi_status fi_inject(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                               uint32_t n, fi_inj* out, fi_store* log, uint32_t log_cap, void* ws, size_t ws_bytes,
                               uint32_t* dev_status, void* stream) {
    if (!p || !image || !t || !sites || !out || !dev_status || (log_cap && !log) || !p->aux) return FI_E_ARG;
    if (t->ckpt && (!t->ckpt_off || !t->ckpt_interval)) return FI_E_ARG;
    if (n == 0) return FI_OK;
    if (!ws || ws_bytes < fi_inject_workspace(n)) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    uint32_t* counter = reinterpret_cast<uint32_t*>(ws);
    uint32_t* order = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + 256);
    const uint32_t ck_iv = t->ckpt ? t->ckpt_interval : 0;
    k_lpt_order<<<1, 1024, 0, s>>>(sites, t->warp_off, ck_iv, n, order, counter, p->code, p->kern, p->n_kern);
    fi_status e = launch_status();
    if (e) return e;
    const size_t smem = golden_smem(p->n_regs);
    e = cuda_status(cudaFuncSetAttribute((const void*)k_inject, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (e) return e;
    int dev = 0, sms = 0, per = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_inject, kWPB * 32, smem);
    const uint32_t grid = (uint32_t)std::min<uint64_t>((n + kWPB - 1) / kWPB, (uint64_t)std::max(1, sms * std::max(1, per)));
    k_inject<<<grid, kWPB * 32, smem, s>>>(make_emu_prog(p), image, t->warp_off, sites, n, out, log, log_cap, t->ckpt,
                                           t->ckpt_off, ck_iv, order, counter, dev_status);
    return launch_status();
}

namespace fi {
size_t propagate_slot_bytes(uint32_t ov_cap, uint32_t pend_cap);
void propagate_caps(uint32_t log_cap, uint32_t ov_words, uint32_t& ov_cap, uint32_t& pend_cap);
fi_status launch_propagate(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                           uint32_t n, fi_inj* out, const fi_store* log, uint32_t log_cap, uint64_t* hist,
                           uint32_t flags, void* ws, size_t ws_bytes, const uint32_t* order, uint32_t* counter,
                           uint32_t* dev_status, cudaStream_t s, const fi_pfault* pf, const uint64_t* opw,
                           uint32_t ov_words, double rtol);
namespace {
__global__ void k_iota(uint32_t* order, uint32_t n, uint32_t* counter) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) order[i] = i;
    if (i == 0) *counter = 0;
}
}  // namespace
}  // namespace fi

extern "C" size_t fi_classify_workspace(uint32_t n_inst, uint32_t n, uint32_t log_cap) {
    if (n_inst <= 1 || n == 0) return 0;
    uint32_t ov_cap, pend_cap;
    propagate_caps(log_cap, 0, ov_cap, pend_cap);
    const size_t sb = propagate_slot_bytes(ov_cap, pend_cap);
    const uint64_t slots = std::min<uint64_t>(((uint64_t)n + 3) / 4 * 4, 148ull * 16);   // <= resident warps
    return 256 + align256((size_t)n * 4) + slots * sb;
}

extern "C" fi_status fi_classify(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                                 uint32_t n, fi_inj* out, const fi_store* log, uint32_t log_cap, uint64_t* hist,
                                 uint32_t flags, double rtol, uint64_t* hist_tol, void* ws, size_t ws_bytes,
                                 uint32_t* dev_status, void* stream) {
    if (!p || !image || !t || !sites || !out || !hist || !dev_status || !p->aux) return FI_E_ARG;
    if (!(rtol >= 0.0)) return FI_E_ARG;
    if (n == 0) return FI_OK;
    if (p->n_inst > 1) {
        // K7: multi-instance programs propagate the faulty warp's effect downstream
        if (!ws || ws_bytes < fi_classify_workspace(p->n_inst, n, log_cap)) return FI_E_ARG;
        cudaStream_t s = (cudaStream_t)stream;
        uint32_t* counter = reinterpret_cast<uint32_t*>(ws);
        uint32_t* order = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + 256);
        const size_t head = 256 + align256((size_t)n * 4);
        k_iota<<<(n + 255) / 256, 256, 0, s>>>(order, n, counter);
        fi_status e = launch_status();
        if (e) return e;
        e = launch_propagate(p, image, t, sites, n, out, log, log_cap, hist, flags, reinterpret_cast<char*>(ws) + head,
                             ws_bytes - head, order, counter, dev_status, s, nullptr, nullptr, 0, rtol);
        if (e || rtol <= 0.0) return e;
        return launch_hist_tol(sites, out, n, hist_tol, s);
    }
    const EmuProg P = make_emu_prog(p);
    ClsArgs A{p->buf, P.gran, image, t->gstore, t->gstore_off, sites, out, n, log, log_cap, hist, flags, dev_status,
              rtol};
    cudaStream_t s = (cudaStream_t)stream;
    k_classify<<<(n + kClsWarps - 1) / kClsWarps, kClsWarps * 32, 0, s>>>(A);
    k_classify_slow<<<std::min<uint32_t>(n, 148u * 8u), kSlowThreads, 0, s>>>(A);
    if (rtol > 0.0) {
        k_classify_tol<<<std::min<uint32_t>(n, 148u * 8u), kSlowThreads, 0, s>>>(A);
        fi_status e = launch_status();
        if (e) return e;
        return launch_hist_tol(sites, out, n, hist_tol, s);
    }
    return launch_status();
}
