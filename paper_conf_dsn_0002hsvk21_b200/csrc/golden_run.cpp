// golden_run.cpp — fi_golden_run: the golden run of PAPER.md:72 Fig. 1 step (1)
// (the run whose dynamic instruction stream the profiler counts) and the golden
// output state of step (4), as ONE call of the C ABI.  Host code only: it
// sequences the golden-pass kernels behind fi_golden_lengths(_jit) /
// fi_scan_u64 / fi_ckpt_layout / fi_golden_trace(_jit) on one stream and owns
// the trace arrays it sizes from pass 1.
#include <algorithm>
#include <new>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/fi.h"
#include "common.cuh"

struct fi_golden {
    cudaStream_t s = nullptr;
    std::vector<void*> ptrs;                 // stream-ordered allocations owned by the handle
    fi_trace t{};
    uint64_t* warp_len = nullptr;
    uint64_t n_gstore = 0;
    std::vector<uint64_t> gstore_off_h;      // host copy [n_warps + 1]
    uint64_t rec_begin = 0, rec_end = 0;     // this rank's record shard (owner-computes run), else all
    uint32_t w_lo = 0, w_hi = 0;             // warps pass 2 ran
    uint64_t* inst_counts = nullptr;         // the run's profile (world 1): [n_inst][8]
    uint32_t* chunk_counts = nullptr;        // ... [ceil(n_rec / FI_CHUNK)][8]
    template <class T>
    fi_status alloc(T** out, size_t bytes) {
        void* p = nullptr;
        cudaError_t e = cudaMallocAsync(&p, std::max<size_t>(bytes, 16), s);
        if (e != cudaSuccess) return fi::cuda_status(e);
        ptrs.push_back(p);
        *out = static_cast<T*>(p);
        return FI_OK;
    }
    void release(cudaStream_t on) {
        for (void* p : ptrs) cudaFreeAsync(p, on);
        ptrs.clear();
    }
};

namespace {
#define GR_TRY(x)                          \
    do {                                   \
        fi_status _s = (x);                \
        if (_s != FI_OK) return _s;        \
    } while (0)

fi_status cu(cudaError_t e) { return fi::cuda_status(e); }

fi_status read_status(const uint32_t* dev_status, cudaStream_t s) {
    uint32_t v = 0;
    GR_TRY(cu(cudaMemcpyAsync(&v, dev_status, 4, cudaMemcpyDeviceToHost, s)));
    GR_TRY(cu(cudaStreamSynchronize(s)));
    if (!v) return FI_OK;
    for (int b = 0; b < 32; ++b)
        if (v & (1u << b)) return (fi_status)b;
    return FI_E_ARG;
}

fi_status run(const fi_program* p, const fi_jit* jit, uint8_t* image, uint32_t ckpt_interval, double budget_frac,
              fi_golden* g, int rank = 0, int world = 1) {
    cudaStream_t s = g->s;
    fi::keep_pool();
    const uint32_t W = p->n_warps;
    uint32_t* st;
    uint64_t *wn, *woff, *goff;
    GR_TRY(g->alloc(&st, 4));
    GR_TRY(g->alloc(&g->warp_len, 8ull * W));
    GR_TRY(g->alloc(&wn, 8ull * W));
    GR_TRY(g->alloc(&woff, 8ull * (W + 1)));
    GR_TRY(g->alloc(&goff, 8ull * (W + 1)));
    GR_TRY(cu(cudaMemsetAsync(st, 0, 4, s)));
    GR_TRY(cu(cudaMemsetAsync(g->warp_len, 0, 8ull * W, s)));
    GR_TRY(cu(cudaMemsetAsync(wn, 0, 8ull * W, s)));
    // pass 1: per-warp lengths and stored-word counts, golden final image
    if (jit) GR_TRY(fi_golden_lengths_jit(jit, p, image, g->warp_len, wn, st, s));
    else GR_TRY(fi_golden_lengths(p, image, g->warp_len, wn, st, s));
    const size_t scan_ws = fi_scan_u64_workspace(W);
    void* sws;
    GR_TRY(g->alloc(&sws, scan_ws));
    GR_TRY(fi_scan_u64(g->warp_len, woff, W, sws, scan_ws, s));
    GR_TRY(fi_scan_u64(wn, goff, W, sws, scan_ws, s));
    GR_TRY(read_status(st, s));                                       // synchronizes
    g->gstore_off_h.assign(W + 1, 0);
    uint64_t n_rec = 0;
    GR_TRY(cu(cudaMemcpyAsync(&n_rec, woff + W, 8, cudaMemcpyDeviceToHost, s)));
    GR_TRY(cu(cudaMemcpyAsync(g->gstore_off_h.data(), goff, 8ull * (W + 1), cudaMemcpyDeviceToHost, s)));
    GR_TRY(cu(cudaStreamSynchronize(s)));
    g->n_gstore = g->gstore_off_h[W];
    fi_record* rec;
    fi_store* gst;
    GR_TRY(g->alloc(&rec, 16ull * std::max<uint64_t>(n_rec, 1)));
    GR_TRY(g->alloc(&gst, 16ull * std::max<uint64_t>(g->n_gstore, 1)));
    // checkpoint layout: warp w gets ceil(len_w / interval) register-file checkpoints
    uint32_t* ck = nullptr;
    uint64_t* ckoff = nullptr;
    uint32_t interval = 0;
    if (ckpt_interval) {
        interval = ckpt_interval == FI_CKPT_AUTO ? 8192u : ckpt_interval;
        const size_t ck_bytes = fi_ckpt_bytes(p->n_regs);
        const size_t lws = fi_ckpt_layout_workspace(W);
        void* lw;
        GR_TRY(g->alloc(&lw, lws));
        GR_TRY(g->alloc(&ckoff, 8ull * (W + 1)));
        size_t free_b = 0, total_b = 0;
        GR_TRY(cu(cudaMemGetInfo(&free_b, &total_b)));
        const double frac = budget_frac > 0 ? budget_frac : 0.2;
        uint64_t n_ck = 0;
        for (;;) {
            GR_TRY(fi_ckpt_layout(g->warp_len, W, interval, ckoff, lw, lws, s));
            GR_TRY(cu(cudaMemcpyAsync(&n_ck, ckoff + W, 8, cudaMemcpyDeviceToHost, s)));
            GR_TRY(cu(cudaStreamSynchronize(s)));
            if (ckpt_interval != FI_CKPT_AUTO || (double)(n_ck * ck_bytes) <= frac * (double)free_b ||
                interval >= (1u << 24))
                break;
            interval *= 2;
        }
        GR_TRY(g->alloc(&ck, n_ck * ck_bytes));
    }
    g->t = fi_trace{rec, n_rec, woff, gst, goff, ck, ckoff, interval, W};
    g->rec_begin = 0; g->rec_end = n_rec; g->w_lo = 0; g->w_hi = W;
    if (world > 1) {
        // owner-computes: this rank's chunk-aligned record shard (fi_campaign's profile
        // shard); pass 2 runs the warps holding those records (a warp straddling two
        // shards runs on both, bit-identically), the image takes the stores of the
        // warps whose FIRST record is in the shard (each warp has exactly one owner)
        std::vector<uint64_t> wo(W + 1);
        GR_TRY(cu(cudaMemcpyAsync(wo.data(), woff, 8ull * (W + 1), cudaMemcpyDeviceToHost, s)));
        GR_TRY(cu(cudaStreamSynchronize(s)));
        uint64_t r0 = 0, r1 = 0;
        uint32_t wa = 0, wb = 0, oa = 0, ob = 0;
        GR_TRY(fi_shard_warps(wo.data(), W, rank, world, &r0, &r1, &wa, &wb, &oa, &ob));
        g->rec_begin = r0; g->rec_end = r1; g->w_lo = wa; g->w_hi = wb;
        GR_TRY(fi_golden_trace_jit_range(jit, p, image, &g->t, wa, wb, oa, ob, nullptr, nullptr, st, s));
        return read_status(st, s);
    }
    // pass 2: trace records, golden store log, checkpoints — and the profile (K1's
    // counts): fused into the JIT pass (JProf), else K1 over the written trace
    const uint64_t n_chunks = (n_rec + FI_CHUNK - 1) / FI_CHUNK;
    GR_TRY(g->alloc(&g->inst_counts, 64ull * std::max<uint32_t>(p->n_inst, 1)));
    GR_TRY(g->alloc(&g->chunk_counts, 32ull * std::max<uint64_t>(n_chunks, 1)));
    GR_TRY(cu(cudaMemsetAsync(g->inst_counts, 0, 64ull * std::max<uint32_t>(p->n_inst, 1), s)));
    GR_TRY(cu(cudaMemsetAsync(g->chunk_counts, 0, 32ull * std::max<uint64_t>(n_chunks, 1), s)));
    if (jit) {
        GR_TRY(fi_golden_trace_jit_range(jit, p, image, &g->t, 0, W, 0, W, g->inst_counts, g->chunk_counts, st, s));
    } else {
        GR_TRY(fi_golden_trace(p, image, &g->t, st, s));
        GR_TRY(fi_profile(&g->t, 0, n_rec, p->n_inst, g->inst_counts, g->chunk_counts, s));
    }
    return read_status(st, s);                                        // synchronizes
}
}  // namespace

extern "C" fi_status fi_golden_run(const fi_program* p, const fi_jit* jit, uint8_t* image, uint32_t ckpt_interval,
                                   double ckpt_budget_frac, fi_golden** out, void* stream) {
    if (!p || !image || !out || !p->n_warps || !p->aux) return FI_E_ARG;
    *out = nullptr;
    fi_golden* g = new (std::nothrow) fi_golden;
    if (!g) return FI_E_ARG;
    g->s = (cudaStream_t)stream;
    const fi_status e = run(p, jit, image, ckpt_interval, ckpt_budget_frac, g);
    if (e != FI_OK) {
        g->release(g->s);
        cudaStreamSynchronize(g->s);
        delete g;
        return e;
    }
    *out = g;
    return FI_OK;
}

extern "C" fi_status fi_shard_warps(const uint64_t* warp_off, uint32_t n_warps, int rank, int world,
                                    uint64_t* rec_begin, uint64_t* rec_end, uint32_t* w_lo, uint32_t* w_hi,
                                    uint32_t* own_lo, uint32_t* own_hi) {
    if (!warp_off || world < 1 || rank < 0 || rank >= world || !rec_begin || !rec_end || !w_lo || !w_hi || !own_lo ||
        !own_hi)
        return FI_E_ARG;
    const uint64_t* b = warp_off;
    const uint64_t* e = warp_off + n_warps;                  // warp_off[0 .. n_warps) (the last entry is n_rec)
    const uint64_t n_rec = warp_off[n_warps];
    const uint64_t C = (n_rec + FI_CHUNK - 1) / FI_CHUNK;
    const uint64_t r0 = std::min<uint64_t>(C * (uint64_t)rank / world * FI_CHUNK, n_rec);
    const uint64_t r1 = std::min<uint64_t>(C * (uint64_t)(rank + 1) / world * FI_CHUNK, n_rec);
    uint32_t wa = 0, wb = 0;
    if (r0 < r1) {
        wa = (uint32_t)(std::upper_bound(b, e, r0) - b) - 1;     // last warp starting at or before r0
        wb = (uint32_t)(std::lower_bound(b, e, r1) - b);         // first warp starting at or after r1
    }
    *rec_begin = r0; *rec_end = r1; *w_lo = wa; *w_hi = wb;
    *own_lo = (uint32_t)(std::lower_bound(b, e, r0) - b);        // warps whose first record is in [r0, r1)
    *own_hi = (uint32_t)(std::lower_bound(b, e, r1) - b);
    return FI_OK;
}

extern "C" fi_status fi_golden_run_shard(const fi_program* p, const fi_jit* jit, uint8_t* image, uint32_t ckpt_interval,
                                         double ckpt_budget_frac, int rank, int world, fi_golden** out, void* stream) {
    if (!p || !jit || !image || !out || !p->n_warps || !p->aux || world < 1 || rank < 0 || rank >= world ||
        p->n_inst != 1)
        return FI_E_ARG;
    *out = nullptr;
    fi_golden* g = new (std::nothrow) fi_golden;
    if (!g) return FI_E_ARG;
    g->s = (cudaStream_t)stream;
    const fi_status e = run(p, jit, image, ckpt_interval, ckpt_budget_frac, g, rank, world);
    if (e != FI_OK) {
        g->release(g->s);
        cudaStreamSynchronize(g->s);
        delete g;
        return e;
    }
    *out = g;
    return FI_OK;
}

extern "C" void fi_golden_shard_range(const fi_golden* g, uint64_t* rec_begin, uint64_t* rec_end, uint32_t* w_lo,
                                      uint32_t* w_hi) {
    if (!g) return;
    if (rec_begin) *rec_begin = g->rec_begin;
    if (rec_end) *rec_end = g->rec_end;
    if (w_lo) *w_lo = g->w_lo;
    if (w_hi) *w_hi = g->w_hi;
}

extern "C" const fi_trace* fi_golden_trace_of(const fi_golden* g) { return g ? &g->t : nullptr; }
extern "C" fi_status fi_golden_profile(const fi_golden* g, const uint64_t** inst_counts, const uint32_t** chunk_counts) {
    if (!g || !inst_counts || !chunk_counts || !g->inst_counts) return FI_E_ARG;
    *inst_counts = g->inst_counts;
    *chunk_counts = g->chunk_counts;
    return FI_OK;
}
extern "C" const uint64_t* fi_golden_warp_len(const fi_golden* g) { return g ? g->warp_len : nullptr; }
extern "C" const uint64_t* fi_golden_gstore_off_host(const fi_golden* g) {
    return g ? g->gstore_off_h.data() : nullptr;
}

extern "C" fi_status fi_golden_free(fi_golden* g, void* stream) {
    if (!g) return FI_OK;
    g->release(stream ? (cudaStream_t)stream : g->s);
    delete g;
    return FI_OK;
}
