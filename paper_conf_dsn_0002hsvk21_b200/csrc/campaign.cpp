// campaign.cpp — fi_campaign, the native campaign driver of one rank
// (Fig. 1 steps (1)-(4); SURVEY §8(e) sharding), and the profile
// file writer of PAPER.md:78.  Host code only: every step of the path runs in
// the CUDA kernels behind the other fi_* entry points, which this file calls
// in order on one stream.  The exchanges are the two integer all-reduces of
// DESIGN.md §9, done by the caller's callback (torch.distributed / NCCL).
#include <algorithm>
#include <chrono>
#include <cstdio>
#include <map>
#include <mutex>
#include <cstring>
#include <string>
#include <vector>

#include <cuda_runtime.h>

#include "../../include/fi.h"
#include "common.cuh"

// Device allocations of one fi_campaign call, stream-ordered from the device's
// default memory pool and freed on every return path.  The pool keeps what it
// holds between calls (release threshold raised once per device), so a repeated
// campaign reuses its ~48 GB instead of paying cudaMalloc/cudaFree each time;
// fi_campaign_release_memory() hands it back to the driver.
void fi::keep_pool() {
    static std::once_flag once[64];
    int dev = -1;
    if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return;
    std::call_once(once[dev], [dev] {
        cudaMemPool_t pool;
        if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
            uint64_t keep = ~0ull;
            cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
        }
    });
}

namespace {
struct Arena {
    cudaStream_t s = nullptr;
    std::vector<void*> ptrs;
    ~Arena() {
        for (void* p : ptrs) cudaFreeAsync(p, s);
        if (!ptrs.empty()) cudaStreamSynchronize(s);
    }
    template <class T>
    fi_status alloc(T** out, size_t bytes) {
        void* p = nullptr;
        cudaError_t e = cudaMallocAsync(&p, std::max<size_t>(bytes, 16), s);
        if (e != cudaSuccess) return fi::cuda_status(e);
        ptrs.push_back(p);
        *out = static_cast<T*>(p);
        return FI_OK;
    }
};

#define FI_TRY(x)                          \
    do {                                   \
        fi_status _s = (x);                \
        if (_s != FI_OK) return _s;        \
    } while (0)

fi_status cu(cudaError_t e) { return fi::cuda_status(e); }

// First set error bit of the device status word (FI_DEV_ERR convention of fi.h).
fi_status check_status(const uint32_t* dev_status, cudaStream_t s) {
    uint32_t v = 0;
    FI_TRY(cu(cudaMemcpyAsync(&v, dev_status, 4, cudaMemcpyDeviceToHost, s)));
    FI_TRY(cu(cudaStreamSynchronize(s)));
    if (!v) return FI_OK;
    for (int b = 0; b < 32; ++b)
        if (v & (1u << b)) return (fi_status)b;
    return FI_E_ARG;
}

struct Events {
    cudaEvent_t e[10] = {};
    int n = 0;
    ~Events() {
        for (int i = 0; i < n; ++i) cudaEventDestroy(e[i]);
    }
    fi_status mark(cudaStream_t s) {
        FI_TRY(cu(cudaEventCreate(&e[n])));
        FI_TRY(cu(cudaEventRecord(e[n], s)));
        ++n;
        return FI_OK;
    }
    float ms(int a, int b) const {
        float t = 0.f;
        if (b < n) cudaEventElapsedTime(&t, e[a], e[b]);
        return t;
    }
};

struct GoldenGuard {                 // the golden run's trace arrays, freed on every return path
    fi_golden* g = nullptr;
    cudaStream_t s = nullptr;
    ~GoldenGuard() { fi_golden_free(g, s); }
};

struct OwnedStream {
    cudaStream_t s = nullptr;
    bool own = false;
    ~OwnedStream() {
        if (own) cudaStreamDestroy(s);
    }
};

// JIT modules built by fi_campaign, per (program code, kernel table, register
// rows, device): compiled once per process, reused by later campaigns.
fi_status cached_jit(const fi_program& p, const fi_kernel* kern_host, int dev, uint32_t modes, fi_jit** out,
                     float* ms) {
    static std::mutex mu;
    static std::map<std::string, fi_jit*> cache;
    std::string key((const char*)p.code_host, sizeof(fi_insn) * p.n_code);
    key.append((const char*)kern_host, sizeof(fi_kernel) * p.n_kern);
    key.append((const char*)&p.n_regs, 4);
    key.append((const char*)&dev, sizeof dev);
    key.append((const char*)&modes, sizeof modes);
    std::lock_guard<std::mutex> g(mu);
    auto it = cache.find(key);
    if (it != cache.end()) { *out = it->second; *ms = 0.f; return FI_OK; }
    const auto t0 = std::chrono::steady_clock::now();
    fi_jit* j = nullptr;
    FI_TRY(fi_jit_build(&p, kern_host, modes, &j));
    *ms = std::chrono::duration<float, std::milli>(std::chrono::steady_clock::now() - t0).count();
    cache[key] = j;
    *out = j;
    return FI_OK;
}

}  // namespace

extern "C" fi_status fi_campaign(const fi_campaign_cfg* cfg, int rank, int world, fi_allreduce_fn allreduce,
                                 void* ctx, fi_campaign_result* res) {
    if (!cfg || !res || world < 1 || rank < 0 || rank >= world) return FI_E_ARG;
    if (world > 1 && !allreduce) return FI_E_ARG;
    if (!cfg->code || !cfg->n_code || !cfg->kern || !cfg->n_kern || !cfg->inst || !cfg->n_inst || !cfg->buf ||
        !cfg->n_buf || (cfg->image_bytes && !cfg->init_image) || !cfg->n_warps)
        return FI_E_ARG;
    if (cfg->sched.n_groups < 1 || cfg->sched.n_groups > 8 || cfg->sched.n_bfms < 1 || cfg->sched.n_bfms > 4)
        return FI_E_ARG;
    if (cfg->propagation > FI_PROPAGATION_K8 || cfg->engine > FI_ENGINE_JIT || !(cfg->rtol >= 0.0)) return FI_E_ARG;
    if (cfg->device >= 0) FI_TRY(cu(cudaSetDevice(cfg->device)));

    OwnedStream os;
    if (cfg->stream) {
        os.s = (cudaStream_t)cfg->stream;
    } else {
        FI_TRY(cu(cudaStreamCreateWithFlags(&os.s, cudaStreamNonBlocking)));
        os.own = true;
    }
    cudaStream_t s = os.s;
    fi::keep_pool();
    Arena A;
    A.s = s;
    Events ev;
    const uint32_t W = cfg->n_warps, K = cfg->n_inst;

    // ---- H2D of the program (caller's host arrays; pinned or pageable) ------
    FI_TRY(ev.mark(s));                                                    // 0
    fi_insn* code;
    fi_kernel* kern;
    fi_instance* inst;
    uint32_t* cbank;
    fi_buffer* buf;
    uint8_t* image;
    FI_TRY(A.alloc(&code, sizeof(fi_insn) * cfg->n_code));
    FI_TRY(A.alloc(&kern, sizeof(fi_kernel) * cfg->n_kern));
    FI_TRY(A.alloc(&inst, sizeof(fi_instance) * K));
    FI_TRY(A.alloc(&cbank, 4ull * cfg->n_cbank));
    FI_TRY(A.alloc(&buf, sizeof(fi_buffer) * cfg->n_buf));
    FI_TRY(A.alloc(&image, cfg->image_bytes));
    FI_TRY(cu(cudaMemcpyAsync(code, cfg->code, sizeof(fi_insn) * cfg->n_code, cudaMemcpyHostToDevice, s)));
    FI_TRY(cu(cudaMemcpyAsync(kern, cfg->kern, sizeof(fi_kernel) * cfg->n_kern, cudaMemcpyHostToDevice, s)));
    FI_TRY(cu(cudaMemcpyAsync(inst, cfg->inst, sizeof(fi_instance) * K, cudaMemcpyHostToDevice, s)));
    if (cfg->n_cbank)
        FI_TRY(cu(cudaMemcpyAsync(cbank, cfg->cbank, 4ull * cfg->n_cbank, cudaMemcpyHostToDevice, s)));
    FI_TRY(cu(cudaMemcpyAsync(buf, cfg->buf, sizeof(fi_buffer) * cfg->n_buf, cudaMemcpyHostToDevice, s)));
    if (cfg->image_bytes) {
        // Buffers with a writer start zeroed (SSA: the emulator never
        // reads their initial content), so only the other buffers cross PCIe: the
        // image is zeroed on the device and the writer-less buffers copied, nearby
        // ones (gap < 1 MiB) merged into one copy.
        FI_TRY(cu(cudaMemsetAsync(image, 0, cfg->image_bytes, s)));
        std::vector<std::pair<uint64_t, uint64_t>> rng;
        for (uint32_t b = 0; b < cfg->n_buf; ++b) {
            const fi_buffer& B = cfg->buf[b];
            if (B.writer >= 0 || !B.size || B.off >= cfg->image_bytes) continue;
            const uint64_t e = std::min<uint64_t>(B.off + B.size, cfg->image_bytes);
            if (!rng.empty() && B.off >= rng.back().second && B.off - rng.back().second < (1u << 20))
                rng.back().second = std::max(rng.back().second, e);
            else
                rng.push_back({B.off, e});
        }
        for (auto& r : rng)
            FI_TRY(cu(cudaMemcpyAsync(image + r.first, cfg->init_image + r.first, r.second - r.first,
                                      cudaMemcpyHostToDevice, s)));
    }

    void* aux;
    FI_TRY(A.alloc(&aux, fi_program_aux_bytes(cfg->image_bytes, cfg->n_code, K)));
    fi_program p{code,  cfg->n_code, kern, cfg->n_kern, inst,   K, cbank, cfg->n_cbank, buf, cfg->n_buf,
                 aux,   cfg->image_bytes, W, fi_program_regs(cfg->code, cfg->n_code), cfg->code, cfg->inst};
    FI_TRY(fi_program_prepare(&p, aux, s));
    // JIT engine: the program's module (golden passes + K4), built once per process
    fi_jit* jit = nullptr;
    float ms_jit = 0.f;
    const bool k8 = cfg->propagation == FI_PROPAGATION_K8 || (cfg->propagation == FI_PROPAGATION_AUTO && K >= 64);
    if (cfg->engine == FI_ENGINE_JIT) {
        int dev = 0;
        FI_TRY(cu(cudaGetDevice(&dev)));
        FI_TRY(cached_jit(p, cfg->kern, dev, FI_JIT_INJECT | FI_JIT_GOLDEN | (k8 ? FI_JIT_PAGE : 0u), &jit, &ms_jit));
    }
    FI_TRY(ev.mark(s));                                                    // 1

    // ---- golden run (fi_golden_run: pass 1, scans, checkpoint layout, pass 2) ----
    GoldenGuard gg;
    gg.s = s;
    // owner-computes: a single-launch program's golden run is sharded
    // like the profile — this rank emulates (pass 2) only the warps of its record
    // shard, and the golden image is completed by one SUM over the writer buffers
    const bool owner = cfg->owner_computes && world > 1 && K == 1 && jit && !cfg->approximate;
    if (owner) FI_TRY(fi_golden_run_shard(&p, jit, image, cfg->ckpt_interval, 0.2, rank, world, &gg.g, s));
    else FI_TRY(fi_golden_run(&p, jit, image, cfg->ckpt_interval, 0.2, &gg.g, s));
    if (owner && fi_jit_len_sliced(jit)) {
        // writer buffers start zeroed (SSA, §3.5) and each word is stored by one warp,
        // owned by one rank: the sum over the ranks is the golden final image
        std::vector<std::pair<uint64_t, uint64_t>> wr;
        for (uint32_t b = 0; b < cfg->n_buf; ++b) {
            const fi_buffer& B = cfg->buf[b];
            if (B.writer < 0 || !B.size) continue;
            const uint64_t o = B.off & ~3ull, e = std::min<uint64_t>((B.off + B.size + 3) & ~3ull, cfg->image_bytes);
            if (!wr.empty() && o <= wr.back().second) wr.back().second = std::max(wr.back().second, e);
            else wr.push_back({o, e});
        }
        for (auto& r : wr)
            if (allreduce(image + r.first, (r.second - r.first) / 4, 4, ctx, s)) return FI_E_COLLECTIVE;
    }
    const fi_trace t = *fi_golden_trace_of(gg.g);
    const uint64_t n_rec = t.n_rec;
    const uint64_t* goff_h = fi_golden_gstore_off_host(gg.g);
    uint32_t* st;
    FI_TRY(A.alloc(&st, 4));
    FI_TRY(cu(cudaMemsetAsync(st, 0, 4, s)));
    FI_TRY(ev.mark(s));                                                    // 2

    // ---- profile: the golden run's (fused), else K1 over this rank's chunk-aligned
    // shard + count exchange (owner-computes, approximate profiling) ------------
    const uint64_t n_chunks = (n_rec + FI_CHUNK - 1) / FI_CHUNK;
    const uint64_t c0 = n_chunks * (uint64_t)rank / world, c1 = n_chunks * (uint64_t)(rank + 1) / world;
    const uint64_t r0 = std::min(c0 * FI_CHUNK, n_rec), r1 = std::min(c1 * FI_CHUNK, n_rec);
    uint64_t* ic;
    uint32_t* cc;
    const uint64_t* gic = nullptr;
    const uint32_t* gcc = nullptr;
    if (!cfg->approximate && fi_golden_profile(gg.g, &gic, &gcc) == FI_OK) {
        // the golden run counted (fused into pass 2 on the JIT engine): every rank
        // holds the whole profile, nothing to scan or exchange
        ic = const_cast<uint64_t*>(gic);
        cc = const_cast<uint32_t*>(gcc);
        FI_TRY(ev.mark(s));                                                // 3
        FI_TRY(ev.mark(s));                                                // 4
    } else {
        FI_TRY(A.alloc(&ic, 64ull * K));
        FI_TRY(A.alloc(&cc, 32ull * std::max<uint64_t>(n_chunks, 1)));
        FI_TRY(cu(cudaMemsetAsync(cc, 0, 32ull * std::max<uint64_t>(n_chunks, 1), s)));
        if (cfg->approximate) {
            // first instance of every static kernel only; every rank
            // computes the same (small) counts, so there is nothing to exchange.
            const size_t aws = fi_profile_approx_workspace(cfg->n_kern, K);
            void* aw;
            FI_TRY(A.alloc(&aw, aws));
            FI_TRY(fi_profile_approx(&p, &t, ic, aw, aws, s));
            FI_TRY(ev.mark(s));                                                // 3
            FI_TRY(ev.mark(s));                                                // 4
        } else {
            FI_TRY(fi_profile(&t, r0, r1, K, ic, cc, s));
            FI_TRY(ev.mark(s));                                                // 3
            if (world > 1) {
                if (allreduce(ic, 8ull * K, 8, ctx, s)) return FI_E_COLLECTIVE;
                if (allreduce(cc, 8ull * n_chunks, 4, ctx, s)) return FI_E_COLLECTIVE;
            }
            FI_TRY(ev.mark(s));                                                // 4
        }
    }

    // ---- K2 index + totals ---------------------------------------------------
    void* index;
    const uint64_t idx_chunks = cfg->approximate ? 0 : n_chunks;
    FI_TRY(A.alloc(&index, fi_site_index_bytes(K, idx_chunks)));
    if (cfg->approximate)
        FI_TRY(fi_build_instance_index(ic, K, index, st, s));
    else
        FI_TRY(fi_build_site_index(ic, K, cc, n_chunks, index, st, s));
    uint64_t totals[8];
    FI_TRY(fi_site_totals(index, K, totals, s));                           // synchronizes
    FI_TRY(check_status(st, s));
    FI_TRY(ev.mark(s));                                                    // 5

    // ---- K3 select / K4 inject / classify of this rank's replicas -------------
    // replica block [r*n/G, (r+1)*n/G); owner-computes: every replica is drawn, the
    // rank keeps those whose site lies in its record shard (fi_select_sites_shard)
    const uint64_t j0 = owner ? 0 : cfg->n_replicas * (uint64_t)rank / world;
    const uint64_t j1 = owner ? cfg->n_replicas : cfg->n_replicas * (uint64_t)(rank + 1) / world;
    if (j1 - j0 > 0xFFFFFFFFull) return FI_E_ARG;
    uint32_t n = (uint32_t)(j1 - j0);
    fi_site* sites;
    fi_inj* inj;
    uint64_t* jidx = nullptr;
    FI_TRY(A.alloc(&sites, 64ull * std::max(n, 1u)));
    FI_TRY(A.alloc(&inj, 24ull * std::max(n, 1u)));
    if (owner && n) {
        fi_site* drawn;
        uint32_t* n_dev;
        FI_TRY(A.alloc(&drawn, 64ull * n));
        FI_TRY(A.alloc(&jidx, 8ull * n));
        FI_TRY(A.alloc(&n_dev, 4));
        FI_TRY(fi_select_sites_shard(&p, &t, cc, index, K, n_chunks, totals, &cfg->sched, 0, n, r0, r1, drawn, st, s));
        FI_TRY(fi_compact_sites(drawn, n, 0, sites, jidx, n_dev, s));
        FI_TRY(cu(cudaMemcpyAsync(&n, n_dev, 4, cudaMemcpyDeviceToHost, s)));
        FI_TRY(cu(cudaStreamSynchronize(s)));
    } else if (n) {
        if (cfg->approximate)
            FI_TRY(fi_select_sites_approx(&p, &t, index, K, totals, &cfg->sched, j0, n, sites, st, s));
        else
            FI_TRY(fi_select_sites(&p, &t, cc, index, K, n_chunks, totals, &cfg->sched, j0, n, sites, st, s));
    }
    FI_TRY(ev.mark(s));                                                    // 6

    // per-replica faulty-store log: 2x the largest golden per-warp store count + 4096
    uint64_t mx_w = 0;
    for (uint32_t w = 0; w < W; ++w) mx_w = std::max(mx_w, goff_h[w + 1] - goff_h[w]);
    const uint32_t log_cap = (uint32_t)std::min<uint64_t>(2 * mx_w + 4096, 0x7FFFFFFFull);
    fi_store* log;
    FI_TRY(A.alloc(&log, 16ull * std::max<uint64_t>((uint64_t)n * log_cap, 1)));
    const size_t iws = fi_inject_workspace(n);
    void* iw;
    FI_TRY(A.alloc(&iw, iws));
    if (n && jit) {
        FI_TRY(fi_inject_jit(jit, &p, image, &t, sites, n, inj, log, log_cap, iw, iws, st, s));
    } else if (n) {
        FI_TRY(fi_inject(&p, image, &t, sites, n, inj, log, log_cap, iw, iws, st, s));
    }
    FI_TRY(ev.mark(s));                                                    // 7

    uint64_t *hist, *hist_tol;
    FI_TRY(A.alloc(&hist, 2 * sizeof(res->hist)));
    hist_tol = hist + 96;
    FI_TRY(cu(cudaMemsetAsync(hist, 0, 2 * sizeof(res->hist), s)));
    const double rtol = cfg->rtol;
    if (n && k8) {
        // pend_cap: 2x the largest launch's golden stores + 4096 (fi.py pend_capacity)
        uint64_t mx_l = 0;
        for (uint32_t k = 0; k < K; ++k)
            mx_l = std::max(mx_l, goff_h[cfg->inst[k].warp_end] - goff_h[cfg->inst[k].warp_begin]);
        const uint32_t pend = (uint32_t)std::min<uint64_t>(2 * mx_l + 4096, 0x7FFFFFFFull);
        const uint64_t budget = cfg->k8_mem_budget ? cfg->k8_mem_budget : (24ull << 30);
        const size_t w1 = fi_classify_batched_workspace(&p, n, log_cap, 1, 1, pend);
        const size_t w2 = fi_classify_batched_workspace(&p, n, log_cap, 2, 1, pend);
        int64_t b = ((int64_t)(budget / 2) - (int64_t)w1) / (int64_t)std::max<size_t>(w2 - w1, 1) + 1;
        const uint32_t batch = (uint32_t)std::max<int64_t>(1, std::min<int64_t>({(int64_t)n, 512, b}));
        const size_t fixed = fi_classify_batched_workspace(&p, n, log_cap, batch, 1, pend);
        const uint32_t pool = (uint32_t)std::max<int64_t>(
            1024, std::min<int64_t>(((int64_t)budget - (int64_t)fixed) / (4096 + 12), 0x7FFFFFFF));
        const size_t kws = fi_classify_batched_workspace(&p, n, log_cap, batch, pool, pend);
        void* kw;
        FI_TRY(A.alloc(&kw, kws));
        if (jit)
            FI_TRY(fi_classify_batched_jit(jit, &p, image, &t, sites, n, inj, log, log_cap, hist, cfg->flags, rtol,
                                           hist_tol, batch, pool, pend, kw, kws, st, s));
        else
            FI_TRY(fi_classify_batched(&p, image, &t, sites, n, inj, log, log_cap, hist, cfg->flags, rtol, hist_tol,
                                       batch, pool, pend, kw, kws, st, s));
    } else if (n) {
        const size_t cws = fi_classify_workspace(K, n, log_cap);
        void* cw = nullptr;
        if (cws) FI_TRY(A.alloc(&cw, cws));
        FI_TRY(fi_classify(&p, image, &t, sites, n, inj, log, log_cap, hist, cfg->flags, rtol, hist_tol, cw, cws, st,
                           s));
    }
    // one exchange of both histograms (the secondary one stays zero when rtol == 0)
    if (world > 1 && allreduce(hist, rtol > 0.0 ? 192 : 96, 8, ctx, s)) return FI_E_COLLECTIVE;
    FI_TRY(ev.mark(s));                                                    // 8

    // ---- D2H of the results ----------------------------------------------------
    FI_TRY(cu(cudaMemcpyAsync(res->hist, hist, sizeof(res->hist), cudaMemcpyDeviceToHost, s)));
    FI_TRY(cu(cudaMemcpyAsync(res->hist_tol, hist_tol, sizeof(res->hist_tol), cudaMemcpyDeviceToHost, s)));
    if (res->sites && n) FI_TRY(cu(cudaMemcpyAsync(res->sites, sites, 64ull * n, cudaMemcpyDeviceToHost, s)));
    if (res->j && n) {                                   // the replica index of every returned row
        if (jidx) FI_TRY(cu(cudaMemcpyAsync(res->j, jidx, 8ull * n, cudaMemcpyDeviceToHost, s)));
        else for (uint32_t i = 0; i < n; ++i) res->j[i] = j0 + i;
    }
    std::vector<fi_inj> inj_h(n);
    fi_inj* inj_dst = res->inj ? res->inj : inj_h.data();
    if (n) FI_TRY(cu(cudaMemcpyAsync(inj_dst, inj, 24ull * n, cudaMemcpyDeviceToHost, s)));
    std::vector<uint64_t> ic_h(8ull * K);
    FI_TRY(cu(cudaMemcpyAsync(ic_h.data(), ic, 64ull * K, cudaMemcpyDeviceToHost, s)));
    FI_TRY(ev.mark(s));                                                    // 9
    FI_TRY(cu(cudaStreamSynchronize(s)));
    fi_status dev = check_status(st, s);

    if (res->inst_counts) std::memcpy(res->inst_counts, ic_h.data(), 64ull * K);
    std::memcpy(res->totals, totals, sizeof(totals));
    uint64_t counted = 0;
    for (uint32_t k = 0; k < K; ++k) counted += ic_h[8ull * k + FI_G_NODEST] + ic_h[8ull * k + FI_G_GPPR];
    res->counted = counted;
    res->n_rec = n_rec;
    res->j0 = j0;
    res->n_local = n;
    res->rec_begin = cfg->approximate ? 0 : r0;
    res->rec_end = cfg->approximate ? n_rec : r1;
    res->n_unclassified = res->n_not_injected = 0;
    for (uint32_t i = 0; i < n; ++i) {
        res->n_unclassified += inj_dst[i].outcome == 0xFF;
        res->n_not_injected += inj_dst[i].outcome == FI_NOT_INJECTED;
    }
    res->ms_h2d = ev.ms(0, 1);
    res->ms_golden = ev.ms(1, 2);
    res->ms_profile = ev.ms(2, 3);
    res->ms_exchange = ev.ms(3, 4);
    res->ms_index = ev.ms(4, 5);
    res->ms_select = ev.ms(5, 6);
    res->ms_inject = ev.ms(6, 7);
    res->ms_classify = ev.ms(7, 8);
    res->ms_d2h = ev.ms(8, 9);
    res->ms_jit = ms_jit;
    // a capacity overflow is reported per replica (outcome 0xFF), not as a failure
    return dev == FI_E_CAPACITY ? FI_OK : dev;
}

// "a profile containing one line for every dynamic kernel".
extern "C" fi_status fi_write_profile_txt(const uint64_t* ic, const fi_instance* inst, uint32_t n_inst,
                                          const char* const* names, uint32_t n_kern, char* buf, size_t buf_bytes,
                                          size_t* needed) {
    if ((n_inst && (!ic || !inst)) || (!names && n_kern) || (!buf && buf_bytes)) return FI_E_ARG;
    std::string out;
    char line[512];
    for (uint32_t k = 0; k < n_inst; ++k) {
        if (inst[k].kernel >= n_kern || !names[inst[k].kernel]) return FI_E_ARG;
        const uint64_t* c = ic + 8ull * k;
        int w = std::snprintf(line, sizeof line, "%s; kernel_count: %u; %llu %llu %llu %llu %llu %llu %llu %llu\n",
                              names[inst[k].kernel], inst[k].kernel_count, (unsigned long long)c[0],
                              (unsigned long long)c[1], (unsigned long long)c[2], (unsigned long long)c[3],
                              (unsigned long long)c[4], (unsigned long long)c[5], (unsigned long long)c[6],
                              (unsigned long long)c[7]);
        if (w < 0 || (size_t)w >= sizeof line) return FI_E_ARG;
        out.append(line, (size_t)w);
    }
    if (needed) *needed = out.size() + 1;
    if (!buf) return buf_bytes ? FI_E_ARG : FI_OK;
    if (out.size() + 1 > buf_bytes) return FI_E_ARG;
    std::memcpy(buf, out.c_str(), out.size() + 1);
    return FI_OK;
}

extern "C" fi_status fi_campaign_release_memory(int device) {
    int dev = device;
    if (dev < 0 && cudaGetDevice(&dev) != cudaSuccess) return FI_E_CUDA;
    cudaMemPool_t pool;
    FI_TRY(cu(cudaDeviceGetDefaultMemPool(&pool, dev)));
    FI_TRY(cu(cudaDeviceSynchronize()));
    return cu(cudaMemPoolTrimTo(pool, 0));
}
