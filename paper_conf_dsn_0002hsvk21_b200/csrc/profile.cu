// profile.cu — K1, the exact profiler (§III-A) as an HBM scan.
//
// "a profile containing one line for every dynamic kernel and the total dynamic
// instruction counts ... in every thread ... Instructions that are not executed
// based on a predicate register are not included" [PAPER.md:78], grouped by the
// Table II arch state ids [PAPER.md:94-104]:
//   inst_counts[k][g]  += popc(active & pred) for every record of instance k in group g
//   chunk_counts[c][g]  = the same sum over the 1,024-record chunk c
// One 16-B record per warp-instruction (App. A.3) is the only input, read once
// with 128-bit streaming loads (L1::no_allocate), 8 loads in flight per lane.
// Each warp owns a contiguous run of chunks; per-lane u32 counters are reduced
// with REDUX (__reduce_add_sync) once per chunk, chunk counts are plain stores,
// and instance counts stay in lanes 0-7 until the instance changes (one u64
// atomic per group per instance per warp).  Chunks that straddle instances
// (rare: instance boundaries) attribute per record.
#include <algorithm>
#include <cstring>
#include <vector>

#include "common.cuh"

namespace fi {
namespace {

constexpr int kThreads = 256;
constexpr int kUnroll = 8;
constexpr uint32_t kNone = 0xFFFFFFFFu;

__device__ __forceinline__ uint4 ld_stream(const uint4* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// PEERS (fi_profile_peers, the multi-GPU path fused with its exchange): every
// chunk-count row also goes straight into each peer rank's chunk_counts over
// NVLink (P.cc[r], IPC-mapped), as the chunk is finished
struct PeerOut {
    uint32_t* cc[FI_MAX_PEERS];
    uint32_t world, rank;
};

template <bool PEERS>
__global__ void __launch_bounds__(kThreads)
k_profile(const uint4* __restrict__ rec, uint64_t r_begin, uint64_t r_end, uint64_t c_begin, uint64_t c_end,
          uint64_t* __restrict__ inst_counts, uint32_t* __restrict__ chunk_counts, const PeerOut P) {
    const uint32_t lane = threadIdx.x & 31;
    const uint64_t gw = ((uint64_t)blockIdx.x * kThreads + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * kThreads) >> 5;
    const uint64_t nch = c_end - c_begin;
    const uint64_t per = (nch + nwarps - 1) / nwarps;
    const uint64_t c0 = c_begin + gw * per;
    const uint64_t c1 = min(c0 + per, c_end);

    uint32_t cur_k = kNone;
    uint64_t acc = 0;                         // lane g < 8: running count of group g for cur_k
    for (uint64_t c = c0; c < c1; ++c) {
        const uint64_t a = max(c * FI_CHUNK, r_begin);
        const uint64_t b = min(c * FI_CHUNK + FI_CHUNK, r_end);
        const uint32_t n = (uint32_t)(b - a);
        const uint4* base = rec + a;
        const uint32_t kf = __ldg(&base[0].x), kl = __ldg(&base[n - 1].x);
        uint32_t cnt[8];
#pragma unroll
        for (int g = 0; g < 8; ++g) cnt[g] = 0;
        for (uint32_t i = lane; i < n; i += 32 * kUnroll) {
            uint4 r[kUnroll];
#pragma unroll
            for (int u = 0; u < kUnroll; ++u)
                r[u] = (i + u * 32 < n) ? ld_stream(base + i + u * 32) : make_uint4(0, 0, 0, 0);
#pragma unroll
            for (int u = 0; u < kUnroll; ++u) {
                const uint32_t cc = __popc(r[u].z & r[u].w);
                const uint32_t gm = r[u].y >> 24;
#pragma unroll
                for (int g = 0; g < 8; ++g) cnt[g] += ((gm >> g) & 1u) ? cc : 0u;
            }
        }
        uint32_t mine = 0;
#pragma unroll
        for (int g = 0; g < 8; ++g) {
            const uint32_t s = __reduce_add_sync(0xFFFFFFFFu, cnt[g]);
            if (lane == (uint32_t)g) mine = s;
        }
        if (lane < 8) {
            chunk_counts[c * 8 + lane] = mine;
            if (PEERS)
                for (uint32_t r = 0; r < P.world; ++r)
                    if (r != P.rank) P.cc[r][c * 8 + lane] = mine;
        }
        if (kf == kl) {
            if (kf != cur_k) {
                if (cur_k != kNone && lane < 8 && acc) atomicAdd((unsigned long long*)&inst_counts[(uint64_t)cur_k * 8 + lane], acc);
                cur_k = kf;
                acc = 0;
            }
            acc += mine;
        } else {
            for (uint32_t i = lane; i < n; i += 32) {
                const uint4 r = __ldg(base + i);
                const uint32_t cc = __popc(r.z & r.w);
                const uint32_t gm = r.y >> 24;
                if (cc)
                    for (int g = 0; g < 8; ++g)
                        if ((gm >> g) & 1u) atomicAdd((unsigned long long*)&inst_counts[(uint64_t)r.x * 8 + g], (unsigned long long)cc);
            }
        }
    }
    if (cur_k != kNone && lane < 8 && acc) atomicAdd((unsigned long long*)&inst_counts[(uint64_t)cur_k * 8 + lane], acc);
}

int g_grid = 0;

// ---- §8 row f1: per-opcode profile ("counts for every opcode") ----
// One warp per contiguous run of records; a per-warp shared-memory histogram over
// the 32 opcode slots for the current instance, flushed with one u64 atomic per
// nonzero opcode when the instance changes (records of a chunk that straddles an
// instance boundary go straight to global atomics).
constexpr int kOpThreads = 256;

__global__ void __launch_bounds__(kOpThreads)
k_profile_opcodes(const uint4* __restrict__ rec, uint64_t r_begin, uint64_t r_end, uint64_t* __restrict__ op_counts) {
    __shared__ uint32_t hist[kOpThreads / 32][FI_NOPS];
    const uint32_t lane = threadIdx.x & 31, wib = threadIdx.x >> 5;
    const uint64_t gw = ((uint64_t)blockIdx.x * kOpThreads + threadIdx.x) >> 5;
    const uint64_t nwarps = ((uint64_t)gridDim.x * kOpThreads) >> 5;
    const uint64_t n = r_end - r_begin;
    const uint64_t per = ((n + nwarps - 1) / nwarps + 31) & ~31ull;
    const uint64_t a = r_begin + gw * per, b = min(a + per, r_end);
    uint32_t* h = hist[wib];
    h[lane] = 0;
    __syncwarp();
    uint32_t cur = kNone;
    for (uint64_t base = a; base < b; base += 32) {
        const uint64_t r = base + lane;
        const uint4 x = r < b ? ld_stream(rec + r) : make_uint4(kNone, 0, 0, 0);
        const uint32_t k0 = __shfl_sync(0xFFFFFFFFu, x.x, 0);
        if (k0 != cur) {                                  // flush the finished instance
            __syncwarp();
            if (cur != kNone && h[lane]) atomicAdd((unsigned long long*)&op_counts[(uint64_t)cur * FI_NOPS + lane], (unsigned long long)h[lane]);
            h[lane] = 0;
            __syncwarp();
            cur = k0;
        }
        const uint32_t c = __popc(x.z & x.w);
        const uint32_t op = (x.y >> 16) & (FI_NOPS - 1);
        if (r < b && c) {
            if (x.x == cur) atomicAdd(&h[op], c);
            else atomicAdd((unsigned long long*)&op_counts[(uint64_t)x.x * FI_NOPS + op], (unsigned long long)c);
        }
    }
    __syncwarp();
    if (cur != kNone && h[lane]) atomicAdd((unsigned long long*)&op_counts[(uint64_t)cur * FI_NOPS + lane], (unsigned long long)h[lane]);
}

// ---- §8 row f1: approximate profiling ----------------------------
// Count only the records of the first dynamic instance of each static kernel
// (one instance's record range per blockIdx.y) ...
__global__ void __launch_bounds__(kThreads)
k_profile_first(const uint4* __restrict__ rec, const uint64_t* __restrict__ warp_off,
                const fi_instance* __restrict__ inst, const uint32_t* __restrict__ firsts,
                uint64_t* __restrict__ inst_counts) {
    const uint32_t k = firsts[blockIdx.y];
    const uint64_t r0 = warp_off[inst[k].warp_begin], r1 = warp_off[inst[k].warp_end];
    const uint32_t lane = threadIdx.x & 31;
    uint32_t cnt[8];
#pragma unroll
    for (int g = 0; g < 8; ++g) cnt[g] = 0;
    for (uint64_t r = r0 + (uint64_t)blockIdx.x * kThreads + threadIdx.x; r < r1; r += (uint64_t)gridDim.x * kThreads) {
        const uint4 x = ld_stream(rec + r);
        const uint32_t c = __popc(x.z & x.w), gm = x.y >> 24;
#pragma unroll
        for (int g = 0; g < 8; ++g) cnt[g] += ((gm >> g) & 1u) ? c : 0u;
    }
#pragma unroll
    for (int g = 0; g < 8; ++g) {
        const uint32_t s = __reduce_add_sync(0xFFFFFFFFu, cnt[g]);
        if (lane == 0 && s) atomicAdd((unsigned long long*)&inst_counts[(uint64_t)k * 8 + g], (unsigned long long)s);
    }
}

// ... and assume every later instance of the same static kernel has the same counts.
__global__ void k_expand_first(const fi_instance* __restrict__ inst, uint32_t n_inst,
                               const uint32_t* __restrict__ first_of_kernel, uint64_t* __restrict__ counts,
                               uint32_t width) {
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n_inst) return;
    const uint32_t f = first_of_kernel[inst[k].kernel];
    if (f == k) return;
    for (uint32_t g = 0; g < width; ++g) counts[(uint64_t)k * width + g] = counts[(uint64_t)f * width + g];
}

}  // namespace
}  // namespace fi

using namespace fi;

extern "C" fi_status fi_profile(const fi_trace* t, uint64_t rec_begin, uint64_t rec_end, uint32_t n_inst,
                                uint64_t* inst_counts, uint32_t* chunk_counts, void* stream) {
    if (!t || !inst_counts || !chunk_counts || rec_end > t->n_rec || rec_begin > rec_end) return FI_E_ARG;
    if (rec_begin % FI_CHUNK) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    fi_status e = cuda_status(cudaMemsetAsync(inst_counts, 0, (size_t)n_inst * 8 * sizeof(uint64_t), s));
    if (e || rec_begin == rec_end) return e;
    if (!g_grid) {
        int dev = 0, sms = 0, per = 0;
        cudaGetDevice(&dev);
        cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
        cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_profile<false>, kThreads, 0);
        g_grid = std::max(1, sms * std::max(1, per));
    }
    const uint64_t c_begin = rec_begin / FI_CHUNK, c_end = (rec_end + FI_CHUNK - 1) / FI_CHUNK;
    const uint64_t warps_needed = c_end - c_begin;
    const int grid = (int)std::min<uint64_t>((uint64_t)g_grid, (warps_needed * 32 + kThreads - 1) / kThreads);
    k_profile<false><<<grid, kThreads, 0, s>>>(reinterpret_cast<const uint4*>(t->rec), rec_begin, rec_end, c_begin,
                                                c_end, inst_counts, chunk_counts, PeerOut{});
    return launch_status();
}

// ---- multi-GPU profile fused with its exchange -------------------
namespace fi {
namespace {
// this rank's partial instance counts into slot [rank] of every rank's partials
__global__ void k_push_partials(const uint64_t* __restrict__ part, uint64_t n, fi_peers P) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        const uint64_t v = part[i];
        for (uint32_t r = 0; r < P.world; ++r) P.partials[r][(uint64_t)P.rank * n + i] = v;
    }
}
// release: everything this rank wrote to its peers is visible before its flag
// increment reaches them (system scope)
__global__ void k_signal(fi_peers P) {
    __threadfence_system();
    for (uint32_t r = 0; r < P.world; ++r) atomicAdd_system(P.flags[r], 1u);
}
// acquire: wait until every rank's increment of this epoch arrived.  Bounded: a
// rank that has not signalled after 60 s (it died, or is skewed by more than
// that) makes the wait give up and set FI_E_COLLECTIVE in the caller's status
// word — the call's counts are then not valid, but the context stays usable.
__device__ __forceinline__ uint64_t globaltimer_ns() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}
__global__ void k_wait(const uint32_t* flag, uint32_t target, uint32_t* status) {
    const uint64_t t0 = globaltimer_ns();
    while (*reinterpret_cast<const volatile uint32_t*>(flag) < target) {
        __nanosleep(200);
        if (globaltimer_ns() - t0 > 60ull * 1000000000ull) { FI_DEV_ERR(status, FI_E_COLLECTIVE); return; }
    }
    __threadfence_system();
}
__global__ void k_sum_partials(const uint64_t* __restrict__ part, uint64_t n, uint32_t world, uint64_t* __restrict__ out) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
        uint64_t s = 0;
        for (uint32_t r = 0; r < world; ++r) s += part[(uint64_t)r * n + i];
        out[i] = s;
    }
}
}  // namespace
}  // namespace fi

extern "C" fi_status fi_ipc_alloc(size_t bytes, void** dev_ptr, void* handle) {
    if (!dev_ptr || !handle) return FI_E_ARG;
    void* p = nullptr;
    fi_status e = cuda_status(cudaMalloc(&p, std::max<size_t>(bytes, 256)));
    if (e) return e;
    if ((e = cuda_status(cudaMemset(p, 0, std::max<size_t>(bytes, 256))))) { cudaFree(p); return e; }
    cudaIpcMemHandle_t h;
    if ((e = cuda_status(cudaIpcGetMemHandle(&h, p)))) { cudaFree(p); return e; }
    std::memcpy(handle, &h, sizeof h);
    *dev_ptr = p;
    return FI_OK;
}
extern "C" fi_status fi_ipc_open(const void* handle, void** dev_ptr) {
    if (!handle || !dev_ptr) return FI_E_ARG;
    cudaIpcMemHandle_t h;
    std::memcpy(&h, handle, sizeof h);
    return cuda_status(cudaIpcOpenMemHandle(dev_ptr, h, cudaIpcMemLazyEnablePeerAccess));
}
extern "C" fi_status fi_ipc_close(void* dev_ptr) { return cuda_status(cudaIpcCloseMemHandle(dev_ptr)); }
extern "C" fi_status fi_ipc_free(void* dev_ptr) { return cuda_status(cudaFree(dev_ptr)); }

extern "C" fi_status fi_profile_peers(const fi_trace* t, uint64_t rec_begin, uint64_t rec_end, uint32_t n_inst,
                                      const fi_peers* peers, uint64_t* part_local, uint32_t epoch,
                                      uint64_t* inst_counts, uint32_t* chunk_counts, uint32_t* dev_status,
                                      void* stream) {
    if (!t || !peers || !part_local || !inst_counts || !chunk_counts || !dev_status || rec_end > t->n_rec ||
        rec_begin > rec_end)
        return FI_E_ARG;
    if (rec_begin % FI_CHUNK || peers->world < 1 || peers->world > FI_MAX_PEERS || peers->rank >= peers->world ||
        epoch == 0)
        return FI_E_ARG;
    const fi_peers P = *peers;
    for (uint32_t r = 0; r < P.world; ++r)
        if (!P.chunk_counts[r] || !P.partials[r] || !P.flags[r]) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    const uint64_t n = (uint64_t)n_inst * 8;
    fi_status e = cuda_status(cudaMemsetAsync(part_local, 0, n * sizeof(uint64_t), s));
    if (e) return e;
    if (rec_begin < rec_end) {
        if (!g_grid) {
            int dev = 0, sms = 0, per = 0;
            cudaGetDevice(&dev);
            cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
            cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, k_profile<false>, kThreads, 0);
            g_grid = std::max(1, sms * std::max(1, per));
        }
        const uint64_t c_begin = rec_begin / FI_CHUNK, c_end = (rec_end + FI_CHUNK - 1) / FI_CHUNK;
        const int grid = (int)std::min<uint64_t>((uint64_t)g_grid, ((c_end - c_begin) * 32 + kThreads - 1) / kThreads);
        PeerOut po{};
        for (uint32_t r = 0; r < P.world; ++r) po.cc[r] = P.chunk_counts[r];
        po.world = P.world;
        po.rank = P.rank;
        k_profile<true><<<grid, kThreads, 0, s>>>(reinterpret_cast<const uint4*>(t->rec), rec_begin, rec_end, c_begin,
                                                   c_end, part_local, P.chunk_counts[P.rank], po);
        if ((e = launch_status())) return e;
    }
    const uint32_t pg = (uint32_t)std::min<uint64_t>(std::max<uint64_t>(1, (n + 255) / 256), 1184);
    k_push_partials<<<pg, 256, 0, s>>>(part_local, n, P);
    k_signal<<<1, 1, 0, s>>>(P);
    k_wait<<<1, 1, 0, s>>>(P.flags[P.rank], epoch * P.world, dev_status);
    k_sum_partials<<<pg, 256, 0, s>>>(P.partials[P.rank], n, P.world, inst_counts);
    if ((e = launch_status())) return e;
    const uint64_t C = (t->n_rec + FI_CHUNK - 1) / FI_CHUNK;  // every rank's rows, now complete, to the caller's array
    return cuda_status(cudaMemcpyAsync(chunk_counts, P.chunk_counts[P.rank], C * 8 * sizeof(uint32_t),
                                       cudaMemcpyDeviceToDevice, s));
}

extern "C" fi_status fi_profile_opcodes(const fi_trace* t, uint64_t rec_begin, uint64_t rec_end, uint32_t n_inst,
                                        uint64_t* op_counts, void* stream) {
    if (!t || !op_counts || rec_end > t->n_rec || rec_begin > rec_end) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    fi_status e = cuda_status(cudaMemsetAsync(op_counts, 0, (size_t)n_inst * FI_NOPS * sizeof(uint64_t), s));
    if (e || rec_begin == rec_end) return e;
    int dev = 0, sms = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const uint64_t warps = (rec_end - rec_begin + 1023) / 1024;
    const int grid = (int)std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)sms * 8, (warps * 32 + kOpThreads - 1) / kOpThreads));
    k_profile_opcodes<<<grid, kOpThreads, 0, s>>>(reinterpret_cast<const uint4*>(t->rec), rec_begin, rec_end, op_counts);
    return launch_status();
}

extern "C" size_t fi_profile_approx_workspace(uint32_t n_kern, uint32_t n_inst) {
    (void)n_inst;
    return 256 + 2 * (size_t)std::max<uint32_t>(n_kern, 1) * sizeof(uint32_t);
}

extern "C" fi_status fi_profile_approx(const fi_program* p, const fi_trace* t, uint64_t* inst_counts, void* ws,
                                       size_t ws_bytes, void* stream) {
    if (!p || !t || !inst_counts || !p->inst_host || !ws || ws_bytes < fi_profile_approx_workspace(p->n_kern, p->n_inst))
        return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<uint32_t> first_of(std::max<uint32_t>(p->n_kern, 1), 0xFFFFFFFFu), firsts;
    for (uint32_t k = 0; k < p->n_inst; ++k) {
        const fi_instance& in = p->inst_host[k];
        if (in.kernel < p->n_kern && first_of[in.kernel] == 0xFFFFFFFFu) {
            first_of[in.kernel] = k;
            firsts.push_back(k);
        }
    }
    uint32_t* d_first_of = reinterpret_cast<uint32_t*>(reinterpret_cast<char*>(ws) + 256);
    uint32_t* d_firsts = d_first_of + std::max<uint32_t>(p->n_kern, 1);
    fi_status e = cuda_status(cudaMemsetAsync(inst_counts, 0, (size_t)p->n_inst * 8 * sizeof(uint64_t), s));
    if (e || firsts.empty()) return e;
    if ((e = cuda_status(cudaMemcpyAsync(d_first_of, first_of.data(), first_of.size() * 4, cudaMemcpyHostToDevice, s)))) return e;
    if ((e = cuda_status(cudaMemcpyAsync(d_firsts, firsts.data(), firsts.size() * 4, cudaMemcpyHostToDevice, s)))) return e;
    if ((e = cuda_status(cudaStreamSynchronize(s)))) return e;      // host vectors go out of scope
    dim3 grid(64, (unsigned)firsts.size());
    k_profile_first<<<grid, kThreads, 0, s>>>(reinterpret_cast<const uint4*>(t->rec), t->warp_off, p->inst, d_firsts,
                                              inst_counts);
    if ((e = launch_status())) return e;
    k_expand_first<<<(p->n_inst + 127) / 128, 128, 0, s>>>(p->inst, p->n_inst, d_first_of, inst_counts, 8);
    return launch_status();
}
