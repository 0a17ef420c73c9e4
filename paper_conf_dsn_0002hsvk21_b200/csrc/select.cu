// select.cu — K2 site index (prefix sums) and K3 site selection.
//
// "A dynamic instruction will be selected from the set of executed
// instructions by choosing a random number n from the set 1..N ... This n-th
// instruction is then translated into a tuple of <kernel_name, kernel_count,
// instruction_count>"; Table II [PAPER.md:110-121] adds the destination register
// and bit-pattern values.  The random index is drawn with Philox4x32-10 + Lemire
// (C-5) and located with two prefix arrays instead of a walk over
// the trace: P_k over instances gives the instance and instruction_count, P_c
// over 1,024-record chunks gives the chunk; one warp then scans that chunk's
// records (warp inclusive scan + ballot) and picks the lane with __fns.
#include <algorithm>

#include "scan.cuh"

namespace fi {
namespace {

// Lemire's nearly-divisionless unbiased draw of s in [0, n) for replica j (C-5).
__device__ void draw(uint64_t seed, uint64_t j, uint64_t n, uint64_t& s, uint32_t& u_dst, uint32_t& u_bit) {
    const uint2 key = make_uint2((uint32_t)seed, (uint32_t)(seed >> 32));
    uint4 b = philox4x32_10(make_uint4((uint32_t)j, (uint32_t)(j >> 32), 0u, 0x46490001u), key);
    u_dst = b.z;
    u_bit = b.w;
    uint64_t x = (uint64_t)b.x | ((uint64_t)b.y << 32);
    uint64_t lo = x * n;
    if (lo < n) {
        const uint64_t t = (0ull - n) % n;
        for (uint32_t a = 1; lo < t; ++a) {
            b = philox4x32_10(make_uint4((uint32_t)j, (uint32_t)(j >> 32), a, 0x46490001u), key);
            x = (uint64_t)b.x | ((uint64_t)b.y << 32);
            lo = x * n;
        }
    }
    s = __umul64hi(x, n);
}

// Largest i in [0, m) with arr[i*stride + g] <= s, given arr[0] <= s < arr[m*stride+g]
// (monotone).  32-ary warp search: 31 probes per round, ballot narrows the range.
__device__ uint64_t warp_upper_search(const uint64_t* __restrict__ arr, uint64_t m, uint32_t stride, uint32_t g,
                                      uint64_t s) {
    const uint32_t lane = threadIdx.x & 31;
    uint64_t lo = 0, hi = m;
    while (hi - lo > 1) {
        const uint64_t d = hi - lo;
        const uint64_t p = lo + ((uint64_t)(lane + 1) * d) / 32;
        const bool le = lane < 31 && p > lo && p < hi && __ldg(&arr[p * stride + g]) <= s;
        const bool gt = lane < 31 && p > lo && p < hi && !le;
        const uint32_t bl = __ballot_sync(0xFFFFFFFFu, le), bg = __ballot_sync(0xFFFFFFFFu, gt);
        uint64_t nlo = lo, nhi = hi;
        if (bl) nlo = __shfl_sync(0xFFFFFFFFu, p, 31 - __clz(bl));
        if (bg) nhi = __shfl_sync(0xFFFFFFFFu, p, __ffs(bg) - 1);
        lo = nlo;
        hi = nhi;
    }
    return lo;
}

struct SelArgs {
    const fi_insn* code; const fi_kernel* kern; const fi_instance* inst;
    const uint4* rec; uint64_t n_rec; const uint64_t* warp_off; uint32_t n_warps;
    const uint64_t* Pk; uint32_t n_inst;
    const uint64_t* Pt; uint64_t n_tiles;         // prefix over 64-chunk tiles
    const uint32_t* cc; uint64_t n_chunks;        // chunk counts [C][8]
    uint64_t totals[8];
    fi_schedule sched;
    uint64_t j0; uint32_t n;
    fi_site* sites; uint32_t* status;
    uint64_t own_c0, own_c1;                      // owner-computes shard: chunks this rank holds the records of
};

constexpr int kWarps = 4;
constexpr uint32_t kTileChunks = 64;          // chunks per index tile (two-level chunk index)

__device__ void finish_site(const SelArgs& A, uint32_t i, uint32_t g, uint32_t bfm, uint64_t s, uint64_t ic,
                            uint32_t k, uint32_t w, uint64_t rec_idx, uint32_t rinsn, uint32_t lane_sel,
                            uint32_t u_dst, uint32_t u_bit);

__global__ void __launch_bounds__(kWarps * 32) k_select(const SelArgs A) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t i = blockIdx.x * kWarps + (threadIdx.x >> 5);
    if (i >= A.n) return;
    const uint64_t j = A.j0 + i;
    const uint32_t g = A.sched.groups[j % A.sched.n_groups];
    const uint32_t bfm = A.sched.bfms[(j / A.sched.n_groups) % A.sched.n_bfms];
    const uint64_t N = A.totals[g];

    uint64_t s = 0;
    uint32_t u_dst = 0, u_bit = 0;
    if (lane == 0) draw(A.sched.seed, j, N, s, u_dst, u_bit);
    s = __shfl_sync(0xFFFFFFFFu, s, 0);
    u_dst = __shfl_sync(0xFFFFFFFFu, u_dst, 0);
    u_bit = __shfl_sync(0xFFFFFFFFu, u_bit, 0);

    // instance: last k with P_k[k][g] <= s ; tile: last t with P_t[t][g] <= s
    const uint32_t k = (uint32_t)warp_upper_search(A.Pk, A.n_inst, 8, g, s);
    const uint64_t t = warp_upper_search(A.Pt, A.n_tiles, 8, g, s);
    uint64_t r = s - __ldg(&A.Pt[t * 8 + g]);
    // chunk inside the tile: warp scan of its (up to 64) chunk counts of group g
    uint64_t c = t * kTileChunks;
    for (uint32_t half = 0; half < kTileChunks; half += 32) {
        const uint64_t ci = t * kTileChunks + half + lane;
        const uint32_t cnt = ci < A.n_chunks ? __ldg(&A.cc[ci * 8 + g]) : 0u;
        uint32_t incl = cnt;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, d);
            if (lane >= (uint32_t)d) incl += y;
        }
        const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
        if (r < total) {
            const uint32_t L = __ffs(__ballot_sync(0xFFFFFFFFu, incl > r)) - 1;
            r -= __shfl_sync(0xFFFFFFFFu, incl - cnt, L);
            c = t * kTileChunks + half + L;
            break;
        }
        r -= total;
    }

    if (c < A.own_c0 || c >= A.own_c1) {          // another rank's records: drawn here, located there
        if (lane == 0) {
            fi_site S{};
            S.s = s; S.group = (uint8_t)g; S.bfm = (uint8_t)bfm; S.u_dst = u_dst; S.u_bit = u_bit;
            S.mask = bfm_mask(bfm, u_bit); S.flags = FI_SITE_REMOTE;
            A.sites[i] = S;
        }
        return;
    }
    // scan the chunk's records for the r-th counted lane-instruction of group g
    const uint64_t base = c * FI_CHUNK;
    const uint32_t nrec = (uint32_t)min((uint64_t)FI_CHUNK, A.n_rec - base);
    bool found = false;
    uint64_t rec_idx = 0;
    uint32_t rinst = 0, rinsn = 0, lane_sel = 0;
    for (uint32_t off = 0; off < nrec; off += 32) {
        const uint32_t idx = off + lane;
        const uint4 x = idx < nrec ? __ldg(&A.rec[base + idx]) : make_uint4(0, 0, 0, 0);
        const uint32_t ex = x.z & x.w;
        const uint32_t cnt = ((x.y >> (24 + g)) & 1u) ? __popc(ex) : 0u;
        uint32_t incl = cnt;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, d);
            if (lane >= (uint32_t)d) incl += y;
        }
        const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
        if (r < total) {
            const uint32_t hit = __ballot_sync(0xFFFFFFFFu, incl > r);
            const uint32_t L = __ffs(hit) - 1;
            const uint32_t before = __shfl_sync(0xFFFFFFFFu, incl - cnt, L);
            const uint32_t exL = __shfl_sync(0xFFFFFFFFu, ex, L);
            rinst = __shfl_sync(0xFFFFFFFFu, x.x, L);
            rinsn = __shfl_sync(0xFFFFFFFFu, x.y, L);
            lane_sel = __fns(exL, 0, (int)(r - before) + 1);      // (r-before)-th set bit, ascending (C-3)
            rec_idx = base + off + L;
            found = true;
            break;
        }
        r -= total;
    }
    if (!found || rinst != k) {
        if (lane == 0) FI_DEV_ERR(A.status, FI_E_SITE);
        return;
    }
    const uint32_t w = (uint32_t)warp_upper_search(A.warp_off, A.n_warps, 1, 0, rec_idx);
    if (lane != 0) return;
    finish_site(A, i, g, bfm, s, s - __ldg(&A.Pk[(uint64_t)k * 8 + g]), k, w, rec_idx, rinsn, lane_sel, u_dst, u_bit);
}

// Record the located site: warp-local step, thread, destination slot (C-6) and
// Table II mask (C-5, C-8).  Lane 0 only.
__device__ void finish_site(const SelArgs& A, uint32_t i, uint32_t g, uint32_t bfm, uint64_t s, uint64_t ic,
                            uint32_t k, uint32_t w, uint64_t rec_idx, uint32_t rinsn, uint32_t lane_sel,
                            uint32_t u_dst, uint32_t u_bit) {
    const fi_instance in = A.inst[k];
    const uint32_t wpc = (in.block + 31) / 32, lw = w - in.warp_begin;
    const uint32_t pc = rinsn & 0xFFFFu;
    const fi_insn I = A.code[A.kern[in.kernel].code_off + pc];
    const Dests d = dests_of(I.op, I.d0, I.d1, I.mod);
    const uint32_t ne = n_slots(d, g);
    if (ne == 0) { FI_DEV_ERR(A.status, FI_E_SITE); return; }
    const uint32_t slot = (uint32_t)(((uint64_t)ne * u_dst) >> 32);        // floor(n x value), C-5/C-6
    uint32_t kind, reg;
    slot_reg(d, g, slot, kind, reg);

    fi_site S;
    S.s = s;
    S.instruction_count = ic;
    S.instance = k;
    S.kernel_id = in.kernel;
    S.kernel_count = in.kernel_count;
    S.warp = w;
    S.step = (uint32_t)(rec_idx - __ldg(&A.warp_off[w]));
    S.thread = (lw / wpc) * in.block + (lw % wpc) * 32 + lane_sel;
    S.pc = pc;
    S.u_dst = u_dst;
    S.u_bit = u_bit;
    S.mask = bfm_mask(bfm, u_bit);
    S.lane = (uint8_t)lane_sel;
    S.group = (uint8_t)g;
    S.bfm = (uint8_t)bfm;
    S.slot = (uint8_t)slot;
    S.dst_kind = (uint8_t)kind;
    S.dst_reg = (uint8_t)reg;
    S.n_elig = (uint8_t)ne;
    S.flags = 0;
    A.sites[i] = S;
}

// Row f1: the approximate profile's P_k names (instance, instruction_count); the
// site is then found by counting through the instance's own records, as the
// injector does at run time (C-17: not injected when the instance is shorter).
__global__ void __launch_bounds__(kWarps * 32) k_select_approx(const SelArgs A) {
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t i = blockIdx.x * kWarps + (threadIdx.x >> 5);
    if (i >= A.n) return;
    const uint64_t j = A.j0 + i;
    const uint32_t g = A.sched.groups[j % A.sched.n_groups];
    const uint32_t bfm = A.sched.bfms[(j / A.sched.n_groups) % A.sched.n_bfms];
    uint64_t s = 0;
    uint32_t u_dst = 0, u_bit = 0;
    if (lane == 0) draw(A.sched.seed, j, A.totals[g], s, u_dst, u_bit);
    s = __shfl_sync(0xFFFFFFFFu, s, 0);
    u_dst = __shfl_sync(0xFFFFFFFFu, u_dst, 0);
    u_bit = __shfl_sync(0xFFFFFFFFu, u_bit, 0);
    const uint32_t k = (uint32_t)warp_upper_search(A.Pk, A.n_inst, 8, g, s);
    const uint64_t ic = s - __ldg(&A.Pk[(uint64_t)k * 8 + g]);
    const fi_instance in = A.inst[k];
    const uint64_t r0 = __ldg(&A.warp_off[in.warp_begin]), r1 = __ldg(&A.warp_off[in.warp_end]);
    uint64_t r = ic, rec_idx = 0;
    uint32_t rinsn = 0, lane_sel = 0;
    bool found = false;
    for (uint64_t base = r0; base < r1; base += 32) {
        const uint64_t idx = base + lane;
        const uint4 x = idx < r1 ? __ldg(&A.rec[idx]) : make_uint4(0, 0, 0, 0);
        const uint32_t ex = x.z & x.w;
        const uint32_t cnt = ((x.y >> (24 + g)) & 1u) ? __popc(ex) : 0u;
        uint32_t incl = cnt;
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, incl, d);
            if (lane >= (uint32_t)d) incl += y;
        }
        const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
        if (r < total) {
            const uint32_t L = __ffs(__ballot_sync(0xFFFFFFFFu, incl > r)) - 1;
            const uint32_t before = __shfl_sync(0xFFFFFFFFu, incl - cnt, L);
            const uint32_t exL = __shfl_sync(0xFFFFFFFFu, ex, L);
            rinsn = __shfl_sync(0xFFFFFFFFu, x.y, L);
            lane_sel = __fns(exL, 0, (int)(r - before) + 1);
            rec_idx = base + L;
            found = true;
            break;
        }
        r -= total;
    }
    if (!found) {                                      // C-17: the site does not exist in this instance
        if (lane == 0) {
            fi_site S = {};
            S.s = s; S.instruction_count = ic; S.instance = k; S.kernel_id = in.kernel;
            S.kernel_count = in.kernel_count; S.u_dst = u_dst; S.u_bit = u_bit; S.mask = bfm_mask(bfm, u_bit);
            S.group = (uint8_t)g; S.bfm = (uint8_t)bfm; S.flags = FI_SITE_NOT_INJECTED;
            A.sites[i] = S;
        }
        return;
    }
    const uint32_t w = (uint32_t)warp_upper_search(A.warp_off, A.n_warps, 1, 0, rec_idx);
    if (lane == 0) finish_site(A, i, g, bfm, s, ic, k, w, rec_idx, rinsn, lane_sel, u_dst, u_bit);
}

size_t align256(size_t x) { return (x + 255) & ~(size_t)255; }

uint64_t n_tiles_of(uint64_t n_chunks) { return (n_chunks + kTileChunks - 1) / kTileChunks; }

struct IndexLayout {
    size_t pk, pt, tsum, ws_k, ws_t, total;
};
IndexLayout layout(uint32_t n_inst, uint64_t n_chunks) {
    const uint64_t T = n_tiles_of(n_chunks);
    IndexLayout L;
    L.pk = 0;
    L.pt = align256(((size_t)n_inst + 1) * 8 * sizeof(uint64_t));
    L.tsum = L.pt + align256(((size_t)T + 1) * 8 * sizeof(uint64_t));
    L.ws_k = L.tsum + align256((size_t)std::max<uint64_t>(T, 1) * 8 * sizeof(uint64_t));
    L.ws_t = L.ws_k + align256(scan_rows_ws(n_inst, 8));
    L.total = L.ws_t + align256(scan_rows_ws(T, 8));
    return L;
}

// Table II identities [PAPER.md:101-104] (§8 row a3), checked on every count row:
// GP = FP64 + FP32 + LD + OTHERS, GPPR = GP + PR, and no group exceeds 32 lanes per record.
template <class T>
__device__ __forceinline__ bool identities_hold(const T c[8], uint64_t max_count) {
    bool ok = (uint64_t)c[FI_G_GP] == (uint64_t)c[FI_G_FP64] + c[FI_G_FP32] + c[FI_G_LD] + c[FI_G_OTHERS];
    ok = ok && (uint64_t)c[FI_G_GPPR] == (uint64_t)c[FI_G_GP] + c[FI_G_PR];
    for (int g = 0; g < 8; ++g) ok = ok && (uint64_t)c[g] <= max_count;
    return ok;
}

__global__ void k_inst_identities(const uint64_t* __restrict__ ic, uint32_t n_inst, uint32_t* status) {
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n_inst) return;
    uint64_t c[8];
    for (int g = 0; g < 8; ++g) c[g] = ic[(uint64_t)k * 8 + g];
    if (!identities_hold(c, ~0ull)) FI_DEV_ERR(status, FI_E_INVARIANT);
}

// per-tile sums of the chunk counts: one warp per 64-chunk tile (and the a3
// identities of every chunk row on the way)
__global__ void k_tile_sums(const uint32_t* __restrict__ cc, uint64_t n_chunks, uint64_t n_tiles,
                            uint64_t* __restrict__ tsum, uint32_t* status) {
    const uint64_t t = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t lane = threadIdx.x & 31;
    if (t >= n_tiles) return;
    uint64_t acc[8];
#pragma unroll
    for (int g = 0; g < 8; ++g) acc[g] = 0;
#pragma unroll
    for (uint32_t half = 0; half < kTileChunks; half += 32) {
        const uint64_t ci = t * kTileChunks + half + lane;
        if (ci < n_chunks) {
            const uint4 a = __ldg(reinterpret_cast<const uint4*>(cc + ci * 8));
            const uint4 b = __ldg(reinterpret_cast<const uint4*>(cc + ci * 8 + 4));
            acc[0] += a.x; acc[1] += a.y; acc[2] += a.z; acc[3] += a.w;
            acc[4] += b.x; acc[5] += b.y; acc[6] += b.z; acc[7] += b.w;
            const uint32_t row[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
            if (!identities_hold(row, 32ull * FI_CHUNK)) FI_DEV_ERR(status, FI_E_INVARIANT);
        }
    }
#pragma unroll
    for (int g = 0; g < 8; ++g) {
        const uint64_t v = __reduce_add_sync(0xFFFFFFFFu, (uint32_t)acc[g]);  // per-tile sum < 2^32 (64 x 1024 x 32)
        if (lane == (uint32_t)g) tsum[t * 8 + g] = v;
    }
}

}  // namespace
}  // namespace fi

using namespace fi;

extern "C" size_t fi_site_index_bytes(uint32_t n_inst, uint64_t n_chunks) { return layout(n_inst, n_chunks).total; }

extern "C" fi_status fi_build_site_index(const uint64_t* inst_counts, uint32_t n_inst, const uint32_t* chunk_counts,
                                         uint64_t n_chunks, void* index, uint32_t* dev_status, void* stream) {
    if (!inst_counts || !chunk_counts || !index || !dev_status) return FI_E_ARG;
    const IndexLayout L = layout(n_inst, n_chunks);
    char* b = reinterpret_cast<char*>(index);
    cudaStream_t s = (cudaStream_t)stream;
    fi_status e = scan_rows_u64x8(inst_counts, reinterpret_cast<uint64_t*>(b + L.pk), n_inst, b + L.ws_k,
                                  L.ws_t - L.ws_k, s);
    if (e) return e;
    const uint64_t T = n_tiles_of(n_chunks);
    uint64_t* tsum = reinterpret_cast<uint64_t*>(b + L.tsum);
    if (n_inst) {
        k_inst_identities<<<(n_inst + 127) / 128, 128, 0, s>>>(inst_counts, n_inst, dev_status);
        if ((e = launch_status())) return e;
    }
    if (T) {
        k_tile_sums<<<(unsigned)((T * 32 + 255) / 256), 256, 0, s>>>(chunk_counts, n_chunks, T, tsum, dev_status);
        if ((e = launch_status())) return e;
    }
    return scan_rows_u64x8(tsum, reinterpret_cast<uint64_t*>(b + L.pt), T, b + L.ws_t, L.total - L.ws_t, s);
}

extern "C" fi_status fi_site_totals(const void* index, uint32_t n_inst, uint64_t totals_host[8], void* stream) {
    if (!index || !totals_host) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    const uint64_t* pk = reinterpret_cast<const uint64_t*>(index);
    fi_status e = cuda_status(cudaMemcpyAsync(totals_host, pk + (size_t)n_inst * 8, 8 * sizeof(uint64_t),
                                              cudaMemcpyDeviceToHost, s));
    if (e) return e;
    return cuda_status(cudaStreamSynchronize(s));
}

static fi_status check_schedule(const fi_schedule* sched, const uint64_t totals_host[8]) {
    if (sched->n_groups == 0 || sched->n_groups > 8 || sched->n_bfms == 0 || sched->n_bfms > 4) return FI_E_ARG;
    for (uint32_t i = 0; i < sched->n_groups; ++i) {
        if (sched->groups[i] >= FI_NGROUPS) return FI_E_ARG;
        if (sched->groups[i] == FI_G_NODEST) return FI_E_NOT_INJECTABLE;     // C-16
        if (totals_host[sched->groups[i]] == 0) return FI_E_EMPTY_GROUP;
    }
    for (uint32_t i = 0; i < sched->n_bfms; ++i)
        if (sched->bfms[i] > FI_ZERO_VALUE) return FI_E_ARG;
    return FI_OK;
}

extern "C" fi_status fi_build_instance_index(const uint64_t* inst_counts, uint32_t n_inst, void* index,
                                             uint32_t* dev_status, void* stream) {
    if (!inst_counts || !index || !dev_status) return FI_E_ARG;
    const IndexLayout L = layout(n_inst, 0);
    char* b = reinterpret_cast<char*>(index);
    cudaStream_t s = (cudaStream_t)stream;
    if (n_inst) {
        k_inst_identities<<<(n_inst + 127) / 128, 128, 0, s>>>(inst_counts, n_inst, dev_status);
        fi_status e = launch_status();
        if (e) return e;
    }
    return scan_rows_u64x8(inst_counts, reinterpret_cast<uint64_t*>(b + L.pk), n_inst, b + L.ws_k, L.ws_t - L.ws_k, s);
}

extern "C" fi_status fi_select_sites_approx(const fi_program* p, const fi_trace* t, const void* index, uint32_t n_inst,
                                            const uint64_t totals_host[8], const fi_schedule* sched, uint64_t j0,
                                            uint32_t n, fi_site* sites, uint32_t* dev_status, void* stream) {
    if (!p || !t || !index || !totals_host || !sched || !sites || !dev_status) return FI_E_ARG;
    fi_status e = check_schedule(sched, totals_host);
    if (e || n == 0) return e;
    const IndexLayout L = layout(n_inst, 0);
    SelArgs A = {};
    A.code = p->code; A.kern = p->kern; A.inst = p->inst;
    A.rec = reinterpret_cast<const uint4*>(t->rec); A.n_rec = t->n_rec; A.warp_off = t->warp_off; A.n_warps = t->n_warps;
    A.Pk = reinterpret_cast<const uint64_t*>(reinterpret_cast<const char*>(index) + L.pk); A.n_inst = n_inst;
    for (int g = 0; g < 8; ++g) A.totals[g] = totals_host[g];
    A.sched = *sched;
    A.j0 = j0; A.n = n; A.sites = sites; A.status = dev_status;
    k_select_approx<<<(n + kWarps - 1) / kWarps, kWarps * 32, 0, (cudaStream_t)stream>>>(A);
    return launch_status();
}

extern "C" fi_status fi_select_sites(const fi_program* p, const fi_trace* t, const uint32_t* chunk_counts,
                                     const void* index, uint32_t n_inst, uint64_t n_chunks,
                                     const uint64_t totals_host[8], const fi_schedule* sched, uint64_t j0, uint32_t n,
                                     fi_site* sites, uint32_t* dev_status, void* stream) {
    if (!p || !t || !index || !chunk_counts || !totals_host || !sched || !sites || !dev_status) return FI_E_ARG;
    fi_status e = check_schedule(sched, totals_host);
    if (e || n == 0) return e;
    const IndexLayout L = layout(n_inst, n_chunks);
    const char* b = reinterpret_cast<const char*>(index);
    SelArgs A;
    A.code = p->code; A.kern = p->kern; A.inst = p->inst;
    A.rec = reinterpret_cast<const uint4*>(t->rec); A.n_rec = t->n_rec; A.warp_off = t->warp_off; A.n_warps = t->n_warps;
    A.Pk = reinterpret_cast<const uint64_t*>(b + L.pk); A.n_inst = n_inst;
    A.Pt = reinterpret_cast<const uint64_t*>(b + L.pt); A.n_tiles = n_tiles_of(n_chunks);
    A.cc = chunk_counts; A.n_chunks = n_chunks;
    for (int g = 0; g < 8; ++g) A.totals[g] = totals_host[g];
    A.sched = *sched;
    A.j0 = j0; A.n = n; A.sites = sites; A.status = dev_status;
    A.own_c0 = 0; A.own_c1 = ~0ull;
    k_select<<<(n + kWarps - 1) / kWarps, kWarps * 32, 0, (cudaStream_t)stream>>>(A);
    return launch_status();
}

extern "C" fi_status fi_select_sites_shard(const fi_program* p, const fi_trace* t, const uint32_t* chunk_counts,
                                           const void* index, uint32_t n_inst, uint64_t n_chunks,
                                           const uint64_t totals_host[8], const fi_schedule* sched, uint64_t j0,
                                           uint32_t n, uint64_t rec_begin, uint64_t rec_end, fi_site* sites,
                                           uint32_t* dev_status, void* stream) {
    if (!p || !t || !index || !chunk_counts || !totals_host || !sched || !sites || !dev_status) return FI_E_ARG;
    if (rec_begin % FI_CHUNK || rec_begin > rec_end || (rec_end % FI_CHUNK && rec_end != t->n_rec)) return FI_E_ARG;
    fi_status e = check_schedule(sched, totals_host);
    if (e || n == 0) return e;
    const IndexLayout L = layout(n_inst, n_chunks);
    const char* b = reinterpret_cast<const char*>(index);
    SelArgs A;
    A.code = p->code; A.kern = p->kern; A.inst = p->inst;
    A.rec = reinterpret_cast<const uint4*>(t->rec); A.n_rec = t->n_rec; A.warp_off = t->warp_off; A.n_warps = t->n_warps;
    A.Pk = reinterpret_cast<const uint64_t*>(b + L.pk); A.n_inst = n_inst;
    A.Pt = reinterpret_cast<const uint64_t*>(b + L.pt); A.n_tiles = n_tiles_of(n_chunks);
    A.cc = chunk_counts; A.n_chunks = n_chunks;
    for (int g = 0; g < 8; ++g) A.totals[g] = totals_host[g];
    A.sched = *sched;
    A.j0 = j0; A.n = n; A.sites = sites; A.status = dev_status;
    A.own_c0 = rec_begin / FI_CHUNK;
    A.own_c1 = (rec_end + FI_CHUNK - 1) / FI_CHUNK;
    k_select<<<(n + kWarps - 1) / kWarps, kWarps * 32, 0, (cudaStream_t)stream>>>(A);
    return launch_status();
}

// Stable compaction of the sites this rank located (flags without FI_SITE_REMOTE):
// one CTA, 1,024 sites per pass, a block-wide scan of the keep flags; the
// replica index j0 + i of each kept site goes to out_j.
namespace fi {
namespace {
__global__ void __launch_bounds__(1024) k_compact_sites(const fi_site* __restrict__ in, uint32_t n, uint64_t j0,
                                                        fi_site* __restrict__ out, uint64_t* __restrict__ out_j,
                                                        uint32_t* n_out) {
    __shared__ uint32_t wsum[32];
    __shared__ uint32_t carry;
    const uint32_t t = threadIdx.x, lane = t & 31, wid = t >> 5;
    if (t == 0) carry = 0;
    __syncthreads();
    for (uint32_t base = 0; base < n; base += 1024) {
        const uint32_t i = base + t;
        const bool keep = i < n && !(in[i].flags & FI_SITE_REMOTE);
        const uint32_t m = __ballot_sync(0xFFFFFFFFu, keep);
        if (lane == 0) wsum[wid] = __popc(m);
        __syncthreads();
        if (wid == 0) {
            uint32_t v = wsum[lane], x = v;
#pragma unroll
            for (int d = 1; d < 32; d <<= 1) {
                const uint32_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
                if (lane >= (uint32_t)d) x += y;
            }
            wsum[lane] = x - v;                       // exclusive prefix of the warps' counts
        }
        __syncthreads();
        const uint32_t pos = carry + wsum[wid] + __popc(m & ((1u << lane) - 1));
        if (keep) { out[pos] = in[i]; out_j[pos] = j0 + i; }
        __syncthreads();
        if (t == 1023) carry = pos + (keep ? 1u : 0u);
        __syncthreads();
    }
    if (t == 0) *n_out = carry;
}
}  // namespace
}  // namespace fi

extern "C" fi_status fi_compact_sites(const fi_site* sites, uint32_t n, uint64_t j0, fi_site* out, uint64_t* out_j,
                                      uint32_t* n_out, void* stream) {
    if (!n_out || (n && (!sites || !out || !out_j))) return FI_E_ARG;
    fi::k_compact_sites<<<1, 1024, 0, (cudaStream_t)stream>>>(sites, n, j0, out, out_j, n_out);
    return launch_status();
}
