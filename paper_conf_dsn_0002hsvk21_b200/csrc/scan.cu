// scan.cu — K2: exclusive prefix sums with a hand-written decoupled lookback
// (Merrill & Garland single-pass scan), no CUB.  Used for
//   P_k[n_inst+1][8]   over inst_counts  (u64 rows of 8)   — "1..N" of PAPER.md:78
//   P_c[n_chunks+1][8] over chunk_counts (u32 rows of 8)
//   warp_off / gstore_off over per-warp lengths (u64, width 1)
// HBM-bound: one read of the input and one write of the output per row.
#include "scan.cuh"

namespace fi {

namespace {

constexpr int kThreads = 256;

template <int W>
struct TileState {
    uint64_t agg[W];
    uint64_t inc[W];
    uint32_t flag;           // 0 = not ready (X), 1 = aggregate (A), 2 = inclusive prefix (P)
    uint32_t pad[3];
};

template <typename Tin, int W, int ITEMS>
__global__ void __launch_bounds__(kThreads)
k_scan_rows(const Tin* __restrict__ in, uint64_t* __restrict__ out, uint64_t n_rows,
            TileState<W>* __restrict__ st, uint32_t* __restrict__ counter) {
    __shared__ uint32_t s_tile;
    __shared__ uint64_t s_warp[kThreads / 32][W];
    __shared__ uint64_t s_prefix[W];
    if (threadIdx.x == 0) s_tile = atomicAdd(counter, 1u);      // tiles start in launch order
    __syncthreads();
    const uint32_t tile = s_tile;
    const uint64_t row0 = (uint64_t)tile * kThreads * ITEMS + (uint64_t)threadIdx.x * ITEMS;
    const uint32_t lane = threadIdx.x & 31, wid = threadIdx.x >> 5;

    uint64_t v[ITEMS][W];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i)
#pragma unroll
        for (int g = 0; g < W; ++g)
            v[i][g] = (row0 + i < n_rows) ? (uint64_t)__ldg(&in[(row0 + i) * W + g]) : 0ull;

    uint64_t tot[W];
#pragma unroll
    for (int g = 0; g < W; ++g) {
        uint64_t s = 0;
#pragma unroll
        for (int i = 0; i < ITEMS; ++i) s += v[i][g];
        tot[g] = s;
    }
    // warp inclusive scan of the per-thread totals
    uint64_t inc[W];
#pragma unroll
    for (int g = 0; g < W; ++g) {
        uint64_t x = tot[g];
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
            uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
            if (lane >= (uint32_t)d) x += y;
        }
        inc[g] = x;
        if (lane == 31) s_warp[wid][g] = x;
    }
    __syncthreads();
    if (wid == 0) {                                   // scan the 8 warp totals
#pragma unroll
        for (int g = 0; g < W; ++g) {
            uint64_t x = lane < kThreads / 32 ? s_warp[lane][g] : 0ull;
#pragma unroll
            for (int d = 1; d < kThreads / 32; d <<= 1) {
                uint64_t y = __shfl_up_sync(0xFFFFFFFFu, x, d);
                if (lane >= (uint32_t)d) x += y;
            }
            if (lane < kThreads / 32) s_warp[lane][g] = x;   // inclusive over warps
        }
    }
    __syncthreads();
    if (wid == 0) {
        // decoupled lookback, one warp: publish this tile's aggregate, then look at
        // 32 predecessors per probe; the nearest one with an inclusive prefix (P)
        // ends the walk, the aggregate-only (A) ones in front of it are added.
        uint64_t agg[W];
#pragma unroll
        for (int g = 0; g < W; ++g) agg[g] = s_warp[kThreads / 32 - 1][g];
        if (tile == 0) {
            if (lane == 0) {
#pragma unroll
                for (int g = 0; g < W; ++g) { st[0].inc[g] = agg[g]; s_prefix[g] = 0; }
                __threadfence();
                *(volatile uint32_t*)&st[0].flag = 2u;
            }
        } else {
            if (lane == 0) {
#pragma unroll
                for (int g = 0; g < W; ++g) st[tile].agg[g] = agg[g];
                __threadfence();
                *(volatile uint32_t*)&st[tile].flag = 1u;
            }
            uint64_t pre[W];
#pragma unroll
            for (int g = 0; g < W; ++g) pre[g] = 0;
            for (int64_t base = (int64_t)tile - 1;; base -= 32) {
                const int64_t p = base - (int64_t)lane;
                uint32_t f = p >= 0 ? *(volatile uint32_t*)&st[p].flag : 2u;
                while (__any_sync(0xFFFFFFFFu, f == 0u))
                    if (f == 0u) f = *(volatile uint32_t*)&st[p].flag;
                __threadfence();
                const uint32_t pm = __ballot_sync(0xFFFFFFFFu, f == 2u);
                const uint32_t stop = pm ? (uint32_t)(__ffs(pm) - 1) : 32u;
                if (p >= 0 && lane <= stop) {
#pragma unroll
                    for (int g = 0; g < W; ++g) pre[g] += lane == stop ? __ldcg(&st[p].inc[g]) : __ldcg(&st[p].agg[g]);
                }
                if (pm) break;
            }
#pragma unroll
            for (int g = 0; g < W; ++g)
#pragma unroll
                for (int d = 16; d > 0; d >>= 1) pre[g] += __shfl_xor_sync(0xFFFFFFFFu, pre[g], d);
            if (lane == 0) {
#pragma unroll
                for (int g = 0; g < W; ++g) { st[tile].inc[g] = pre[g] + agg[g]; s_prefix[g] = pre[g]; }
                __threadfence();
                *(volatile uint32_t*)&st[tile].flag = 2u;
            }
        }
    }
    __syncthreads();
    // exclusive prefix of this thread's first row
    uint64_t run[W];
#pragma unroll
    for (int g = 0; g < W; ++g)
        run[g] = s_prefix[g] + (wid ? s_warp[wid - 1][g] : 0ull) + inc[g] - tot[g];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
        if (row0 + i < n_rows) {
#pragma unroll
            for (int g = 0; g < W; ++g) out[(row0 + i) * W + g] = run[g];
        }
#pragma unroll
        for (int g = 0; g < W; ++g) run[g] += v[i][g];
        if (row0 + i + 1 == n_rows) {
#pragma unroll
            for (int g = 0; g < W; ++g) out[n_rows * W + g] = run[g];
        }
    }
}

template <int W>
size_t ws_bytes(uint64_t n_rows, int items) {
    uint64_t tiles = (n_rows + (uint64_t)kThreads * items - 1) / ((uint64_t)kThreads * items);
    if (tiles == 0) tiles = 1;
    return 256 + tiles * sizeof(TileState<W>);
}

}  // namespace

size_t scan_rows_ws(uint64_t n_rows, int width) {
    return width == 8 ? ws_bytes<8>(n_rows, 4) : ws_bytes<1>(n_rows, 16);
}

template <typename Tin, int W, int ITEMS>
static fi_status launch(const Tin* in, uint64_t* out, uint64_t n_rows, void* ws, size_t ws_n, cudaStream_t s) {
    if (ws_n < ws_bytes<W>(n_rows, ITEMS)) return FI_E_ARG;
    uint64_t tiles = (n_rows + (uint64_t)kThreads * ITEMS - 1) / ((uint64_t)kThreads * ITEMS);
    if (n_rows == 0) {
        return cuda_status(cudaMemsetAsync(out, 0, sizeof(uint64_t) * W, s));
    }
    auto* counter = reinterpret_cast<uint32_t*>(ws);
    auto* st = reinterpret_cast<TileState<W>*>(reinterpret_cast<char*>(ws) + 256);
    fi_status e = cuda_status(cudaMemsetAsync(ws, 0, ws_bytes<W>(n_rows, ITEMS), s));
    if (e) return e;
    k_scan_rows<Tin, W, ITEMS><<<(unsigned)tiles, kThreads, 0, s>>>(in, out, n_rows, st, counter);
    return launch_status();
}

fi_status scan_rows_u32x8(const uint32_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_n, cudaStream_t s) {
    return launch<uint32_t, 8, 4>(in, out, n, ws, ws_n, s);
}
fi_status scan_rows_u64x8(const uint64_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_n, cudaStream_t s) {
    return launch<uint64_t, 8, 4>(in, out, n, ws, ws_n, s);
}
fi_status scan_rows_u64x1(const uint64_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_n, cudaStream_t s) {
    return launch<uint64_t, 1, 16>(in, out, n, ws, ws_n, s);
}

}  // namespace fi

extern "C" size_t fi_scan_u64_workspace(uint64_t n) { return fi::scan_rows_ws(n, 1); }

extern "C" fi_status fi_scan_u64(const uint64_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_bytes, void* stream) {
    if (!out || (n && !in)) return FI_E_ARG;
    return fi::scan_rows_u64x1(in, out, n, ws, ws_bytes, (cudaStream_t)stream);
}
