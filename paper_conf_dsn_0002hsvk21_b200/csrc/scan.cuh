#pragma once
#include "common.cuh"

namespace fi {
size_t scan_rows_ws(uint64_t n_rows, int width);
fi_status scan_rows_u32x8(const uint32_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_n, cudaStream_t s);
fi_status scan_rows_u64x8(const uint64_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_n, cudaStream_t s);
fi_status scan_rows_u64x1(const uint64_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_n, cudaStream_t s);
}  // namespace fi
