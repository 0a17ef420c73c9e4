// jit_k8.h — host mirror of JK8 (jit_prelude.cuh): the K8 state k8_exec_jit
// reads, filled by propagate8.cu from its K8Args.  Field order and types must
// match JK8 exactly (the K8 parity tests compare both engines).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/fi.h"

namespace fi {
struct JK8Host {
    const uint64_t* warp_off; const uint64_t* gst_off; const fi_store* gst;
    void* slot;
    const uint32_t* ptab; uint32_t total_pages;
    const uint32_t* pool; const uint32_t* page_base; const uint32_t* last_ref; const uint32_t* dropped; uint32_t dwords;
    fi_store* pend; uint32_t pend_cap;
    fi_store* forn; uint32_t foreign_cap;
    const uint32_t* active; const uint32_t* n_active; uint32_t* work;
    fi_store* scratch; uint32_t log_cap;
    uint32_t flags; uint32_t* status;
    unsigned long long* steps;                      // emulated warp-steps of the re-executed warps (summed)
    const uint32_t* bcount; uint32_t n_buf;         // [slot][buffer] page counts
};
fi_status jit_k8_exec(const fi_jit* j, const fi_program* p, const uint8_t* image, const JK8Host& K, uint32_t t,
                      uint32_t max_grid, cudaStream_t s);
}  // namespace fi
