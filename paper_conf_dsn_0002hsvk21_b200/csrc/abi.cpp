// abi.cpp — host-only entry points of libfi: status strings, version, and the
// Table II parameter-file writer ("Each parameter is specified in
// the parameter file as a separate line").
#include <cstdio>
#include <cstring>
#include <string>

#include <cuda_runtime.h>

#include "../../include/fi.h"

namespace fi {
static thread_local std::string g_cuda_err;
void set_cuda_error(cudaError_t e) { g_cuda_err = std::string(cudaGetErrorName(e)) + ": " + cudaGetErrorString(e); }
}  // namespace fi

extern "C" const char* fi_last_cuda_error(void) { return fi::g_cuda_err.c_str(); }

extern "C" const char* fi_version(void) { return "libfi 0.1 (sm_100a)"; }

extern "C" const char* fi_status_str(fi_status s) {
    switch (s) {
        case FI_OK: return "ok";
        case FI_E_ARG: return "bad argument";
        case FI_E_EMPTY_GROUP: return "scheduled instruction group has no dynamic instances (N_g == 0)";
        case FI_E_NOT_INJECTABLE: return "G_NODEST has no destination register and cannot be injected (C-16)";
        case FI_E_PROGRAM: return "golden run faulted or the program violates the SSA/race-free model";
        case FI_E_CUDA: return "CUDA error";
        case FI_E_SITE: return "site does not match the re-executed warp / trace";
        case FI_E_CAPACITY: return "faulty store log overflow";
        case FI_E_INVARIANT: return "Table II identity violated by a count row (GP = FP64+FP32+LD+OTHERS, GPPR = GP+PR)";
        case FI_E_COLLECTIVE: return "all-reduce callback failed";
    }
    return "unknown status";
}

// Seven lines in Table II order [PAPER.md:92-122]: arch state id, bit-flip
// model, kernel name, kernel count, instruction count, destination register
// value, bit-pattern value; the two [0,1) values are u/2^32 (C-5).
extern "C" fi_status fi_write_params_txt(const fi_site* s, const char* kernel_name, char* buf, size_t n) {
    if (!s || !kernel_name || !buf || !n) return FI_E_ARG;
    int w = std::snprintf(buf, n, "%u\n%u\n%s\n%u\n%llu\n%.10f\n%.10f\n", (unsigned)s->group, (unsigned)s->bfm,
                          kernel_name, s->kernel_count, (unsigned long long)s->instruction_count,
                          (double)s->u_dst / 4294967296.0, (double)s->u_bit / 4294967296.0);
    return (w < 0 || (size_t)w >= n) ? FI_E_ARG : FI_OK;
}
