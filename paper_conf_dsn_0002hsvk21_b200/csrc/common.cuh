// common.cuh — libfi internals shared by the CUDA translation units.
// Independent of oracle/ (no shared code); semantics from DESIGN.md §3-§4.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

#include "../../include/fi.h"

namespace fi {

enum Op : uint32_t {
    NOP = 0, EXIT, BRA, MOV, S2R, IADD3, IMAD, IMAD_WIDE, SHF, LOP3, SEL,
    ISETP, FSETP, DSETP, FADD, FMUL, FFMA, FMNMX, DADD, DMUL, DFMA,
    LDG, LDC, STG, I2F, F2I, F2F_F64_F32, F2F_F32_F64, SHFL, IMNMX, MUFU_RCP64
};
constexpr uint32_t kRZ = 127, kPT = 7;
constexpr uint64_t kVaBase = 0x00007F0000000000ull;          // C-15
constexpr uint32_t kNoBuf = 0xFFFFFFFFu;
constexpr uint32_t kQNaN32 = 0x7FFFFFFFu;                      // C-13
constexpr uint64_t kQNaN64 = 0x7FFFFFFFFFFFFFFFull;

// Architectural destinations of an instruction (DESIGN.md §3.2 "dest"):
// n_gp consecutive GP registers from d0 (0 if d0 == RZ) and at most one predicate.
struct Dests { uint32_t gp_base, n_gp, pr; bool has_pr; };

__host__ __device__ inline Dests dests_of(uint32_t op, uint32_t d0, uint32_t d1, uint32_t mod) {
    Dests d{d0, 0, 0, false};
    uint32_t n = 0;
    switch (op) {
        case MOV: case S2R: case IMAD: case SHF: case LOP3: case SEL: case I2F: case F2I:
        case F2F_F32_F64: case SHFL: case IMNMX: case FADD: case FMUL: case FFMA: case FMNMX: case IADD3:
            n = 1; break;
        case IMAD_WIDE: case DADD: case DMUL: case DFMA: case F2F_F64_F32: case MUFU_RCP64: n = 2; break;
        case LDG: n = 1u << ((mod & 3) > 2 ? 2 : (mod & 3)); break;
        case LDC: n = (mod & 1) ? 2 : 1; break;
        default: n = 0;
    }
    d.n_gp = (d0 == kRZ) ? 0 : n;
    if (op == IADD3 && (d1 & 7) != kPT) { d.has_pr = true; d.pr = d1 & 7; }
    if ((op == ISETP || op == FSETP || op == DSETP) && (d0 & 7) != kPT) { d.has_pr = true; d.pr = d0 & 7; }
    return d;
}

// Table II membership (reading C-2): bit g set iff the instruction is in group g.
__host__ __device__ inline uint32_t groupmask_of(uint32_t op, uint32_t d0, uint32_t d1, uint32_t mod) {
    Dests d = dests_of(op, d0, d1, mod);
    if (d.n_gp == 0 && !d.has_pr) return 1u << FI_G_NODEST;
    if (d.n_gp == 0) return (1u << FI_G_PR) | (1u << FI_G_GPPR);
    uint32_t base = (op == DADD || op == DMUL || op == DFMA) ? FI_G_FP64
                  : (op == FADD || op == FMUL || op == FFMA || op == FMNMX) ? FI_G_FP32
                  : (op == LDG || op == LDC) ? FI_G_LD : FI_G_OTHERS;
    return (1u << base) | (1u << FI_G_GPPR) | (1u << FI_G_GP);
}

// Eligible destination slots for group g (C-6): GP registers ascending for the
// GP-type groups, the predicate for G_PR, GP then predicate for G_GPPR.
__host__ __device__ inline uint32_t n_slots(const Dests& d, uint32_t g) {
    if (g == FI_G_NODEST) return 0;
    if (g == FI_G_PR) return d.has_pr ? 1 : 0;
    if (g == FI_G_GPPR) return d.n_gp + (d.has_pr ? 1 : 0);
    return d.n_gp;
}
__host__ __device__ inline void slot_reg(const Dests& d, uint32_t g, uint32_t slot, uint32_t& kind, uint32_t& reg) {
    if (g == FI_G_PR || slot >= d.n_gp) { kind = 1; reg = d.pr; }
    else { kind = 0; reg = d.gp_base + slot; }
}

// Table II masks with value = u / 2^32 (C-5, C-8); ZERO_VALUE resolved at injection.
__host__ __device__ inline uint32_t bfm_mask(uint32_t bfm, uint32_t u) {
    switch (bfm) {
        case FI_FLIP_SINGLE_BIT: return 1u << (uint32_t)((32ull * u) >> 32);
        case FI_FLIP_TWO_BITS: return 3u << (uint32_t)((31ull * u) >> 32);
        case FI_RANDOM_VALUE: return (uint32_t)((0xFFFFFFFFull * u) >> 32);
        default: return 0;
    }
}

#ifdef __CUDACC__
// Philox4x32-10 (Salmon et al. 2011), the counter-based RNG of every draw (C-5)
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
    for (int r = 0; r < 10; ++r) {
        if (r) { k.x += 0x9E3779B9u; k.y += 0xBB67AE85u; }
        const uint32_t hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
        const uint32_t hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
        c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
    }
    return c;
}

// C-12 secondary numeric classification: does the faulty element
// fv differ from the golden element gv beyond the relative tolerance rtol
// (atol = 0)?  Equal bits: no.  U32 buffers: any difference.  F32 / F64: yes
// unless both are finite and |f - g| <= rtol * |g| in IEEE double, round to
// nearest (so NaN or an infinity against anything else always differs).
__device__ __forceinline__ bool beyond_tol(uint32_t dtype, uint64_t fv, uint64_t gv, double rtol) {
    if (fv == gv) return false;
    double f, g;
    if (dtype == 1) {
        f = (double)__uint_as_float((uint32_t)fv);
        g = (double)__uint_as_float((uint32_t)gv);
    } else if (dtype == 2) {
        f = __longlong_as_double((long long)fv);
        g = __longlong_as_double((long long)gv);
    } else {
        return true;
    }
    if (!isfinite(f) || !isfinite(g)) return true;
    return !(fabs(__dsub_rn(f, g)) <= __dmul_rn(rtol, fabs(g)));
}
__device__ __forceinline__ uint32_t buf_dtype(uint32_t flags) { return (flags >> 8) & 0xFFu; }
#endif

// hist_tol[group][bfm][outcome] over replicas [0, n): the secondary histogram, a
// bitwise SDC flagged FI_SDC_WITHIN_TOL counted as Masked (C-12).
fi_status launch_hist_tol(const fi_site* sites, const fi_inj* inj, uint32_t n, uint64_t* hist_tol, cudaStream_t s);

}  // namespace fi

// error plumbing for the host side of the ABI
namespace fi {
void set_cuda_error(cudaError_t e);
inline fi_status cuda_status(cudaError_t e) {
    if (e == cudaSuccess) return FI_OK;
    set_cuda_error(e);
    return FI_E_CUDA;
}
inline fi_status launch_status() { return cuda_status(cudaGetLastError()); }
// raise the release threshold of the current device's default memory pool once, so
// the stream-ordered allocations of fi_campaign / fi_golden_run stay mapped between
// calls (fi_campaign_release_memory hands them back)
void keep_pool();
}  // namespace fi

#define FI_DEV_ERR(ptr, code) atomicOr((ptr), 1u << (code))
