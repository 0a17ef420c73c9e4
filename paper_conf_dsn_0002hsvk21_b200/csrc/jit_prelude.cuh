// jit_prelude.cuh — device helpers of the JIT-specialised emulator (jit.cpp).
//
// This header is embedded as text into libfi.so and prepended to the CUDA
// source jit.cpp generates per program, which NVRTC compiles for sm_100a.  It is
// self-contained (NVRTC sees no system headers).  The semantics are DESIGN.md
// §3 — the same as emu.cuh's interpreter, which the generated code must match
// bit for bit (both are checked against the CPU oracle by the parity tests).
typedef unsigned char u8;
typedef unsigned int u32;
typedef int i32;
typedef unsigned long long u64;
typedef long long i64;

#define JFULL 0xFFFFFFFFu
#define JQNAN32 0x7FFFFFFFu
#define JQNAN64 0x7FFFFFFFFFFFFFFFull
#define JVA_BASE 0x00007F0000000000ull
#define JNOBUF 0xFFFFFFFFu

// layouts identical to include/fi.h
struct jfi_instance { u32 kernel, kernel_count, grid, block, cbank_off, cbank_len, warp_begin, warp_end; };
struct jfi_buffer { u64 off, size; i32 writer; u32 flags; };
struct jfi_store { u64 va; u32 value, step; };
struct jfi_site {
    u64 s, instruction_count;
    u32 instance, kernel_id, kernel_count, warp, step, thread;
    u32 pc, u_dst, u_bit, mask;
    u8 lane, group, bfm, slot, dst_kind, dst_reg, n_elig, flags;
};
struct jfi_inj {
    u32 before, after, mask, fault_pc;
    u8 fault_kind, outcome, overflow, flags;
    u32 n_faulty_stores;
};

struct JArgs {
    const u8* img;               // golden final image
    const u32* gran;             // buffer id per 256-B granule
    const jfi_buffer* buf;
    const jfi_instance* inst;
    const u32* cbank;
    u64 image_bytes;
};

struct JOut {
    u32 steps, fault, fault_pc, nstore, before, after, mask;
    bool fired, bad;
};

__device__ __forceinline__ float ju2f(u32 x) { return __uint_as_float(x); }
__device__ __forceinline__ u32 jfbits(float f) { return f != f ? JQNAN32 : __float_as_uint(f); }
__device__ __forceinline__ double ju2d(u64 x) { return __longlong_as_double((long long)x); }
__device__ __forceinline__ u64 jdbits(double d) { return d != d ? JQNAN64 : (u64)__double_as_longlong(d); }
__device__ __forceinline__ u64 jpair(u32 lo, u32 hi) { return (u64)lo | ((u64)hi << 32); }

__device__ __forceinline__ u32 jfmnmx(u32 a, u32 b, bool mx) {
    const float x = ju2f(a), y = ju2f(b);
    const bool xn = x != x, yn = y != y;
    if (xn && yn) return JQNAN32;
    if (xn) return b;
    if (yn) return a;
    if (x == y) {                                   // -0 < +0 (C-13)
        const bool xneg = a >> 31;
        return mx ? (xneg ? b : a) : (xneg ? a : b);
    }
    return mx ? (x > y ? a : b) : (x < y ? a : b);
}

__device__ __forceinline__ bool jcmp_f(double x, double y, u32 c) {
    if (x != x || y != y) return false;             // ordered compares
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}
__device__ __forceinline__ bool jcmp_s(i32 x, i32 y, u32 c) {
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}
__device__ __forceinline__ bool jcmp_u(u32 x, u32 y, u32 c) {
    switch (c) {
        case 0: return x < y; case 1: return x <= y; case 2: return x > y;
        case 3: return x >= y; case 4: return x == y; case 5: return x != y;
    }
    return false;
}

__device__ __forceinline__ u32 jf2i(u32 a) {
    const float f = ju2f(a);
    if (f != f) return 0;
    if (f >= 2147483648.0f) return 0x7FFFFFFFu;
    if (f < -2147483648.0f) return 0x80000000u;
    return (u32)__float2int_rz(f);
}

template <u32 LUT>
__device__ __forceinline__ u32 jlop3(u32 a, u32 b, u32 c) {
    u32 r = 0;
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const u32 t = ((i & 4) ? a : ~a) & ((i & 2) ? b : ~b) & ((i & 1) ? c : ~c);
        r |= ((LUT >> i) & 1u) ? t : 0u;
    }
    return r;
}

__device__ __forceinline__ u32 jshf(u32 a, u32 bv, u32 m) {
    const u32 s = bv > 32 ? 32 : bv;
    if (m == 0) return s >= 32 ? 0u : a << s;
    if (m == 1) return s >= 32 ? 0u : a >> s;
    return (u32)((i32)a >> (s >= 32 ? 31 : s));
}

__device__ __forceinline__ u32 jshfl_src(u32 lane, u32 bv, u32 m) {
    i64 src;
    switch (m) {
        case 0: src = bv & 31; break;
        case 1: src = lane ^ (bv & 31); break;
        case 2: src = (i64)lane + (i64)bv; if (src > 31) src = lane; break;
        default: src = (i64)lane - (i64)bv; if (src < 0) src = lane; break;
    }
    return (u32)src;
}

__device__ __forceinline__ u32 jld32(const u8* p) {
    u32 r;
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
    return r;
}
__device__ __forceinline__ uint2 jld64(const u8* p) {
    uint2 r;
    asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0, %1}, [%2];" : "=r"(r.x), "=r"(r.y) : "l"(p));
    return r;
}
__device__ __forceinline__ uint4 jld128(const u8* p) {
    uint4 r;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0, %1, %2, %3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
    return r;
}

// per-lane two-entry cache of buffer bounds (image offsets)
struct JBufCache {
    u64 lo0, hi0, lo1, hi1;
    bool z0, z1;
    __device__ __forceinline__ JBufCache() : lo0(1), hi0(0), lo1(1), hi1(0), z0(false), z1(false) {}
};

// 0 ok, 1 misaligned, 2 unmapped (C-15); *zero = writer rule for instance k
__device__ __forceinline__ u32 jcheck(const JArgs& A, JBufCache& C, u64 va, u32 w, u32 k, bool* zero) {
    if (va & (w - 1)) return 1;
    const u64 off = va - JVA_BASE;
    // (off < hi first: an address just below the VA base wraps off + w around)
    if (off >= C.lo0 && off < C.hi0 && off + w <= C.hi0) { *zero = C.z0; return 0; }
    if (off >= C.lo1 && off < C.hi1 && off + w <= C.hi1) { *zero = C.z1; return 0; }
    if (va < JVA_BASE || off >= A.image_bytes) return 2;
    const u32 b = __ldg(&A.gran[off >> 8]);
    if (b == JNOBUF) return 2;
    const u64 lo = __ldg(&A.buf[b].off), hi = lo + __ldg(&A.buf[b].size);
    if (off + w > hi) return 2;
    const i32 wr = __ldg(&A.buf[b].writer);
    C.lo1 = C.lo0; C.hi1 = C.hi0; C.z1 = C.z0;
    C.lo0 = lo; C.hi0 = hi; C.z0 = wr >= 0 && (u32)wr >= k;
    *zero = C.z0;
    return 0;
}

// cache-only check: true iff the access is aligned and inside one of the two
// cached buffers (then *zero is that buffer's writer-rule flag); no state change
__device__ __forceinline__ bool jhit(const JBufCache& C, u64 va, u32 w, bool* zero) {
    const u64 off = va - JVA_BASE;
    const bool h0 = off >= C.lo0 && off < C.hi0 && off + w <= C.hi0;
    const bool h1 = off >= C.lo1 && off < C.hi1 && off + w <= C.hi1;
    *zero = h0 ? C.z0 : C.z1;
    return ((va & (w - 1)) == 0) && (h0 || h1);
}

// one LDG of 1/2/4 words for this lane; returns the fault code (0 ok)
template <u32 LW>
__device__ __forceinline__ u32 jldg(const JArgs& A, JBufCache& C, u64 va, u32 k, bool ex, uint4& v) {
    bool zero = false;
    const u32 c = ex ? jcheck(A, C, va, 4u << LW, k, &zero) : 0u;
    v = make_uint4(0, 0, 0, 0);
    if (ex && !c && !zero) {
        const u8* src = A.img + (va - JVA_BASE);
        if (LW == 0) v.x = jld32(src);
        else if (LW == 1) { const uint2 t = jld64(src); v.x = t.x; v.y = t.y; }
        else v = jld128(src);
    }
    return c;
}
