// golden.cu — program preparation and the golden run that makes the trace
// resident in HBM (§8 row a1).
//
// PAPER.md:72 step (1) profiles a fault-free run and step (4) compares with the
// golden output state.  Here the golden run is the emulator in two passes:
//   pass 1 (fi_golden_lengths): instances in launch order, one launch each;
//          stores go straight into the image, which ends as the golden final
//          image; per-warp step and stored-word counts come out.
//   pass 2 (fi_golden_trace): every warp of every instance in ONE launch over the
//          final image (DESIGN.md §3.5 writer rule), writing the App. A.3 records,
//          the golden store log and register-file checkpoints at the offsets
//          scanned from pass 1.
#include <algorithm>
#include <vector>

#include "emu.cuh"
#include "scan.cuh"

namespace fi {
namespace {

constexpr int kWPB = 4;   // emulated warps per CTA

size_t emu_smem(uint32_t n_regs) { return (size_t)kWPB * (n_regs + 1) * 32 * sizeof(uint32_t); }

__global__ void __launch_bounds__(kWPB * 32)
k_golden_len(EmuProg P, uint8_t* img, uint32_t k, uint64_t* warp_len, uint64_t* warp_nst, uint32_t* status) {
    extern __shared__ uint32_t smem[];
    const uint32_t wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const fi_instance in = P.inst[k];
    const uint32_t lw = blockIdx.x * kWPB + wib;
    if (lw >= in.warp_end - in.warp_begin) return;
    const uint32_t wpc = (in.block + 31) / 32;
    uint32_t* R = smem + wib * (P.n_regs + 1) * 32;
    EmuOut o = emulate<EMU_LEN>(P, img, img, k, lw / wpc, lw % wpc, R, 0xFFFFFFFFu, nullptr, nullptr, 0, HookIn{},
                                nullptr, 0);
    if (lane == 0) {
        warp_len[in.warp_begin + lw] = o.steps;
        warp_nst[in.warp_begin + lw] = o.nstore;
        if (o.fault) FI_DEV_ERR(status, FI_E_PROGRAM);
    }
}

__global__ void __launch_bounds__(kWPB * 32)
k_golden_trace(EmuProg P, const uint8_t* img, uint32_t n_warps, const uint64_t* warp_off, const uint64_t* gst_off,
               fi_record* rec, fi_store* gst, uint32_t* ckpt, const uint64_t* ck_off, uint32_t ck_interval,
               uint32_t* status) {
    extern __shared__ uint32_t smem[];
    const uint32_t wib = threadIdx.x >> 5, lane = threadIdx.x & 31;
    const uint32_t w = blockIdx.x * kWPB + wib;
    if (w >= n_warps) return;
    const uint32_t k = instance_of_warp(P.inst, P.n_inst, w);
    const fi_instance in = P.inst[k];
    const uint32_t wpc = (in.block + 31) / 32, lw = w - in.warp_begin;
    uint32_t* R = smem + wib * (P.n_regs + 1) * 32;
    const uint64_t r0 = warp_off[w], g0 = gst_off[w];
    uint32_t* ck = ckpt ? ckpt + ck_off[w] * (ckpt_bytes(P.n_regs) / 4) : nullptr;
    EmuOut o = emulate<EMU_TRACE>(P, nullptr, img, k, lw / wpc, lw % wpc, R, 0xFFFFFFFFu, rec + r0, gst + g0,
                                  0xFFFFFFFFu, HookIn{}, ck, ckpt ? ck_interval : 0);
    if (lane == 0 && (o.fault || o.steps != warp_off[w + 1] - r0 || o.nstore != gst_off[w + 1] - g0))
        FI_DEV_ERR(status, FI_E_PROGRAM);
}

__global__ void k_gran(const fi_buffer* buf, uint32_t n_buf, uint32_t* gran, uint64_t n_gran) {
    for (uint32_t b = blockIdx.y; b < n_buf; b += gridDim.y) {
        const uint64_t g0 = buf[b].off >> 8, g1 = (buf[b].off + buf[b].size + 255) >> 8;
        for (uint64_t g = g0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; g < g1 && g < n_gran;
             g += (uint64_t)gridDim.x * blockDim.x)
            gran[g] = b;
    }
}

// decode every static instruction (register operands -> smem row offsets) and
// precompute its trace insn word pc | op<<16 | groupmask<<24 (Table II, C-2)
__global__ void k_decode(const fi_insn* code, uint32_t n_code, const fi_kernel* kern, uint32_t n_kern, uint32_t zr,
                         uint4* dec, uint4* fdec, uint8_t* fbl, uint32_t* ins, uint32_t* run) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n_code) return;
    const fi_insn I = code[i];
    uint32_t pc = 0, end = i + 1;
    for (uint32_t k = 0; k < n_kern; ++k)
        if (i >= kern[k].code_off && i < kern[k].code_off + kern[k].code_len) {
            pc = i - kern[k].code_off;
            end = kern[k].code_off + kern[k].code_len;
        }
    dec[i] = decode_insn(I, zr);
    ins[i] = pc | ((uint32_t)I.op << 16) | (groupmask_of(I.op, I.d0, I.d1, I.mod) << 24);
    uint32_t r = 0;                                   // straight-line run starting here
    for (uint32_t j = i; j < end && is_plain(code[j].op); ++j) ++r;
    // LDG batch: consecutive LDGs none of whose address pair is written by an
    // earlier LDG of the batch (their loads can be in flight together)
    uint32_t lr = 0;
    for (uint32_t j = i; j < end && code[j].op == LDG && lr < 0xFFFF; ++j) {
        bool hazard = false;
        for (uint32_t q = i; q < j && !hazard; ++q) {
            const Dests d = dests_of(code[q].op, code[q].d0, code[q].d1, code[q].mod);
            for (uint32_t x = 0; x < 2; ++x) {
                const uint32_t a = code[j].a + x;
                if (code[j].a != kRZ && a >= d.gp_base && a < d.gp_base + d.n_gp) hazard = true;
            }
        }
        if (hazard) break;
        ++lr;
    }
    // simple-FFMA run: unguarded FFMAs without operand modifiers (GEMM / conv inner loops)
    uint32_t fr = 0;
    for (uint32_t j = i; j < end && fr < 0xFF && code[j].op == FFMA && code[j].guard == kPT && code[j].mod == 0 &&
                         code[j].d0 < zr; ++j)
        ++fr;
    run[i] = (r > 0xFFFF ? 0xFFFFu : r) | (std::min<uint32_t>(lr, 0xFF) << 16) | (fr << 24);
    // independent batch inside the simple-FFMA run
    uint32_t fb = 0;
    for (uint32_t j = i; j < i + fr && fb < kFfmaBatch; ++j) {
        bool hazard = false;
        for (uint32_t q = i; q < j && !hazard; ++q) {
            const uint32_t d = code[q].d0;
            hazard = code[j].a == d || code[j].b == d || code[j].c == d || code[j].d0 == d;
        }
        if (hazard) break;
        ++fb;
    }
    if (fr) {
        const uint4 D = dec[i];
        fdec[i] = make_uint4(D.y & 0xFFFF, D.y >> 16, D.z & 0xFFFF, D.z >> 16);
    } else {
        fdec[i] = make_uint4(0, 0, 0, 0);
    }
    fbl[i] = (uint8_t)fb;
    if (i + 1 == n_code)
        for (uint32_t q = 0; q < kFfmaBatch; ++q) fdec[n_code + q] = make_uint4(0, 0, 0, 0);
}

// Buffers an instance's constant bank points into (each adjacent word pair read as
// a 64-bit VA): K7 skips a later instance when none of them holds dirty words.
__global__ void k_inst_bufs(const fi_instance* inst, uint32_t n_inst, const uint32_t* cbank, const uint32_t* gran,
                            uint64_t image_bytes, uint32_t* ib) {
    const uint32_t k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= n_inst) return;
    const fi_instance in = inst[k];
    uint32_t* out = ib + (size_t)k * (kInstBufs + 1);
    uint32_t n = 0;
    for (uint32_t j = 0; j + 1 < in.cbank_len && n <= kInstBufs; ++j) {
        const uint64_t va = (uint64_t)cbank[in.cbank_off + j] | ((uint64_t)cbank[in.cbank_off + j + 1] << 32);
        if (va < kVaBase || va - kVaBase >= image_bytes) continue;
        const uint32_t b = gran[(va - kVaBase) >> 8];
        if (b == kNoBuf) continue;
        bool have = false;
        for (uint32_t q = 0; q < n && q < kInstBufs; ++q) have |= out[1 + q] == b;
        if (have) continue;
        if (n < kInstBufs) out[1 + n] = b;
        ++n;
    }
    out[0] = n;                                       // > kInstBufs: too many, treat as unknown
}

__global__ void k_ckpt_counts(const uint64_t* warp_len, uint32_t n, uint32_t interval, uint64_t* cnt) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n) cnt[i] = (warp_len[i] + interval - 1) / interval;
}

}  // namespace

size_t golden_smem(uint32_t n_regs) { return emu_smem(n_regs); }
size_t aux_dec_offset(const fi_program* p) { return aux_layout(p->image_bytes, p->n_code, p->n_inst).dec; }
size_t aux_ins_offset(const fi_program* p) { return aux_layout(p->image_bytes, p->n_code, p->n_inst).ins; }

}  // namespace fi

using namespace fi;

extern "C" uint32_t fi_program_regs(const fi_insn* code, uint32_t n) {
    uint32_t mx = 0;
    for (uint32_t i = 0; i < n; ++i) {
        const fi_insn& I = code[i];
        for (uint32_t f : {(uint32_t)I.d0, (uint32_t)I.a, (uint32_t)I.b, (uint32_t)I.c})
            if (f < kRZ) mx = std::max(mx, f);
    }
    return std::min<uint32_t>(kRZ, mx + 4);        // +3: widest multi-register operand (LDG/STG.128)
}

extern "C" size_t fi_program_aux_bytes(uint64_t image_bytes, uint32_t n_code, uint32_t n_inst) {
    return aux_layout(image_bytes, n_code, n_inst).total;
}

extern "C" fi_status fi_program_prepare(const fi_program* p, void* aux, void* stream) {
    if (!p || !aux || p->n_regs == 0 || p->n_regs > kRZ) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    const AuxLayout L = aux_layout(p->image_bytes, p->n_code, p->n_inst);
    char* a = reinterpret_cast<char*>(aux);
    uint32_t* gran = reinterpret_cast<uint32_t*>(a + L.gran);
    const uint64_t n_gran = (p->image_bytes + 255) >> 8;
    fi_status e = cuda_status(cudaMemsetAsync(gran, 0xFF, std::max<uint64_t>(n_gran, 1) * sizeof(uint32_t), s));
    if (e) return e;
    if (p->n_buf) {
        dim3 grid(64, std::min<uint32_t>(p->n_buf, 4096));
        k_gran<<<grid, 256, 0, s>>>(p->buf, p->n_buf, gran, n_gran);
        if ((e = launch_status())) return e;
    }
    if (p->n_code) {
        k_decode<<<(p->n_code + 127) / 128, 128, 0, s>>>(p->code, p->n_code, p->kern, p->n_kern, p->n_regs,
                                                         reinterpret_cast<uint4*>(a + L.dec),
                                                         reinterpret_cast<uint4*>(a + L.fdec),
                                                         reinterpret_cast<uint8_t*>(a + L.fbl),
                                                         reinterpret_cast<uint32_t*>(a + L.ins),
                                                         reinterpret_cast<uint32_t*>(a + L.run));
        if ((e = launch_status())) return e;
    }
    if (p->n_inst) {
        k_inst_bufs<<<(p->n_inst + 127) / 128, 128, 0, s>>>(p->inst, p->n_inst, p->cbank, gran, p->image_bytes,
                                                            reinterpret_cast<uint32_t*>(a + L.ib));
        if ((e = launch_status())) return e;
    }
    return FI_OK;
}

static fi_status set_smem(const void* f, size_t bytes) {
    return cuda_status(cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bytes));
}

extern "C" fi_status fi_golden_lengths(const fi_program* p, uint8_t* image, uint64_t* warp_len, uint64_t* warp_nstore,
                                       uint32_t* dev_status, void* stream) {
    if (!p || !image || !warp_len || !warp_nstore || !dev_status || !p->inst_host || !p->aux) return FI_E_ARG;
    if (p->n_regs == 0 || p->n_regs > kRZ) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    const size_t smem = emu_smem(p->n_regs);
    fi_status e = set_smem((const void*)k_golden_len, smem);
    if (e) return e;
    const EmuProg P = make_emu_prog(p);
    for (uint32_t k = 0; k < p->n_inst; ++k) {
        const uint32_t nw = p->inst_host[k].warp_end - p->inst_host[k].warp_begin;
        if (!nw) continue;
        k_golden_len<<<(nw + kWPB - 1) / kWPB, kWPB * 32, smem, s>>>(P, image, k, warp_len, warp_nstore, dev_status);
        if ((e = launch_status())) return e;
    }
    return FI_OK;
}

extern "C" size_t fi_ckpt_bytes(uint32_t n_regs) { return ckpt_bytes(n_regs); }

extern "C" size_t fi_ckpt_layout_workspace(uint32_t n_warps) {
    return align256((size_t)n_warps * 8) + scan_rows_ws(n_warps, 1);
}

extern "C" fi_status fi_ckpt_layout(const uint64_t* warp_len, uint32_t n_warps, uint32_t interval, uint64_t* ckpt_off,
                                    void* ws, size_t ws_bytes, void* stream) {
    if (!warp_len || !ckpt_off || !ws || interval == 0 || ws_bytes < fi_ckpt_layout_workspace(n_warps)) return FI_E_ARG;
    cudaStream_t s = (cudaStream_t)stream;
    uint64_t* cnt = reinterpret_cast<uint64_t*>(ws);
    const size_t head = align256((size_t)n_warps * 8);
    if (n_warps) {
        k_ckpt_counts<<<(n_warps + 255) / 256, 256, 0, s>>>(warp_len, n_warps, interval, cnt);
        fi_status e = launch_status();
        if (e) return e;
    }
    return scan_rows_u64x1(cnt, ckpt_off, n_warps, reinterpret_cast<char*>(ws) + head, ws_bytes - head, s);
}

extern "C" fi_status fi_golden_trace(const fi_program* p, const uint8_t* image, const fi_trace* t,
                                     uint32_t* dev_status, void* stream) {
    if (!p || !image || !t || !t->warp_off || !t->gstore_off || !t->rec || !dev_status || !p->aux) return FI_E_ARG;
    if (t->ckpt && (!t->ckpt_off || !t->ckpt_interval)) return FI_E_ARG;
    if (!p->n_warps) return FI_OK;
    cudaStream_t s = (cudaStream_t)stream;
    const size_t smem = emu_smem(p->n_regs);
    fi_status e = set_smem((const void*)k_golden_trace, smem);
    if (e) return e;
    k_golden_trace<<<(p->n_warps + kWPB - 1) / kWPB, kWPB * 32, smem, s>>>(
        make_emu_prog(p), image, p->n_warps, t->warp_off, t->gstore_off, t->rec, t->gstore, t->ckpt, t->ckpt_off,
        t->ckpt_interval, dev_status);
    return launch_status();
}
