/* oracle.h — CPU ORACLE for the NVBitFI hot path.  TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * `--impl reference` legs may load this library.  It shares no code, header,
 * table or constant with the CUDA library (paper_conf_dsn_0002hsvk21_b200/csrc,
 * include/fi.h); both are written independently from PAPER.md and the readings
 * in DESIGN.md.  The only thing both sides consume is the seeded program format
 * produced by fi_inputs/ (DESIGN.md §3).
 *
 * What it computes, by plain definition (PAPER.md = /root/reference/PAPER.md):
 *   golden run + counting   PAPER.md:78 §III-A "dynamic instruction counts for every
 *                           opcode in every thread ... Instructions that are not
 *                           executed based on a predicate register are not included"
 *                           grouped by Table II arch state ids.
 *   selection               PAPER.md:78 "choosing a random number n from the set 1..N"
 *                           -> enumeration of group-g sites in canonical order (C-3)
 *   injection               PAPER.md:78,138 corrupt the destination register of one
 *                           dynamic instruction; masks PAPER.md:116-121 (Table II)
 *   classification          PAPER.md:184-196 (Table V), :206 — DUE > SDC > Masked
 * Every function below is pinned by tests/test_oracle_*.py.
 */
#ifndef FI_ORACLE_H
#define FI_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* ---- program (input format) — oracle's own declarations ---- */
typedef struct { uint8_t op, guard, d0, d1, a, b, c, mod; uint32_t imm, ext; } orc_insn;
typedef struct { uint32_t code_off, code_len, nregs, pad; } orc_kernel;
typedef struct { uint32_t kernel, kernel_count, grid, block, cbank_off, cbank_len, warp_begin, warp_end; } orc_instance;
typedef struct { uint64_t off, size; int32_t writer; uint32_t flags; } orc_buffer;
typedef struct {
    const orc_insn* code; uint32_t n_code;
    const orc_kernel* kern; uint32_t n_kern;
    const orc_instance* inst; uint32_t n_inst;
    const uint32_t* cbank; uint32_t n_cbank;
    const orc_buffer* buf; uint32_t n_buf;
    const uint8_t* init_image; uint64_t image_bytes;
} orc_program;

/* trace record (App. A.3): {instance, pc | op<<16 | groupmask<<24, active, pred} */
typedef struct { uint32_t instance, insn, active, pred; } orc_record;

typedef struct {
    uint64_t s, instruction_count;
    uint32_t instance, kernel_id, kernel_count, warp, step, thread;
    uint32_t pc, u_dst, u_bit, mask;
    uint8_t lane, group, bfm, slot, dst_kind, dst_reg, n_elig, flags /* bit0: not injected (C-17) */;
} orc_site;                                           /* 64 B */

typedef struct {
    uint32_t before, after, mask, fault_pc;
    uint8_t fault_kind, outcome, flags /* bit0: potential DUE (f4) */, pad;
    uint32_t n_faulty_stores;
} orc_inj;                                            /* 24 B */

/* groups (Table II order, C-1) and outcomes (Table V) */
enum { ORC_G_FP64 = 0, ORC_G_FP32, ORC_G_LD, ORC_G_PR, ORC_G_NODEST, ORC_G_OTHERS, ORC_G_GPPR, ORC_G_GP };
enum { ORC_MASKED = 0, ORC_SDC = 1, ORC_DUE = 2, ORC_NOT_INJECTED = 3 };
enum { ORC_MODE_FULL = 0, ORC_MODE_WARP_LOCAL = 1, ORC_UNCHECKED = 0x100 /* f4 potential-DUE semantics */ };
enum { ORC_POTENTIAL_DUE = 1, ORC_SDC_WITHIN_TOL = 8 /* C-12 secondary: bitwise SDC, every element within rtol */ };

/* status: 0 ok; 1 arg; 2 empty group; 3 not injectable; 4 program error */
const char* orc_error(void* h);

/* golden run.  keep_trace=1 keeps the App. A.3 trace in RAM.  Returns a handle
 * (NULL on error; orc_last_error() explains). */
void* orc_golden_run(const orc_program* p, int n_threads, int keep_trace);
const char* orc_last_error(void);
void orc_free(void* h);
uint32_t orc_n_warps(void* h);
uint64_t orc_n_records(void* h);
void orc_counts(void* h, uint64_t* out /*[n_inst][8]*/);
void orc_warp_counts(void* h, uint64_t* out /*[n_warps][8]*/);
void orc_warp_len(void* h, uint64_t* out /*[n_warps]*/);
void orc_final_image(void* h, uint8_t* out /*[image_bytes]*/);
int orc_trace(void* h, orc_record* out /*[n_records]*/);
uint64_t orc_n_golden_stores(void* h);

/* count only (no memory/trace kept): interpret the warps [w0, w1) of a
 * single-instance program from the initial image; used for bounded CPU
 * baselines.  Returns records interpreted. */
uint64_t orc_count_warps(const orc_program* p, uint32_t w0, uint32_t w1, int n_threads, uint64_t* counts8);

/* the profiler's count over a trace already in host RAM (K1's CPU baseline):
 * counts[k][g] = sum over records of instance k with g in groupmask of
 * popc(active & pred).  Returns 1 if a record names an instance >= n_inst. */
int orc_scan_trace(const orc_record* rec, uint64_t n, uint32_t n_inst, int n_threads, uint64_t* counts);

/* selection by enumeration (C-3..C-6).  With keep_trace=0 (single-
 * instance programs only) the site's warp comes from the per-warp counts and the
 * rank inside it from a re-interpretation of that warp — the same canonical order. */
int orc_select(void* h, uint64_t seed, const uint8_t* groups, uint32_t n_groups,
               const uint8_t* bfms, uint32_t n_bfms, uint64_t j0, uint32_t n, orc_site* out);

int orc_locate(void* h, int group, const uint64_t* s, uint32_t n, orc_site* out);

/* row f1: per-opcode profile and approximate profiling */
int orc_opcode_counts(void* h, uint64_t* out /*[n_inst][32]*/);
int orc_approx_counts(void* h, uint64_t* out /*[n_inst][8]*/);
int orc_select_approx(void* h, uint64_t seed, const uint8_t* groups, uint32_t n_groups,
                      const uint8_t* bfms, uint32_t n_bfms, uint64_t j0, uint32_t n, orc_site* out);

/* injection + classification; mode ORC_MODE_FULL re-runs the whole program.
 * rtol > 0: also the C-12 secondary numeric classification — ORC_SDC_WITHIN_TOL
 * in flags of every SDC whose output elements all satisfy |f-g| <= rtol*|g|
 * (both finite; u32 buffers bitwise). */
int orc_inject(void* h, const orc_site* sites, uint32_t n, int mode, int n_threads, double rtol, orc_inj* out);

/* rows f2/f3: permanent / intermittent faults (Table III) */
typedef struct { uint32_t opcode, sm, lane, mask, q32, n_sm; uint64_t seed; } orc_pfault;   /* 32 B */
int orc_inject_permanent(void* h, const orc_pfault* pf, uint32_t n, int mode, int n_threads, orc_inj* out);
int orc_permanent_image(void* h, const orc_pfault* pf, uint32_t rep, int mode, uint8_t* out_image);

/* faulty final image of one transient site, full mode (multi-launch propagation pins);
 * returns the fault kind, -1 if the site was not reached */
int orc_inject_image(void* h, const orc_site* site, int mode, uint8_t* out_image);

/* single-instance, no golden handle (full-size sampled parity, CPU baselines) */
int orc_warp_site_rank(const orc_program* p, uint32_t w, int g, uint32_t step, uint32_t lane,
                       uint64_t* rank, uint64_t* total);
int orc_warp_site_at(const orc_program* p, uint32_t w, int g, uint64_t rank,
                     uint32_t* step, uint32_t* lane, uint32_t* pc);
int orc_inject_local(const orc_program* p, const orc_site* sites, uint32_t n, int n_threads,
                     orc_inj* out, uint8_t* decided);

/* RNG / mask primitives */
void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);
void orc_draw(uint64_t seed, uint64_t j, uint64_t n_g, uint64_t* s, uint32_t* u_dst, uint32_t* u_bit, uint32_t* attempts);
uint32_t orc_mask(int bfm, uint32_t u_bit);
uint32_t orc_group_mask(const orc_insn* insn);
uint32_t orc_dest_slots(const orc_insn* insn, int group, uint8_t* kind, uint8_t* reg);

#ifdef __cplusplus
}
#endif
#endif
