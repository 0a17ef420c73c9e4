/* fi.h — C ABI of libfi.so, the B200 (sm_100a) NVBitFI hot path.
 *
 * PAPER.md = /root/reference/PAPER.md (Tsai et al., "NVBitFI: Dynamic Fault
 * Injection for GPUs", DSN 2021).  DESIGN.md §3 defines the program model,
 * §4 the readings C-1..C-20 of the paper that these calls implement.
 *
 * Conventions (all entry points):
 *   - Pointers are DEVICE pointers owned by the caller unless marked host.
 *     libfi allocates nothing persistent; scratch is the caller's.
 *   - Calls are asynchronous and ordered on `stream` (a cudaStream_t passed as
 *     void*; NULL = legacy default stream).  Only calls documented as
 *     "synchronizes" block the host.
 *   - Every call returns fi_status; nothing throws or exits across the ABI.
 *     Launch/CUDA errors return FI_E_CUDA (fi_last_cuda_error() has the text).
 *     Errors found by device code (a golden-run fault, a site that does not
 *     match the trace) are OR-ed into the caller's device word `dev_status`
 *     as (1u << fi_status) bits; read it after the stream completes.
 *   - Reentrant given distinct output / scratch buffers.
 */
#ifndef FI_H
#define FI_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    FI_OK = 0,
    FI_E_ARG = 1,              /* bad argument / size */
    FI_E_EMPTY_GROUP = 2,      /* N_g == 0 for a scheduled group */
    FI_E_NOT_INJECTABLE = 3,   /* G_NODEST scheduled (C-16) */
    FI_E_PROGRAM = 4,          /* golden run faulted / program violates DESIGN.md §3.5 */
    FI_E_CUDA = 5,
    FI_E_SITE = 6,             /* a site does not match the re-executed warp */
    FI_E_CAPACITY = 8,         /* faulty store log overflow (replica must be re-run with a larger log) */
    FI_E_INVARIANT = 9,        /* a Table II identity does not hold for a count row (§8 row a3) */
    FI_E_COLLECTIVE = 10       /* fi_campaign: the caller's all-reduce callback failed */
} fi_status;

/* Table II arch state ids [PAPER.md:94-104], 0-based (C-1) */
typedef enum { FI_G_FP64 = 0, FI_G_FP32 = 1, FI_G_LD = 2, FI_G_PR = 3, FI_G_NODEST = 4,
               FI_G_OTHERS = 5, FI_G_GPPR = 6, FI_G_GP = 7, FI_NGROUPS = 8 } fi_group;
/* Table II bit-flip models [PAPER.md:105-109], 0-based (C-1) */
typedef enum { FI_FLIP_SINGLE_BIT = 0, FI_FLIP_TWO_BITS = 1, FI_RANDOM_VALUE = 2, FI_ZERO_VALUE = 3 } fi_bfm;
/* Table V outcomes [PAPER.md:184-196] */
typedef enum { FI_MASKED = 0, FI_SDC = 1, FI_DUE = 2,
               FI_NOT_INJECTED = 3 /* approximate profile named a site the instance does not have (C-17) */ } fi_outcome;
#define FI_NOPS 32                                   /* opcode slots of the per-opcode profile */

/* ---- program ------------------------------------------- */
typedef struct { uint8_t op, guard, d0, d1, a, b, c, mod; uint32_t imm, ext; } fi_insn;          /* 16 B */
typedef struct { uint32_t code_off, code_len, nregs, pad; } fi_kernel;                             /* 16 B */
typedef struct { uint32_t kernel, kernel_count, grid, block, cbank_off, cbank_len,
                 warp_begin, warp_end; } fi_instance;                                                /* 32 B */
typedef struct { uint64_t off, size; int32_t writer; uint32_t flags; } fi_buffer;                  /* 24 B; flags bit0 = output */

typedef struct {
    const fi_insn* code;      uint32_t n_code;       /* device */
    const fi_kernel* kern;    uint32_t n_kern;       /* device */
    const fi_instance* inst;  uint32_t n_inst;       /* device */
    const uint32_t* cbank;    uint32_t n_cbank;      /* device */
    const fi_buffer* buf;     uint32_t n_buf;        /* device, sorted by off */
    const void* aux;                                 /* device, fi_program_aux_bytes(): written by fi_program_prepare */
    uint64_t image_bytes;
    uint32_t n_warps;
    uint32_t n_regs;                                 /* register rows the emulator keeps: from fi_program_regs() */
    const fi_insn* code_host;                        /* host mirrors (launch geometry, validation) */
    const fi_instance* inst_host;
} fi_program;

/* ---- trace (App. A.3) ---------------------------------- */
typedef struct { uint32_t instance, insn, active, pred; } fi_record;   /* insn = pc | op<<16 | groupmask<<24 */
typedef struct { uint64_t va; uint32_t value, step; } fi_store;        /* one stored 32-bit word, 16 B */

/* The trace and the golden-run side data.  fi_golden_trace writes rec, gstore
 * and ckpt; every other call only reads them. */
typedef struct {
    fi_record* rec;           uint64_t n_rec;        /* device */
    const uint64_t* warp_off;                        /* device [n_warps+1]: first record of each warp */
    fi_store* gstore;                                /* device: golden store log, per warp contiguous */
    const uint64_t* gstore_off;                      /* device [n_warps+1] */
    uint32_t* ckpt;                                  /* device: golden register-file checkpoints, or NULL */
    const uint64_t* ckpt_off;                        /* device [n_warps+1], in checkpoints (fi_ckpt_layout) */
    uint32_t ckpt_interval;                          /* steps between checkpoints (0 = none) */
    uint32_t n_warps;
} fi_trace;

/* ---- sites, schedule, injection results -------------------------------- */
typedef struct {
    uint64_t s, instruction_count;                   /* s in [0, N_g) (C-4); instruction_count = s - P_k[instance] */
    uint32_t instance, kernel_id, kernel_count, warp, step, thread;   /* kernel_count: ordinal of the instance among its static kernel's */
    uint32_t pc, u_dst, u_bit, mask;                 /* mask = Table II pattern (0 for ZERO_VALUE: resolved at injection) */
    uint8_t lane, group, bfm, slot, dst_kind /*0 GP, 1 PR*/, dst_reg, n_elig,
            flags /* bit0 FI_SITE_NOT_INJECTED */;
} fi_site;                                           /* 64 B */
#define FI_SITE_NOT_INJECTED 1u
#define FI_SITE_REMOTE 0x80u      /* fi_select_sites_shard: drawn here, located by the rank holding its records */

typedef struct {
    uint64_t seed;                                   /* campaign seed (Philox key) */
    uint32_t n_groups, n_bfms;
    uint8_t groups[8];                               /* group(j) = groups[j % n_groups] */
    uint8_t bfms[4];                                 /* bfm(j) = bfms[(j / n_groups) % n_bfms] */
} fi_schedule;

typedef struct {
    uint32_t before, after, mask, fault_pc;          /* mask actually applied (ZERO_VALUE: = before) */
    uint8_t fault_kind /*0 none, 1 misaligned, 2 unmapped, 3 watchdog, 4 illegal pc*/, outcome, overflow,
            flags /* bit0 FI_POTENTIAL_DUE: fault not fatal under FI_UNCHECKED (f4) */;
    uint32_t n_faulty_stores;                        /* faulty stores after the site (words) */
} fi_inj;                                            /* 24 B */

/* ======================================================================== */
const char* fi_status_str(fi_status s);
const char* fi_last_cuda_error(void);
const char* fi_version(void);

/* Register rows the emulator must keep for this program: 1 + the largest
 * register index the code can touch (host scan of code_host).  Host only. */
uint32_t fi_program_regs(const fi_insn* code_host, uint32_t n_code);

/* Prepared program data, built once per program into `aux` (then set
 * p->aux = aux): the granule map (buffer id per 256-B granule of the image,
 * for the C-15 access check) and the pre-decoded code the emulator executes. */
size_t fi_program_aux_bytes(uint64_t image_bytes, uint32_t n_code, uint32_t n_inst);
fi_status fi_program_prepare(const fi_program* p, void* aux, void* stream);

/* Golden run, pass 1 — PAPER.md:72 step (1)/(4) golden state.  Executes the
 * instances in launch order on `image` (in: initial image, out: golden final
 * image), writing per-warp step counts warp_len[n_warps] and
 * stored-word counts warp_nstore[n_warps].  One launch per instance. */
fi_status fi_golden_lengths(const fi_program* p, uint8_t* image, uint64_t* warp_len, uint64_t* warp_nstore,
                            uint32_t* dev_status, void* stream);

/* Exclusive scan of n u64 values into out[n+1] (out[n] = total).  Scratch:
 * fi_scan_u64_workspace(n) bytes. */
size_t fi_scan_u64_workspace(uint64_t n);
fi_status fi_scan_u64(const uint64_t* in, uint64_t* out, uint64_t n, void* ws, size_t ws_bytes, void* stream);

/* Checkpoint layout: warp w gets ceil(warp_len[w] / interval) checkpoints
 * (before steps 0, interval, 2*interval, ...); ckpt_off[n_warps+1] is their
 * exclusive scan.  Each checkpoint is fi_ckpt_bytes(n_regs) bytes.  Scratch:
 * fi_ckpt_layout_workspace(n_warps) bytes. */
size_t fi_ckpt_bytes(uint32_t n_regs);
size_t fi_ckpt_layout_workspace(uint32_t n_warps);
fi_status fi_ckpt_layout(const uint64_t* warp_len, uint32_t n_warps, uint32_t interval, uint64_t* ckpt_off,
                         void* ws, size_t ws_bytes, void* stream);

/* Golden run, pass 2: re-executes every warp of every instance in ONE launch
 * over the golden final image and writes, through t, the trace records
 * (App. A.3), the golden store log and (if t->ckpt) the checkpoints, at
 * t->warp_off / t->gstore_off / t->ckpt_off (exclusive scans of pass 1). */
fi_status fi_golden_trace(const fi_program* p, const uint8_t* image, const fi_trace* t,
                          uint32_t* dev_status, void* stream);

/* K1 — profile, "dynamic instruction counts for every opcode in
 * every thread ... Instructions that are not executed based on a predicate
 * register are not included", grouped by Table II (C-2):
 *   inst_counts[k][g] = sum over records r of instance k in [rec_begin, rec_end)
 *                       of popc(active & pred) * [g in groupmask(r)]      (u64)
 *   chunk_counts[c][g] = same sum over chunk c = records [1024c, 1024c+1024)
 *                       (u32), written for every chunk overlapping the range.
 * rec_begin must be a multiple of 1024 (shards own whole chunks).
 * inst_counts is zeroed and accumulated by the call (n_inst x 8 u64). */
fi_status fi_profile(const fi_trace* t, uint64_t rec_begin, uint64_t rec_end, uint32_t n_inst,
                     uint64_t* inst_counts, uint32_t* chunk_counts, void* stream);
#define FI_CHUNK 1024

/* §8 row f1 — per-opcode profile, "a profile containing one line
 * for every dynamic kernel and the total dynamic instruction counts for every
 * opcode in every thread": op_counts[k][op] = sum over the records of instance k
 * in [rec_begin, rec_end) with opcode op of popc(active & pred) (u64 [n_inst][32],
 * zeroed by the call).  The executed-opcode set [PAPER.md:82] is its nonzero
 * columns. */
/* ---- multi-GPU profile fused with its exchange ------------------
 * One rank of G (<= FI_MAX_PEERS) GPUs: K1 over this rank's chunk-aligned record
 * shard that ALSO stores every finished chunk-count row straight into each peer's
 * chunk_counts (peer memory mapped over NVLink with fi_ipc_open), then pushes its
 * partial instance counts into slot [rank] of every peer's partials, signals every
 * peer's flag (system-scope release), waits until its own flag reaches
 * epoch * G (all ranks' rows and partials arrived), sums the G partial slots
 * into inst_counts [K][8] and copies the completed rows into chunk_counts [C][8]
 * (caller's device arrays, as fi_profile's).  Replaces fi_profile + two all-reduces with one
 * stream-ordered call: no host round trip, no separate collective.
 * peers (host struct): chunk_counts[r] ([C][8] u32), partials[r] ([G][K][8] u64),
 * flags[r] (u32, zero-initialised, never reset) of every rank r, this rank's own
 * at [rank]; part_local: [K][8] u64 scratch of this rank; epoch: 1, 2, ... — the
 * number of fi_profile_peers calls this rank has made, the same on every rank.
 * Every rank must call it for every epoch (the wait spins on the device until the
 * others do; after 60 s without them it gives up and ORs FI_E_COLLECTIVE into
 * dev_status — that epoch's counts are then invalid; no trap, the context lives on).  A rank must not start epoch e+1 before every rank has consumed the
 * chunk_counts / partials of epoch e (the bench's per-step barrier).
 * Errors: FI_E_ARG, FI_E_CUDA. */
#define FI_MAX_PEERS 8
typedef struct {
    uint32_t* chunk_counts[FI_MAX_PEERS];
    uint64_t* partials[FI_MAX_PEERS];
    uint32_t* flags[FI_MAX_PEERS];
    uint32_t world, rank;
} fi_peers;
fi_status fi_profile_peers(const fi_trace* t, uint64_t rec_begin, uint64_t rec_end, uint32_t n_inst,
                           const fi_peers* peers, uint64_t* part_local, uint32_t epoch, uint64_t* inst_counts,
                           uint32_t* chunk_counts, uint32_t* dev_status, void* stream);
/* Device memory shareable with the other ranks' processes (cudaMalloc +
 * cudaIpcGetMemHandle): *dev_ptr (zero-filled) and its 64-B handle; fi_ipc_open
 * maps a peer's handle into this process (peer access enabled lazily);
 * fi_ipc_close unmaps it, fi_ipc_free frees this process's allocation. */
fi_status fi_ipc_alloc(size_t bytes, void** dev_ptr, void* handle /* 64 B out */);
fi_status fi_ipc_open(const void* handle /* 64 B */, void** dev_ptr);
fi_status fi_ipc_close(void* dev_ptr);
fi_status fi_ipc_free(void* dev_ptr);

fi_status fi_profile_opcodes(const fi_trace* t, uint64_t rec_begin, uint64_t rec_end, uint32_t n_inst,
                             uint64_t* op_counts, void* stream);

/* §8 row f1 — approximate profiling: "only counts the dynamic
 * instructions in the first instance of every static kernel and assumes that the
 * instruction counts for subsequent instances of the same static kernel are the
 * same".  Fills inst_counts[n_inst][8] that way (synchronizes once to upload the
 * first-instance table).  Scratch: fi_profile_approx_workspace() bytes. */
size_t fi_profile_approx_workspace(uint32_t n_kern, uint32_t n_inst);
fi_status fi_profile_approx(const fi_program* p, const fi_trace* t, uint64_t* inst_counts, void* ws,
                            size_t ws_bytes, void* stream);

/* K2 — site index ("1..N" of PAPER.md:78 as prefix sums): exclusive prefix
 * sums P_k[n_inst+1][8] of inst_counts and P_t[T+1][8] of the chunk counts
 * summed per tile of 64 chunks (T = ceil(n_chunks/64)), both u64 with the
 * decoupled-lookback scan; the chunk level itself is resolved at selection time
 * by a warp scan of the tile's chunk counts (no per-chunk prefix array).
 * `index` must hold fi_site_index_bytes(n_inst, n_chunks) bytes.
 * §8 row a3: on the way it checks the Table II identities [PAPER.md:101-104]
 * (GP = FP64+FP32+LD+OTHERS, GPPR = GP+PR) and count <= 32 x records on every
 * instance row and every chunk row; a violation sets FI_E_INVARIANT. */
size_t fi_site_index_bytes(uint32_t n_inst, uint64_t n_chunks);
fi_status fi_build_site_index(const uint64_t* inst_counts, uint32_t n_inst, const uint32_t* chunk_counts,
                              uint64_t n_chunks, void* index, uint32_t* dev_status, void* stream);
/* The instance level alone (P_k + a3 identities), e.g. over approximate counts;
 * `index` sized fi_site_index_bytes(n_inst, 0). */
fi_status fi_build_instance_index(const uint64_t* inst_counts, uint32_t n_inst, void* index, uint32_t* dev_status,
                                  void* stream);
/* Totals N_g (host, synchronizes): copies P_k[n_inst][*] */
fi_status fi_site_totals(const void* index, uint32_t n_inst, uint64_t totals_host[8], void* stream);

/* K3 — draw + search ("random number n from the set 1..N ...
 * translated into a tuple of <kernel_name, kernel_count, instruction_count>";
 * Table II destination register / bit-pattern value [PAPER.md:114-121]).
 * Replica j = j0 + i for i < n: s by Philox4x32-10 + Lemire,
 * then instance, chunk, record, lane, warp, step, slot and mask.
 * `sched` is a host pointer.  totals_host from fi_site_totals. */
fi_status fi_select_sites(const fi_program* p, const fi_trace* t, const uint32_t* chunk_counts, const void* index,
                          uint32_t n_inst, uint64_t n_chunks, const uint64_t totals_host[8],
                          const fi_schedule* sched, uint64_t j0, uint32_t n, fi_site* sites, uint32_t* dev_status,
                          void* stream);

/* Owner-computes K3: the same draw for replicas [j0, j0+n), but
 * only sites whose chunk lies in this rank's record shard [rec_begin, rec_end)
 * (chunk-aligned; the rank whose golden pass wrote those records) are located;
 * the others are written with FI_SITE_REMOTE set and only s / u_dst / u_bit /
 * group / bfm / mask filled.  fi_compact_sites then keeps the located ones. */
fi_status fi_select_sites_shard(const fi_program* p, const fi_trace* t, const uint32_t* chunk_counts,
                                const void* index, uint32_t n_inst, uint64_t n_chunks, const uint64_t totals_host[8],
                                const fi_schedule* sched, uint64_t j0, uint32_t n, uint64_t rec_begin,
                                uint64_t rec_end, fi_site* sites, uint32_t* dev_status, void* stream);
/* Stable compaction of sites[0, n) without FI_SITE_REMOTE into out[0, *n_out)
 * (device count), their replica indices j0 + i into out_j.  One CTA. */
fi_status fi_compact_sites(const fi_site* sites, uint32_t n, uint64_t j0, fi_site* out, uint64_t* out_j,
                           uint32_t* n_out, void* stream);

/* K3 with an approximate profile (row f1): s is drawn over the approximate
 * totals and mapped to (instance k, instruction_count) by the approximate P_k;
 * the site is then located like NVBitFI's injector does at run time — by
 * counting group-g lane-instructions through instance k's records.  When
 * instruction_count >= the instance's real count the site gets
 * FI_SITE_NOT_INJECTED (C-17); K4/K5 skip it (outcome FI_NOT_INJECTED). */
fi_status fi_select_sites_approx(const fi_program* p, const fi_trace* t, const void* index, uint32_t n_inst,
                                 const uint64_t totals_host[8], const fi_schedule* sched, uint64_t j0, uint32_t n,
                                 fi_site* sites, uint32_t* dev_status, void* stream);

/* K4 — inject: one CUDA warp re-executes the site's
 * synthetic warp over the golden final image — from its first instruction, or
 * from the golden checkpoint at or before the site when t->ckpt is set (the
 * prefix is fault-free, so both start states are the same); after
 * the site's instruction writes its destinations, lane `lane`'s destination
 * `dst_reg` is XOR-ed with the mask (ZERO_VALUE: mask = before; predicates C-7).
 * Stores after the site are logged to log[i*log_cap ...] (fi_store words).
 * Memory faults and the watchdog (C-9, C-10) end the replica.
 * Scheduling only (results do not depend on it): persistent warps take
 * replicas from a queue ordered longest-expected-first (counting sort of the
 * steps left after the restart point); scratch: fi_inject_workspace(n) bytes.
 * After the call, bytes 8..15 of ws hold the number of warp-instructions the
 * replicas emulated (u64, from their restart points; measurement only). */
size_t fi_inject_workspace(uint32_t n);
fi_status fi_inject(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                    uint32_t n, fi_inj* out, fi_store* log, uint32_t log_cap, void* ws, size_t ws_bytes,
                    uint32_t* dev_status, void* stream);

/* K5 — classify (Table V [PAPER.md:184-196], [PAPER.md:206]; C-9, C-12, C-14):
 * DUE if a fault/watchdog ended the replica; else SDC if the final value of any
 * output-buffer word differs bitwise from the golden run; else Masked.
 * Writes out[i].outcome and adds 1 to hist[group][bfm][outcome] (u64 [8][4][3]).
 * Replicas with overflow set get outcome 0xFF and FI_E_CAPACITY in dev_status.
 * flags & FI_UNCHECKED (§8 row f4, "potential DUE" [PAPER.md:195-196], [PAPER.md:208]):
 * the application does not check CUDA errors, so a memory fault or illegal
 * instruction only ends the faulting warp — its earlier stores stand — and the
 * replica is classified SDC/Masked by its outputs with FI_POTENTIAL_DUE set;
 * a hang (watchdog) stays DUE.
 * Multi-instance programs (K7): the faulty warp's effect in its instance is
 * propagated through the later instances — every later instance that references
 * a buffer holding a dirty word is re-executed against the replica's faulty
 * overlay, its stores diffed against its golden store log — and the replica is
 * classified on the whole program's outputs (PAPER.md:72 step (4), :206).
 * Scratch: fi_classify_workspace(n_inst, n, log_cap) bytes (0 for one instance).
 * Replicas whose overlay or update lists overflow get outcome 0xFF + FI_E_CAPACITY.
 * K7 CONSUMES `log`: a replica's log slot is reused as scratch for the stores of
 * the later launches it re-executes (classify a log once; K5 and K8 only read it). */
#define FI_UNCHECKED 1u
#define FI_POTENTIAL_DUE 1u
/* K8 outcome 0xFF (not classified) reasons in fi_inj.flags: a capacity was
 * exceeded (also FI_E_CAPACITY), or the replica loaded a corrupted word of a
 * buffer whose pages were dropped after its last launch reference (wild load) */
#define FI_UNCLASSIFIED_CAPACITY 2u
#define FI_UNCLASSIFIED_WILD 4u
/* C-12 secondary numeric classification ("rtol = 1e-6, atol = 0,
 * NaN != number", reported beside the graded bitwise one; the paper leaves the
 * SDC check to the user, "Output file is different" [PAPER.md:189], "both
 * application and user dependent" [PAPER.md:204]).  With rtol > 0 the classify
 * calls also set FI_SDC_WITHIN_TOL in fi_inj.flags of every bitwise SDC whose
 * differing output ELEMENTS (buffer dtype, fi_buffer.flags bits 8..15: 0 u32,
 * 1 f32, 2 f64) all satisfy: both finite and |f - g| <= rtol * |g| (IEEE double,
 * round to nearest; u32 elements never do), and, when hist_tol is not NULL,
 * accumulate hist_tol[8][4][3] with those replicas counted as Masked.  The
 * graded outcome and hist are unchanged.  rtol = 0 (hist_tol ignored): bitwise only. */
#define FI_SDC_WITHIN_TOL 8u
size_t fi_classify_workspace(uint32_t n_inst, uint32_t n, uint32_t log_cap);
fi_status fi_classify(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                      uint32_t n, fi_inj* out, const fi_store* log, uint32_t log_cap, uint64_t* hist,
                      uint32_t flags, double rtol, uint64_t* hist_tol, void* ws, size_t ws_bytes,
                      uint32_t* dev_status, void* stream);

/* K8 — fi_classify for long multi-instance programs (thousands of launches,
 * SURVEY C3/C4/C5): same definition and result as fi_classify's K7 (C-12, C-14,
 * C-19), computed instance-major over batches of `batch` replicas: for every
 * later launch, the (replica, warp) pairs of the replicas whose corrupted words
 * it may read are re-executed across the whole GPU.  Faulty memory lives in
 * copy-on-write 4 KB pages from a pool of `pool_pages`; pages that equal the
 * golden state are returned (a replica with none is Masked early) and pages of a
 * buffer past its last launch reference are dropped.  pend_cap = update slots per
 * replica and launch (>= the launch's golden stores, plus faulty extras).
 * Replicas that exceed a capacity, or that later load a dropped corrupted word,
 * get outcome 0xFF and FI_E_CAPACITY — never a wrong class.  Fills out[].outcome
 * / flags (and fault_kind/fault_pc of the first downstream fault when K4 had
 * none), accumulates hist[8][4][3].  Scratch: fi_classify_batched_workspace();
 * after fi_classify_batched_jit its first 8 bytes hold the u64 count of emulated
 * warp-steps of every warp K8 re-executed (the work behind its issue roofline). */
size_t fi_classify_batched_workspace(const fi_program* p, uint32_t n, uint32_t log_cap, uint32_t batch,
                                     uint32_t pool_pages, uint32_t pend_cap);
fi_status fi_classify_batched(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_site* sites,
                              uint32_t n, fi_inj* out, const fi_store* log, uint32_t log_cap, uint64_t* hist,
                              uint32_t flags, double rtol, uint64_t* hist_tol, uint32_t batch, uint32_t pool_pages,
                              uint32_t pend_cap, void* ws, size_t ws_bytes, uint32_t* dev_status, void* stream);

/* §8 rows f2/f3 — permanent faults (Table III
 * [PAPER.md:128-134]) and intermittent faults.  A fault is
 * {opcode id, SM id, lane id, XOR bit mask}: the destination registers of every
 * dynamic instance of the opcode executed in that lane by the CTAs on that SM
 * (CTA c of an instance runs on SM c mod n_sm, reading C-21) are XOR-ed with the
 * same mask (a predicate destination flips iff mask bit 0 is set).  q32 != 0
 * makes it intermittent: an instance is corrupted only when
 * Philox4x32-10(ctr = {warp, step, replica, 0x46490002}, key = seed).x < q32
 * (reading C-22).  Every run re-executes the affected warps of every instance
 * (plus, as in K7, every later instance that may read corrupted words) and is
 * classified on the whole program (Table V).  hist[3] (u64) accumulates
 * op_weights[opcode] per outcome — the opcode-weighted outcomes of PAPER.md:228
 * (1 per run when op_weights is NULL).
 * A permanent fault can corrupt many words: ov_words bounds the distinct
 * corrupted words one run may hold (e.g. image_bytes/4; 0 = the transient
 * default, max(log_cap, 4096)); a run that exceeds it gets outcome 0xFF and
 * FI_E_CAPACITY.  Scratch: fi_inject_permanent_workspace(n, log_cap, ov_words,
 * max_slots) bytes — max_slots (0 = as many as can be resident, else >= 4)
 * caps the replicas in flight and so the scratch; the call uses as many slots
 * as ws_bytes holds (at least 4).  faults/op_weights/out/log/hist/ws/dev_status
 * are device pointers; out[i].mask = faults[i].mask, fault_kind/fault_pc the
 * first fault (DUE) or the first non-fatal one (FI_POTENTIAL_DUE). */
typedef struct {
    uint32_t opcode, sm, lane, mask;
    uint32_t q32;                                    /* 0 = permanent; else activation probability * 2^32 */
    uint32_t n_sm;                                   /* SMs of the modelled GPU (148 for B200) */
    uint64_t seed;
} fi_pfault;                                         /* 32 B */
size_t fi_inject_permanent_workspace(uint32_t n, uint32_t log_cap, uint32_t ov_words, uint32_t max_slots);
fi_status fi_inject_permanent(const fi_program* p, const uint8_t* image, const fi_trace* t, const fi_pfault* faults,
                              uint32_t n, const uint64_t* op_weights, fi_inj* out, fi_store* log, uint32_t log_cap,
                              uint32_t ov_words, uint64_t* hist, uint32_t flags, void* ws, size_t ws_bytes,
                              uint32_t* dev_status, void* stream);

/* Rows f2/f3 on K8: fi_inject_permanent for long multi-launch programs — same
 * faults, definition and outputs (out[i], opcode-weighted hist[3]); every replica
 * runs from the first launch with the opcode hook armed on the faulty SM's CTAs,
 * launches re-executed where the opcode runs on that SM or corrupted pages are
 * referenced.  Scratch: fi_classify_batched_workspace(p, n, log_cap, batch,
 * pool_pages, pend_cap); capacities as for fi_classify_batched. */
fi_status fi_inject_permanent_batched(const fi_program* p, const uint8_t* image, const fi_trace* t,
                                      const fi_pfault* faults, uint32_t n, const uint64_t* op_weights, fi_inj* out,
                                      uint32_t log_cap, uint64_t* hist, uint32_t flags, uint32_t batch,
                                      uint32_t pool_pages, uint32_t pend_cap, void* ws, size_t ws_bytes,
                                      uint32_t* dev_status, void* stream);

/* ---- JIT-specialised emulator (K4 on per-program generated code) --------
 * fi_jit_build generates CUDA source from the program's code (p->code_host and
 * the HOST kernel table kern_host[p->n_kern]) — every static instruction
 * becomes straight-line device code with the synthetic registers in hardware
 * registers — compiles it with NVRTC for sm_100a (libnvrtc.so.12, loaded at
 * run time) and loads it into the current device's primary context.  The
 * semantics are DESIGN.md §3, identical to the interpreter behind fi_inject.
 * Synchronous; FI_E_PROGRAM if NVRTC rejects the source (fi_jit_log() has the
 * log), FI_E_CUDA if NVRTC / the driver is unavailable.  Free with fi_jit_free.
 * fi_jit_compile_check compiles without loading (no GPU needed); fi_jit_source
 * returns the generated source (buf may be NULL; returns the bytes needed, 0 on
 * bad arguments). */
typedef struct fi_jit fi_jit;
#define FI_JIT_INJECT 1u                            /* k_inject_jit (fi_inject_jit) */
#define FI_JIT_GOLDEN 2u                            /* golden passes (fi_golden_lengths_jit, fi_golden_trace_jit) */
#define FI_JIT_PAGE 4u                              /* K8 re-execution over replica pages (fi_classify_batched_jit) */
fi_status fi_jit_build(const fi_program* p, const fi_kernel* kern_host, uint32_t modes, fi_jit** out);
void fi_jit_free(fi_jit* j);
double fi_jit_compile_seconds(const fi_jit* j);
const char* fi_jit_log(void);
fi_status fi_jit_compile_check(const fi_insn* code_host, uint32_t n_code, const fi_kernel* kern_host, uint32_t n_kern,
                               uint32_t n_regs, uint32_t modes, size_t* cubin_bytes);
/* (fi_jit_source / fi_jit_compile_check also accept modes | 0x100: pass 1 as the
 * control slice, as fi_jit_build picks it.) */
size_t fi_jit_source(const fi_insn* code_host, uint32_t n_code, const fi_kernel* kern_host, uint32_t n_kern,
                     uint32_t n_regs, uint32_t modes, char* buf, size_t buf_bytes);
/* K4 on the JIT module `j` built for p: same arguments, scratch, scheduling and
 * results as fi_inject (bit-identical outputs), asynchronous on `stream`. */
fi_status fi_inject_jit(const fi_jit* j, const fi_program* p, const uint8_t* image, const fi_trace* t,
                        const fi_site* sites, uint32_t n, fi_inj* out, fi_store* log, uint32_t log_cap, void* ws,
                        size_t ws_bytes, uint32_t* dev_status, void* stream);
/* The golden passes on a module built with FI_JIT_GOLDEN: same results (trace
 * records, store log, checkpoints, final image, lengths) as fi_golden_lengths /
 * fi_golden_trace, bit for bit, with one difference in who writes the image.
 * fi_jit_build generates pass 1 as the CONTROL SLICE of each kernel (only the
 * instructions that can reach a BRA / EXIT / STG guard, jit.cpp control_slice)
 * when the program has one launch or no slice loads memory: that length pass
 * leaves `image` untouched.  Pass 2 (fi_golden_trace_jit, one launch per instance
 * in launch order) always stores into `image` (in: pass 1's image, out: the
 * golden final image), so after both calls `image` is the golden final image
 * either way. */
fi_status fi_golden_lengths_jit(const fi_jit* j, const fi_program* p, uint8_t* image, uint64_t* warp_len,
                                uint64_t* warp_nstore, uint32_t* dev_status, void* stream);
fi_status fi_golden_trace_jit(const fi_jit* j, const fi_program* p, uint8_t* image, const fi_trace* t,
                              uint32_t* dev_status, void* stream);
/* Pass 2 for the warps [w_lo, w_hi) only, image stores only from the warps
 * [own_lo, own_hi) (the owner-computes golden run of fi_golden_run_shard), and
 * optionally the profile of those warps' records fused into the pass: with
 * inst_counts ([n_inst][8] u64) and chunk_counts ([ceil(n_rec/FI_CHUNK)][8] u32),
 * both device and ZEROED by the caller, the call ADDS what fi_profile over the
 * records of warps [w_lo, w_hi) would write (PAPER.md:78 — the profiler counts
 * during the golden run); both NULL = no profile; one NULL = FI_E_ARG. */
fi_status fi_golden_trace_jit_range(const fi_jit* j, const fi_program* p, uint8_t* image, const fi_trace* t,
                                    uint32_t w_lo, uint32_t w_hi, uint32_t own_lo, uint32_t own_hi,
                                    uint64_t* inst_counts, uint32_t* chunk_counts,
                                    uint32_t* dev_status, void* stream);
/* 1 when fi_jit_build generated golden pass 1 as the control slice (it then leaves
 * the image untouched; pass 2 writes it), else 0. */
int fi_jit_len_sliced(const fi_jit* j);
/* fi_classify_batched with K8's per-launch re-execution on a module built with
 * FI_JIT_PAGE: same arguments, scratch and results (transient faults). */
fi_status fi_classify_batched_jit(const fi_jit* j, const fi_program* p, const uint8_t* image, const fi_trace* t,
                                  const fi_site* sites, uint32_t n, fi_inj* out, const fi_store* log, uint32_t log_cap,
                                  uint64_t* hist, uint32_t flags, double rtol, uint64_t* hist_tol, uint32_t batch,
                                  uint32_t pool_pages, uint32_t pend_cap, void* ws, size_t ws_bytes,
                                  uint32_t* dev_status, void* stream);

/* fi_golden_run — the golden run as ONE call: Fig. 1 step (1) (the
 * run whose dynamic instructions the profiler counts) and the golden
 * output state step (4) compares against.  Runs pass 1
 * (per-warp lengths and stored-word counts, golden final image), the scans, the
 * checkpoint layout and pass 2 (App. A.3 trace records, golden store log,
 * register-file checkpoints) on `jit` (a module built with FI_JIT_GOLDEN) or, with
 * jit = NULL, on the shared-memory interpreter — bit-identical results.
 *   image         device, caller's: in = the initial image, out = golden final image
 *   ckpt_interval 0 = no checkpoints, FI_CKPT_AUTO = 8192 steps doubled while the
 *                 checkpoints exceed ckpt_budget_frac (<= 0: 0.2) of free HBM
 *   *out          the trace: fi_golden_trace_of(*out) is the fi_trace every later
 *                 call reads (fi_profile, fi_select_sites, fi_inject*, fi_classify*),
 *                 and the run's profile (fi_golden_profile, Fig. 1 step
 *                 (2)): counted inside pass 2 on the JIT engine, K1 on the interpreter
 * Memory: UNLIKE the calls above, the trace arrays (records, store log,
 * checkpoints, offsets) are sized by pass 1 and allocated by this call,
 * stream-ordered from the current device's default memory pool; *out owns them
 * until fi_golden_free(*out, stream).  SYNCHRONIZES (the record totals size the
 * allocations).  Errors: FI_E_ARG, FI_E_PROGRAM (the golden run faulted: the
 * program violates DESIGN.md §3.5), FI_E_CUDA; nothing is allocated on error. */
typedef struct fi_golden fi_golden;
fi_status fi_golden_run(const fi_program* p, const fi_jit* jit, uint8_t* image, uint32_t ckpt_interval,
                        double ckpt_budget_frac, fi_golden** out, void* stream);
/* Owner-computes golden run of rank `rank` of `world` (a
 * single-launch program and the JIT engine): pass 1 for every warp (the layout
 * is global), pass 2 only for the warps holding the records of this rank's
 * chunk-aligned shard [r0, r1) = fi_campaign's profile shard, and into `image`
 * only the stores of the warps whose first record lies in it.  The trace of
 * that shard, its checkpoints and store log are valid; the rest of the arrays is
 * not written.  With a sliced pass 1 (fi_jit_len_sliced) the image then holds
 * the golden words of this rank's warps only: the SUM over the ranks of the
 * writer buffers (zero-initialised, SSA) is the golden final image.
 * world = 1 is fi_golden_run. */
fi_status fi_golden_run_shard(const fi_program* p, const fi_jit* jit, uint8_t* image, uint32_t ckpt_interval,
                              double ckpt_budget_frac, int rank, int world, fi_golden** out, void* stream);
void fi_golden_shard_range(const fi_golden* g, uint64_t* rec_begin, uint64_t* rec_end, uint32_t* w_lo, uint32_t* w_hi);
/* The owner-computes partition (host only): from warp_off_host[n_warps+1], rank
 * r of G's chunk-aligned record shard [rec_begin, rec_end) (fi_campaign's profile
 * shard), the warps [w_lo, w_hi) holding its records (pass 2 runs them) and the
 * warps [own_lo, own_hi) whose first record lies in it (they store into the
 * image).  Over the ranks the own ranges partition every warp with a record. */
fi_status fi_shard_warps(const uint64_t* warp_off_host, uint32_t n_warps, int rank, int world, uint64_t* rec_begin,
                         uint64_t* rec_end, uint32_t* w_lo, uint32_t* w_hi, uint32_t* own_lo, uint32_t* own_hi);
const fi_trace* fi_golden_trace_of(const fi_golden* g);          /* host struct of device pointers */
/* The golden run's profile, Fig. 1 step (2): device pointers (owned by
 * g) to inst_counts [n_inst][8] u64 and chunk_counts [ceil(n_rec/FI_CHUNK)][8] u32,
 * equal to what fi_profile(trace, 0, n_rec, ...) writes — counted inside pass 2 on
 * the JIT engine, by K1 over the finished trace on the interpreter.  FI_E_ARG for
 * a handle of fi_golden_run_shard with world > 1 (no whole-trace profile). */
fi_status fi_golden_profile(const fi_golden* g, const uint64_t** inst_counts, const uint32_t** chunk_counts);
const uint64_t* fi_golden_warp_len(const fi_golden* g);          /* device [n_warps] golden steps per warp */
const uint64_t* fi_golden_gstore_off_host(const fi_golden* g);   /* HOST [n_warps+1] copy of gstore_off */
fi_status fi_golden_free(fi_golden* g, void* stream);            /* stream-ordered release; NULL g is a no-op */

/* Table II parameter file, one parameter per line in Table II order
 * [PAPER.md:88]: arch state id, bit-flip model, kernel name, kernel count,
 * instruction count, destination register value, bit-pattern value (the two
 * [0,1) values printed as u/2^32 with 10 digits).  Host only. */
fi_status fi_write_params_txt(const fi_site* site_host, const char* kernel_name, char* buf, size_t buf_bytes);

/* The profile file of PAPER.md:78 ("a profile containing one line for every
 * dynamic kernel"): one line per dynamic kernel instance k, in launch order,
 *   <kernel_name>; kernel_count: <c>; <G_FP64> <G_FP32> <G_LD> <G_PR> <G_NODEST> <G_OTHERS> <G_GPPR> <G_GP>
 * with the eight Table II counts of inst_counts_host[k][0..7] (u64, host).
 * kernel_names[n_kern] (host) names the static kernels; inst_host[n_inst] gives
 * each instance's static kernel and kernel_count.  Writes at most buf_bytes
 * (NUL-terminated); *needed (if not NULL) receives the full length + 1, so a
 * call with buf = NULL, buf_bytes = 0 sizes the buffer.  FI_E_ARG if it does
 * not fit.  Host only. */
fi_status fi_write_profile_txt(const uint64_t* inst_counts_host, const fi_instance* inst_host, uint32_t n_inst,
                               const char* const* kernel_names, uint32_t n_kern, char* buf, size_t buf_bytes,
                               size_t* needed);

/* ---- fi_campaign: the whole campaign of one rank, host buffers in and out ----
 * PAPER.md:72 Fig. 1 steps (1)-(4) end to end, as the driver of SURVEY §8(e):
 * H2D of the program (from HOST arrays; buffers with a writer are zeroed on the
 * device instead of copied — they start zeroed), golden run (passes 1 + 2, golden
 * checkpoints), K1 profile of this rank's chunk-aligned record shard
 * [chunk r*C/G, (r+1)*C/G), all-reduce(SUM) of inst_counts (u64) and
 * chunk_counts (u32) through `allreduce`, K2 index (+ a3 identities), K3 select
 * / K4 inject / K5|K7|K8 classify of this rank's replica block
 * [r*n/G, (r+1)*n/G) (replica RNG keyed by the global index j, so results do
 * not depend on G), all-reduce(SUM) of the u64 histogram, D2H of the results.
 * With cfg->approximate the profile is PAPER.md:80's approximate one
 * (fi_profile_approx, first instance per static kernel; no record sharding,
 * no count all-reduce) and sites come from fi_select_sites_approx (C-17).
 *
 * allreduce(dev, count, elem_bytes, ctx, stream): in-place SUM over the ranks of
 * `count` integers of elem_bytes (4 or 8) at device pointer dev, ordered on
 * `stream`; returns 0 on success.  May be NULL when world == 1.  Typically
 * torch.distributed all_reduce on NCCL (paper_conf_dsn_0002hsvk21_b200.fi.campaign).
 *
 * Memory: unlike the other calls, fi_campaign allocates its device memory itself
 * (stream-ordered, from cfg->device's default memory pool; all freed before it
 * returns, but the pool keeps the memory reserved for the next call — see
 * fi_campaign_release_memory) and SYNCHRONIZES.
 * Host arrays in cfg are read only; result arrays marked optional may be NULL.
 * Errors: FI_E_ARG (bad cfg), FI_E_PROGRAM / FI_E_INVARIANT / FI_E_SITE /
 * FI_E_CAPACITY from device status, FI_E_EMPTY_GROUP / FI_E_NOT_INJECTABLE from
 * selection, FI_E_CUDA, FI_E_COLLECTIVE when allreduce returns non-zero. */
typedef int (*fi_allreduce_fn)(void* dev, uint64_t count, uint32_t elem_bytes, void* ctx, void* stream);
#define FI_PROPAGATION_AUTO 0u      /* K8 from 64 launches on, else K5/K7 (fi_classify) */
#define FI_PROPAGATION_K7 1u        /* fi_classify */
#define FI_PROPAGATION_K8 2u        /* fi_classify_batched */
#define FI_CKPT_AUTO 0xFFFFFFFFu    /* 8192 steps, doubled until the checkpoints fit 20% of free HBM */
#define FI_ENGINE_INTERP 0u
#define FI_ENGINE_JIT 1u
typedef struct {
    /* the program, HOST arrays */
    const fi_insn* code;         uint32_t n_code;
    const fi_kernel* kern;       uint32_t n_kern;
    const fi_instance* inst;     uint32_t n_inst;
    const uint32_t* cbank;       uint32_t n_cbank;
    const fi_buffer* buf;        uint32_t n_buf;
    const uint8_t* init_image;   uint64_t image_bytes;
    uint32_t n_warps;
    /* the campaign */
    fi_schedule sched;           /* seed + per-replica group / bit-flip model */
    uint64_t n_replicas;         /* whole campaign, all ranks */
    uint32_t flags;              /* FI_UNCHECKED (row f4) */
    uint32_t propagation;        /* FI_PROPAGATION_* */
    uint32_t approximate;        /* 1 = approximate profile (row f1) */
    uint32_t ckpt_interval;      /* steps between golden checkpoints, 0 = none, FI_CKPT_AUTO */
    uint32_t engine;             /* K4 engine: FI_ENGINE_INTERP, or FI_ENGINE_JIT (fi_inject_jit; the module is
                                    built once per program and device and cached for the process) */
    uint64_t k8_mem_budget;      /* device bytes for K8 scratch (0 = 24 GiB) */
    int device;                  /* CUDA device ordinal (< 0 = current) */
    void* stream;                /* cudaStream_t (NULL = a stream fi_campaign creates) */
    double rtol;                 /* > 0: also the C-12 secondary numeric classification (hist_tol) */
    uint32_t owner_computes;     /* world > 1, one launch, JIT: the golden run is sharded with the profile
                                    (fi_golden_run_shard) and each rank injects the replicas whose site lies in
                                    its record shard (fi_select_sites_shard) instead of the block [r*n/G, (r+1)*n/G) */
} fi_campaign_cfg;

typedef struct {
    uint64_t hist[8][4][3];      /* [group][bfm][Masked, SDC, DUE], summed over all ranks */
    uint64_t totals[8];          /* N_g over the whole trace (exact or approximate) */
    uint64_t n_rec;              /* trace records (warp-instructions) */
    uint64_t counted;            /* thread-level dynamic instructions counted (NODEST + GPPR) */
    uint64_t j0, n_local;        /* this rank's replica block */
    uint64_t rec_begin, rec_end; /* this rank's profile shard */
    uint64_t n_unclassified;     /* replicas with outcome 0xFF (capacity), this rank */
    uint64_t n_not_injected;     /* approximate sites that do not exist (C-17), this rank */
    /* CUDA-event times on the stream, ms: H2D + prepare, golden run, profile,
     * count exchange, index, select, inject, classify + histogram exchange, D2H */
    float ms_h2d, ms_golden, ms_profile, ms_exchange, ms_index, ms_select, ms_inject, ms_classify, ms_d2h;
    float ms_jit;                /* host time building the JIT module (0 when cached or not used) */
    /* optional host outputs (NULL = not returned) */
    fi_site* sites;              /* [n_local] */
    fi_inj* inj;                 /* [n_local] */
    uint64_t* inst_counts;       /* [n_inst][8] (after the exchange) */
    uint64_t hist_tol[8][4][3];  /* cfg->rtol > 0: secondary histogram (FI_SDC_WITHIN_TOL counted Masked), all ranks */
    uint64_t* j;                 /* optional [n_local]: the replica index of each returned site / result row */
} fi_campaign_result;

fi_status fi_campaign(const fi_campaign_cfg* cfg, int rank, int world, fi_allreduce_fn allreduce, void* ctx,
                      fi_campaign_result* res);
/* Return the device memory fi_campaign's calls left reserved in `device`'s default
 * memory pool (device < 0: the current device) to the driver.  Synchronizes the
 * device.  FI_E_CUDA on failure. */
fi_status fi_campaign_release_memory(int device);

#ifdef __cplusplus
}
#endif
#endif
