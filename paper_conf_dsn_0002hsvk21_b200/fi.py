"""ctypes binding of libfi.so (include/fi.h) — argument marshalling only.

Every step of the path runs in the CUDA kernels behind the C ABI; PyTorch only
allocates device memory and supplies the current stream.  There is no CPU
fallback: if libfi.so is missing or no CUDA device is present, calls raise.
The function names mirror fi.h (fi_golden_lengths, fi_profile, fi_select_sites,
fi_inject, fi_classify, ...).
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np
import torch

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libfi.so")

FI_OK, FI_E_ARG, FI_E_EMPTY_GROUP, FI_E_NOT_INJECTABLE, FI_E_PROGRAM, FI_E_CUDA, FI_E_SITE = 0, 1, 2, 3, 4, 5, 6
FI_E_CAPACITY, FI_E_INVARIANT = 8, 9
FI_CHUNK = 1024
FI_UNCHECKED, FI_POTENTIAL_DUE = 1, 1
FI_SDC_WITHIN_TOL = 8                          # fi_inj.flags: bitwise SDC within rtol (C-12 secondary)
G_FP64, G_FP32, G_LD, G_PR, G_NODEST, G_OTHERS, G_GPPR, G_GP = range(8)
GROUP_NAMES = ["G_FP64", "G_FP32", "G_LD", "G_PR", "G_NODEST", "G_OTHERS", "G_GPPR", "G_GP"]
BFM_NAMES = ["FLIP_SINGLE_BIT", "FLIP_TWO_BITS", "RANDOM_VALUE", "ZERO_VALUE"]
MASKED, SDC, DUE, NOT_INJECTED = 0, 1, 2, 3
FI_NOPS = 32

SITE_DTYPE = np.dtype([
    ("s", "<u8"), ("instruction_count", "<u8"),
    ("instance", "<u4"), ("kernel_id", "<u4"), ("kernel_count", "<u4"), ("warp", "<u4"),
    ("step", "<u4"), ("thread", "<u4"), ("pc", "<u4"), ("u_dst", "<u4"), ("u_bit", "<u4"), ("mask", "<u4"),
    ("lane", "u1"), ("group", "u1"), ("bfm", "u1"), ("slot", "u1"), ("dst_kind", "u1"), ("dst_reg", "u1"),
    ("n_elig", "u1"), ("flags", "u1"),
])
INJ_DTYPE = np.dtype([("before", "<u4"), ("after", "<u4"), ("mask", "<u4"), ("fault_pc", "<u4"),
                      ("fault_kind", "u1"), ("outcome", "u1"), ("overflow", "u1"), ("flags", "u1"),
                      ("n_faulty_stores", "<u4")])
RECORD_DTYPE = np.dtype([("instance", "<u4"), ("insn", "<u4"), ("active", "<u4"), ("pred", "<u4")])
STORE_DTYPE = np.dtype([("va", "<u8"), ("value", "<u4"), ("step", "<u4")])
PFAULT_DTYPE = np.dtype([("opcode", "<u4"), ("sm", "<u4"), ("lane", "<u4"), ("mask", "<u4"), ("q32", "<u4"),
                         ("n_sm", "<u4"), ("seed", "<u8")])
assert SITE_DTYPE.itemsize == 64 and INJ_DTYPE.itemsize == 24 and PFAULT_DTYPE.itemsize == 32


class FIError(RuntimeError):
    def __init__(self, code: int, where: str, detail: str = ""):
        self.code = code
        super().__init__(f"{where}: {status_str(code)} ({code}){' — ' + detail if detail else ''}")


class fi_program(C.Structure):
    _fields_ = [("code", C.c_void_p), ("n_code", C.c_uint32),
                ("kern", C.c_void_p), ("n_kern", C.c_uint32),
                ("inst", C.c_void_p), ("n_inst", C.c_uint32),
                ("cbank", C.c_void_p), ("n_cbank", C.c_uint32),
                ("buf", C.c_void_p), ("n_buf", C.c_uint32),
                ("aux", C.c_void_p),
                ("image_bytes", C.c_uint64),
                ("n_warps", C.c_uint32), ("n_regs", C.c_uint32),
                ("code_host", C.c_void_p), ("inst_host", C.c_void_p)]


class fi_trace(C.Structure):
    _fields_ = [("rec", C.c_void_p), ("n_rec", C.c_uint64), ("warp_off", C.c_void_p),
                ("gstore", C.c_void_p), ("gstore_off", C.c_void_p),
                ("ckpt", C.c_void_p), ("ckpt_off", C.c_void_p), ("ckpt_interval", C.c_uint32),
                ("n_warps", C.c_uint32)]


class fi_schedule(C.Structure):
    _fields_ = [("seed", C.c_uint64), ("n_groups", C.c_uint32), ("n_bfms", C.c_uint32),
                ("groups", C.c_uint8 * 8), ("bfms", C.c_uint8 * 4)]


FI_MAX_PEERS = 8


class fi_peers(C.Structure):
    _fields_ = [("chunk_counts", C.c_void_p * FI_MAX_PEERS), ("partials", C.c_void_p * FI_MAX_PEERS),
                ("flags", C.c_void_p * FI_MAX_PEERS), ("world", C.c_uint32), ("rank", C.c_uint32)]


class fi_campaign_cfg(C.Structure):
    _fields_ = [("code", C.c_void_p), ("n_code", C.c_uint32),
                ("kern", C.c_void_p), ("n_kern", C.c_uint32),
                ("inst", C.c_void_p), ("n_inst", C.c_uint32),
                ("cbank", C.c_void_p), ("n_cbank", C.c_uint32),
                ("buf", C.c_void_p), ("n_buf", C.c_uint32),
                ("init_image", C.c_void_p), ("image_bytes", C.c_uint64),
                ("n_warps", C.c_uint32),
                ("sched", fi_schedule),
                ("n_replicas", C.c_uint64),
                ("flags", C.c_uint32), ("propagation", C.c_uint32), ("approximate", C.c_uint32),
                ("ckpt_interval", C.c_uint32), ("engine", C.c_uint32), ("k8_mem_budget", C.c_uint64),
                ("device", C.c_int), ("stream", C.c_void_p), ("rtol", C.c_double), ("owner_computes", C.c_uint32)]


class fi_campaign_result(C.Structure):
    _fields_ = [("hist", C.c_uint64 * 96), ("totals", C.c_uint64 * 8),
                ("n_rec", C.c_uint64), ("counted", C.c_uint64), ("j0", C.c_uint64), ("n_local", C.c_uint64),
                ("rec_begin", C.c_uint64), ("rec_end", C.c_uint64),
                ("n_unclassified", C.c_uint64), ("n_not_injected", C.c_uint64),
                ("ms_h2d", C.c_float), ("ms_golden", C.c_float), ("ms_profile", C.c_float),
                ("ms_exchange", C.c_float), ("ms_index", C.c_float), ("ms_select", C.c_float),
                ("ms_inject", C.c_float), ("ms_classify", C.c_float), ("ms_d2h", C.c_float), ("ms_jit", C.c_float),
                ("sites", C.c_void_p), ("inj", C.c_void_p), ("inst_counts", C.c_void_p),
                ("hist_tol", C.c_uint64 * 96), ("j", C.c_void_p)]


# int allreduce(void* dev, uint64_t count, uint32_t elem_bytes, void* ctx, void* stream)
ALLREDUCE_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_uint64, C.c_uint32, C.c_void_p, C.c_void_p)
FI_PROPAGATION = {"auto": 0, "k7": 1, "k8": 2}
FI_CKPT_AUTO = 0xFFFFFFFF
FI_JIT_INJECT, FI_JIT_GOLDEN, FI_JIT_PAGE = 1, 2, 4

_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise FIError(FI_E_CUDA, "load", f"{LIB_PATH} not built (run __graft_entry__.build())")
        L = C.CDLL(LIB_PATH)
        vp, u32, u64, sz = C.c_void_p, C.c_uint32, C.c_uint64, C.c_size_t
        st = C.c_int
        sig = {
            "fi_status_str": (C.c_char_p, [st]),
            "fi_last_cuda_error": (C.c_char_p, []),
            "fi_version": (C.c_char_p, []),
            "fi_program_regs": (u32, [vp, u32]),
            "fi_program_aux_bytes": (sz, [u64, u32, u32]),
            "fi_program_prepare": (st, [vp, vp, vp]),
            "fi_golden_lengths": (st, [vp, vp, vp, vp, vp, vp]),
            "fi_scan_u64_workspace": (sz, [u64]),
            "fi_scan_u64": (st, [vp, vp, u64, vp, sz, vp]),
            "fi_ckpt_bytes": (sz, [u32]),
            "fi_ckpt_layout_workspace": (sz, [u32]),
            "fi_ckpt_layout": (st, [vp, u32, u32, vp, vp, sz, vp]),
            "fi_golden_trace": (st, [vp, vp, vp, vp, vp]),
            "fi_profile": (st, [vp, u64, u64, u32, vp, vp, vp]),
            "fi_site_index_bytes": (sz, [u32, u64]),
            "fi_build_site_index": (st, [vp, u32, vp, u64, vp, vp, vp]),
            "fi_site_totals": (st, [vp, u32, vp, vp]),
            "fi_select_sites": (st, [vp, vp, vp, vp, u32, u64, vp, vp, u64, u32, vp, vp, vp]),
            "fi_inject_workspace": (sz, [u32]),
            "fi_inject": (st, [vp, vp, vp, vp, u32, vp, vp, u32, vp, sz, vp, vp]),
            "fi_classify_workspace": (sz, [u32, u32, u32]),
            "fi_classify": (st, [vp, vp, vp, vp, u32, vp, vp, u32, vp, u32, C.c_double, vp, vp, sz, vp, vp]),
            "fi_write_params_txt": (st, [vp, C.c_char_p, C.c_char_p, sz]),
            "fi_profile_opcodes": (st, [vp, u64, u64, u32, vp, vp]),
            "fi_profile_approx_workspace": (sz, [u32, u32]),
            "fi_profile_approx": (st, [vp, vp, vp, vp, sz, vp]),
            "fi_build_instance_index": (st, [vp, u32, vp, vp, vp]),
            "fi_select_sites_approx": (st, [vp, vp, vp, u32, vp, vp, u64, u32, vp, vp, vp]),
            "fi_inject_permanent_workspace": (sz, [u32, u32, u32, u32]),
            "fi_classify_batched_workspace": (sz, [vp, u32, u32, u32, u32, u32]),
            "fi_inject_permanent_batched": (st, [vp, vp, vp, vp, u32, vp, vp, u32, vp, u32, u32, u32, u32, vp, sz,
                                                 vp, vp]),
            "fi_classify_batched": (st, [vp, vp, vp, vp, u32, vp, vp, u32, vp, u32, C.c_double, vp, u32, u32, u32, vp,
                                         sz, vp, vp]),
            "fi_classify_batched_jit": (st, [vp, vp, vp, vp, vp, u32, vp, vp, u32, vp, u32, C.c_double, vp, u32, u32,
                                             u32, vp, sz, vp, vp]),
            "fi_inject_permanent": (st, [vp, vp, vp, vp, u32, vp, vp, vp, u32, u32, vp, u32, vp, sz, vp, vp]),
            "fi_jit_build": (st, [vp, vp, u32, C.POINTER(vp)]),
            "fi_jit_free": (None, [vp]),
            "fi_jit_compile_seconds": (C.c_double, [vp]),
            "fi_jit_log": (C.c_char_p, []),
            "fi_jit_compile_check": (st, [vp, u32, vp, u32, u32, u32, C.POINTER(C.c_size_t)]),
            "fi_jit_source": (sz, [vp, u32, vp, u32, u32, u32, vp, sz]),
            "fi_golden_lengths_jit": (st, [vp, vp, vp, vp, vp, vp, vp]),
            "fi_golden_trace_jit": (st, [vp, vp, vp, vp, vp, vp]),
            "fi_golden_trace_jit_range": (st, [vp, vp, vp, vp, u32, u32, u32, u32, vp, vp, vp, vp]),
            "fi_golden_run": (st, [vp, vp, vp, u32, C.c_double, C.POINTER(vp), vp]),
            "fi_golden_trace_of": (C.POINTER(fi_trace), [vp]),
            "fi_golden_warp_len": (vp, [vp]),
            "fi_golden_gstore_off_host": (C.POINTER(C.c_uint64), [vp]),
            "fi_golden_free": (st, [vp, vp]),
            "fi_golden_profile": (st, [vp, C.POINTER(vp), C.POINTER(vp)]),
            "fi_golden_run_shard": (st, [vp, vp, vp, u32, C.c_double, C.c_int, C.c_int, C.POINTER(vp), vp]),
            "fi_golden_shard_range": (None, [vp, vp, vp, vp, vp]),
            "fi_jit_len_sliced": (C.c_int, [vp]),
            "fi_shard_warps": (st, [vp, u32, C.c_int, C.c_int, vp, vp, vp, vp, vp, vp]),
            "fi_inject_jit": (st, [vp, vp, vp, vp, vp, u32, vp, vp, u32, vp, sz, vp, vp]),
            "fi_write_profile_txt": (st, [vp, vp, u32, vp, u32, vp, sz, C.POINTER(C.c_size_t)]),
            "fi_campaign": (st, [C.POINTER(fi_campaign_cfg), C.c_int, C.c_int, ALLREDUCE_FN, vp,
                                 C.POINTER(fi_campaign_result)]),
            "fi_campaign_release_memory": (st, [C.c_int]),
            "fi_profile_peers": (st, [vp, u64, u64, u32, vp, vp, u32, vp, vp, vp, vp]),
            "fi_ipc_alloc": (st, [sz, C.POINTER(C.c_void_p), vp]),
            "fi_ipc_open": (st, [vp, C.POINTER(C.c_void_p)]),
            "fi_ipc_close": (st, [vp]),
            "fi_ipc_free": (st, [vp]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype, f.argtypes = res, args
        _lib = L
    return _lib


def status_str(code: int) -> str:
    try:
        return lib().fi_status_str(code).decode()
    except Exception:
        return "unknown"


def _check(rc: int, where: str):
    if rc != FI_OK:
        detail = lib().fi_last_cuda_error().decode() if rc == FI_E_CUDA else ""
        raise FIError(rc, where, detail)


def _stream() -> int:
    return torch.cuda.current_stream().cuda_stream


def _p(t: torch.Tensor | None) -> int | None:
    return None if t is None else t.data_ptr()


def _to_dev(a: np.ndarray, device) -> torch.Tensor:
    b = np.ascontiguousarray(a).view(np.uint8).reshape(-1)
    if b.size == 0:
        return torch.empty(16, dtype=torch.uint8, device=device)
    return torch.from_numpy(b.copy()).to(device, non_blocking=False)


class DeviceStatus:
    """The caller-owned device word that kernels OR error bits into."""

    def __init__(self, device):
        self.t = torch.zeros(1, dtype=torch.int32, device=device)

    @property
    def ptr(self):
        return self.t.data_ptr()

    def check(self, where: str):
        v = int(self.t.item()) & 0xFFFFFFFF
        if v:
            code = (v & -v).bit_length() - 1
            raise FIError(code, where, f"device status bits {v:#x}")


class DeviceProgram:
    """A program (fi_inputs.Program) resident on the GPU, plus its fi_program struct."""

    def __init__(self, prog, device="cuda", host: dict | None = None):
        """host: optional pinned uint8 CPU tensors keyed code/kernels/instances/
        cbank/buffers/init_image (asynchronous H2D copies from pinned memory)."""
        self.prog = prog
        self.device = torch.device(device)

        def up(key, arr):
            if host is not None and host[key].numel():
                return host[key].to(self.device, non_blocking=True)
            return _to_dev(arr, self.device)
        self.code = up("code", prog.code)
        self.kern = up("kernels", prog.kernels)
        self.inst = up("instances", prog.instances)
        self.cbank = up("cbank", prog.cbank)
        self.buf = up("buffers", prog.buffers)
        self.init_image = up("init_image", prog.init_image)
        self.aux = torch.empty(lib().fi_program_aux_bytes(prog.image_bytes, len(prog.code), len(prog.instances)),
                               dtype=torch.uint8,
                               device=self.device)
        self._code_host = np.ascontiguousarray(prog.code)
        self._inst_host = np.ascontiguousarray(prog.instances)
        self._kern_host = np.ascontiguousarray(prog.kernels)
        self._jit = {}
        self.n_regs = int(lib().fi_program_regs(self._code_host.ctypes.data, len(self._code_host)))
        self.c = fi_program(
            _p(self.code), len(prog.code), _p(self.kern), len(prog.kernels), _p(self.inst), len(prog.instances),
            _p(self.cbank), len(prog.cbank), _p(self.buf), len(prog.buffers), _p(self.aux),
            prog.image_bytes, prog.n_warps, self.n_regs, self._code_host.ctypes.data, self._inst_host.ctypes.data)
        _check(lib().fi_program_prepare(C.byref(self.c), _p(self.aux), _stream()), "fi_program_prepare")

    @property
    def n_inst(self):
        return len(self.prog.instances)

    def jit(self, modes: int = FI_JIT_INJECT) -> "Jit":
        """The program's JIT-specialised emulator module (fi_jit_build) holding
        `modes` — any module already built with a superset is reused; else one is
        built and cached per (code, kernel table, register rows, modes, device)."""
        for m, j in self._jit.items():
            if m & modes == modes:
                return j
        import hashlib
        base = (hashlib.sha1(self._code_host.tobytes() + self._kern_host.tobytes()).hexdigest(), self.n_regs,
                self.device.index if self.device.index is not None else torch.cuda.current_device())
        for (b, m), j in _JIT_CACHE.items():
            if b == base and m & modes == modes:
                self._jit[m] = j
                return j
        j = Jit(self, modes)
        _JIT_CACHE[(base, modes)] = j
        self._jit[modes] = j
        return j

    @property
    def n_warps(self):
        return self.prog.n_warps


_JIT_CACHE: dict = {}


class Jit:
    """fi_jit_build: per-program generated CUDA, NVRTC-compiled for sm_100a."""

    def __init__(self, dp: "DeviceProgram", modes: int = FI_JIT_INJECT):
        h = C.c_void_p()
        rc = lib().fi_jit_build(C.byref(dp.c), dp._kern_host.ctypes.data, modes, C.byref(h))
        if rc != FI_OK:
            raise FIError(rc, "fi_jit_build", lib().fi_jit_log().decode()[-4000:])
        self.h = h
        self.compile_seconds = float(lib().fi_jit_compile_seconds(h))

    def __del__(self):
        try:
            if self.h:
                lib().fi_jit_free(self.h)
                self.h = None
        except Exception:
            pass


def jit_source(prog, modes: int = FI_JIT_INJECT, n_regs: int | None = None) -> str:
    code, kern = np.ascontiguousarray(prog.code), np.ascontiguousarray(prog.kernels)
    nr = n_regs or int(lib().fi_program_regs(code.ctypes.data, len(code)))
    n = lib().fi_jit_source(code.ctypes.data, len(code), kern.ctypes.data, len(kern), nr, modes, None, 0)
    buf = C.create_string_buffer(n)
    lib().fi_jit_source(code.ctypes.data, len(code), kern.ctypes.data, len(kern), nr, modes, buf, n)
    return buf.value.decode()


def jit_compile_check(prog, modes: int = FI_JIT_INJECT) -> int:
    """NVRTC-compile the program's generated emulator without loading it (no GPU); returns cubin bytes."""
    code, kern = np.ascontiguousarray(prog.code), np.ascontiguousarray(prog.kernels)
    nr = int(lib().fi_program_regs(code.ctypes.data, len(code)))
    cb = C.c_size_t(0)
    rc = lib().fi_jit_compile_check(code.ctypes.data, len(code), kern.ctypes.data, len(kern), nr, modes, C.byref(cb))
    if rc != FI_OK:
        raise FIError(rc, "fi_jit_compile_check", lib().fi_jit_log().decode()[-4000:])
    return int(cb.value)


@dataclass
class GoldenTrace:
    dp: DeviceProgram
    image: torch.Tensor          # golden final image (u8)
    warp_len: torch.Tensor
    warp_off: torch.Tensor       # [W+1] u64 (int64 tensor)
    gstore_off: torch.Tensor
    rec: torch.Tensor            # [R*16] u8
    gstore: torch.Tensor
    n_rec: int
    n_gstore: int
    c: fi_trace
    ckpt: torch.Tensor | None = None
    ckpt_off: torch.Tensor | None = None
    ckpt_interval: int = 0
    owner: object = None         # _GoldenHandle: keeps fi_golden_run's arrays alive
    shard: tuple = ()            # (rec_begin, rec_end, w_lo, w_hi) of the records / warps pass 2 wrote
    inst_counts: torch.Tensor | None = None    # fi_golden_profile (world 1): [K][8] i64
    chunk_counts: torch.Tensor | None = None   # ... [C][8] i32

    @property
    def n_chunks(self):
        return (self.n_rec + FI_CHUNK - 1) // FI_CHUNK


def scan_u64(x: torch.Tensor) -> torch.Tensor:
    n = x.numel()
    out = torch.empty(n + 1, dtype=torch.int64, device=x.device)
    ws_n = lib().fi_scan_u64_workspace(n)
    ws = torch.empty(max(ws_n, 1), dtype=torch.uint8, device=x.device)
    _check(lib().fi_scan_u64(_p(x), _p(out), n, _p(ws), ws_n, _stream()), "fi_scan_u64")
    return out


class _GoldenHandle:
    """Owns an fi_golden (the trace arrays fi_golden_run allocated)."""

    def __init__(self, h: C.c_void_p):
        self.h = h

    def __del__(self):
        try:
            if self.h:
                lib().fi_golden_free(self.h, None)
                self.h = None
        except Exception:
            pass


def golden_run(dp: DeviceProgram, ckpt_interval: int | str = "auto", ckpt_budget_frac: float = 0.2,
               engine: str = "jit", rank: int = 0, world: int = 1) -> GoldenTrace:
    """fi_golden_run (one C-ABI call): pass 1 (lengths) -> scans + checkpoint
    layout -> pass 2 (trace records, golden store log, checkpoints).

    ckpt_interval: steps between golden register-file checkpoints (0 = none);
    "auto" = 8192 (a replica restarts from the checkpoint at or
    before its site), doubled until the checkpoints fit ckpt_budget_frac of free HBM.
    engine: "jit" (the golden passes on the program's JIT module built with
    FI_JIT_GOLDEN) or "interp" (emu.cuh): bit-identical results.  The trace
    arrays are owned by the returned GoldenTrace (freed with it).
    world > 1 (single-launch program, JIT): fi_golden_run_shard — pass 2 of rank
    `rank`'s record shard only (GoldenTrace.shard = (rec_begin, rec_end, w_lo, w_hi));
    the image then holds that rank's warps' golden stores only."""
    jit = dp.jit(FI_JIT_GOLDEN) if engine == "jit" else None
    if engine not in ("jit", "interp"):
        raise ValueError(engine)
    image = dp.init_image.clone()
    W = dp.n_warps
    h = C.c_void_p()
    ci = FI_CKPT_AUTO if ckpt_interval == "auto" else int(ckpt_interval)
    if world > 1:
        if jit is None:
            raise ValueError("the owner-computes golden run needs the JIT engine")
        _check(lib().fi_golden_run_shard(C.byref(dp.c), jit.h, _p(image), ci, float(ckpt_budget_frac), rank, world,
                                         C.byref(h), _stream()), "fi_golden_run_shard")
    else:
        _check(lib().fi_golden_run(C.byref(dp.c), jit.h if jit is not None else None, _p(image), ci,
                                   float(ckpt_budget_frac), C.byref(h), _stream()), "fi_golden_run")
    owner = _GoldenHandle(h)
    sh = (C.c_uint64(), C.c_uint64(), C.c_uint32(), C.c_uint32())
    lib().fi_golden_shard_range(h, *(C.byref(x) for x in sh))
    tc = fi_trace.from_buffer_copy(lib().fi_golden_trace_of(h).contents)
    d = dp.device
    n_rec, n_gst = int(tc.n_rec), int(lib().fi_golden_gstore_off_host(h)[W])
    rec = device_view(tc.rec, max(n_rec, 1) * 16, 1, d)
    gst = device_view(tc.gstore, max(n_gst, 1) * 16, 1, d)
    woff = device_view(tc.warp_off, W + 1, 8, d)
    goff = device_view(tc.gstore_off, W + 1, 8, d)
    wl = device_view(lib().fi_golden_warp_len(h), W, 8, d)
    ck = ckoff = None
    if tc.ckpt:
        ckoff = device_view(tc.ckpt_off, W + 1, 8, d)
        n_ck = int(ckoff[W].item())
        ck = device_view(tc.ckpt, max(n_ck * lib().fi_ckpt_bytes(dp.n_regs), 16), 1, d)
    ic = cc = None
    pi, pc = C.c_void_p(), C.c_void_p()
    if lib().fi_golden_profile(h, C.byref(pi), C.byref(pc)) == FI_OK:
        ic = device_view(pi.value, max(dp.n_inst, 1) * 8, 8, d).view(max(dp.n_inst, 1), 8)
        cc = device_view(pc.value, max((n_rec + FI_CHUNK - 1) // FI_CHUNK, 1) * 8, 4, d).view(-1, 8)
    return GoldenTrace(dp, image, wl, woff, goff, rec, gst, n_rec, n_gst, tc, ck, ckoff, int(tc.ckpt_interval),
                       owner, tuple(int(x.value) for x in sh), ic, cc)


def golden_profile(gt: GoldenTrace):
    """fi_golden_profile: the golden run's own profile (inst_counts [K][8] i64,
    chunk_counts [C][8] i32) — fused into pass 2 on the JIT engine, K1 on the
    interpreter; what profile(gt) computes over the whole trace.  Views of
    arrays the GoldenTrace owns."""
    if gt.inst_counts is None:
        raise FIError(FI_E_ARG, "fi_golden_profile", "no whole-trace profile (owner-computes shard)")
    return gt.inst_counts, gt.chunk_counts


def profile(gt: GoldenTrace, rec_begin: int = 0, rec_end: int | None = None,
            inst_counts: torch.Tensor | None = None, chunk_counts: torch.Tensor | None = None):
    """fi_profile (K1) over records [rec_begin, rec_end)."""
    rec_end = gt.n_rec if rec_end is None else rec_end
    K = gt.dp.n_inst
    if inst_counts is None:
        inst_counts = torch.empty((K, 8), dtype=torch.int64, device=gt.dp.device)
    if chunk_counts is None:
        chunk_counts = torch.zeros((max(gt.n_chunks, 1), 8), dtype=torch.int32, device=gt.dp.device)
    _check(lib().fi_profile(C.byref(gt.c), rec_begin, rec_end, K, _p(inst_counts), _p(chunk_counts), _stream()),
           "fi_profile")
    return inst_counts, chunk_counts


class PeerExchange:
    """The buffers of fi_profile_peers for one rank: this rank's
    chunk_counts [C][8] u32, partials [G][K][8] u64 and flag, allocated shareable
    (fi_ipc_alloc), their handles exchanged through torch.distributed
    (all_gather_object), every peer's mapped here (fi_ipc_open)."""

    def __init__(self, n_chunks: int, n_inst: int, rank: int, world: int, device, group=None):
        import torch.distributed as dist
        assert 1 <= world <= FI_MAX_PEERS
        self.world, self.rank, self.n_inst, self.device = world, rank, n_inst, torch.device(device)
        self.epoch = 0
        sizes = (max(n_chunks, 1) * 8 * 4, world * max(n_inst, 1) * 8 * 8, 256)
        self.own, handles = [], []
        for b in sizes:
            ptr, h = C.c_void_p(), C.create_string_buffer(64)
            _check(lib().fi_ipc_alloc(b, C.byref(ptr), h), "fi_ipc_alloc")
            self.own.append(ptr.value)
            handles.append(h.raw)
        allh = [None] * world
        dist.all_gather_object(allh, handles, group=group)
        self.opened = []
        self.peers = fi_peers()
        self.peers.world, self.peers.rank = world, rank
        for r in range(world):
            for q, arr in enumerate((self.peers.chunk_counts, self.peers.partials, self.peers.flags)):
                if r == rank:
                    arr[r] = self.own[q]
                else:
                    ptr = C.c_void_p()
                    _check(lib().fi_ipc_open(C.create_string_buffer(allh[r][q], 64), C.byref(ptr)), "fi_ipc_open")
                    self.opened.append(ptr.value)
                    arr[r] = ptr.value
        self.part_local = torch.empty((max(n_inst, 1), 8), dtype=torch.int64, device=self.device)
        self.chunk_counts = torch.zeros((max(n_chunks, 1), 8), dtype=torch.int32, device=self.device)

    def profile(self, gt: "GoldenTrace", rec_begin: int, rec_end: int, inst_counts: torch.Tensor,
                status: "DeviceStatus | None" = None) -> None:
        """One epoch; a peer that never signals sets FI_E_COLLECTIVE in `status`
        (checked here when no status is given)."""
        self.epoch += 1
        st = status or DeviceStatus(self.device)
        _check(lib().fi_profile_peers(C.byref(gt.c), rec_begin, rec_end, gt.dp.n_inst, C.byref(self.peers),
                                      _p(self.part_local), self.epoch, _p(inst_counts), _p(self.chunk_counts),
                                      st.ptr, _stream()), "fi_profile_peers")
        if status is None:
            st.check("fi_profile_peers")

    def close(self, group=None):
        """Unmap the peers' buffers, wait for every rank to have done the same, then
        free this rank's (collective: every rank calls it)."""
        import torch.distributed as dist
        torch.cuda.synchronize(self.device)
        for p in self.opened:
            lib().fi_ipc_close(p)
        self.opened = []
        if dist.is_available() and dist.is_initialized():
            dist.barrier(group=group)
        for p in self.own:
            lib().fi_ipc_free(p)
        self.own = []


class SiteIndex:
    """fi_build_site_index (K2): P_k and 64-chunk-tile prefix sums; totals N_g."""

    def __init__(self, gt: GoldenTrace, inst_counts: torch.Tensor, chunk_counts: torch.Tensor,
                 status: DeviceStatus | None = None):
        self.gt = gt
        self.chunk_counts = chunk_counts
        self.n_inst = gt.dp.n_inst
        self.n_chunks = gt.n_chunks
        nb = lib().fi_site_index_bytes(self.n_inst, self.n_chunks)
        self.buf = torch.empty(nb, dtype=torch.uint8, device=gt.dp.device)
        st = status or DeviceStatus(gt.dp.device)
        _check(lib().fi_build_site_index(_p(inst_counts), self.n_inst, _p(chunk_counts), self.n_chunks,
                                         _p(self.buf), st.ptr, _stream()), "fi_build_site_index")
        tot = (C.c_uint64 * 8)()
        _check(lib().fi_site_totals(_p(self.buf), self.n_inst, tot, _stream()), "fi_site_totals")
        self.totals = [int(x) for x in tot]
        self._tot = tot
        if status is None:
            st.check("fi_build_site_index")      # totals already synchronized the stream

    def prefix_inst(self) -> torch.Tensor:
        return self.buf[: (self.n_inst + 1) * 64].view(torch.int64).view(self.n_inst + 1, 8)


def schedule(seed: int, groups, bfms) -> fi_schedule:
    s = fi_schedule()
    s.seed = seed
    s.n_groups, s.n_bfms = len(groups), len(bfms)
    for i, g in enumerate(groups):
        s.groups[i] = g
    for i, b in enumerate(bfms):
        s.bfms[i] = b
    return s


def select_sites(idx: SiteIndex, sched: fi_schedule, j0: int, n: int, sites: torch.Tensor | None = None,
                 status: DeviceStatus | None = None) -> torch.Tensor:
    """fi_select_sites (K3): returns a [n*64] u8 tensor of fi_site."""
    gt = idx.gt
    if sites is None:
        sites = torch.empty(max(n, 1) * 64, dtype=torch.uint8, device=gt.dp.device)
    st = status or DeviceStatus(gt.dp.device)
    _check(lib().fi_select_sites(C.byref(gt.dp.c), C.byref(gt.c), _p(idx.chunk_counts), _p(idx.buf), idx.n_inst,
                                 idx.n_chunks,
                                 idx._tot, C.byref(sched), j0, n, _p(sites), st.ptr, _stream()), "fi_select_sites")
    if status is None:
        st.check("fi_select_sites")
    return sites


def inject(gt: GoldenTrace, sites: torch.Tensor, n: int, log_cap: int, out: torch.Tensor | None = None,
           log: torch.Tensor | None = None, status: DeviceStatus | None = None, ws: torch.Tensor | None = None,
           engine: str = "jit"):
    """fi_inject (K4).  engine "jit": fi_inject_jit on the program's generated
    emulator (built on first use); "interp": fi_inject (the shared-memory
    interpreter).  Both give bit-identical results."""
    dev = gt.dp.device
    if out is None:
        out = torch.empty(max(n, 1) * 24, dtype=torch.uint8, device=dev)
    if log is None:
        log = torch.empty(max(n * log_cap, 1) * 16, dtype=torch.uint8, device=dev)
    st = status or DeviceStatus(dev)
    ws_n = lib().fi_inject_workspace(n)
    if ws is None or ws.numel() < ws_n:
        ws = torch.empty(ws_n, dtype=torch.uint8, device=dev)
    if engine == "jit":
        _check(lib().fi_inject_jit(gt.dp.jit(FI_JIT_INJECT).h, C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c), _p(sites), n, _p(out),
                                   _p(log), log_cap, _p(ws), ws_n, st.ptr, _stream()), "fi_inject_jit")
    elif engine == "interp":
        _check(lib().fi_inject(C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c), _p(sites), n, _p(out), _p(log), log_cap,
                               _p(ws), ws_n, st.ptr, _stream()), "fi_inject")
    else:
        raise ValueError(engine)
    if status is None:
        st.check("fi_inject")
    return out, log


def classify(gt: GoldenTrace, sites: torch.Tensor, n: int, out: torch.Tensor, log: torch.Tensor, log_cap: int,
             hist: torch.Tensor | None = None, status: DeviceStatus | None = None,
             unchecked: bool = False, ws: torch.Tensor | None = None, rtol: float = 0.0,
             hist_tol: torch.Tensor | None = None) -> torch.Tensor:
    """fi_classify (K5/K7): fills out[].outcome, accumulates hist[8][4][3].
    unchecked=True: potential-DUE semantics (FI_UNCHECKED, row f4).  rtol > 0:
    also the C-12 secondary numeric classification (FI_SDC_WITHIN_TOL in
    out[].flags; hist_tol [8][4][3] accumulated when given)."""
    dev = gt.dp.device
    if hist is None:
        hist = torch.zeros((8, 4, 3), dtype=torch.int64, device=dev)
    st = status or DeviceStatus(dev)
    ws_n = lib().fi_classify_workspace(gt.dp.n_inst, n, log_cap)
    if ws_n and (ws is None or ws.numel() < ws_n):
        ws = torch.empty(ws_n, dtype=torch.uint8, device=dev)
    _check(lib().fi_classify(C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c), _p(sites), n, _p(out), _p(log), log_cap,
                             _p(hist), FI_UNCHECKED if unchecked else 0, float(rtol), _p(hist_tol),
                             _p(ws) if ws_n else None, ws_n, st.ptr, _stream()), "fi_classify")
    if status is None:
        st.check("fi_classify")
    return hist


def profile_opcodes(gt: GoldenTrace, rec_begin: int = 0, rec_end: int | None = None) -> torch.Tensor:
    """fi_profile_opcodes (row f1): per-instance, per-opcode thread-level counts [K][32]."""
    rec_end = gt.n_rec if rec_end is None else rec_end
    out = torch.empty((max(gt.dp.n_inst, 1), FI_NOPS), dtype=torch.int64, device=gt.dp.device)
    _check(lib().fi_profile_opcodes(C.byref(gt.c), rec_begin, rec_end, gt.dp.n_inst, _p(out), _stream()),
           "fi_profile_opcodes")
    return out


def profile_approx(gt: GoldenTrace) -> torch.Tensor:
    """fi_profile_approx (row f1): counts of each static kernel's first instance reused."""
    dp = gt.dp
    out = torch.empty((max(dp.n_inst, 1), 8), dtype=torch.int64, device=dp.device)
    ws_n = lib().fi_profile_approx_workspace(len(dp.prog.kernels), dp.n_inst)
    ws = torch.empty(ws_n, dtype=torch.uint8, device=dp.device)
    _check(lib().fi_profile_approx(C.byref(dp.c), C.byref(gt.c), _p(out), _p(ws), ws_n, _stream()), "fi_profile_approx")
    return out


class InstanceIndex:
    """fi_build_instance_index: P_k only (e.g. over approximate counts) + totals."""

    def __init__(self, gt: GoldenTrace, inst_counts: torch.Tensor, status: DeviceStatus | None = None):
        self.gt = gt
        self.n_inst = gt.dp.n_inst
        nb = lib().fi_site_index_bytes(self.n_inst, 0)
        self.buf = torch.empty(nb, dtype=torch.uint8, device=gt.dp.device)
        st = status or DeviceStatus(gt.dp.device)
        _check(lib().fi_build_instance_index(_p(inst_counts), self.n_inst, _p(self.buf), st.ptr, _stream()),
               "fi_build_instance_index")
        tot = (C.c_uint64 * 8)()
        _check(lib().fi_site_totals(_p(self.buf), self.n_inst, tot, _stream()), "fi_site_totals")
        self.totals = [int(x) for x in tot]
        self._tot = tot
        if status is None:
            st.check("fi_build_instance_index")


def select_sites_approx(idx: InstanceIndex, sched: fi_schedule, j0: int, n: int,
                        sites: torch.Tensor | None = None, status: DeviceStatus | None = None) -> torch.Tensor:
    """fi_select_sites_approx (row f1)."""
    gt = idx.gt
    if sites is None:
        sites = torch.empty(max(n, 1) * 64, dtype=torch.uint8, device=gt.dp.device)
    st = status or DeviceStatus(gt.dp.device)
    _check(lib().fi_select_sites_approx(C.byref(gt.dp.c), C.byref(gt.c), _p(idx.buf), idx.n_inst, idx._tot,
                                        C.byref(sched), j0, n, _p(sites), st.ptr, _stream()), "fi_select_sites_approx")
    if status is None:
        st.check("fi_select_sites_approx")
    return sites


def pend_capacity(gt: GoldenTrace) -> int:
    """Update slots per replica and launch for K8: 2x the largest launch's golden
    stores + 4096 (faulty extras; exceeding it is reported, never mis-classified)."""
    gs = gt.gstore_off.cpu().numpy()
    wb = gt.dp.prog.instances["warp_begin"].astype(np.int64)
    we = gt.dp.prog.instances["warp_end"].astype(np.int64)
    mx = int((gs[we] - gs[wb]).max()) if len(wb) else 0
    return 2 * mx + 4096


def classify_batched(gt: GoldenTrace, sites: torch.Tensor, n: int, out: torch.Tensor, log: torch.Tensor,
                     log_cap: int, hist: torch.Tensor | None = None, unchecked: bool = False, batch: int | None = None,
                     pool_pages: int | None = None, pend_cap: int | None = None, mem_budget: int = 24 << 30,
                     status: DeviceStatus | None = None, engine: str = "interp", rtol: float = 0.0,
                     hist_tol: torch.Tensor | None = None, steps_out: list | None = None) -> torch.Tensor:
    """fi_classify_batched (K8): whole-program outcomes for long multi-instance
    programs, replica batches in lockstep over the launches.  engine "jit":
    fi_classify_batched_jit (re-execution on the program's JIT module).
    rtol / hist_tol: the C-12 secondary numeric classification, as classify().
    steps_out (engine "jit"): appended with the emulated warp-steps of the
    re-executed warps (the workspace's first 8 bytes, fi.h; synchronises)."""
    dev = gt.dp.device
    if hist is None:
        hist = torch.zeros((8, 4, 3), dtype=torch.int64, device=dev)
    pend_cap = pend_capacity(gt) if pend_cap is None else pend_cap
    if batch is None:                                  # per-slot parts within half the budget
        w1 = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, log_cap, 1, 1, pend_cap)
        w2 = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, log_cap, 2, 1, pend_cap)
        batch = int(max(1, min(n, 512, (mem_budget // 2 - w1) // max(w2 - w1, 1) + 1)))
    if pool_pages is None:                             # the rest of the budget after the fixed parts
        fixed = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, log_cap, batch, 1, pend_cap)
        pool_pages = max(1024, (mem_budget - fixed) // (4096 + 12))
    ws_n = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, log_cap, batch, pool_pages, pend_cap)
    ws = torch.empty(ws_n, dtype=torch.uint8, device=dev)
    st = status or DeviceStatus(dev)
    if engine == "jit":
        _check(lib().fi_classify_batched_jit(gt.dp.jit(FI_JIT_PAGE).h, C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c),
                                             _p(sites), n, _p(out), _p(log), log_cap, _p(hist),
                                             FI_UNCHECKED if unchecked else 0, float(rtol), _p(hist_tol), batch,
                                             pool_pages, pend_cap, _p(ws), ws_n, st.ptr, _stream()),
               "fi_classify_batched_jit")
        if steps_out is not None:
            steps_out.append(int(ws[:8].view(torch.int64).item()))
    else:
        _check(lib().fi_classify_batched(C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c), _p(sites), n, _p(out),
                                         _p(log), log_cap, _p(hist), FI_UNCHECKED if unchecked else 0, float(rtol),
                                         _p(hist_tol), batch, pool_pages, pend_cap, _p(ws), ws_n, st.ptr, _stream()),
               "fi_classify_batched")
    if status is None:
        st.check("fi_classify_batched")
    return hist


def inject_permanent_batched(gt: GoldenTrace, faults: np.ndarray, op_weights: torch.Tensor | None = None,
                             unchecked: bool = False, batch: int | None = None, pool_pages: int | None = None,
                             pend_cap: int | None = None, mem_budget: int = 24 << 30):
    """fi_inject_permanent_batched (rows f2/f3 on K8).  Returns (inj [n*24] u8, weighted hist [3] i64)."""
    dev = gt.dp.device
    f = np.ascontiguousarray(faults, dtype=PFAULT_DTYPE)
    n = len(f)
    ft = torch.from_numpy(f.view(np.uint8).copy()).to(dev)
    out = torch.zeros(max(n, 1) * 24, dtype=torch.uint8, device=dev)
    hist = torch.zeros(3, dtype=torch.int64, device=dev)
    cap = log_capacity(gt)
    pend_cap = pend_capacity(gt) if pend_cap is None else pend_cap
    if batch is None:
        w1 = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, cap, 1, 1, pend_cap)
        w2 = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, cap, 2, 1, pend_cap)
        batch = int(max(1, min(n, 512, (mem_budget // 2 - w1) // max(w2 - w1, 1) + 1)))
    if pool_pages is None:
        fixed = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, cap, batch, 1, pend_cap)
        pool_pages = max(1024, (mem_budget - fixed) // (4096 + 12))
    ws_n = lib().fi_classify_batched_workspace(C.byref(gt.dp.c), n, cap, batch, pool_pages, pend_cap)
    ws = torch.empty(ws_n, dtype=torch.uint8, device=dev)
    st = DeviceStatus(dev)
    _check(lib().fi_inject_permanent_batched(C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c), _p(ft), n,
                                             _p(op_weights), _p(out), cap, _p(hist),
                                             FI_UNCHECKED if unchecked else 0, batch, pool_pages, pend_cap, _p(ws),
                                             ws_n, st.ptr, _stream()), "fi_inject_permanent_batched")
    st.check("fi_inject_permanent_batched")
    return out, hist


def inject_permanent(gt: GoldenTrace, faults: np.ndarray, op_weights: torch.Tensor | None = None,
                     unchecked: bool = False, log_cap: int | None = None, ov_words: int | None = None,
                     max_slots: int = 0):
    """fi_inject_permanent (rows f2/f3).  Returns (inj [n*24] u8, weighted hist [3] i64).
    ov_words defaults to every word of the image (a permanent fault may corrupt them all)."""
    dev = gt.dp.device
    f = np.ascontiguousarray(faults, dtype=PFAULT_DTYPE)
    n = len(f)
    cap = log_capacity(gt) if log_cap is None else log_cap
    ft = torch.from_numpy(f.view(np.uint8).copy()).to(dev)
    out = torch.zeros(max(n, 1) * 24, dtype=torch.uint8, device=dev)
    log = torch.empty(max(n * cap, 1) * 16, dtype=torch.uint8, device=dev)
    hist = torch.zeros(3, dtype=torch.int64, device=dev)
    ovw = gt.dp.prog.image_bytes // 4 if ov_words is None else ov_words
    ws_n = lib().fi_inject_permanent_workspace(n, cap, ovw, max_slots)
    if not max_slots:                                 # keep the overlays within 16 GiB of HBM
        ms = 2368
        while ws_n > 16 << 30 and ms > 4:
            ms //= 2
            ws_n = lib().fi_inject_permanent_workspace(n, cap, ovw, ms)
    ws = torch.empty(ws_n, dtype=torch.uint8, device=dev)
    st = DeviceStatus(dev)
    _check(lib().fi_inject_permanent(C.byref(gt.dp.c), _p(gt.image), C.byref(gt.c), _p(ft), n, _p(op_weights),
                                     _p(out), _p(log), cap, ovw, _p(hist), FI_UNCHECKED if unchecked else 0, _p(ws), ws_n,
                                     st.ptr, _stream()), "fi_inject_permanent")
    st.check("fi_inject_permanent")
    return out, hist


def write_params_txt(site_row: np.ndarray, kernel_name: str) -> str:
    a = np.ascontiguousarray(np.asarray(site_row, dtype=SITE_DTYPE).reshape(1))
    buf = C.create_string_buffer(1024)
    _check(lib().fi_write_params_txt(a.ctypes.data, kernel_name.encode(), buf, 1024), "fi_write_params_txt")
    return buf.value.decode()


def write_profile_txt(inst_counts: np.ndarray, prog) -> str:
    """fi_write_profile_txt: PAPER.md:78's profile, one line per dynamic kernel."""
    ic = np.ascontiguousarray(inst_counts, dtype=np.uint64)
    inst = np.ascontiguousarray(prog.instances)
    names = [n.encode() for n in prog.kernel_names]
    arr = (C.c_char_p * max(len(names), 1))(*names)
    need = C.c_size_t(0)
    _check(lib().fi_write_profile_txt(ic.ctypes.data, inst.ctypes.data, len(inst), arr, len(names), None, 0,
                                      C.byref(need)), "fi_write_profile_txt")
    buf = C.create_string_buffer(need.value)
    _check(lib().fi_write_profile_txt(ic.ctypes.data, inst.ctypes.data, len(inst), arr, len(names), buf, need.value,
                                      None), "fi_write_profile_txt")
    return buf.value.decode()


class _DevArray:
    """A device pointer seen through __cuda_array_interface__ (zero-copy into torch)."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False), "version": 3,
                                         "strides": None, "stream": None}


def device_view(ptr: int, n: int, elem_bytes: int, device) -> torch.Tensor:
    return torch.as_tensor(_DevArray(ptr, n, {8: "<i8", 4: "<i4", 1: "|u1"}[elem_bytes]), device=device)


def torch_allreduce(group=None):
    """An fi_allreduce_fn over torch.distributed (NCCL on the GPU box): in-place
    SUM of the device integers, ordered on fi_campaign's stream."""
    import torch.distributed as dist

    def cb(dev, count, elem_bytes, ctx, stream):
        try:
            d = torch.device("cuda", torch.cuda.current_device())
            t = device_view(dev, count, elem_bytes, d)
            with torch.cuda.stream(torch.cuda.ExternalStream(stream, device=d)):
                dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
            return 0
        except Exception as e:                          # never raise across the C ABI
            import sys
            print(f"fi allreduce callback failed: {e!r}", file=sys.stderr)
            return 1
    return ALLREDUCE_FN(cb)


@dataclass
class CampaignResult:
    hist: np.ndarray             # [8][4][3] u64, all ranks
    totals: list
    n_rec: int
    counted: int
    j0: int
    n_local: int
    rec_range: tuple
    n_unclassified: int
    n_not_injected: int
    ms: dict
    sites: np.ndarray | None
    inj: np.ndarray | None
    inst_counts: np.ndarray | None
    hist_tol: np.ndarray | None = None   # rtol > 0: C-12 secondary histogram [8][4][3]
    j: np.ndarray | None = None          # the replica index of each returned row


def campaign(prog, seed: int, groups, bfms, n_replicas: int, rank: int = 0, world: int = 1, allreduce=None,
             unchecked: bool = False, propagation: str = "auto", approximate: bool = False, ckpt="auto",
             k8_mem_budget: int = 0, device: int | None = None, host: dict | None = None,
             return_arrays: bool = True, engine: str = "jit", rtol: float = 0.0,
             owner_computes: bool = False) -> CampaignResult:
    """fi_campaign: the whole campaign of this rank from HOST arrays (golden run,
    sharded profile, count exchange, index, select, inject, classify, histogram
    exchange, D2H).  `host`: optional pinned uint8 tensors keyed code / kernels /
    instances / cbank / buffers / init_image (else the numpy arrays are used).
    allreduce: an ALLREDUCE_FN (torch_allreduce() by default when world > 1)."""
    arrs = {k: np.ascontiguousarray(getattr(prog, k)) for k in
            ("code", "kernels", "instances", "cbank", "buffers", "init_image")}

    def hp(k):
        if host is not None and host[k].numel():
            return host[k].data_ptr()
        return arrs[k].ctypes.data if arrs[k].size else None
    cfg = fi_campaign_cfg()
    cfg.code, cfg.n_code = hp("code"), len(arrs["code"])
    cfg.kern, cfg.n_kern = hp("kernels"), len(arrs["kernels"])
    cfg.inst, cfg.n_inst = hp("instances"), len(arrs["instances"])
    cfg.cbank, cfg.n_cbank = hp("cbank"), len(arrs["cbank"])
    cfg.buf, cfg.n_buf = hp("buffers"), len(arrs["buffers"])
    cfg.init_image, cfg.image_bytes = hp("init_image"), prog.image_bytes
    cfg.n_warps = prog.n_warps
    cfg.sched = schedule(seed, groups, bfms)
    cfg.n_replicas = n_replicas
    cfg.flags = FI_UNCHECKED if unchecked else 0
    cfg.propagation = FI_PROPAGATION[propagation]
    cfg.approximate = 1 if approximate else 0
    cfg.ckpt_interval = FI_CKPT_AUTO if ckpt == "auto" else int(ckpt)
    cfg.engine = {"interp": 0, "jit": 1}[engine]
    cfg.k8_mem_budget = k8_mem_budget
    cfg.rtol = float(rtol)
    cfg.owner_computes = 1 if owner_computes else 0
    cfg.device = torch.cuda.current_device() if device is None else device
    cfg.stream = torch.cuda.current_stream(cfg.device).cuda_stream or None
    # rows this rank may return: its replica block, or (owner-computes) any replica
    n_loc = n_replicas if (owner_computes and world > 1) else \
        n_replicas * (rank + 1) // world - n_replicas * rank // world
    res = fi_campaign_result()
    sites = inj = ic = jj = None
    if return_arrays:
        sites = np.zeros(max(n_loc, 1), dtype=SITE_DTYPE)
        inj = np.zeros(max(n_loc, 1), dtype=INJ_DTYPE)
        ic = np.zeros((max(len(prog.instances), 1), 8), dtype=np.uint64)
        jj = np.zeros(max(n_loc, 1), dtype=np.uint64)
        res.sites, res.inj, res.inst_counts, res.j = sites.ctypes.data, inj.ctypes.data, ic.ctypes.data, jj.ctypes.data
    if world > 1 and allreduce is None:
        allreduce = torch_allreduce()
    cb = allreduce if allreduce is not None else ALLREDUCE_FN()
    _check(lib().fi_campaign(C.byref(cfg), rank, world, cb, None, C.byref(res)), "fi_campaign")
    ms = {k: float(getattr(res, "ms_" + k)) for k in
          ("h2d", "golden", "profile", "exchange", "index", "select", "inject", "classify", "d2h", "jit")}
    return CampaignResult(np.array(res.hist, dtype=np.uint64).reshape(8, 4, 3), [int(x) for x in res.totals],
                          int(res.n_rec), int(res.counted), int(res.j0), int(res.n_local),
                          (int(res.rec_begin), int(res.rec_end)), int(res.n_unclassified), int(res.n_not_injected),
                          ms, None if sites is None else sites[:res.n_local], None if inj is None else inj[:res.n_local],
                          ic, np.array(res.hist_tol, dtype=np.uint64).reshape(8, 4, 3) if rtol > 0 else None,
                          None if jj is None else jj[:res.n_local])


def shard_warps(warp_off: np.ndarray, rank: int, world: int) -> dict:
    """fi_shard_warps (host): the owner-computes partition of rank `rank` of `world`."""
    wo = np.ascontiguousarray(warp_off, dtype=np.uint64)
    r0, r1 = C.c_uint64(), C.c_uint64()
    wa, wb, oa, ob = C.c_uint32(), C.c_uint32(), C.c_uint32(), C.c_uint32()
    _check(lib().fi_shard_warps(wo.ctypes.data, len(wo) - 1, rank, world, C.byref(r0), C.byref(r1), C.byref(wa),
                                C.byref(wb), C.byref(oa), C.byref(ob)), "fi_shard_warps")
    return dict(rec=(r0.value, r1.value), run=(wa.value, wb.value), own=(oa.value, ob.value))


def campaign_release_memory(device: int = -1) -> None:
    """fi_campaign_release_memory: give back the device memory fi_campaign keeps
    reserved in the device's default pool between calls."""
    _check(lib().fi_campaign_release_memory(device), "fi_campaign_release_memory")


def as_numpy(t: torch.Tensor, dtype: np.dtype, n: int | None = None) -> np.ndarray:
    a = t.detach().cpu().numpy().view(np.uint8).reshape(-1).view(dtype)
    return a if n is None else a[:n]


def log_capacity(gt: GoldenTrace) -> int:
    """Per-replica faulty-store log slots: 2x the largest golden per-warp store
    count + 4096 (replicas that exceed it are flagged, never mis-classified)."""
    gs = gt.gstore_off
    mx = int((gs[1:] - gs[:-1]).max().item()) if gt.dp.n_warps else 0
    return 2 * mx + 4096
