"""CPU ORACLE — test infrastructure only.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_dsn_0002hsvk21_b200``) never imports it and shares no code with it.

This module is a thin ctypes wrapper around ``oracle/liboracle.so`` (built from
oracle.cpp with ``-O2 -ffp-contract=off``), plus the confidence-interval formula
of PAPER.md:214 (§IV-B), which is plain arithmetic kept here in Python.

Parity status: every function is pinned by tests/test_oracle_*.py
except the outcome *fractions* of whole campaigns, which the paper does not fix
for synthetic programs ("parity unpinned": the paper's 32.5/4.2/63.3 % needs
SpecACCEL).
"""
from __future__ import annotations

import ctypes as C
import math
import os
import subprocess
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "liboracle.so")
SRC = [os.path.join(HERE, "oracle.cpp"), os.path.join(HERE, "oracle.h")]

G_FP64, G_FP32, G_LD, G_PR, G_NODEST, G_OTHERS, G_GPPR, G_GP = range(8)
GROUP_NAMES = ["G_FP64", "G_FP32", "G_LD", "G_PR", "G_NODEST", "G_OTHERS", "G_GPPR", "G_GP"]
MASKED, SDC, DUE, NOT_INJECTED = 0, 1, 2, 3
MODE_FULL, MODE_WARP_LOCAL = 0, 1
UNCHECKED = 0x100          # OR into mode: potential-DUE semantics (row f4)
POTENTIAL_DUE = 1          # inj["flags"] bit
SDC_WITHIN_TOL = 8         # inj["flags"] bit: C-12 secondary numeric mode

RECORD_DTYPE = np.dtype([("instance", "<u4"), ("insn", "<u4"), ("active", "<u4"), ("pred", "<u4")])
SITE_DTYPE = np.dtype([
    ("s", "<u8"), ("instruction_count", "<u8"),
    ("instance", "<u4"), ("kernel_id", "<u4"), ("kernel_count", "<u4"), ("warp", "<u4"),
    ("step", "<u4"), ("thread", "<u4"), ("pc", "<u4"), ("u_dst", "<u4"), ("u_bit", "<u4"), ("mask", "<u4"),
    ("lane", "u1"), ("group", "u1"), ("bfm", "u1"), ("slot", "u1"), ("dst_kind", "u1"), ("dst_reg", "u1"),
    ("n_elig", "u1"), ("flags", "u1"),
])
INJ_DTYPE = np.dtype([("before", "<u4"), ("after", "<u4"), ("mask", "<u4"), ("fault_pc", "<u4"),
                      ("fault_kind", "u1"), ("outcome", "u1"), ("flags", "u1"), ("pad", "u1"),
                      ("n_faulty_stores", "<u4")])
PFAULT_DTYPE = np.dtype([("opcode", "<u4"), ("sm", "<u4"), ("lane", "<u4"), ("mask", "<u4"), ("q32", "<u4"),
                         ("n_sm", "<u4"), ("seed", "<u8")])
assert SITE_DTYPE.itemsize == 64 and INJ_DTYPE.itemsize == 24 and PFAULT_DTYPE.itemsize == 32


class _Program(C.Structure):
    _fields_ = [("code", C.c_void_p), ("n_code", C.c_uint32),
                ("kern", C.c_void_p), ("n_kern", C.c_uint32),
                ("inst", C.c_void_p), ("n_inst", C.c_uint32),
                ("cbank", C.c_void_p), ("n_cbank", C.c_uint32),
                ("buf", C.c_void_p), ("n_buf", C.c_uint32),
                ("init_image", C.c_void_p), ("image_bytes", C.c_uint64)]


_lock = threading.Lock()
_lib = None


def build(force: bool = False) -> str:
    """Compile liboracle.so (plain g++, no GPU).  Building the checker is not using it."""
    stale = not os.path.exists(LIB_PATH) or any(os.path.getmtime(s) > os.path.getmtime(LIB_PATH) for s in SRC)
    if force or stale:
        subprocess.run(["g++", "-O2", "-std=c++17", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
                        "-pthread", "-Wall", "-o", LIB_PATH, SRC[0]], check=True)
    return LIB_PATH


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = C.CDLL(LIB_PATH)
            vp, u32, u64, i32 = C.c_void_p, C.c_uint32, C.c_uint64, C.c_int
            L.orc_golden_run.restype = vp
            L.orc_golden_run.argtypes = [C.POINTER(_Program), i32, i32]
            L.orc_last_error.restype = C.c_char_p
            L.orc_error.restype = C.c_char_p
            L.orc_error.argtypes = [vp]
            L.orc_free.argtypes = [vp]
            L.orc_n_warps.restype = u32
            L.orc_n_warps.argtypes = [vp]
            L.orc_n_records.restype = u64
            L.orc_n_records.argtypes = [vp]
            L.orc_n_golden_stores.restype = u64
            L.orc_n_golden_stores.argtypes = [vp]
            for f in ("orc_counts", "orc_warp_counts", "orc_warp_len", "orc_final_image"):
                getattr(L, f).argtypes = [vp, vp]
            L.orc_trace.argtypes = [vp, vp]
            L.orc_count_warps.restype = u64
            L.orc_count_warps.argtypes = [C.POINTER(_Program), u32, u32, i32, vp]
            L.orc_scan_trace.argtypes = [vp, u64, u32, i32, vp]
            L.orc_select.argtypes = [vp, u64, vp, u32, vp, u32, u64, u32, vp]
            L.orc_locate.argtypes = [vp, i32, vp, u32, vp]
            L.orc_opcode_counts.argtypes = [vp, vp]
            L.orc_approx_counts.argtypes = [vp, vp]
            L.orc_select_approx.argtypes = [vp, u64, vp, u32, vp, u32, u64, u32, vp]
            L.orc_inject.argtypes = [vp, vp, u32, i32, i32, C.c_double, vp]
            L.orc_inject_permanent.argtypes = [vp, vp, u32, i32, i32, vp]
            L.orc_permanent_image.argtypes = [vp, vp, u32, i32, vp]
            L.orc_inject_image.argtypes = [vp, vp, i32, vp]
            L.orc_warp_site_rank.argtypes = [C.POINTER(_Program), u32, i32, u32, u32, C.POINTER(u64), C.POINTER(u64)]
            L.orc_inject_local.argtypes = [C.POINTER(_Program), vp, u32, i32, vp, vp]
            L.orc_warp_site_at.argtypes = [C.POINTER(_Program), u32, i32, u64, C.POINTER(u32), C.POINTER(u32),
                                           C.POINTER(u32)]
            L.orc_philox4x32_10.argtypes = [vp, vp, vp]
            L.orc_draw.argtypes = [u64, u64, u64, C.POINTER(u64), C.POINTER(u32), C.POINTER(u32), C.POINTER(u32)]
            L.orc_mask.restype = u32
            L.orc_mask.argtypes = [i32, u32]
            L.orc_group_mask.restype = u32
            L.orc_group_mask.argtypes = [vp]
            L.orc_dest_slots.restype = u32
            L.orc_dest_slots.argtypes = [vp, i32, vp, vp]
            _lib = L
    return _lib


def _ptr(a: np.ndarray) -> int:
    return a.ctypes.data if a.size else 0


def _cprog(prog) -> tuple[_Program, list]:
    keep = [np.ascontiguousarray(x) for x in (prog.code, prog.kernels, prog.instances, prog.cbank,
                                                prog.buffers, prog.init_image)]
    code, kern, inst, cb, buf, img = keep
    p = _Program(_ptr(code), len(code), _ptr(kern), len(kern), _ptr(inst), len(inst),
                 _ptr(cb), len(cb), _ptr(buf), len(buf), _ptr(img), img.size)
    return p, keep


def n_threads_default() -> int:
    return os.cpu_count() or 1


class Golden:
    """Golden run of a program by the oracle interpreter (PAPER.md:72 step (1)
    profile and the golden output state of step (4))."""

    def __init__(self, prog, keep_trace: bool = True, n_threads: int | None = None):
        self.prog = prog
        self._p, self._keep = _cprog(prog)
        L = lib()
        self.h = L.orc_golden_run(C.byref(self._p), n_threads or n_threads_default(), int(keep_trace))
        if not self.h:
            raise RuntimeError("oracle golden run failed: " + L.orc_last_error().decode())
        self.n_warps = L.orc_n_warps(self.h)
        self.n_records = L.orc_n_records(self.h)
        self.keep_trace = keep_trace

    def __del__(self):
        if getattr(self, "h", None):
            try:
                lib().orc_free(self.h)
            except TypeError:                          # interpreter shutdown: module globals gone
                pass
            self.h = None

    def counts(self) -> np.ndarray:
        out = np.zeros((len(self.prog.instances), 8), dtype=np.uint64)
        lib().orc_counts(self.h, _ptr(out))
        return out

    def warp_counts(self) -> np.ndarray:
        out = np.zeros((self.n_warps, 8), dtype=np.uint64)
        lib().orc_warp_counts(self.h, _ptr(out))
        return out

    def warp_len(self) -> np.ndarray:
        out = np.zeros(self.n_warps, dtype=np.uint64)
        lib().orc_warp_len(self.h, _ptr(out))
        return out

    def final_image(self) -> np.ndarray:
        out = np.zeros(self.prog.image_bytes, dtype=np.uint8)
        lib().orc_final_image(self.h, _ptr(out))
        return out

    def n_golden_stores(self) -> int:
        return int(lib().orc_n_golden_stores(self.h))

    def trace(self) -> np.ndarray:
        out = np.zeros(self.n_records, dtype=RECORD_DTYPE)
        if lib().orc_trace(self.h, _ptr(out)):
            raise RuntimeError("trace not kept")
        return out

    def select(self, seed: int, groups, bfms, j0: int, n: int) -> np.ndarray:
        g = np.asarray(groups, dtype=np.uint8)
        b = np.asarray(bfms, dtype=np.uint8)
        out = np.zeros(n, dtype=SITE_DTYPE)
        rc = lib().orc_select(self.h, seed, _ptr(g), len(g), _ptr(b), len(b), j0, n, _ptr(out))
        if rc:
            raise OracleError(rc, lib().orc_error(self.h).decode())
        return out

    def opcode_counts(self) -> np.ndarray:
        out = np.zeros((len(self.prog.instances), 32), dtype=np.uint64)
        if lib().orc_opcode_counts(self.h, _ptr(out)):
            raise RuntimeError("trace not kept")
        return out

    def approx_counts(self) -> np.ndarray:
        out = np.zeros((len(self.prog.instances), 8), dtype=np.uint64)
        lib().orc_approx_counts(self.h, _ptr(out))
        return out

    def select_approx(self, seed: int, groups, bfms, j0: int, n: int) -> np.ndarray:
        g = np.asarray(groups, dtype=np.uint8)
        b = np.asarray(bfms, dtype=np.uint8)
        out = np.zeros(n, dtype=SITE_DTYPE)
        rc = lib().orc_select_approx(self.h, seed, _ptr(g), len(g), _ptr(b), len(b), j0, n, _ptr(out))
        if rc:
            raise OracleError(rc, lib().orc_error(self.h).decode())
        return out

    def inject_permanent(self, faults: np.ndarray, mode: int = MODE_FULL, n_threads: int | None = None) -> np.ndarray:
        """Rows f2/f3 by the definition: whole-program re-run per fault."""
        faults = np.ascontiguousarray(faults, dtype=PFAULT_DTYPE)
        out = np.zeros(len(faults), dtype=INJ_DTYPE)
        lib().orc_inject_permanent(self.h, _ptr(faults), len(faults), mode, n_threads or n_threads_default(), _ptr(out))
        return out

    def permanent_image(self, fault, rep: int = 0, mode: int = MODE_FULL):
        """(fault kind, faulty final image) of replica `rep` of one permanent fault."""
        f = np.ascontiguousarray(np.asarray(fault, dtype=PFAULT_DTYPE).reshape(1))
        img = np.zeros_like(self.final_image())
        k = lib().orc_permanent_image(self.h, _ptr(f), rep, mode, _ptr(img))
        return k, img

    def inject_image(self, site, mode: int = MODE_FULL):
        """(fault kind, faulty final image) of one transient site, full mode."""
        s = np.ascontiguousarray(np.asarray(site, dtype=SITE_DTYPE).reshape(1))
        img = np.zeros(self.prog.image_bytes, dtype=np.uint8)
        k = lib().orc_inject_image(self.h, _ptr(s), mode, _ptr(img))
        if k < 0:
            raise OracleError(4, "injection site not reached as selected")
        return k, img

    def locate(self, group: int, s) -> np.ndarray:
        s = np.ascontiguousarray(s, dtype=np.uint64)
        out = np.zeros(len(s), dtype=SITE_DTYPE)
        rc = lib().orc_locate(self.h, group, _ptr(s), len(s), _ptr(out))
        if rc:
            raise OracleError(rc, lib().orc_error(self.h).decode())
        return out

    def inject(self, sites: np.ndarray, mode: int = MODE_FULL, n_threads: int | None = None,
               rtol: float = 0.0) -> np.ndarray:
        """Injection + classification.  rtol > 0: C-12's
        secondary numeric mode sets SDC_WITHIN_TOL in flags."""
        sites = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
        out = np.zeros(len(sites), dtype=INJ_DTYPE)
        rc = lib().orc_inject(self.h, _ptr(sites), len(sites), mode, n_threads or n_threads_default(), float(rtol),
                              _ptr(out))
        if rc:
            raise OracleError(rc, lib().orc_error(self.h).decode())
        return out


class OracleError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"[{code}] {msg}")
        self.code = code


def count_warps(prog, w0: int, w1: int, n_threads: int | None = None) -> tuple[int, np.ndarray]:
    """Interpret warps [w0, w1) of a single-instance program (bounded CPU baseline)."""
    p, keep = _cprog(prog)
    out = np.zeros(8, dtype=np.uint64)
    n = lib().orc_count_warps(C.byref(p), w0, w1, n_threads or n_threads_default(), _ptr(out))
    return int(n), out


def scan_trace(records: np.ndarray, n_inst: int, n_threads: int | None = None) -> np.ndarray:
    """The profiler's count over an App. A.3 trace in host RAM (u64 [n_inst][8])."""
    rec = np.ascontiguousarray(records).view(np.uint8).reshape(-1)
    assert rec.size % 16 == 0
    out = np.zeros((n_inst, 8), dtype=np.uint64)
    if lib().orc_scan_trace(_ptr(rec), rec.size // 16, n_inst, n_threads or n_threads_default(), _ptr(out)):
        raise OracleError(4, "record names an instance beyond n_inst")
    return out


def warp_site_rank(prog, warp: int, group: int, step: int, lane: int) -> tuple[int, int] | None:
    """(rank of (step, lane) among warp `warp`'s group sites, warp total) for a
    single-instance program, or None if (step, lane) is not a site."""
    p, keep = _cprog(prog)
    r, t = C.c_uint64(), C.c_uint64()
    rc = lib().orc_warp_site_rank(C.byref(p), warp, group, step, lane, C.byref(r), C.byref(t))
    if rc == 2:
        raise OracleError(rc, "orc_warp_site_rank: not a single-instance program")
    return None if rc else (r.value, t.value)


def warp_site_at(prog, warp: int, group: int, rank: int) -> tuple[int, int, int] | None:
    """(step, lane, pc) of the rank-th group site of warp `warp` (single-instance)."""
    p, keep = _cprog(prog)
    st, ln, pc = C.c_uint32(), C.c_uint32(), C.c_uint32()
    rc = lib().orc_warp_site_at(C.byref(p), warp, group, rank, C.byref(st), C.byref(ln), C.byref(pc))
    if rc == 2:
        raise OracleError(rc, "orc_warp_site_at: not a single-instance program")
    return None if rc else (st.value, ln.value, pc.value)


def build_site(prog, seed: int, j: int, group: int, bfm: int, per_warp_total: int, n_total: int) -> np.ndarray:
    """The oracle's own site for replica j of a single-instance program whose
    warps all have `per_warp_total` group sites (a closed form the caller pins):
    draw s (C-5), w = s // per_warp_total, locate the rank inside warp w by
    enumeration (C-3), then slot (C-6) and mask (C-8)."""
    s, u_dst, u_bit, _ = draw(seed, j, n_total)
    w, rank = divmod(s, per_warp_total)
    step, lane, pc = warp_site_at(prog, w, group, rank)
    inst = prog.instances[0]
    wpc = (int(inst["block"]) + 31) // 32
    row = np.zeros(1, dtype=SITE_DTYPE)
    slots = dest_slots(prog.code[int(prog.kernels[int(inst["kernel"])]["code_off"]) + pc], group)
    slot = (len(slots) * u_dst) >> 32
    row["s"], row["instruction_count"], row["instance"], row["kernel_id"] = s, s, 0, int(inst["kernel"])
    row["kernel_count"], row["warp"], row["step"], row["pc"] = int(inst["kernel_count"]), w, step, pc
    row["thread"] = (w // wpc) * int(inst["block"]) + (w % wpc) * 32 + lane
    row["u_dst"], row["u_bit"], row["mask"] = u_dst, u_bit, mask(bfm, u_bit)
    row["lane"], row["group"], row["bfm"], row["slot"] = lane, group, bfm, slot
    row["dst_kind"], row["dst_reg"], row["n_elig"] = slots[slot][0], slots[slot][1], len(slots)
    return row


def inject_local(prog, sites: np.ndarray, n_threads: int | None = None) -> tuple[np.ndarray, np.ndarray]:
    """Warp-local injection of a single-instance program without a golden handle.
    Returns (inj, decided)."""
    p, keep = _cprog(prog)
    sites = np.ascontiguousarray(sites, dtype=SITE_DTYPE)
    out = np.zeros(len(sites), dtype=INJ_DTYPE)
    dec = np.zeros(len(sites), dtype=np.uint8)
    rc = lib().orc_inject_local(C.byref(p), _ptr(sites), len(sites), n_threads or n_threads_default(),
                                _ptr(out), _ptr(dec))
    if rc:
        raise OracleError(rc, "orc_inject_local failed")
    return out, dec.astype(bool)


def philox4x32_10(ctr, key) -> list[int]:
    c = np.asarray(ctr, dtype=np.uint32)
    k = np.asarray(key, dtype=np.uint32)
    o = np.zeros(4, dtype=np.uint32)
    lib().orc_philox4x32_10(_ptr(c), _ptr(k), _ptr(o))
    return [int(x) for x in o]


def draw(seed: int, j: int, n_g: int) -> tuple[int, int, int, int]:
    s, ud, ub, at = C.c_uint64(), C.c_uint32(), C.c_uint32(), C.c_uint32()
    lib().orc_draw(seed, j, n_g, C.byref(s), C.byref(ud), C.byref(ub), C.byref(at))
    return s.value, ud.value, ub.value, at.value


def mask(bfm: int, u_bit: int) -> int:
    return int(lib().orc_mask(bfm, u_bit))


def group_mask(insn_row) -> int:
    a = np.ascontiguousarray(np.asarray(insn_row).reshape(1))
    return int(lib().orc_group_mask(_ptr(a)))


def dest_slots(insn_row, group: int) -> list[tuple[int, int]]:
    a = np.ascontiguousarray(np.asarray(insn_row).reshape(1))
    k = np.zeros(8, np.uint8)
    r = np.zeros(8, np.uint8)
    n = lib().orc_dest_slots(_ptr(a), group, _ptr(k), _ptr(r))
    return [(int(k[i]), int(r[i])) for i in range(n)]


# ---- PAPER.md:214 §IV-B confidence margins ----------------------------------
_Z = {0.90: 1.6448536269514722, 0.95: 1.959963984540054, 0.99: 2.5758293035489004}


def ci_margin(n: int, confidence: float, p_hat: float | None = None) -> float:
    """Normal-approximation margin z*sqrt(p(1-p)/n); worst case p = 0.5 when
    p_hat is None ("100 injections ... 90% ... +-8%; 1000 ... 95% ... +-3%")."""
    p = 0.5 if p_hat is None else p_hat
    return _Z[confidence] * math.sqrt(p * (1 - p) / n)


def histogram(sites: np.ndarray, inj: np.ndarray, tol: bool = False) -> np.ndarray:
    """Outcome histogram [group][bfm][M,S,D] (u64), by plain counting.  tol=True:
    the C-12 secondary histogram (an SDC flagged SDC_WITHIN_TOL counts as Masked)."""
    h = np.zeros((8, 4, 3), dtype=np.uint64)
    for s, r in zip(sites, inj):
        o = int(r["outcome"])
        if tol and o == SDC and int(r["flags"]) & SDC_WITHIN_TOL:
            o = MASKED
        if o < 3:                                  # not-injected sites are not outcomes
            h[int(s["group"]), int(s["bfm"]), o] += 1
    return h
