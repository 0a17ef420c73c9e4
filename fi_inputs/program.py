"""Synthetic program container and builder (input format only).

A *program* is what the golden run executes: static kernels in
mini-SASS, a launch schedule of dynamic kernel instances ("one line
for every dynamic kernel"), per-instance constant banks, and a memory image
made of 256-B aligned allocations.  This module only lays the arrays out; it
computes nothing the method computes (no counts, no groups, no selection).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import isa

KERNEL_DTYPE = np.dtype([("code_off", "<u4"), ("code_len", "<u4"), ("nregs", "<u4"), ("pad", "<u4")])
INSTANCE_DTYPE = np.dtype([
    ("kernel", "<u4"), ("kernel_count", "<u4"), ("grid", "<u4"), ("block", "<u4"),
    ("cbank_off", "<u4"), ("cbank_len", "<u4"), ("warp_begin", "<u4"), ("warp_end", "<u4"),
])
BUFFER_DTYPE = np.dtype([("off", "<u8"), ("size", "<u8"), ("writer", "<i4"), ("flags", "<u4")])
assert KERNEL_DTYPE.itemsize == 16 and INSTANCE_DTYPE.itemsize == 32 and BUFFER_DTYPE.itemsize == 24


@dataclass
class Program:
    name: str
    code: np.ndarray            # INSN_DTYPE [n_code]
    kernels: np.ndarray         # KERNEL_DTYPE [n_kern]
    kernel_names: list
    instances: np.ndarray       # INSTANCE_DTYPE [n_inst]
    cbank: np.ndarray           # <u4 [n_cbank]
    buffers: np.ndarray         # BUFFER_DTYPE [n_buf], sorted by off
    buffer_names: list
    init_image: np.ndarray      # u1 [image_bytes]
    meta: dict = field(default_factory=dict)

    @property
    def n_warps(self) -> int:
        return int(self.instances["warp_end"][-1]) if len(self.instances) else 0

    @property
    def image_bytes(self) -> int:
        return int(self.init_image.size)

    def buffer(self, name: str):
        i = self.buffer_names.index(name)
        return self.buffers[i]

    def view(self, image: np.ndarray, name: str, dtype) -> np.ndarray:
        b = self.buffer(name)
        return image[int(b["off"]):int(b["off"]) + int(b["size"])].view(dtype)


def _round_up(x: int, a: int) -> int:
    return (x + a - 1) // a * a


class ProgramBuilder:
    def __init__(self, name: str):
        self.name = name
        self.code_rows: list[np.ndarray] = []
        self.n_code = 0
        self.kernels: list[tuple] = []
        self.kernel_names: list[str] = []
        self.instances: list[tuple] = []
        self.cbank: list[int] = []
        self.buffers: list[dict] = []
        self.image_bytes = 0
        self.n_warps = 0
        self._kcount: dict[int, int] = {}

    def add_kernel(self, name: str, code: np.ndarray, nregs: int = 127) -> int:
        assert code.dtype == isa.INSN_DTYPE
        self.kernels.append((self.n_code, len(code), nregs, 0))
        self.kernel_names.append(name)
        self.code_rows.append(code)
        self.n_code += len(code)
        return len(self.kernels) - 1

    def add_buffer(self, name: str, nbytes: int, init: np.ndarray | None = None,
                   writer: int = -1, output: bool = False, dtype: int = isa.DT_U32) -> int:
        """Allocate a buffer; returns its virtual address.  `writer` is the one
        instance that stores into it (SSA), -1 for none."""
        off = self.image_bytes
        self.buffers.append(dict(name=name, off=off, size=nbytes, writer=writer,
                                 flags=(isa.BUF_OUTPUT if output else 0) | (dtype << 8),
                                 init=None if init is None else np.ascontiguousarray(init).view(np.uint8).ravel()))
        self.image_bytes = _round_up(off + nbytes, isa.ALLOC_ALIGN)
        return isa.VA_BASE + off

    def set_writer(self, va: int, writer: int):
        for b in self.buffers:
            if isa.VA_BASE + b["off"] == va:
                b["writer"] = writer
                return
        raise KeyError(hex(va))

    def add_instance(self, kernel: int, grid: int, block: int, cbank_words: list[int]) -> int:
        kc = self._kcount.get(kernel, 0)
        self._kcount[kernel] = kc + 1
        wpc = (block + 31) // 32
        wb = self.n_warps
        self.n_warps += grid * wpc
        self.instances.append((kernel, kc, grid, block, len(self.cbank), len(cbank_words), wb, self.n_warps))
        self.cbank.extend(int(w) & 0xFFFFFFFF for w in cbank_words)
        return len(self.instances) - 1

    def build(self, **meta) -> Program:
        image = np.zeros(self.image_bytes, dtype=np.uint8)
        for b in self.buffers:
            if b["init"] is not None:
                assert b["init"].size <= b["size"]
                image[b["off"]:b["off"] + b["init"].size] = b["init"]
                assert b["writer"] < 0, "SSA: a buffer written by an instance starts zeroed"
        bufs = np.array([(b["off"], b["size"], b["writer"], b["flags"]) for b in self.buffers], dtype=BUFFER_DTYPE)
        return Program(
            name=self.name,
            code=np.concatenate(self.code_rows) if self.code_rows else np.zeros(0, isa.INSN_DTYPE),
            kernels=np.array(self.kernels, dtype=KERNEL_DTYPE),
            kernel_names=list(self.kernel_names),
            instances=np.array(self.instances, dtype=INSTANCE_DTYPE),
            cbank=np.array(self.cbank, dtype="<u4"),
            buffers=bufs,
            buffer_names=[b["name"] for b in self.buffers],
            init_image=image,
            meta=dict(meta),
        )


def ptr_words(va: int) -> list[int]:
    return [va & 0xFFFFFFFF, va >> 32]


# ---- data recipe ---------------------------------------------
def f32_data(seed: int, n: int) -> np.ndarray:
    """Exact f32 values in [-1, 1): ((w >> 8) - 2^23) * 2^-23 for random u32 w."""
    w = np.random.Generator(np.random.PCG64(seed)).integers(0, 2**32, size=n, dtype=np.uint64)
    return (((w >> np.uint64(8)).astype(np.int64) - (1 << 23)).astype(np.float64) * 2.0**-23).astype(np.float32)


def f64_data(seed: int, n: int) -> np.ndarray:
    w = np.random.Generator(np.random.PCG64(seed)).integers(0, 2**63, size=n, dtype=np.uint64)
    return ((w >> np.uint64(10)).astype(np.int64) - (1 << 52)).astype(np.float64) * 2.0**-52


def u32_data(seed: int, n: int) -> np.ndarray:
    return np.random.Generator(np.random.PCG64(seed)).integers(0, 2**32, size=n, dtype=np.uint64).astype(np.uint32)
