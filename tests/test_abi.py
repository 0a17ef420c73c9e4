"""CPU-side checks of the C ABI: libfi.so builds for sm_100a, loads without a
GPU, exports every entry point include/fi.h declares, and its host-only calls
behave (status strings, register scan, parameter-file writer)."""
import ctypes as C
import os
import re

import numpy as np

from fi_inputs import programs as P

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "fi.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(fi_[a-z0-9_]+)\s*\(", src)))


def test_lib_exports_every_declared_symbol():
    from paper_conf_dsn_0002hsvk21_b200 import build, fi
    build.build()
    L = C.CDLL(fi.LIB_PATH)
    names = _declared()
    assert len(names) >= 17
    for n in names:
        assert hasattr(L, n), n


def test_sass_is_sm100a():
    import subprocess
    from paper_conf_dsn_0002hsvk21_b200 import build
    lib = build.build()
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", lib], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_host_calls():
    from paper_conf_dsn_0002hsvk21_b200 import fi
    assert "sm_100a" in fi.lib().fi_version().decode()
    assert fi.status_str(fi.FI_E_NOT_INJECTABLE).startswith("G_NODEST")
    code = np.ascontiguousarray(P.c2(full=False).code)
    n = fi.lib().fi_program_regs(code.ctypes.data, len(code))
    assert n == 99           # largest register index 95 (+4)
    s = np.zeros(1, dtype=fi.SITE_DTYPE)
    s["group"], s["bfm"], s["kernel_count"], s["instruction_count"] = 7, 0, 3, 12345
    s["u_dst"], s["u_bit"] = 2**31, 2**30
    txt = fi.write_params_txt(s[0], "sgemm_128x128")
    assert txt.split("\n")[:7] == ["7", "0", "sgemm_128x128", "3", "12345", "0.5000000000", "0.2500000000"]


def test_header_constants_match_input_format():
    """The opcode numbers in fi_inputs/isa.py, the libfi sources and the oracle
    are three independent copies of the format; check they agree."""
    from fi_inputs import isa
    names = ["NOP", "EXIT", "BRA", "MOV", "S2R", "IADD3", "IMAD", "IMAD_WIDE", "SHF", "LOP3", "SEL",
             "ISETP", "FSETP", "DSETP", "FADD", "FMUL", "FFMA", "FMNMX", "DADD", "DMUL", "DFMA",
             "LDG", "LDC", "STG", "I2F", "F2I", "F2F_F64_F32", "F2F_F32_F64", "SHFL", "IMNMX", "MUFU_RCP64"]
    for i, n in enumerate(names):
        assert getattr(isa, n) == i
    for path in ("paper_conf_dsn_0002hsvk21_b200/csrc/common.cuh", "oracle/oracle.cpp"):
        src = open(os.path.join(ROOT, path)).read()
        m = re.search(r"NOP = 0, (.*?)\n\s*(.*?)\n\s*(.*?)\n", src, flags=re.S)
        listed = ("NOP, " + m.group(1) + " " + m.group(2) + " " + m.group(3)).replace("\n", " ")
        got = [x.strip() for x in listed.split(",") if x.strip()]
        assert got[:len(names)] == names, path


def test_profile_txt_one_line_per_dynamic_kernel():
    """the profile has one line per dynamic kernel (name, kernel
    count, the eight Table II counts in order)."""
    from paper_conf_dsn_0002hsvk21_b200 import fi
    prog = P.multi_instance_chain(5)
    ic = (np.arange(5 * 8, dtype=np.uint64).reshape(5, 8) * np.uint64(1 << 33))
    txt = fi.write_profile_txt(ic, prog).splitlines()
    assert len(txt) == 5
    for k, line in enumerate(txt):
        name, kc, counts = line.split("; ")
        inst = prog.instances[k]
        assert name == prog.kernel_names[inst["kernel"]]
        assert kc == f"kernel_count: {inst['kernel_count']}"
        assert [int(x) for x in counts.split()] == [int(x) for x in ic[k]]


def test_campaign_argument_errors_without_gpu():
    """fi_campaign validates its host arguments before touching the device."""
    from paper_conf_dsn_0002hsvk21_b200 import fi
    res = fi.fi_campaign_result()
    cfg = fi.fi_campaign_cfg()
    L = fi.lib()
    assert L.fi_campaign(None, 0, 1, fi.ALLREDUCE_FN(), None, C.byref(res)) == fi.FI_E_ARG
    assert L.fi_campaign(C.byref(cfg), 0, 1, fi.ALLREDUCE_FN(), None, C.byref(res)) == fi.FI_E_ARG   # empty program
    assert L.fi_campaign(C.byref(cfg), 2, 2, fi.ALLREDUCE_FN(), None, C.byref(res)) == fi.FI_E_ARG   # rank >= world
    assert L.fi_campaign(C.byref(cfg), 0, 2, fi.ALLREDUCE_FN(), None, C.byref(res)) == fi.FI_E_ARG   # no callback


def test_jit_source_compiles_for_sm100a():
    """The JIT-specialised emulator's generated CUDA compiles with NVRTC for
    sm_100a (no GPU needed) for programs exercising every opcode."""
    from paper_conf_dsn_0002hsvk21_b200 import fi
    for prog in (P.c1(), P.fuzz_program(3, n_ops=120), P.multi_instance_chain(3), P.scatter_chain()):
        assert fi.jit_compile_check(prog) > 1000
    assert fi.jit_compile_check(P.c1(), fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN) > 1000
    src = fi.jit_source(P.c1())
    assert "k_inject_jit" in src and "kern_0" in src
