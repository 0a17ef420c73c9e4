"""Host-side pins of the JIT generator's register liveness (jit.cpp gen_kernel,
DESIGN.md §7.4): the generated CUDA (fi_jit_source, no GPU needed) zeroes
exactly the registers no lane can read again, never a SHFL source, and never in
the trace pass (whose checkpoints copy every register).  The values themselves
are pinned on the GPU by the JIT-vs-interpreter-vs-oracle parity suite."""
import re

import pytest

from fi_inputs import hpc as H
from fi_inputs import programs as P
from paper_conf_dsn_0002hsvk21_b200 import fi

KILLS = re.compile(r"((?:R\d+ = 0u; )+)")


def _functions(src: str, mode: str) -> dict[str, str]:
    """kern_<k>_<mode> bodies, from the block dispatch on (the register
    initialisation before the dispatch loop is not a kill)."""
    out = {}
    for m in re.finditer(r"__forceinline__ void (kern_\d+_%s)\(" % mode, src):
        end = src.find("__forceinline__ void kern_", m.end())
        body = src[m.end(): end if end >= 0 else len(src)]
        out[m.group(1)] = body[body.index(" switch (pcm) {"):]
    return out


def _sets(body: str) -> list[set[int]]:
    return [{int(x) for x in re.findall(r"R(\d+) = 0u;", k)} for k in KILLS.findall(body)]


def test_c2_k_loop_exits():
    """SGEMM (fi_inputs/programs.py sgemm_code): the K loop is pcs 17..89, its BRA
    at 89.  Back edge (chain to B17): R0-R5 (setup) and the 16 fragment registers
    R72-R87 (reloaded at the loop top) are dead; everything the loop or the
    epilogue reads (accumulators R8-R71, pointers, counters, R6/R7) is kept."""
    src = fi.jit_source(P.c2(full=False), fi.FI_JIT_INJECT)
    body = _functions(src, "inj")["kern_0_inj"]
    bra = body[body.index("{ const bool pv = Q0;"):body.index(" B90:")]
    back = re.search(r"pcm = 17u; ((?:R\d+ = 0u; )+)goto B17;", bra)
    assert back, "no kills on the back edge"
    want = set(range(0, 6)) | set(range(72, 88))
    assert {int(x) for x in re.findall(r"R(\d+)", back.group(1))} == want
    # leaving the loop for the epilogue without chaining: the loop-only registers
    # (B pointer R90/R91, counter R92, A stride R93) are dead too; R88/R89 (C
    # pointer, rewritten at 90 but read after), R94 (stride of the STG loop) kept
    ft = re.search(r"goto B90; \} ((?:R\d+ = 0u; )+)upc = 90u;", bra)
    assert ft
    assert {int(x) for x in re.findall(r"R(\d+)", ft.group(1))} == want | {90, 91, 92, 93}
    case17 = body[body.index("  case 17:"):].split("\n")[0]
    for s in _sets(bra) + _sets(case17):               # nor the accumulators, while the loop can run
        assert not s & set(range(8, 72))


@pytest.mark.parametrize("mode,name", [(fi.FI_JIT_INJECT, "inj"), (fi.FI_JIT_GOLDEN, "len"),
                                       (fi.FI_JIT_PAGE, "page")])
def test_shfl_sources_never_zeroed(mode, name):
    """SHFL reads the source register of parked and exited lanes."""
    prog = H.stencil(n=16, iters=2)
    src = fi.jit_source(prog, mode)
    funcs = _functions(src, name)
    assert funcs
    seen = False
    for body in funcs.values():
        srcs = {int(x) for x in re.findall(r"__shfl_sync\(JFULL, R(\d+), src_\)", body)}
        if not srcs:
            continue
        seen = True
        for s in _sets(body):
            assert not s & srcs, (srcs, s)
    assert seen, "no SHFL in the stencil program's kernels"


def test_trace_pass_has_no_kills():
    src = fi.jit_source(P.c2(full=False), fi.FI_JIT_GOLDEN)
    assert _sets(_functions(src, "len")["kern_0_len"]), "pass 1 (lengths) uses liveness"
    assert not _sets(_functions(src, "trace")["kern_0_trace"]), "checkpoints copy every register"


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_kills_only_dead_registers_fuzz(seed):
    """On fuzz programs (branches, guards, loops): a register zeroed on the way into
    a block is not read in that block before an unguarded write of it."""
    prog = P.fuzz_program(seed)
    src = fi.jit_source(prog, fi.FI_JIT_INJECT)
    for body in _functions(src, "inj").values():
        for m in re.finditer(r"((?:R\d+ = 0u; )+)goto B(\d+);", body):
            killed = {int(x) for x in re.findall(r"R(\d+)", m.group(1))}
            blk = body[body.index(" B%s:\n" % m.group(2)):]
            blk = blk[:blk.index("continue;")]
            for stmt in blk.split("\n"):
                reads = {int(x) for x in re.findall(r"\bR(\d+)\b(?! = )", stmt)}
                assert not reads & killed, (m.group(2), reads & killed, stmt[:200])
                # an unguarded instruction's write ends the register's dead range
                if "const bool pv = true;" in stmt:
                    killed -= {int(x) for x in re.findall(r"if \(ex\) R(\d+) = ", stmt)}
