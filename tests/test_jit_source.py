"""Host-side pins of the JIT generator's structure (jit.cpp; the
generated CUDA via fi_jit_source, no GPU needed).  The values are pinned on the
GPU by the JIT-vs-interpreter-vs-oracle parity suite; these keep the
structural choices the measurements rest on from regressing silently."""
import re

from fi_inputs import programs as P
from paper_conf_dsn_0002hsvk21_b200 import fi


def test_emulator_functions_are_inlined():
    """Each per-kernel emulator function is inlined into its one entry kernel
    (as a separate function ptxas reloaded the memory descriptor per load)."""
    src = fi.jit_source(P.c2(full=False), fi.FI_JIT_INJECT | fi.FI_JIT_GOLDEN | fi.FI_JIT_PAGE)
    kerns = re.findall(r"__device__ (\w+) void kern_\d+_(\w+)\(", src)
    assert {m for _, m in kerns} == {"inj", "len", "trace", "page"}
    assert all(q == "__forceinline__" for q, _ in kerns)


def test_template_loop_profile_flushes():
    """Golden pass 2's full-warp template loop (C2's K-loop): the record template
    goes out as one bulk copy from an elected lane; the fused profile's count is
    kept in a register there and flushed before every chunk-crossing pass, before
    every per-lane record round and when the loop is left."""
    src = fi.jit_source(P.c2(full=False), fi.FI_JIT_GOLDEN)
    body = src[src.index("void kern_0_trace("):]
    body = body[:body.index("finish:")]
    assert "if (jelect()) jbulk_st_p(" in body
    assert "JPFLUSH_; jprof_tmpl_cross(" in body
    assert "{ JPFLUSH_; jprof_round(" in body
    full = body.index("full warp, two iterations per trip")
    assert "#define JPFLUSH_ { if (lane < 8u) jx->prof.pcnt_[lane] += jpa_; jpa_ = 0u; }" in body[:full]
    # after the unrolled loop: the exit flush, then the shared-memory versions again
    tail = body[full:]
    assert re.search(r"#define JFW_ 0\n JPFLUSH_;\n#undef JPCC_", tail)
    assert "#define JPFLUSH_ {}" in tail


def test_page_mode_checks_pass_the_slot_view():
    """K8's PAGE mode hands the replica slot's view (JPage) to every cache fill, so
    an entry can record that the slot holds no page of the buffer; the cache
    carried from the previous job is keyed by instance and slot."""
    src = fi.jit_source(P.c3(full=False), fi.FI_JIT_PAGE)
    assert "jcheck<" in src and ", &PG)" in src
    assert "jx->bck == k && jx->bckp == (u32)(size_t)PG.ptab" in src
    assert "jx->bckp = (u32)(size_t)PG.ptab;" in src
