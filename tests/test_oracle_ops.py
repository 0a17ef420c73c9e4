"""Pin the oracle interpreter opcode by opcode (DESIGN.md §3 semantics,
C-13) against numpy IEEE arithmetic, exact rationals and Python integers."""
import numpy as np
import pytest

import oracle as O
import opcases


@pytest.fixture(scope="module")
def all_cases():
    return opcases.cases(seed=1234)


def test_ops_conform(all_cases):
    bad = []
    for name, rows, words, exp in all_cases:
        prog = opcases.build(rows, words, name)
        g = O.Golden(prog, keep_trace=False, n_threads=2)
        y = prog.view(g.final_image(), "Y", "<u4").reshape(-1, 8)
        if not np.array_equal(y, exp):
            i = np.argwhere(y != exp)[0]
            bad.append(f"{name}: thread {i[0]} word {i[1]} got {y[i[0], i[1]]:#x} want {exp[i[0], i[1]]:#x} in {words[i[0]]}")
    assert not bad, "\n".join(bad[:20])


def test_exact_fma_helper_sanity():
    # the rounding helper itself: values exactly representable round to themselves,
    # and a*a - fl(a*a) is the exact error term (the classic FMA identity)
    a = 1.0 + 2.0**-23
    assert opcases.exact_fma(a, 1.0, 0.0, 32) == opcases.bits32(a)
    err = opcases.f32(opcases.exact_fma(a, a, -float(np.float32(a * a)), 32))
    assert err == 2.0**-46
    assert opcases.exact_fma(1e308, 10.0, 0.0, 64) == 0x7FF0000000000000
    assert opcases.exact_fma(2.0**-1074, 0.5, 0.0, 64) == 0          # ties-to-even to zero
    assert opcases.exact_fma(2.0**-1074, 1.5, 0.0, 64) == 2          # 1.5 ulp -> 2 ulp
