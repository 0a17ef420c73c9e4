"""Closed-form Table II counts of the generated kernels, derived by hand from
the listings in fi_inputs/programs.py (pins for the oracle and for full-size
GPU parity)."""
FP64, FP32, LD, PR, NODEST, OTHERS, GPPR, GP = range(8)


def sgemm_per_thread(K: int) -> list[int]:
    """C2 kernel per thread: prologue 17 insns, 73 per k-iteration (4 LDG.128,
    64 FFMA, 2 IMAD.WIDE + IADD3, ISETP, BRA — the last BRA predicated off),
    epilogue 29 insns (LDC.64, LDC, IMAD, IMAD.WIDE, 8 x (2 STG.128 + IMAD.WIDE), EXIT)."""
    per = [0] * 8
    per[LD] = 5 + 4 * K + 2
    per[FP32] = 64 * K
    per[OTHERS] = 12 + 3 * K + 2 + 8
    per[PR] = K
    per[NODEST] = (K - 1) + 16 + 1
    per[GP] = per[FP32] + per[LD] + per[OTHERS]
    per[GPPR] = per[GP] + per[PR]
    return per


def sgemm_closed_form(M: int, N: int, K: int):
    threads = M * N // 64
    return [x * threads for x in sgemm_per_thread(K)], (threads // 32) * (17 + 73 * K + 29)
