"""Pin the oracle on the C5 mixed HPC suite (mini sizes) against numpy and
conservation laws — values fixed by the mathematics, not by the oracle.

stencil  bitwise: the same f32 operation order in numpy (sum of neighbours left
         to right, then one FMA with power-of-two coefficients, exact in f64)
lbm      float64 numpy D3Q19 BGK with pull streaming to 1e-15; mass and momentum
         conserved to rounding
md       float64 numpy velocity Verlet with all-pairs LJ forces to 1e-14; total
         force (Newton's third law) zero to rounding
ep       integer tallies bitwise from a Python LCG; f64 sums to rounding; the
         acceptance rate of a uniform pair in the unit disc is pi/4
"""
import numpy as np
import pytest

import oracle as O
from fi_inputs import hpc as H


def test_stencil_bitwise():
    n, iters = 8, 5
    p = H.stencil(n, iters)
    g = O.Golden(p)
    img = g.final_image()
    P = n + 2
    u = p.view(img, "u0", "<f4").reshape(P, P, P).copy()
    for it in range(iters):
        c = u[1:-1, 1:-1, 1:-1]
        s = (u[1:-1, 1:-1, :-2] + u[1:-1, 1:-1, 2:]).astype(np.float32)
        for nb in (u[1:-1, :-2, 1:-1], u[1:-1, 2:, 1:-1], u[:-2, 1:-1, 1:-1], u[2:, 1:-1, 1:-1]):
            s = (s + nb).astype(np.float32)
        un = np.zeros_like(u)
        un[1:-1, 1:-1, 1:-1] = (s.astype(np.float64) * 0.125 + (c * np.float32(0.25)).astype(np.float64)).astype(np.float32)
        assert np.array_equal(p.view(img, f"u{it + 1}", "<u4").reshape(P, P, P), un.view("<u4"))
        u = un
    ss = p.view(img, "sumsq", "<f4").astype(np.float64).sum()
    assert abs(ss - (u.astype(np.float64) ** 2).sum()) <= 1e-5 * ss


def test_lbm_matches_numpy_and_conserves():
    n, steps = 4, 6
    p = H.lbm(n, steps, 3)
    img = O.Golden(p).final_image()
    c = np.array(H.D3Q19)
    w = np.array(H.D3Q19_W)
    tau = p.meta["tau"]
    f = p.view(img, "f0", "<f8").reshape(19, n, n, n).copy()
    assert np.allclose(f.sum(0), p.view(img, "rho0", "<f8").reshape(n, n, n), rtol=1e-15, atol=0)
    mass0 = f.sum()
    for st in range(steps):
        fs = np.stack([np.roll(f[q], shift=(c[q][2], c[q][1], c[q][0]), axis=(0, 1, 2)) for q in range(19)])
        rho = fs.sum(0)
        u = [(fs * c[:, a][:, None, None, None]).sum(0) / rho for a in range(3)]
        usq = u[0] ** 2 + u[1] ** 2 + u[2] ** 2
        cu = [c[q][0] * u[0] + c[q][1] * u[1] + c[q][2] * u[2] for q in range(19)]
        feq = np.stack([w[q] * rho * (1 + 3 * cu[q] + 4.5 * cu[q] ** 2 - 1.5 * usq) for q in range(19)])
        f = fs - (fs - feq) / tau
        got = p.view(img, f"f{st + 1}", "<f8").reshape(19, n, n, n)
        assert np.abs(got - f).max() <= 1e-15
        assert abs(got.sum() - mass0) <= 1e-13 * mass0
        for a in range(3):
            assert abs((got * c[:, a][:, None, None, None]).sum()) <= 1e-13 * mass0
    m = p.view(img, f"m{steps}", "<f8").reshape(4, n, n, n)
    assert np.abs(m[0] - f.sum(0)).max() <= 1e-14


def test_md_matches_numpy_and_newton3():
    p = H.md(3, 3)
    img = O.Golden(p).final_image()
    N, L, rc, dt = (p.meta[k] for k in ("N", "L", "rc", "dt"))

    def force(x):
        d = x[:, :, None] - x[:, None, :]
        d = np.where(d > L / 2, d - L, d)
        d = np.where(d < -L / 2, d + L, d)
        r2 = (d ** 2).sum(0)
        np.fill_diagonal(r2, np.inf)
        ok = r2 < rc * rc
        inv = np.where(ok, 1 / np.where(ok, r2, 1), 0)
        s6 = inv ** 3
        return (24 * (2 * s6 - 1) * s6 * inv)[None] * d

    x = p.view(img, "x0", "<f8").reshape(3, N).copy()
    v = p.view(img, "v0", "<f8").reshape(3, N).copy()
    f = force(x).sum(2)
    got = p.view(img, "f0", "<f8").reshape(3, N)
    assert np.abs(got - f).max() <= 1e-13 * np.abs(f).max()
    assert np.abs(got.sum(1)).max() <= 1e-13 * np.abs(f).sum()
    for st in range(3):
        vh = v + dt / 2 * f
        x = x + dt * vh
        x = np.where(x >= L, x - L, x)
        x = np.where(x < 0, x + L, x)
        f = force(x).sum(2)
        v = vh + dt / 2 * f
        assert np.abs(p.view(img, f"x{st + 1}", "<f8").reshape(3, N) - x).max() <= 1e-13
        assert np.abs(p.view(img, f"v{st + 1}", "<f8").reshape(3, N) - v).max() <= 1e-13


def test_ep_tallies():
    threads, pairs, chunks = 256, 16, 2
    p = H.ep(threads, pairs, chunks)
    img = O.Golden(p).final_image()
    acc = 0
    for c in range(chunks):
        x0 = (p.meta["seed"] + 7919 * c) & 0xFFFFFFFF
        tot = np.zeros(4, np.int64)
        sx = sy = 0.0
        for t in range(threads):
            xx = (t * 2654435761 + x0) & 0xFFFFFFFF
            for _ in range(pairs):
                us = []
                for _ in range(2):
                    xx = (xx * 1664525 + 1013904223) & 0xFFFFFFFF
                    us.append(2.0 * float(np.float32(np.float32(xx) * np.float32(2.0 ** -32))) - 1.0)
                X, Y = us
                tt = X * X + Y * Y
                if tt <= 1:
                    tot += [1, tt < 0.25, tt < 0.5, tt < 0.75]
                    sx += X * tt
                    sy += Y * tt
        got = p.view(img, f"tally{c}", "<u4")
        assert np.array_equal(got[:4], tot)
        gs = p.view(img, f"tally{c}", "<f8")[2:4]
        assert abs(gs[0] - sx) <= 1e-12 * threads * pairs and abs(gs[1] - sy) <= 1e-12 * threads * pairs
        acc += tot[0]
    assert abs(acc / (threads * pairs * chunks) - np.pi / 4) < 0.03


def test_suite_shapes():
    progs = H.c5(full=False)
    assert [p.meta["config"] for p in progs][:4] == ["C5-stencil", "C5-lbm", "C5-md", "C5-ep"]
    for p in progs:
        g = O.Golden(p)
        c = g.counts()
        assert (c[:, 7] == c[:, 0] + c[:, 1] + c[:, 2] + c[:, 5]).all()
        assert (c[:, 6] == c[:, 7] + c[:, 3]).all()
