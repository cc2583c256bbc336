"""Error-bound pins for EVERY statement form of every app, in every {f64, f32, f16}
configuration (VERDICT r1 "next" #1).

The oracle's low-precision runs are definitions (readings R1-R5);
nothing can reproduce them bit for bit except the definition itself.  What
mathematics does fix is how far each statement may land from the EXACT result
of the same statement on the same stored operands:

  * an fma chain / any summation order over K terms:  |fl - s| <= gamma_K * sum|terms|
    (Higham, Accuracy and Stability, Lemma 3.1 / Eq. 3.4), gamma_K = K u / (1 - K u);
  * one IEEE operation (+ - * / sqrt): relative error <= u;
  * storing a value into a narrower object (R1): <= u_c |v| + half the smallest
    subnormal of c.

For each configuration the test reads the oracle's stored contents of every
object (inputs after a2, temporaries and outputs after their statements), then,
statement by statement, recomputes the exact result in 64-bit-mantissa long
double from the statement's STORED inputs and checks the oracle's stored output
against that bound, with u taken from the statement's compute type T (R2).  A
dropped or duplicated term, a wrong index or transpose, a sign error, a wrong
scalar, a statement computed in the wrong T (f32 where R2 says f64) or an
output stored without rounding to its object's precision all break a bound by
orders of magnitude.  Scalars are the RNE-to-T images of their fp64 literals
(reading R2), formed here with numpy's float32 cast.
"""
import itertools
import math

import numpy as np
import pytest

import oracle
from paper_conf_cgo_kangcp20_b200 import inputs as gen

F64, F32, F16 = 0, 1, 2
LD = np.longdouble
U = {F64: 2.0 ** -53, F32: 2.0 ** -24, F16: 2.0 ** -11}
ETA = {F64: 2.0 ** -1075, F32: 2.0 ** -150, F16: 2.0 ** -25}   # half the smallest subnormal
U_REF = 2.0 ** -63                                               # long double reference
SC = (1.5, 1.2)                                                  # alpha, beta: no fp16 overflow


def gam(k, u):
    return k * u / (1.0 - k * u)


def T_of(*codes):
    """R2: widest touched precision, floored at f32."""
    return F64 if F64 in codes else F32


def lit(T, x):
    """R2: an fp64 literal RNE-rounded to T."""
    return float(np.float32(x)) if T == F32 else float(x)


def stored(x, c):
    """a2: the orig f32 contents RNE-rounded to c (numpy's RNE casts)."""
    x = np.asarray(x, dtype=np.float32)
    return (x.astype(np.float16) if c == F16 else x).astype(np.float64)


def store_err(T, c, mag):
    """Rounding a T result into an object of precision c (R1)."""
    if c == F64 or (c == F32 and T == F32):
        return 0.0 * mag
    return U[c] * mag + ETA[c]


def check(got, exact, arith, T, c, what, ref_terms=None):
    """|got - exact| <= arith + store rounding + long-double reference slack."""
    got = np.asarray(got, dtype=np.float64)
    exact = np.asarray(exact, dtype=LD)
    arith = np.asarray(arith, dtype=np.float64)
    mag = np.abs(exact).astype(np.float64) + arith
    slack = 64 * U_REF * (mag if ref_terms is None else np.asarray(ref_terms, np.float64) + mag)
    bound = arith + store_err(T, c, mag) + slack
    err = np.abs(got.astype(LD) - exact).astype(np.float64)
    assert np.all(np.isfinite(got)), what
    bad = err > bound * (1 + 1e-12)
    assert not bad.any(), "%s: %d/%d entries out of bound, worst err %.3g vs bound %.3g" % (
        what, int(bad.sum()), bad.size, float(err[bad].max()), float(bound[bad][np.argmax(err[bad])]))


def mm(a, b):
    return np.asarray(a, LD) @ np.asarray(b, LD)


def amm(a, b):
    return np.abs(np.asarray(a, LD)) @ np.abs(np.asarray(b, LD))


# rows of R5's row-dot: lane chain of V, butterfly 5, <= 8 slabs per tile, tiles;
# the depth of any term is < K + 14 for every K, so gamma_{K+14} bounds it
RD = 14


def run(kind, dims, prec, ins, sc=None):
    objs = oracle.app_objects(kind, dims)
    fin = oracle.run_config(kind, dims, list(prec), ins, sc)
    F = [oracle.widen(f, p).reshape(o["rows"], o["cols"]) for f, p, o in zip(fin, prec, objs)]
    S = [stored(x, p).reshape(o["rows"], o["cols"]) if x is not None else None
         for x, p, o in zip(ins, prec, objs)]
    return F, S


# --------------------------------------------------------------- per app
def pin_gemm(dims, p, ins):
    F, S = run("gemm", dims, p, ins, SC)
    T = T_of(*p)
    al, be = lit(T, SC[0]), lit(T, SC[1])
    K = dims[2]
    ex = al * mm(S[0], S[1]) + be * S[2].astype(LD)
    ar = gam(K + 2, U[T]) * (abs(al) * amm(S[0], S[1]) + np.abs(be * S[2]))
    check(F[2], ex, ar, T, p[2], "gemm C")


def pin_2mm(dims, p, ins):
    NI, NJ, NK, NL = dims
    F, S = run("2mm", dims, p, ins)
    T1, T2 = T_of(p[0], p[1], p[2]), T_of(p[2], p[3], p[4])
    check(F[2], mm(S[0], S[1]), gam(NK, U[T1]) * amm(S[0], S[1]), T1, p[2], "2mm C")
    check(F[4], mm(F[2], S[3]), gam(NJ, U[T2]) * amm(F[2], S[3]), T2, p[4], "2mm E")


def pin_3mm(dims, p, ins):
    NI, NJ, NK, NL, NM = dims
    F, S = run("3mm", dims, p, ins)
    T1, T2, T3 = T_of(p[0], p[1], p[4]), T_of(p[2], p[3], p[5]), T_of(p[4], p[5], p[6])
    check(F[4], mm(S[0], S[1]), gam(NK, U[T1]) * amm(S[0], S[1]), T1, p[4], "3mm E")
    check(F[5], mm(S[2], S[3]), gam(NM, U[T2]) * amm(S[2], S[3]), T2, p[5], "3mm F")
    check(F[6], mm(F[4], F[5]), gam(NJ, U[T3]) * amm(F[4], F[5]), T3, p[6], "3mm G")


def pin_atax(dims, p, ins):
    NX, NY = dims
    F, S = run("atax", dims, p, ins)
    T1, T2 = T_of(p[0], p[1], p[3]), T_of(p[0], p[3], p[2])
    A, x, tmp = S[0], S[1][0], F[3][0]
    check(tmp, mm(A, x), gam(NY + RD, U[T1]) * amm(A, x), T1, p[3], "atax tmp (row-dot)")
    check(F[2][0], mm(A.T, tmp), gam(NX + 2, U[T2]) * amm(A.T, tmp), T2, p[2], "atax y (column-sum)")


def pin_bicg(dims, p, ins):
    NX, NY = dims
    F, S = run("bicg", dims, p, ins)
    T1, T2 = T_of(p[0], p[1], p[2]), T_of(p[0], p[3], p[4])
    A, r, pv = S[0], S[1][0], S[3][0]
    check(F[2][0], mm(A.T, r), gam(NX + 2, U[T1]) * amm(A.T, r), T1, p[2], "bicg s (column-sum)")
    check(F[4][0], mm(A, pv), gam(NY + RD, U[T2]) * amm(A, pv), T2, p[4], "bicg q (row-dot)")


def pin_gesummv(dims, p, ins):
    N = dims[0]
    F, S = run("gesummv", dims, p, ins, SC)
    A, B, x = S[0], S[1], S[2][0]
    T1, T2, T3 = T_of(p[0], p[2], p[4]), T_of(p[1], p[2], p[3]), T_of(p[4], p[3])
    tmp = F[4][0]
    check(tmp, mm(A, x), gam(N + RD, U[T1]) * amm(A, x), T1, p[4], "gesummv tmp")
    # y1 = RNE_c(y)(B x) is overwritten; bound its error e1, then y = fma(al, tmp, be*y1)
    bx, sbx = mm(B, x), amm(B, x).astype(np.float64)
    e1 = gam(N + RD, U[T2]) * sbx
    e1 = e1 + store_err(T2, p[3], np.abs(bx).astype(np.float64) + e1)
    al, be = lit(T3, SC[0]), lit(T3, SC[1])
    ex = al * tmp.astype(LD) + be * bx
    ar = abs(be) * e1 + gam(2, U[T3]) * (abs(al) * np.abs(tmp) + abs(be) * (sbx + e1))
    check(F[3][0], ex, ar, T3, p[3], "gesummv y")


def pin_mvt(dims, p, ins):
    N = dims[0]
    F, S = run("mvt", dims, p, ins)
    A, x1, x2, y1, y2 = S[0], S[1][0], S[2][0], S[3][0], S[4][0]
    T1, T2 = T_of(p[0], p[1], p[3]), T_of(p[0], p[2], p[4])
    check(F[1][0], x1.astype(LD) + mm(A, y1), gam(N + RD + 1, U[T1]) * (np.abs(x1) + amm(A, y1)), T1,
          p[1], "mvt x1")
    check(F[2][0], x2.astype(LD) + mm(A.T, y2), gam(N + 3, U[T2]) * (np.abs(x2) + amm(A.T, y2)), T2,
          p[2], "mvt x2")


def _col_mean(S0, F1, p, N, what):
    T = T_of(p[0], p[1])
    ex = S0.astype(LD).sum(axis=0) / N
    ar = gam(N + 2, U[T]) * np.abs(S0).sum(axis=0) / N
    check(F1[0], ex, ar, T, p[1], what)


def pin_corr(dims, p, ins, eps=0.005):
    N, M = dims
    F, S = run("corr", dims, p, ins)
    d, mean, std, X = S[0], F[1][0], F[2][0], F[0]
    _col_mean(d, F[1], p, N, "corr mean")
    T2 = T_of(p[0], p[1], p[2])
    dev = d.astype(LD) - mean.astype(LD)
    s_ex = np.sqrt((dev * dev).sum(axis=0) / N)
    rel = gam(N + 4, U[T2]) / 2 + U[T2]
    assert np.all(s_ex.astype(np.float64) > 10 * eps)      # the eps guard stays off here
    check(std, s_ex, rel * s_ex.astype(np.float64), T2, p[2], "corr stddev")
    sqn = lit(T2, math.sqrt(N))
    den = sqn * std.astype(LD)
    ex = dev / den
    check(X, ex, gam(3, U[T2]) * np.abs(ex).astype(np.float64), T2, p[0], "corr normalise")
    T4 = T_of(p[0], p[3])
    sy = mm(X.T, X)
    ar = gam(N, U[T4]) * amm(X.T, X)
    np.fill_diagonal(sy, 1.0)
    np.fill_diagonal(ar, 0.0)
    check(F[3], sy, ar, T4, p[3], "corr symmat")
    assert np.array_equal(F[3], F[3].T)


def pin_covar(dims, p, ins):
    N, M = dims
    F, S = run("covar", dims, p, ins)
    d, mean, X = S[0], F[1][0], F[0]
    _col_mean(d, F[1], p, N, "covar mean")
    T2 = T_of(p[0], p[1])
    ex = d.astype(LD) - mean.astype(LD)
    check(X, ex, U[T2] * np.abs(ex).astype(np.float64), T2, p[0], "covar centre")
    T3 = T_of(p[0], p[2])
    dv = lit(T3, N - 1.0)
    check(F[2], mm(X.T, X) / dv, gam(N + 1, U[T3]) * amm(X.T, X) / dv, T3, p[2], "covar symmat")
    assert np.array_equal(F[2], F[2].T)


def pin_syrk(dims, p, ins):
    N, M = dims
    F, S = run("syrk", dims, p, ins, SC)
    T = T_of(p[0], p[1])
    al, be = lit(T, SC[0]), lit(T, SC[1])
    up = al * mm(S[0].T, S[0]) + be * S[1].astype(LD)
    ar = gam(N + 2, U[T]) * (abs(al) * amm(S[0].T, S[0]) + np.abs(be * S[1]))
    iu = np.triu_indices(M)
    check(F[1][iu], up[iu], ar[iu], T, p[1], "syrk C (upper)")
    assert np.array_equal(F[1], F[1].T)                   # lower = mirror of upper


def pin_syr2k(dims, p, ins):
    N, M = dims
    F, S = run("syr2k", dims, p, ins, SC)
    T = T_of(*p)
    al, be = lit(T, SC[0]), lit(T, SC[1])
    A, B, C0 = S[0], S[1], S[2]
    c1 = al * mm(A.T, B) + be * C0.astype(LD)
    e1 = gam(N + 2, U[T]) * (abs(al) * amm(A.T, B) + np.abs(be * C0))
    e1 = e1 + store_err(T, p[2], np.abs(c1).astype(np.float64) + e1)
    ex = c1 + al * mm(B.T, A)
    ar = e1 + gam(N + 2, U[T]) * (abs(al) * amm(B.T, A) + np.abs(c1).astype(np.float64) + e1)
    check(F[2], ex, ar, T, p[2], "syr2k C")


CONV2D_C = [0.2, -0.3, 0.4, 0.5, 0.6, 0.7, -0.8, -0.9, 0.10]
DI2 = [-1, 0, 1, -1, 0, 1, -1, 0, 1]
DJ2 = [-1, -1, -1, 0, 0, 0, 1, 1, 1]


def pin_conv2d(dims, p, ins):
    NI, NJ = dims
    F, S = run("conv2d", dims, p, ins)
    T = T_of(*p)
    A = S[0].astype(LD)
    ex = np.zeros((NI - 2, NJ - 2), LD)
    mag = np.zeros((NI - 2, NJ - 2), np.float64)
    for c, di, dj in zip(CONV2D_C, DI2, DJ2):
        t = lit(T, c) * A[1 + di:NI - 1 + di, 1 + dj:NJ - 1 + dj]
        ex += t
        mag += np.abs(t).astype(np.float64)
    check(F[1][1:-1, 1:-1], ex, gam(10, U[T]) * mag, T, p[1], "conv2d interior")
    border = F[1].copy()
    border[1:-1, 1:-1] = 0
    assert not border.any()


def pin_conv3d(dims, p, ins):
    NI, NJ, NK = dims
    F, S = run("conv3d", dims, p, ins)
    T = T_of(*p)
    A = S[0].reshape(NI, NJ, NK).astype(LD)
    ex = np.zeros((NI - 2, NJ - 2, NK - 2), LD)
    mag = np.zeros(ex.shape, np.float64)
    for q, g in enumerate((0.25, 0.5, 0.25)):
        for k, c in enumerate(CONV2D_C):
            di, dj, dk = q - 1, k % 3 - 1, k // 3 - 1
            t = lit(T, g * c) * A[1 + di:NI - 1 + di, 1 + dj:NJ - 1 + dj, 1 + dk:NK - 1 + dk]
            ex += t
            mag += np.abs(t).astype(np.float64)
    out = F[1].reshape(NI, NJ, NK)
    check(out[1:-1, 1:-1, 1:-1], ex, gam(28, U[T]) * mag, T, p[1], "conv3d interior")
    border = out.copy()
    border[1:-1, 1:-1, 1:-1] = 0
    assert not border.any()


def pin_fdtd2d(dims, p, ins):
    """Per time step: state t+1 (a run of t+1 steps) against one exact step applied
    to state t (a run of t steps) -- the runs share their first t steps."""
    TM, NX, NY = dims
    objs = oracle.app_objects("fdtd2d", dims)
    fict = stored(ins[0], p[0])[0]
    state = [None, stored(ins[1], p[1]).reshape(NX, NY), stored(ins[2], p[2]).reshape(NX, NY),
             stored(ins[3], p[3]).reshape(NX, NY)]
    T1, T2, T3, T4 = T_of(p[0], p[2]), T_of(p[2], p[3]), T_of(p[1], p[3]), T_of(p[3], p[1], p[2])
    for t in range(TM):
        d = [t + 1, NX, NY]
        sub = [ins[0][:, :t + 1], ins[1], ins[2], ins[3]]
        F, _ = run("fdtd2d", d, p, sub)
        ex0, ey0, hz0 = (state[k].astype(LD) for k in (1, 2, 3))
        ex1, ey1, hz1 = F[1], F[2], F[3]
        check(ey1[0], np.full(NY, fict[t], LD), np.zeros(NY), T1, p[2], "fdtd ey[0] = fict[t]")
        e_ey = ey0[1:] - LD(0.5) * (hz0[1:] - hz0[:-1])
        a_ey = gam(3, U[T2]) * (np.abs(ey0[1:]) + 0.5 * (np.abs(hz0[1:]) + np.abs(hz0[:-1]))).astype(np.float64)
        check(ey1[1:], e_ey, a_ey, T2, p[2], "fdtd ey step %d" % t)
        e_ex = ex0[:, 1:] - LD(0.5) * (hz0[:, 1:] - hz0[:, :-1])
        a_ex = gam(3, U[T3]) * (np.abs(ex0[:, 1:]) + 0.5 * (np.abs(hz0[:, 1:]) + np.abs(hz0[:, :-1]))).astype(np.float64)
        check(ex1[:, 1:], e_ex, a_ex, T3, p[1], "fdtd ex step %d" % t)
        assert np.array_equal(ex1[:, 0], state[1][:, 0])
        c4 = lit(T4, 0.7)
        X, Y = ex1.astype(LD), ey1.astype(LD)
        s = (X[:-1, 1:] - X[:-1, :-1]) + Y[1:, :-1] - Y[:-1, :-1]
        sa = (np.abs(X[:-1, 1:]) + np.abs(X[:-1, :-1]) + np.abs(Y[1:, :-1]) + np.abs(Y[:-1, :-1])).astype(np.float64)
        e_hz = hz0[:-1, :-1] - c4 * s
        a_hz = gam(5, U[T4]) * (np.abs(hz0[:-1, :-1]).astype(np.float64) + c4 * sa)
        check(F[3][:-1, :-1], e_hz, a_hz, T4, p[3], "fdtd hz step %d" % t)
        assert np.array_equal(F[3][-1], state[3][-1]) and np.array_equal(F[3][:, -1], state[3][:, -1])
        state = [None, ex1, ey1, hz1]


PINS = {
    "gemm": (pin_gemm, [13, 17, 21]),
    "2mm": (pin_2mm, [9, 14, 11, 7]),
    "3mm": (pin_3mm, [6, 9, 8, 10, 7]),
    "atax": (pin_atax, [270, 300]),
    "bicg": (pin_bicg, [261, 290]),
    "gesummv": (pin_gesummv, [300]),
    "mvt": (pin_mvt, [290]),
    "corr": (pin_corr, [60, 23]),
    "covar": (pin_covar, [55, 19]),
    "syrk": (pin_syrk, [31, 18]),
    "syr2k": (pin_syr2k, [27, 15]),
    "conv2d": (pin_conv2d, [17, 23]),
    "conv3d": (pin_conv3d, [7, 9, 11]),
    "fdtd2d": (pin_fdtd2d, [4, 13, 17]),
}


@pytest.mark.parametrize("kind", sorted(PINS))
def test_every_statement_within_its_rounding_bound(oracle_lib, kind):
    """All 3^M configurations (f64 / f32 / f16 objects), random inputs (P:160 Random
    set, values 0-1), every statement against its exact value on the stored operands."""
    fn, dims = PINS[kind]
    objs = oracle.app_objects(kind, dims)
    ins = gen.make_inputs(kind, objs, "random", seed=9)
    for prec in itertools.product([F64, F32, F16], repeat=len(objs)):
        fn(dims, list(prec), ins)


def test_bounds_catch_planted_mistakes(oracle_lib):
    """The bounds are tight enough to see the mistakes they exist for: a dropped
    term, a transposed operand, a sign flip and an unrounded store all fail."""
    dims = [13, 17, 21]
    objs = oracle.app_objects("gemm", dims)
    ins = gen.make_inputs("gemm", objs, "random", seed=9)
    p = [F32, F32, F16]
    F, S = run("gemm", dims, p, ins, SC)
    T = F32
    al, be = lit(T, SC[0]), lit(T, SC[1])
    ar = gam(23, U[T]) * (abs(al) * amm(S[0], S[1]) + np.abs(be * S[2]))
    good = al * mm(S[0], S[1]) + be * S[2].astype(LD)
    check(F[2], good, ar, T, p[2], "reference")
    A_drop = S[0].copy()
    A_drop[:, 5] = 0
    planted = [al * mm(A_drop, S[1]) + be * S[2].astype(LD),                # dropped k = 5
               al * mm(S[0], S[1][::-1]) + be * S[2].astype(LD),            # wrong index order
               al * mm(S[0], S[1]) - be * S[2].astype(LD)]                  # sign error
    for bad in planted:
        with pytest.raises(AssertionError):
            check(F[2], bad, ar, T, p[2], "planted")
    with pytest.raises(AssertionError):         # f32 value where R1 stores f16
        F32res, _ = run("gemm", dims, [F32, F32, F32], ins, SC)
        check(F32res[2], good, np.zeros_like(ar), T, F32, "unrounded store")
        check(F[2], good, np.zeros_like(ar), T, F32, "f16 result vs exact without its store error")
