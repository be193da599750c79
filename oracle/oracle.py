"""ctypes front-end of the plain C oracle (oracle/aabft_oracle.c).

TEST INFRASTRUCTURE ONLY: only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs may import this module.  It performs
argument marshalling only; every step of the method is in aabft_oracle.c, which
cites the PAPER.md passage it follows.  It never imports the CUDA package.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "aabft_oracle.c")
LIB = os.path.join(HERE, "libaabft_oracle.so")
CFLAGS = ["-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-pthread", "-shared",
          "-fPIC", "-Wall"]

STATUS_NAMES = {0: "CLEAN", 1: "CORRECTED", 2: "CHECKSUM_ONLY", 3: "UNCORRECTABLE", 4: "SINGLE"}

_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(LIB) or os.path.getmtime(LIB) < os.path.getmtime(SRC):
        subprocess.check_call(["gcc", *CFLAGS, "-o", LIB, SRC, "-lm"])
    return LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        i64, i32, dbl, vp = C.c_int64, C.c_int, C.c_double, C.c_void_p
        L.oracle_encode_cols.argtypes = [i32, i64, i64, i32, vp, i64, vp, i64]
        L.oracle_encode_rows.argtypes = [i32, i64, i64, i32, vp, i64, vp, i64]
        L.oracle_topp_vector.argtypes = [i32, vp, i64, i64, i32, vp, vp]
        L.oracle_topp_rows.argtypes = [i32, i64, i64, i32, i32, vp, i64, vp, i64, vp, vp]
        L.oracle_topp_cols.argtypes = [i32, i64, i64, i32, i32, vp, i64, vp, i64, vp, vp]
        L.oracle_gemm.argtypes = [i32, i32, i64, i64, i64, vp, i64, vp, i64, vp, i64, i32]
        L.oracle_dot_fault.argtypes = [i32, i32, i64, vp, vp, i64, i32, i64, C.c_uint64, dbl]
        L.oracle_dot_fault.restype = dbl
        L.oracle_y.argtypes = [i32, vp, vp, vp, vp]
        L.oracle_y.restype = dbl
        L.oracle_sigma_coeff.argtypes = [i64, i32]
        L.oracle_sigma_coeff.restype = dbl
        L.oracle_bound.argtypes = [i64, i32, i32, dbl, dbl, vp, vp]
        L.oracle_bounds_all.argtypes = [i64, i64, i64, i32, i32, dbl, i32, i32, vp, vp, vp, vp,
                                        vp, vp, vp, vp]
        L.oracle_check.argtypes = [i32, i64, i64, i64, i32, i32, dbl, i32, i32, vp, i64, vp, i64,
                                   vp, i64, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp,
                                   vp, vp]
        L.oracle_correct.argtypes = [i32, i64, i64, i64, i32, i32, dbl, i32, i32, vp, i64, vp,
                                     i64, vp, i64, vp, vp, vp, vp, vp, vp, vp, vp]
        L.oracle_check_ext.argtypes = [i32, i64, i64, i32, vp, i64, vp, i64, vp, i64, vp, vp, dbl,
                                       vp, vp, vp, vp, vp, vp, vp, vp, vp, vp, vp]
        L.oracle_correct_ext.argtypes = [i32, i64, i64, i32, vp, i64, vp, i64, vp, i64, vp, dbl,
                                         vp, vp, vp, vp]
        L.oracle_norms_rows.argtypes = [i32, i64, i64, vp, i64, vp]
        L.oracle_norms_cols.argtypes = [i32, i64, i64, vp, i64, vp]
        L.oracle_sea_bounds.argtypes = [i64, i64, i64, i32, i32, vp, vp, vp, vp, vp, vp, vp]
        _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _dt(a) -> int:
    if a.dtype == np.float64:
        return 0
    if a.dtype == np.float32:
        return 1
    raise TypeError("oracle supports float64 / float32 only")


def _c(a):
    return np.ascontiguousarray(a)


def default_t(dtype) -> int:
    """Reading R1: t = 52 (FP64) / 23 (FP32), eps_M = 2^-t."""
    return 52 if np.dtype(dtype) == np.float64 else 23


# ---------------------------------------------------------------- steps (O2..O8)
def encode_cols(A, bs):
    A = _c(A)
    M, K = A.shape
    Acs = np.zeros((M // bs, K), dtype=A.dtype)
    lib().oracle_encode_cols(_dt(A), M, K, bs, _p(A), K, _p(Acs), K)
    return Acs


def encode_rows(B, bs):
    B = _c(B)
    K, N = B.shape
    Bcs = np.zeros((K, N // bs), dtype=B.dtype)
    lib().oracle_encode_rows(_dt(B), K, N, bs, _p(B), N, _p(Bcs), N // bs)
    return Bcs


def topp_vector(x, p):
    x = _c(x)
    val = np.zeros(p, dtype=np.float64)
    idx = np.zeros(p, dtype=np.int32)
    lib().oracle_topp_vector(_dt(x), _p(x), x.shape[0], 1, p, _p(val), _p(idx))
    return val, idx


def topp_rows(A, Acs, bs, p):
    A, Acs = _c(A), _c(Acs)
    M, K = A.shape
    val = np.zeros((M + M // bs, p), dtype=np.float64)
    idx = np.zeros((M + M // bs, p), dtype=np.int32)
    lib().oracle_topp_rows(_dt(A), M, K, bs, p, _p(A), K, _p(Acs), K, _p(val), _p(idx))
    return val, idx


def topp_cols(B, Bcs, bs, p):
    B, Bcs = _c(B), _c(Bcs)
    K, N = B.shape
    val = np.zeros((N + N // bs, p), dtype=np.float64)
    idx = np.zeros((N + N // bs, p), dtype=np.int32)
    lib().oracle_topp_cols(_dt(B), K, N, bs, p, _p(B), N, _p(Bcs), N // bs, _p(val), _p(idx))
    return val, idx


def gemm(A, B, fma_model=1, nthreads=None):
    A, B = _c(A), _c(B)
    M, K = A.shape
    K2, N = B.shape
    assert K == K2 and A.dtype == B.dtype
    Cm = np.zeros((M, N), dtype=A.dtype)
    nt = nthreads or os.cpu_count() or 1
    lib().oracle_gemm(_dt(A), fma_model, M, N, K, _p(A), K, _p(B), N, _p(Cm), N, nt)
    return Cm


def dot_fault(a, b, fma_model=1, site=-1, k_step=0, xor_mask=0, add=0.0):
    """One element sum_k a[k]*b[k] (ascending k) with an Alg-3 style fault (site -1: none)."""
    a, b = _c(a), _c(b)
    return lib().oracle_dot_fault(_dt(a), fma_model, a.shape[0], _p(a), _p(b), 1, site, k_step,
                                  C.c_uint64(xor_mask), add)


def y_of(va, ia, vb, ib):
    va, vb = _c(np.asarray(va, np.float64)), _c(np.asarray(vb, np.float64))
    ia, ib = _c(np.asarray(ia, np.int32)), _c(np.asarray(ib, np.int32))
    return lib().oracle_y(va.shape[0], _p(va), _p(ia), _p(vb), _p(ib))


def sigma_coeff(n, fma_model=1):
    return lib().oracle_sigma_coeff(n, fma_model)


def bound(n, y, *, fma_model=1, t=52, omega=3.0):
    sg = np.zeros(1)
    e = np.zeros(1)
    lib().oracle_bound(n, fma_model, t, omega, y, _p(sg), _p(e))
    return float(sg[0]), float(e[0])


def bounds_all(M, N, K, bs, p, topA, topB, *, omega=3.0, t=52, fma_model=1):
    (av, ai), (bv, bi) = topA, topB
    eps_col = np.zeros((M // bs, N))
    sig_col = np.zeros((M // bs, N))
    eps_row = np.zeros((M, N // bs))
    sig_row = np.zeros((M, N // bs))
    lib().oracle_bounds_all(M, N, K, bs, p, omega, t, fma_model, _p(_c(av)), _p(_c(ai)),
                            _p(_c(bv)), _p(_c(bi)), _p(eps_col), _p(sig_col), _p(eps_row),
                            _p(sig_row))
    return dict(eps_col=eps_col, sig_col=sig_col, eps_row=eps_row, sig_row=sig_row)


@dataclass
class CheckResult:
    status: np.ndarray
    worst: np.ndarray
    nrows: np.ndarray
    ncols: np.ndarray
    row: np.ndarray
    col: np.ndarray
    ratio: np.ndarray
    counts: np.ndarray
    max_ratio: float
    d_col: np.ndarray
    d_row: np.ndarray
    extra: dict = field(default_factory=dict)


def check(Cm, Ccol, Crow, K, bs, p, topA, topB, *, omega=3.0, t=None, fma_model=1):
    Cm, Ccol, Crow = _c(Cm), _c(Ccol), _c(Crow)
    M, N = Cm.shape
    t = default_t(Cm.dtype) if t is None else t
    nb = (M // bs) * (N // bs)
    ints = [np.zeros(nb, np.int32) for _ in range(6)]
    ratio = np.zeros(nb)
    counts = np.zeros(8, np.int64)
    mr = np.zeros(1)
    d_col = np.zeros((M // bs, N))
    d_row = np.zeros((M, N // bs))
    (av, ai), (bv, bi) = topA, topB
    lib().oracle_check(_dt(Cm), M, N, K, bs, p, omega, t, fma_model, _p(Cm), N, _p(Ccol), N,
                       _p(Crow), N // bs, _p(_c(av)), _p(_c(ai)), _p(_c(bv)), _p(_c(bi)),
                       *[_p(x) for x in ints], _p(ratio), _p(counts), _p(mr), _p(d_col),
                       _p(d_row))
    shp = (M // bs, N // bs)
    return CheckResult(*(x.reshape(shp) for x in ints), ratio.reshape(shp), counts,
                       float(mr[0]), d_col, d_row)


def correct(Cm, Ccol, Crow, K, bs, p, topA, topB, res: CheckResult, *, omega=3.0, t=None,
            fma_model=1):
    """In-place correction of Cm; updates res.status / res.counts."""
    assert Cm.flags.c_contiguous
    M, N = Cm.shape
    t = default_t(Cm.dtype) if t is None else t
    (av, ai), (bv, bi) = topA, topB
    st = _c(res.status.reshape(-1)).copy()
    lib().oracle_correct(_dt(Cm), M, N, K, bs, p, omega, t, fma_model, _p(Cm), N,
                         _p(_c(Ccol)), N, _p(_c(Crow)), N // bs, _p(_c(av)), _p(_c(ai)),
                         _p(_c(bv)), _p(_c(bi)), _p(st), _p(_c(res.row.reshape(-1))),
                         _p(_c(res.col.reshape(-1))), _p(res.counts))
    res.status = st.reshape(res.status.shape)
    return res


def check_ext(Cm, Ccol, Crow, bs, *, eps_col=None, eps_row=None, eps_fixed=0.0):
    """O7 against an external eps (NEXT-3, reading R26): per-checksum eps arrays (e.g. SEA) or
    one fixed eps for every check."""
    Cm, Ccol, Crow = _c(Cm), _c(Ccol), _c(Crow)
    M, N = Cm.shape
    nb = (M // bs) * (N // bs)
    ints = [np.zeros(nb, np.int32) for _ in range(6)]
    ratio = np.zeros(nb)
    counts = np.zeros(8, np.int64)
    mr = np.zeros(1)
    d_col = np.zeros((M // bs, N))
    d_row = np.zeros((M, N // bs))
    ec = None if eps_col is None else _c(np.asarray(eps_col, np.float64))
    er = None if eps_row is None else _c(np.asarray(eps_row, np.float64))
    lib().oracle_check_ext(_dt(Cm), M, N, bs, _p(Cm), N, _p(Ccol), N, _p(Crow), N // bs, _p(ec),
                           _p(er), float(eps_fixed), *[_p(x) for x in ints], _p(ratio),
                           _p(counts), _p(mr), _p(d_col), _p(d_row))
    shp = (M // bs, N // bs)
    return CheckResult(*(x.reshape(shp) for x in ints), ratio.reshape(shp), counts,
                       float(mr[0]), d_col, d_row)


def correct_ext(Cm, Ccol, Crow, bs, res: CheckResult, *, eps_row=None, eps_fixed=0.0):
    assert Cm.flags.c_contiguous
    M, N = Cm.shape
    st = _c(res.status.reshape(-1)).copy()
    er = None if eps_row is None else _c(np.asarray(eps_row, np.float64))
    lib().oracle_correct_ext(_dt(Cm), M, N, bs, _p(Cm), N, _p(_c(Ccol)), N, _p(_c(Crow)), N // bs,
                             _p(er), float(eps_fixed), _p(st), _p(_c(res.row.reshape(-1))),
                             _p(_c(res.col.reshape(-1))), _p(res.counts))
    res.status = st.reshape(res.status.shape)
    return res


def norms_rows(X):
    X = _c(X)
    R, L = X.shape
    out = np.zeros(R)
    lib().oracle_norms_rows(_dt(X), R, L, _p(X), L, _p(out))
    return out


def norms_cols(X):
    X = _c(X)
    L, Cn = X.shape
    out = np.zeros(Cn)
    lib().oracle_norms_cols(_dt(X), L, Cn, _p(X), Cn, _p(out))
    return out


def sea_bounds(A, B, Acs, Bcs, bs, *, t=None):
    """O11 SEA-ABFT comparator bound (§III): eps_col, eps_row and the corner."""
    M, K = A.shape
    N = B.shape[1]
    t = default_t(A.dtype) if t is None else t
    nA, nAcs, nB, nBcs = norms_rows(A), norms_rows(Acs), norms_cols(B), norms_cols(Bcs)
    eps_col = np.zeros((M // bs, N))
    eps_row = np.zeros((M, N // bs))
    eps_corner = np.zeros((M // bs, N // bs))
    lib().oracle_sea_bounds(M, N, K, bs, t, _p(nA), _p(nAcs), _p(nB), _p(nBcs), _p(eps_col),
                            _p(eps_row), _p(eps_corner))
    return dict(eps_col=eps_col, eps_row=eps_row, eps_corner=eps_corner, nA=nA, nAcs=nAcs,
                nB=nB, nBcs=nBcs)


# ---------------------------------------------------------------- whole path
def encode(A, B, bs, p):
    Acs = encode_cols(A, bs)
    Bcs = encode_rows(B, bs)
    return dict(Acs=Acs, Bcs=Bcs, topA=topp_rows(A, Acs, bs, p), topB=topp_cols(B, Bcs, bs, p))


def apply_faults(A, B, enc, Cm, Ccol, Crow, faults, fma_model=1):
    """O9: recompute each faulted C_fc element with its fault.  A fault is a dict with keys
    row, col (C_fc coordinates: row >= M -> Ccol row row-M; col >= N -> Crow col col-N),
    site (0 xor final, 1 xor after k_step, 2 add final, 3 add after k_step, 4 xor of the
    separately rounded product at k_step -- Alg 3 errorVecMul), k_step, xor_mask, add."""
    M, K = A.shape
    N = B.shape[1]
    for f in faults:
        r, c = f["row"], f["col"]
        a = enc["Acs"][r - M] if r >= M else A[r]
        b = enc["Bcs"][:, c - N] if c >= N else B[:, c]
        v = dot_fault(np.ascontiguousarray(a), np.ascontiguousarray(b), fma_model,
                      f.get("site", 0), f.get("k_step", 0), f.get("xor_mask", 0),
                      f.get("add", 0.0))
        if r >= M:
            Ccol[r - M, c] = v
        elif c >= N:
            Crow[r, c - N] = v
        else:
            Cm[r, c] = v


def protected_matmul(A, B, *, bs, p=2, omega=3.0, t=None, fma_model=1, faults=(), do_correct=True,
                     nthreads=None):
    """Full oracle path O2..O8 (+ O9 faults).  Returns dict with every intermediate."""
    t = default_t(A.dtype) if t is None else t
    enc = encode(A, B, bs, p)
    Cm = gemm(A, B, fma_model, nthreads)
    Ccol = gemm(enc["Acs"], B, fma_model, nthreads)
    Crow = gemm(A, enc["Bcs"], fma_model, nthreads)
    if faults:
        apply_faults(A, B, enc, Cm, Ccol, Crow, faults, fma_model)
    K = A.shape[1]
    res = check(Cm, Ccol, Crow, K, bs, p, enc["topA"], enc["topB"], omega=omega, t=t,
                fma_model=fma_model)
    if do_correct:
        correct(Cm, Ccol, Crow, K, bs, p, enc["topA"], enc["topB"], res, omega=omega, t=t,
                fma_model=fma_model)
    return dict(enc=enc, C=Cm, Ccol=Ccol, Crow=Crow, check=res)


def abft_matmul_ext(A, B, *, bs, mode="sea", eps_fixed=0.0, t=None, fma_model=1, faults=(),
                    do_correct=True, nthreads=None):
    """Comparator paths (NEXT-3): plain checksums (no top-p) + GEMM + check/correct against
    the SEA-ABFT bound (mode "sea") or one fixed eps (mode "fixed")."""
    enc = dict(Acs=encode_cols(A, bs), Bcs=encode_rows(B, bs))
    Cm = gemm(A, B, fma_model, nthreads)
    Ccol = gemm(enc["Acs"], B, fma_model, nthreads)
    Crow = gemm(A, enc["Bcs"], fma_model, nthreads)
    if faults:
        apply_faults(A, B, enc, Cm, Ccol, Crow, faults, fma_model)
    if mode == "sea":
        sea = sea_bounds(A, B, enc["Acs"], enc["Bcs"], bs, t=t)
        ec, er = sea["eps_col"], sea["eps_row"]
    elif mode == "fixed":
        sea, ec, er = None, None, None
    else:
        raise ValueError(mode)
    res = check_ext(Cm, Ccol, Crow, bs, eps_col=ec, eps_row=er, eps_fixed=eps_fixed)
    if do_correct:
        correct_ext(Cm, Ccol, Crow, bs, res, eps_row=er, eps_fixed=eps_fixed)
    return dict(enc=enc, C=Cm, Ccol=Ccol, Crow=Crow, check=res, sea=sea)
