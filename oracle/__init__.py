"""ctypes wrapper around the serial CPU oracle (oracle/hccmf_oracle.c).

TEST INFRASTRUCTURE ONLY.  Only tests/, ``__graft_entry__.smoke()`` and bench.py's
``cpu_baseline`` / ``--impl reference`` legs may import this module.  The product
package ``paper_conf_icpp_huangylhbl21_b200`` never imports it, and it imports
nothing from the product package: the two share no code (only the seeded input
generators in ``synth/`` feed both).

Every function forwards to the C oracle, which follows PAPER.md
(Huang et al., ICPP '21) step by step in fp64; see the C file's header for the
per-function citations and DESIGN.md section 3 for the readings of the paper.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "hccmf_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

# strict IEEE build: no contraction of a*b+c into FMA, no fast-math, no OpenMP
CFLAGS = ["-O2", "-ffp-contract=off", "-fno-fast-math", "-std=c99", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (strict fp).  Returns the .so path."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        P = ctypes.c_void_p
        i32, i64, u64, f64 = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_double
        sig = {
            "orc_splitmix": (u64, [u64]),
            "orc_hash": (u64, [u64, u64, u64, u64]),
            "orc_uniform": (f64, [u64]),
            "orc_perm": (ctypes.c_int, [u64, u64, i64, P]),
            "orc_perm_balanced": (ctypes.c_int, [i64, i64, P, i32, P]),
            "orc_dp0": (None, [i32, P, P]),
            "orc_dp0_affine": (None, [i32, P, P, P]),
            "orc_dp1": (i32, [i32, P, P, P]),
            "orc_dp2": (None, [i32, P, P, f64, P]),
            "orc_row_prefix": (None, [i64, i64, P, P, P]),
            "orc_bounds": (None, [i64, i64, P, i32, P, P]),
            "orc_block_sort": (ctypes.c_int, [i64, i64, i64, P, P, P, i32, i32, i32, P, P, P, u64, P, P, P, P]),
            "orc_init": (None, [u64, i64, i64, i32, P, P, P, P]),
            "orc_sgd_update": (f64, [i32, f64, f64, P, P, f64]),
            "orc_run": (None, [i64, i64, i32, f64, f64, P, P, P, P, P]),
            "orc_epoch": (ctypes.c_int, [i32, i32, i32, i32, i32, P, i64, i32, f64, f64, P, P, P, P, P]),
            "orc_rmse": (f64, [i64, P, P, P, i32, P, P, P, P]),
            "orc_objective": (f64, [i64, P, P, P, i32, f64, P, P, P, P]),
            "orc_unpermute": (None, [i64, i32, P, P, P]),
            "orc_epoch_phased": (ctypes.c_int, [i32, i32, i32, i32, P, i64, i32, f64, f64, P, P, P, P, P]),
            "orc_round_half": (f64, [f64]),
            "orc_epoch_wire16": (ctypes.c_int, [i32, i32, i32, i32, i32, P, i64, i32, f64, f64, P, P, P, P, P]),
            "orc_epoch_q16": (ctypes.c_int, [i32, i32, i32, i32, i32, P, i64, i32, f64, f64, P, P, P, P, P, i32, i32,
                                             ctypes.c_uint32]),
            "orc_round_half_sr": (f64, [f64, ctypes.c_uint32]),
            "orc_sr_word": (ctypes.c_uint32, [i64, ctypes.c_uint32, ctypes.c_uint32]),
            "orc_cost_model": (i32, [i32, i64, i64, i64, i32, P, P, f64, i32, i32, i32, f64, P, P, P, P]),
        }
        for name, (res, args) in sig.items():
            fn = getattr(L, name)
            fn.restype = res
            fn.argtypes = args
        _lib = L
    return _lib


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"], "oracle arrays must be C-contiguous"
    return a.ctypes.data_as(ctypes.c_void_p)


def _i32(a):
    return np.ascontiguousarray(a, dtype=np.int32)


def _f32(a):
    return np.ascontiguousarray(a, dtype=np.float32)


def _f64(a):
    return np.ascontiguousarray(a, dtype=np.float64)


# ---------------------------------------------------------------- hash / perm
def splitmix(x: int) -> int:
    return int(lib().orc_splitmix(x))


def hash4(seed: int, tag: int, a: int, b: int) -> int:
    return int(lib().orc_hash(seed, tag, a, b))


def uniform(h: int) -> float:
    return float(lib().orc_uniform(h))


def perm(seed: int, tag: int, count: int) -> np.ndarray:
    out = np.empty(max(count, 0), dtype=np.int32)
    rc = lib().orc_perm(seed, tag, count, _p(out))
    assert rc == 0
    return out


def perm_balanced(n: int, v, B: int) -> np.ndarray:
    """Degree-balanced column permutation (R30): v' of every item."""
    vv = _i32(v)
    out = np.empty(n, dtype=np.int32)
    rc = lib().orc_perm_balanced(n, len(vv), _p(vv), B, _p(out))
    assert rc == 0
    return out


# ------------------------------------------------------------------ partition
def dp0(t_e) -> np.ndarray:
    t = _f64(t_e)
    x = np.empty_like(t)
    lib().orc_dp0(len(t), _p(t), _p(x))
    return x


def dp0_affine(a, b) -> np.ndarray:
    a, b = _f64(a), _f64(b)
    x = np.empty_like(a)
    lib().orc_dp0_affine(len(a), _p(a), _p(b), _p(x))
    return x


def dp1(x, t):
    x, t = _f64(x), _f64(t)
    out = np.empty_like(x)
    it = lib().orc_dp1(len(x), _p(x), _p(t), _p(out))
    return out, int(it)


def dp2(x, t, t_sync: float) -> np.ndarray:
    x, t = _f64(x), _f64(t)
    out = np.empty_like(x)
    lib().orc_dp2(len(x), _p(x), _p(t), float(t_sync), _p(out))
    return out


def cost_model(m, n, nnz, k, B, Bbus, B_server, t=1, q_only=1, elem=4, lambda_sync=10.0):
    """Eq. 1-5 time cost model; returns (x, T_i, T_sync, T, branch) with branch 1 = DP1, 2 = DP2."""
    B, Bbus = _f64(B), _f64(Bbus)
    p = len(B)
    x = np.empty(p)
    Ti = np.empty(p)
    Ts = ctypes.c_double()
    T = ctypes.c_double()
    br = lib().orc_cost_model(p, m, n, nnz, k, _p(B), _p(Bbus), B_server, t, q_only, elem, lambda_sync, _p(x),
                              _p(Ti), ctypes.byref(Ts), ctypes.byref(T))
    return x, Ti, Ts.value, T.value, int(br)


def row_prefix(m: int, u, perm_row) -> np.ndarray:
    u, pr = _i32(u), _i32(perm_row)
    S = np.empty(m + 1, dtype=np.int64)
    lib().orc_row_prefix(m, len(u), _p(u), _p(pr), _p(S))
    return S


def bounds(m: int, nnz: int, S, G: int, x) -> np.ndarray:
    S = np.ascontiguousarray(S, dtype=np.int64)
    x = _f64(x)
    b = np.empty(G + 1, dtype=np.int32)
    lib().orc_bounds(m, nnz, _p(S), G, _p(x), _p(b))
    return b


def block_sort(m, n, u, v, r, G, Br, Bc, b, perm_row, perm_col, seed=0):
    u, v, r = _i32(u), _i32(v), _f32(r)
    b, pr, pc = _i32(b), _i32(perm_row), _i32(perm_col)
    nnz = len(u)
    ou = np.empty(nnz, np.int32)
    ov = np.empty(nnz, np.int32)
    orr = np.empty(nnz, np.float32)
    off = np.empty(G * Br * Bc + 1, np.int64)
    rc = lib().orc_block_sort(m, n, nnz, _p(u), _p(v), _p(r), G, Br, Bc, _p(b), _p(pr), _p(pc), seed,
                              _p(ou), _p(ov), _p(orr), _p(off))
    assert rc == 0
    return ou, ov, orr, off


# ---------------------------------------------------------------- SGD / eval
def init(seed, m, n, k, perm_row, perm_col):
    P = np.empty((m, k), np.float64)
    Q = np.empty((n, k), np.float64)
    lib().orc_init(seed, m, n, k, _p(_i32(perm_row)), _p(_i32(perm_col)), _p(P), _p(Q))
    return P, Q


def sgd_update(gamma, lam, p, q, r):
    """One update in place on fp64 vectors p, q; returns e."""
    assert p.dtype == np.float64 and q.dtype == np.float64
    return float(lib().orc_sgd_update(len(p), gamma, lam, _p(p), _p(q), float(r)))


def run(lo, hi, k, gamma, lam, ru, rv, rr, P, Q):
    lib().orc_run(lo, hi, k, gamma, lam, _p(ru), _p(rv), _p(rr), _p(P), _p(Q))


SCHED = {"det": 0, "serial": 1, "hogwild": 1}
SYNC = {"none": 0, "ring": 1, "allreduce": 2}


def epoch(sched, sync, G, Br, Bc, off, n, k, gamma, lam, ru, rv, rr, P, Q):
    """One epoch in place on fp64 P (m x k) and Q (n x k), permuted-id order."""
    assert P.dtype == np.float64 and Q.dtype == np.float64
    off = np.ascontiguousarray(off, dtype=np.int64)
    rc = lib().orc_epoch(SCHED[sched], SYNC[sync], G, Br, Bc, _p(off), n, P.shape[1], gamma, lam,
                         _p(ru), _p(rv), _p(rr), _p(P), _p(Q))
    if rc != 0:
        raise ValueError("oracle epoch: invalid grid for this schedule")


def epoch_phased(G, Br, Bc, phases, off, n, k, gamma, lam, ru, rv, rr, P, Q):
    """All-reduce epoch with `phases` sub-epoch syncs (serial inside each replica)."""
    off = np.ascontiguousarray(off, dtype=np.int64)
    rc = lib().orc_epoch_phased(G, Br, Bc, phases, _p(off), n, P.shape[1], gamma, lam, _p(ru), _p(rv), _p(rr),
                                _p(P), _p(Q))
    if rc != 0:
        raise ValueError("oracle phased epoch: Br must be a multiple of phases")


def round_half(x: float) -> float:
    return float(lib().orc_round_half(float(x)))


def round_half_sr(x: float, r13: int) -> float:
    return float(lib().orc_round_half_sr(float(x), int(r13)))


def sr_word(i: int, t: int, c: int) -> int:
    return int(lib().orc_sr_word(int(i), int(t), int(c)))


def epoch_wire16(sched, sync, G, Br, Bc, off, n, k, gamma, lam, ru, rv, rr, P, Q):
    """Ring / all-reduce epoch with FP16 transmission of Q (Strategy 2, R25)."""
    off = np.ascontiguousarray(off, dtype=np.int64)
    rc = lib().orc_epoch_wire16(SCHED[sched], SYNC[sync], G, Br, Bc, _p(off), n, P.shape[1], gamma, lam, _p(ru),
                                _p(rv), _p(rr), _p(P), _p(Q))
    if rc != 0:
        raise ValueError("oracle wire16 epoch: invalid grid or sync")


def epoch_q16(sched, sync, G, Br, Bc, off, n, k, gamma, lam, ru, rv, rr, P, Q, add16=False, sr=False, t=0):
    """Epoch with Q stored in binary16 (every q_v write rounded; add16: the write is a
    binary16 add of the rounded increment, as atomic Hogwild does; R26; sr:
    stochastic rounding with the random words of epoch t, R27)."""
    off = np.ascontiguousarray(off, dtype=np.int64)
    rc = lib().orc_epoch_q16(SCHED[sched], SYNC[sync], G, Br, Bc, _p(off), n, P.shape[1], gamma, lam, _p(ru),
                             _p(rv), _p(rr), _p(P), _p(Q), int(bool(add16)), int(bool(sr)), int(t))
    if rc != 0:
        raise ValueError("oracle q16 epoch: invalid grid for this schedule")


def rmse(tu, tv, tr, perm_row, perm_col, P, Q) -> float:
    tu, tv, tr = _i32(tu), _i32(tv), _f32(tr)
    return float(lib().orc_rmse(len(tu), _p(tu), _p(tv), _p(tr), P.shape[1], _p(_i32(perm_row)),
                                _p(_i32(perm_col)), _p(P), _p(Q)))


def objective(u, v, r, lam, perm_row, perm_col, P, Q) -> float:
    u, v, r = _i32(u), _i32(v), _f32(r)
    return float(lib().orc_objective(len(u), _p(u), _p(v), _p(r), P.shape[1], lam, _p(_i32(perm_row)),
                                     _p(_i32(perm_col)), _p(P), _p(Q)))


def unpermute(perm_, Xp) -> np.ndarray:
    X = np.empty_like(Xp)
    lib().orc_unpermute(Xp.shape[0], Xp.shape[1], _p(_i32(perm_)), _p(Xp), _p(X))
    return X


class Problem:
    """Convenience: the whole oracle pipeline for one problem (tests only)."""

    def __init__(self, m, n, k, gamma, lam, u, v, r, G=1, Br=1, Bc=1, seed=0, x=None, col_balance=0):
        self.m, self.n, self.k, self.gamma, self.lam = m, n, k, gamma, lam
        self.u, self.v, self.r = _i32(u), _i32(v), _f32(r)
        self.G, self.Br, self.Bc = G, Br, Bc
        self.perm_row = perm(seed, 1, m)
        self.perm_col = perm_balanced(n, self.v, Bc) if col_balance else perm(seed, 2, n)
        self.S = row_prefix(m, self.u, self.perm_row)
        self.x = np.full(G, 1.0 / G) if x is None else _f64(x)
        self.b = bounds(m, len(self.u), self.S, G, self.x)
        self.ru, self.rv, self.rr, self.off = block_sort(m, n, self.u, self.v, self.r, G, Br, Bc, self.b,
                                                         self.perm_row, self.perm_col, seed)
        self.P = None
        self.Q = None

    def init(self, seed):
        self.P, self.Q = init(seed, self.m, self.n, self.k, self.perm_row, self.perm_col)

    def set_factors(self, P_orig, Q_orig):
        """Factors given in ORIGINAL id order (as hccmf_set_factors takes them)."""
        self.P = np.empty((self.m, self.k), np.float64)
        self.Q = np.empty((self.n, self.k), np.float64)
        self.P[self.perm_row] = np.asarray(P_orig, np.float64)
        self.Q[self.perm_col] = np.asarray(Q_orig, np.float64)

    def epoch(self, sched="det", sync="none"):
        epoch(sched, sync, self.G, self.Br, self.Bc, self.off, self.n, self.k, self.gamma, self.lam,
              self.ru, self.rv, self.rr, self.P, self.Q)

    def epoch_q16(self, sched="det", sync="none", add16=False, sr=False, t=0):
        epoch_q16(sched, sync, self.G, self.Br, self.Bc, self.off, self.n, self.k, self.gamma, self.lam,
                  self.ru, self.rv, self.rr, self.P, self.Q, add16, sr, t)

    def epoch_wire16(self, sched="det", sync="ring"):
        epoch_wire16(sched, sync, self.G, self.Br, self.Bc, self.off, self.n, self.k, self.gamma, self.lam,
                     self.ru, self.rv, self.rr, self.P, self.Q)

    def epoch_phased(self, phases):
        epoch_phased(self.G, self.Br, self.Bc, phases, self.off, self.n, self.k, self.gamma, self.lam, self.ru,
                     self.rv, self.rr, self.P, self.Q)

    def factors(self):
        return unpermute(self.perm_row, self.P), unpermute(self.perm_col, self.Q)

    def rmse(self, tu, tv, tr):
        return rmse(tu, tv, tr, self.perm_row, self.perm_col, self.P, self.Q)
