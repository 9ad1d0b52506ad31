"""oracle — plain, slow, obviously-correct CPU implementation of the hot path.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  The product package ``paper_conf_icpp_wangzll21_b200`` never imports it
and shares no code with it (no kernels, headers, helpers or constants).

Two independent formulations live here:

* ``tid_oracle.c`` (C, int64, OpenMP over pairs) — the definition written out:
  direct sum of squared differences, one streaming top-2 scan per query row,
  integer ratio test, count, sort-based ranking.  Passages cited per function.
* ``np_*`` (NumPy, int64, full stable sort per row) — a second formulation used
  only to pin the C oracle on tiny inputs.

Readings where the paper is silent are listed in the C header and in DESIGN.md.
Every function here is pinned by tests/test_oracle.py (no "parity unpinned" entries).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "tid_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

DIM = 128


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def _L():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        vp, i32, i64, u32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_uint32
        lib.oracle_sqdist.argtypes = [vp, vp]
        lib.oracle_sqdist.restype = i64
        lib.oracle_dist_matrix.argtypes = [vp, i32, vp, i32, vp]
        lib.oracle_two_nn.argtypes = [vp, vp, i32, vp]
        lib.oracle_ratio_pass.argtypes = [i64, i64, i32, u32, u32]
        lib.oracle_ratio_pass.restype = ctypes.c_int
        lib.oracle_match_count.argtypes = [vp, i32, vp, i32, u32, u32, vp]
        lib.oracle_match_count.restype = i32
        lib.oracle_verify.argtypes = [vp, i32, vp, i32, i64, vp, vp, u32, u32, vp, vp]
        lib.oracle_search_counts.argtypes = [vp, vp, i32, i64, vp, vp, i32, i64, u32, u32, vp]
        lib.oracle_topk.argtypes = [vp, i64, i64, i64, i32, vp, vp]
        lib.oracle_merge_topk.argtypes = [vp, vp, i32, i64, i32, vp, vp]
        _lib = lib
    return _lib


def _c(a, dt):
    return np.ascontiguousarray(np.asarray(a), dtype=dt)


def _p(a):
    return None if a is None else a.ctypes.data


# ---------------------------------------------------------------- C oracle wrappers
def sqdist(q, r) -> int:
    q, r = _c(q, np.uint8), _c(r, np.uint8)
    assert q.shape == (DIM,) and r.shape == (DIM,)
    return int(_L().oracle_sqdist(_p(q), _p(r)))


def dist_matrix(Q, R) -> np.ndarray:
    Q, R = _c(Q, np.uint8), _c(R, np.uint8)
    D = np.empty((Q.shape[0], R.shape[0]), np.int64)
    _L().oracle_dist_matrix(_p(Q), Q.shape[0], _p(R), R.shape[0], _p(D))
    return D


def two_nn(q, R, m_r: int | None = None) -> tuple[int, int, int, int]:
    q, R = _c(q, np.uint8), _c(R, np.uint8)
    out = np.empty(4, np.int64)
    _L().oracle_two_nn(_p(q), _p(R), R.shape[0] if m_r is None else m_r, _p(out))
    return tuple(int(x) for x in out)


def ratio_pass(d1: int, d2: int, m_r: int = 2, num: int = 4, den: int = 5) -> bool:
    return bool(_L().oracle_ratio_pass(d1, d2, m_r, num, den))


def match_count(Q, R, num: int = 4, den: int = 5, n_q: int | None = None, m_r: int | None = None,
                want_nn: bool = False):
    Q, R = _c(Q, np.uint8), _c(R, np.uint8)
    nq = Q.shape[0] if n_q is None else n_q
    mr = R.shape[0] if m_r is None else m_r
    nn = np.empty((nq, 4), np.int64) if want_nn else None
    c = int(_L().oracle_match_count(_p(Q), nq, _p(R), mr, num, den, _p(nn)))
    return (c, nn) if want_nn else c


def verify(Q, R, num: int = 4, den: int = 5, n_q=None, m_r=None, want_nn: bool = True):
    """Q [P][n][128], R [P][m][128] -> counts int32 [P], nn int64 [P][n][4] (rows >= n_q[p] = -1)."""
    Q, R = _c(Q, np.uint8), _c(R, np.uint8)
    P, n, m = Q.shape[0], Q.shape[1], R.shape[1]
    nq = None if n_q is None else _c(n_q, np.int32)
    mr = None if m_r is None else _c(m_r, np.int32)
    counts = np.empty(P, np.int32)
    nn = np.full((P, n, 4), -1, np.int64) if want_nn else None
    _L().oracle_verify(_p(Q), n, _p(R), m, P, _p(nq), _p(mr), num, den, _p(counts), _p(nn))
    return counts, nn


def search_counts(Qs, Rs, num: int = 4, den: int = 5, n_q=None, kp=None) -> np.ndarray:
    """Qs [B][n][128], Rs [R][m][128] -> counts int32 [B][R]."""
    Qs, Rs = _c(Qs, np.uint8), _c(Rs, np.uint8)
    B, n = Qs.shape[0], Qs.shape[1]
    R, m = Rs.shape[0], Rs.shape[1]
    nq = None if n_q is None else _c(n_q, np.int32)
    kpa = None if kp is None else _c(kp, np.int32)
    counts = np.empty((B, R), np.int32)
    _L().oracle_search_counts(_p(Qs), _p(nq), n, B, _p(Rs), _p(kpa), m, R, num, den, _p(counts))
    return counts


def topk(counts, k: int, id_base: int = 0):
    counts = _c(counts, np.int32)
    B, R = counts.shape
    assert 0 < k <= R
    ids = np.empty((B, k), np.int64)
    cn = np.empty((B, k), np.int32)
    _L().oracle_topk(_p(counts), B, R, id_base, k, _p(ids), _p(cn))
    return ids, cn


def merge_topk(ids, cnts):
    """ids/cnts [G][B][k] -> merged [B][k] in (count desc, id asc) order."""
    ids, cnts = _c(ids, np.int64), _c(cnts, np.int32)
    G, B, k = ids.shape
    io = np.empty((B, k), np.int64)
    co = np.empty((B, k), np.int32)
    _L().oracle_merge_topk(_p(ids), _p(cnts), G, B, k, _p(io), _p(co))
    return io, co


def search(Qs, Rs, k: int, num: int = 4, den: int = 5, n_q=None, kp=None, id_base: int = 0):
    c = search_counts(Qs, Rs, num, den, n_q, kp)
    ids, cn = topk(c, k, id_base)
    return ids, cn, c


# ------------------------------------------------------- NumPy brute force (2nd formulation)
def np_dist_matrix(Q, R) -> np.ndarray:
    """Direct broadcast (q - r)^2 sum, int64.  Tiny inputs only."""
    Q = np.asarray(Q, np.int64)
    R = np.asarray(R, np.int64)
    return ((Q[:, None, :] - R[None, :, :]) ** 2).sum(-1)


def np_two_nn(Q, R) -> np.ndarray:
    """Per row: full stable sort of (d, i) — first two entries.  Returns int64 [n][4]."""
    D = np_dist_matrix(Q, R)
    n, m = D.shape
    out = np.full((n, 4), -1, np.int64)
    out[:, 0] = np.iinfo(np.int64).max
    out[:, 2] = np.iinfo(np.int64).max
    for j in range(n):
        order = np.argsort(D[j], kind="stable")  # ties -> lower index first
        if m >= 1:
            out[j, 0], out[j, 1] = D[j, order[0]], order[0]
        if m >= 2:
            out[j, 2], out[j, 3] = D[j, order[1]], order[1]
    return out


def np_match_count(Q, R, num: int = 4, den: int = 5) -> int:
    nn = np_two_nn(Q, R)
    if R.shape[0] < 2:
        return 0
    return int(np.sum(den * den * nn[:, 0] < num * num * nn[:, 2]))


def np_rank(counts, k: int, id_base: int = 0):
    counts = np.asarray(counts)
    B, R = counts.shape
    ids = np.arange(id_base, id_base + R)
    out_i = np.empty((B, k), np.int64)
    out_c = np.empty((B, k), np.int32)
    for b in range(B):
        order = np.lexsort((ids, -counts[b].astype(np.int64)))  # primary: count desc, then id asc
        out_i[b] = ids[order[:k]]
        out_c[b] = counts[b, order[:k]]
    return out_i, out_c
