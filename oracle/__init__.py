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
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-shared", "-fPIC", "-o", tmp, _SRC])
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
        lib.oracle_f64_search_counts.argtypes = [vp, vp, i32, i64, vp, vp, i32, i64, u32, u32, vp]
        f32 = ctypes.c_float
        lib.oracle_geometric.argtypes = [vp, i32, i32, i64, vp, vp, vp, vp, f32, f32, f32, f32, f32, f32, i32,
                                         ctypes.c_uint64, u32, u32, vp, vp, vp]
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


# ------------------------------------------------- f1: RootSIFT + FP16 float path (§4.2, §5.1, Alg. 2)
def rootsift(X) -> np.ndarray:
    """RootSIFT: L1-normalise each SIFT vector, then take the element-wise square
    root; the result has unit L2 norm and Euclidean distance = Hellinger kernel distance."""
    X = np.asarray(X, np.float64)
    s = X.sum(-1, keepdims=True)
    return np.sqrt(np.divide(X, s, out=np.zeros_like(X), where=s > 0))


def to_fp16(X, scale: float = 1.0) -> np.ndarray:
    """FP16 storage with a scale factor applied before the conversion (2^-7 in
    practice).  Round-to-nearest-even (IEEE)."""
    return (np.asarray(X, np.float64) * scale).astype(np.float16)


def fp16_accumulate_sq_norm(x_fp16) -> np.float16:
    """||x||^2 accumulated in FP16 arithmetic (each product and partial sum rounded to fp16), the
    arithmetic of an fp16-accumulating HGEMM.  Pins the Table 2 overflow boundary."""
    acc = np.float16(0)
    with np.errstate(over="ignore"):
        for v in np.asarray(x_fp16, np.float16):
            acc = np.float16(acc + np.float16(v * v))
    return acc


def f16_dist_matrix(Q16, R16) -> np.ndarray:
    """Squared distances of fp16-stored descriptors, computed exactly in float64 (the oracle
    of what the GPU's fp16 x fp16 -> fp32 path approximates)."""
    Q = np.asarray(Q16, np.float16).astype(np.float64)
    R = np.asarray(R16, np.float16).astype(np.float64)
    return ((Q[:, None, :] - R[None, :, :]) ** 2).sum(-1)


def f16_match_count(Q16, R16, num: int = 4, den: int = 5, n_q=None, m_r=None) -> int:
    """2-NN per query row + ratio test on squared distances in the rational form of
    reading R1, den^2 * d1 < num^2 * d2 (strict), in float64 for fp16-stored
    descriptors (num/den = 4/5: no rounding of the threshold itself)."""
    nq = len(Q16) if n_q is None else n_q
    mr = len(R16) if m_r is None else m_r
    if mr < 2 or nq == 0:
        return 0
    D = f16_dist_matrix(Q16[:nq], R16[:mr])
    part = np.partition(D, 1, axis=1)[:, :2]
    d1, d2 = part[:, 0], part[:, 1]
    return int(np.sum(den * den * d1 < num * num * d2))


def f16_search_counts(Qs16, Rs16, num: int = 4, den: int = 5, n_q=None, kp=None) -> np.ndarray:
    B, R = len(Qs16), len(Rs16)
    out = np.zeros((B, R), np.int32)
    for b in range(B):
        for r in range(R):
            out[b, r] = f16_match_count(Qs16[b], Rs16[r], num, den, None if n_q is None else n_q[b],
                                        None if kp is None else kp[r])
    return out


def f16_search_counts_c(Qs16, Rs16, num: int = 4, den: int = 5, n_q=None, kp=None) -> np.ndarray:
    """The same counts as ``f16_search_counts`` from the C oracle (float64 direct sums, OpenMP over
    pairs; oracle_f64_search_counts) — for sizes the NumPy formulation cannot reach.  Pinned
    against the NumPy formulation and the exact integer oracle in tests/test_oracle_f16.py."""
    Q = np.ascontiguousarray(np.asarray(Qs16, np.float16).astype(np.float64))
    R = np.ascontiguousarray(np.asarray(Rs16, np.float16).astype(np.float64))
    B, n = Q.shape[0], Q.shape[1]
    Rn, m = R.shape[0], R.shape[1]
    nq = None if n_q is None else _c(n_q, np.int32)
    kpa = None if kp is None else _c(kp, np.int32)
    counts = np.empty((B, Rn), np.int32)
    _L().oracle_f64_search_counts(_p(Q), _p(nq), n, B, _p(R), _p(kpa), m, Rn, num, den, _p(counts))
    return counts


def geometric(nn, q_xy, r_xy, *, border=0.0, q_size=(1e9, 1e9), r_size=(1e9, 1e9), inlier_px=3.0,
              iterations=256, seed=2021, num=4, den=5, n_q=None, m_r=None):
    """f4 post-match verification (readings R14-R16 in the C
    header): from verify's nn [P][n][4], query / reference keypoint coordinates [P][n][2] /
    [P][m][2] -> (good [P] = ratio-test matches surviving edge removal, inliers [P] of the best
    2-point similarity hypothesis, model [P][4] = (a, b, tx, ty))."""
    nn = _c(nn, np.int64)
    P, n = nn.shape[0], nn.shape[1]
    q_xy, r_xy = _c(q_xy, np.float32), _c(r_xy, np.float32)
    m = r_xy.shape[1]
    assert q_xy.shape == (P, n, 2) and r_xy.shape[0] == P and r_xy.shape[2] == 2
    nq = None if n_q is None else _c(n_q, np.int32)
    mr = None if m_r is None else _c(m_r, np.int32)
    good, inl = np.empty(P, np.int32), np.empty(P, np.int32)
    model = np.empty((P, 4), np.float64)
    _L().oracle_geometric(_p(nn), n, m, P, _p(nq), _p(mr), _p(q_xy), _p(r_xy), border, q_size[0], q_size[1],
                          r_size[0], r_size[1], inlier_px, iterations, seed, num, den, _p(good), _p(inl),
                          _p(model))
    return good, inl, model


def compression_error(Qf, Rf, Q16, R16) -> float:
    """Eq. 2: mean over all (i, j) of |rho(R_i, Q_j) - rho_FP16(R_i, Q_j)| / rho(R_i, Q_j),
    rho = Euclidean distance; the fp16 distances are those of the fp16-stored (scaled)
    descriptors, un-scaled by the caller's scale factor (pass Q16/R16 already divided), computed
    exactly in float64 (reading R13).  Pairs with rho = 0 (0/0 in Eq. 2) are left out of the mean
    (reading R12).  Pinned in closed form by tests/test_oracle_f16.py."""
    rho = np.sqrt(((np.asarray(Rf, np.float64)[:, None, :] - np.asarray(Qf, np.float64)[None, :, :]) ** 2).sum(-1))
    rho16 = np.sqrt(((np.asarray(R16, np.float64)[:, None, :] - np.asarray(Q16, np.float64)[None, :, :]) ** 2).sum(-1))
    ok = rho > 0
    return float(np.mean(np.abs(rho - rho16)[ok] / rho[ok]))
