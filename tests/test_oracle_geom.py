"""Pins for the f4 oracle (post-match verification: edge-feature removal + geometric
verification, §3.1, §4.1; readings R14-R16 in DESIGN.md /
oracle/tid_oracle.c).  nn rows are built by hand here: row j passes the ratio test with
(d1, d2) = (0, 100) or fails with (50, 50), and its nearest reference keypoint is i1."""
import numpy as np

import oracle


def _nn(P, n, passing, i1):
    nn = np.zeros((P, n, 4), np.int64)
    nn[..., 0], nn[..., 2] = 50, 50
    nn[..., 0][passing], nn[..., 2][passing] = 0, 100
    nn[..., 1] = i1
    nn[..., 3] = 0
    return nn


def _brute(Pq, Qr, thr):
    """NumPy exhaustive search over all pairs u < v (float64, each operation rounded once):
    the largest inlier count and its (earliest) model."""
    M = len(Pq)
    best, bm = -1, np.zeros(4)
    for u in range(M):
        for v in range(u + 1, M):
            dp, dq = Pq[v] - Pq[u], Qr[v] - Qr[u]
            den = dp[0] * dp[0] + dp[1] * dp[1]
            if den == 0:
                continue
            a = (dp[0] * dq[0] + dp[1] * dq[1]) / den
            b = (dp[0] * dq[1] - dp[1] * dq[0]) / den
            tx = Qr[u, 0] - (a * Pq[u, 0] - b * Pq[u, 1])
            ty = Qr[u, 1] - (b * Pq[u, 0] + a * Pq[u, 1])
            ex = a * Pq[:, 0] - b * Pq[:, 1] + tx - Qr[:, 0]
            ey = b * Pq[:, 0] + a * Pq[:, 1] + ty - Qr[:, 1]
            c = int(np.sum(ex * ex + ey * ey < np.float64(thr) * np.float64(thr)))
            if c > best:
                best, bm = c, np.array([a, b, tx, ty])
    return max(best, 0), bm


def test_exact_similarity_recovered(rng):
    """Query points mapped by X = -2y + 500, Y = 2x + 6 (a = 0, b = 2: rotation by 90 degrees and
    scale 2, all exact in binary) plus 12 outliers: the exhaustive search and RANSAC find the
    model exactly and count exactly the 30 planted inliers."""
    P, n, m = 1, 42, 42
    q = rng.integers(0, 200, (P, n, 2)).astype(np.float32)
    r = np.empty((P, m, 2), np.float32)
    r[0, :, 0] = -2 * q[0, :, 1] + 500
    r[0, :, 1] = 2 * q[0, :, 0] + 6
    r[0, 30:] = rng.integers(1000, 2000, (12, 2))  # outliers far away
    nn = _nn(P, n, np.ones((P, n), bool), np.arange(n))
    for iters in (0, 200):
        good, inl, model = oracle.geometric(nn, q, r, inlier_px=1.0, iterations=iters)
        assert good[0] == 42 and inl[0] == 30, (iters, inl)
        np.testing.assert_array_equal(model[0], [0.0, 2.0, 500.0, 6.0])


def test_exhaustive_equals_numpy_brute_force(rng):
    """Noisy data, several pairs, ragged n_q: exhaustive mode == NumPy brute force (inliers and
    the model bit for bit); RANSAC never beats it and matches it with enough hypotheses."""
    P, n, m = 4, 40, 30
    q = (rng.random((P, n, 2)) * 300).astype(np.float32)
    i1 = rng.integers(0, m, (P, n))
    r = (rng.random((P, m, 2)) * 300).astype(np.float32)
    for p in range(P):  # half the rows follow a similarity + noise
        ang, sc = rng.random() * 6.28, 0.5 + rng.random()
        a, b = sc * np.cos(ang), sc * np.sin(ang)
        for j in range(0, n, 2):
            x, y = q[p, j]
            r[p, i1[p, j]] = (a * x - b * y + 700 + rng.normal(0, 0.3), b * x + a * y + 650 + rng.normal(0, 0.3))
    passing = rng.random((P, n)) < 0.8
    nn = _nn(P, n, passing, i1)
    n_q = np.array([40, 33, 2, 1], np.int32)
    good, inl, model = oracle.geometric(nn, q, r, inlier_px=2.0, iterations=0, n_q=n_q)
    g2, inl2, _ = oracle.geometric(nn, q, r, inlier_px=2.0, iterations=4000, n_q=n_q)
    np.testing.assert_array_equal(g2, good)
    for p in range(P):
        rows = [j for j in range(n_q[p]) if passing[p, j]]
        assert good[p] == len(rows)
        Pq = q[p, rows].astype(np.float64)
        Qr = r[p, i1[p, rows]].astype(np.float64)
        bi, bm = _brute(Pq, Qr, 2.0) if len(rows) >= 2 else (0, np.zeros(4))
        assert inl[p] == bi
        np.testing.assert_array_equal(model[p], bm)
        assert inl2[p] <= inl[p]
    assert inl2[0] == inl[0] and inl[0] >= 5
    assert inl[2] in (0, 2) and inl[3] == 0 and good[3] <= 1  # M < 2: no hypothesis


def test_edge_feature_removal(rng):
    """Reading R14: matches whose query or reference keypoint lies within `border` px of its
    image edge are dropped before the geometric step (x < b, y < b, x >= W - b, y >= H - b)."""
    P, n = 1, 8
    q = np.array([[[5, 50], [50, 5], [50, 50], [95, 50], [50, 94.9], [50, 50], [20, 20], [80, 80]]], np.float32)
    r = np.array([[[50, 50], [50, 50], [50, 50], [50, 50], [50, 50], [3, 50], [50, 196], [100, 100]]], np.float32)
    nn = _nn(P, n, np.ones((P, n), bool), np.arange(n))
    # query image 100 x 100, reference 200 x 200, border 10:
    # rows 0, 1 (query x or y < 10), 3 (x >= 90), 4 (y >= 90), 5 (reference x < 10) and 6
    # (reference y >= 190) are dropped; rows 2 and 7 survive
    good, inl, _ = oracle.geometric(nn, q, r, border=10, q_size=(100, 100), r_size=(200, 200), iterations=0)
    assert good[0] == 2 and inl[0] == 2
    good0, _, _ = oracle.geometric(nn, q, r, border=0, q_size=(100, 100), r_size=(200, 200), iterations=0)
    assert good0[0] == 8


def test_ratio_test_gates_matches(rng):
    """Only rows passing the ratio test (reading R1) enter: the good count equals the
    number of passing rows; a reference with fewer than 2 keypoints (R3) contributes none."""
    P, n, m = 2, 20, 20
    q = (rng.random((P, n, 2)) * 50 + 10).astype(np.float32)
    r = q.copy()
    passing = np.zeros((P, n), bool)
    passing[:, :7] = True
    nn = _nn(P, n, passing, np.arange(n))
    good, inl, model = oracle.geometric(nn, q, r, iterations=0, m_r=np.array([20, 1], np.int32))
    assert good.tolist() == [7, 0] and inl.tolist() == [7, 0]
    np.testing.assert_array_equal(model[0], [1.0, 0.0, 0.0, 0.0])
