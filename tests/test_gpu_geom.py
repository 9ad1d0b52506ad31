"""GPU parity of SURVEY §8 row f4 (post-match verification: edge-feature removal + geometric
verification; readings R14-R16): tid_verify_geometric vs the
oracle (oracle.verify's (d1, i1, d2, i2) -> oracle.geometric), exactly: ratio-test counts, the
good matches left after edge removal, the best hypothesis' inlier count and its model bit for
bit (fp64 with every operation rounded separately on both sides)."""
import numpy as np
import pytest

import oracle
import tidgen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def tid():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    from paper_conf_icpp_wangzll21_b200 import build
    build.build()
    import paper_conf_icpp_wangzll21_b200 as t
    return t


def _scene(P, n, m, seed, n_planted=120):
    """Verification pairs (half planted) with keypoint coordinates: reference keypoints uniform in
    a 640 x 480 image; for a planted pair the query keypoints that match (oracle 2-NN) sit where
    a similarity (scale 0.8, rotation 0.3 rad, shift) maps them, plus 0.5 px noise; the rest are
    uniform in the 512 x 512 query image."""
    rng = np.random.default_rng(seed)
    Q, R, pos = tidgen.pairs(P, n, m, seed=seed, n_planted=n_planted)
    _, onn = oracle.verify(Q, R)
    r_xy = np.stack([rng.random((P, m)) * 640, rng.random((P, m)) * 480], -1).astype(np.float32)
    q_xy = np.stack([rng.random((P, n)) * 512, rng.random((P, n)) * 512], -1).astype(np.float32)
    a, b = 0.8 * np.cos(0.3), 0.8 * np.sin(0.3)
    for p in np.nonzero(pos)[0]:
        for j in range(n):
            d1, i1, d2 = onn[p, j, 0], onn[p, j, 1], onn[p, j, 2]
            if 25 * d1 < 16 * d2:
                # q = S^-1(r): solve the 2x2 system of the similarity
                X, Y = r_xy[p, i1] - np.array([40.0, 30.0], np.float32)
                det = a * a + b * b
                q_xy[p, j] = ((a * X + b * Y) / det + rng.normal(0, 0.5), (-b * X + a * Y) / det + rng.normal(0, 0.5))
    return Q, R, pos, q_xy, r_xy, onn


@pytest.mark.parametrize("iters,border", [(256, 0.0), (0, 16.0)])
def test_geometric_verify_equals_oracle(tid, iters, border):
    P, n, m = 24, 300, 260
    Q, R, pos, q_xy, r_xy, onn = _scene(P, n, m, seed=7)
    rng = np.random.default_rng(3)
    n_q = rng.integers(150, n + 1, P).astype(np.int32)
    m_r = rng.integers(200, m + 1, P).astype(np.int32)
    m_r[5] = 1  # reading R3: fewer than 2 reference keypoints, nothing matches
    _, onn = oracle.verify(Q, R, n_q=n_q, m_r=m_r)
    ec, _ = oracle.verify(Q, R, n_q=n_q, m_r=m_r, want_nn=False)
    kw = dict(border=border, q_size=(512, 512), r_size=(640, 480), inlier_px=2.0, iterations=iters, seed=11)
    eg, ei, em = oracle.geometric(onn, q_xy, r_xy, n_q=n_q, m_r=m_r, **kw)
    with tid.Index(query_kp_max=1024) as idx:
        c, g, i, mdl = idx.verify_geometric(Q, R, q_xy, r_xy, border=border, query_size=(512, 512),
                                            ref_size=(640, 480), inlier_px=2.0, iterations=iters, seed=11,
                                            n_q=n_q, m_r=m_r)
    np.testing.assert_array_equal(c.astype(np.int64), ec)
    np.testing.assert_array_equal(g.astype(np.int64), eg)
    np.testing.assert_array_equal(i.astype(np.int64), ei)
    np.testing.assert_array_equal(mdl, em)
    # planted pairs keep most of their matches as inliers; unrelated pairs have (almost) none
    planted = pos & (m_r >= 2)
    assert np.mean(i[planted] >= 0.5 * g[planted]) > 0.9
    assert i[~pos].max() <= 6 and i[planted].min() > 4 * max(1, i[~pos].max())


def test_geometric_recovers_the_similarity(tid):
    """The best hypothesis of a planted pair approximates the planted similarity (scale 0.8,
    rotation 0.3 rad, shift (40, 30)) to within the 0.5 px noise."""
    Q, R, pos, q_xy, r_xy, _ = _scene(4, 400, 256, seed=9, n_planted=150)
    with tid.Index(query_kp_max=1024) as idx:
        _, g, inl, mdl = idx.verify_geometric(Q, R, q_xy, r_xy, inlier_px=2.0, iterations=512)
    for p in np.nonzero(pos)[0]:
        a, b, tx, ty = mdl[p]
        assert abs(a - 0.8 * np.cos(0.3)) < 0.02 and abs(b - 0.8 * np.sin(0.3)) < 0.02
        assert abs(tx - 40) < 5 and abs(ty - 30) < 5 and inl[p] > 80
