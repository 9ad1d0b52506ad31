"""Pins for the CPU oracle (oracle/) against what the paper and the mathematics fix.

Each test names the PAPER.md passage (P:a-b) it pins.  None of these re-types the
oracle's formula: they use a second formulation (NumPy full sort), closed forms,
hand-computed worked cases (tests/golden/), invariants, and brute force on tiny
inputs, chosen so that a dropped term, a wrong sign/index or a transposed operand
in the oracle fails at least one of them.
"""
import os

import numpy as np
import pytest

import oracle
import tidgen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
I64MAX = np.iinfo(np.int64).max


def rand_u8(rng, *shape, hi=256):
    return rng.integers(0, hi, size=shape, dtype=np.uint8)


# --------------------------------------------------------------------------- distance
def test_sqdist_hand_cases():
    """Squared Euclidean distance (Eq. 1 LHS P:353-354): closed forms."""
    z = np.zeros(128, np.uint8)
    f = np.full(128, 255, np.uint8)
    assert oracle.sqdist(z, f) == 128 * 255 * 255 == 8_323_200
    assert oracle.sqdist(f, z) == 8_323_200
    r = np.arange(128, dtype=np.uint8)
    assert oracle.sqdist(z, r) == int((np.arange(128, dtype=np.int64) ** 2).sum())  # q = 0 => ||r||^2
    assert oracle.sqdist(r, r) == 0
    e = z.copy(); e[7] = 3
    g = z.copy(); g[9] = 4
    assert oracle.sqdist(e, g) == 25  # orthogonal one-hots: 3^2 + 4^2


def test_dist_matrix_vs_numpy_bruteforce(rng):
    """Second formulation: NumPy broadcast brute force on random tiny inputs."""
    for n, m in [(1, 1), (3, 5), (17, 9)]:
        Q, R = rand_u8(rng, n, 128), rand_u8(rng, m, 128)
        np.testing.assert_array_equal(oracle.dist_matrix(Q, R), oracle.np_dist_matrix(Q, R))


def test_dist_eq1_identity(rng):
    """Eq. 1: rho^2(R,Q) = N_R + N_Q - 2 R^T Q, computed the OTHER way
    (norms + dot product) must equal the oracle's direct sum for every pair."""
    Q, R = rand_u8(rng, 40, 128), rand_u8(rng, 70, 128)
    Qi, Ri = Q.astype(np.int64), R.astype(np.int64)
    eq1 = (Qi ** 2).sum(1)[:, None] + (Ri ** 2).sum(1)[None, :] - 2 * Qi @ Ri.T
    np.testing.assert_array_equal(oracle.dist_matrix(Q, R), eq1)


def test_dist_symmetry(rng):
    Q, R = rand_u8(rng, 6, 128), rand_u8(rng, 8, 128)
    np.testing.assert_array_equal(oracle.dist_matrix(Q, R), oracle.dist_matrix(R, Q).T)


# --------------------------------------------------------------------------- 2-NN
def test_two_nn_vs_full_sort(rng):
    """Streaming top-2 scan vs full stable sort per row (NumPy): same (d1,i1,d2,i2)."""
    for hi in (256, 4):  # hi=4 -> many ties, exercises the lowest-index tie-break
        Q, R = rand_u8(rng, 50, 128, hi=hi), rand_u8(rng, 33, 128, hi=hi)
        c, nn = oracle.match_count(Q, R, want_nn=True)
        np.testing.assert_array_equal(nn, oracle.np_two_nn(Q, R))
        assert c == oracle.np_match_count(Q, R)


def test_two_nn_alg1_order_invariant(rng):
    """Alg. 1 adds N_Q only AFTER the per-column sort: the top-2 indices of
    N_R - 2 R^T Q (no query norm) must equal the oracle's 2-NN on full distances."""
    Q, R = rand_u8(rng, 30, 128), rand_u8(rng, 40, 128)
    Qi, Ri = Q.astype(np.int64), R.astype(np.int64)
    key = (Ri ** 2).sum(1)[None, :] - 2 * Qi @ Ri.T
    _, nn = oracle.match_count(Q, R, want_nn=True)
    for j in range(30):
        order = np.argsort(key[j], kind="stable")
        assert (nn[j, 1], nn[j, 3]) == (order[0], order[1])
        assert nn[j, 0] == key[j, order[0]] + (Qi[j] ** 2).sum()
        assert nn[j, 2] == key[j, order[1]] + (Qi[j] ** 2).sum()


def test_two_nn_permutation(rng):
    """Permuting reference keypoints permutes indices consistently, distances unchanged."""
    Q, R = rand_u8(rng, 20, 128), rand_u8(rng, 25, 128)
    perm = rng.permutation(25)
    _, a = oracle.match_count(Q, R, want_nn=True)
    _, b = oracle.match_count(Q, R[perm], want_nn=True)
    np.testing.assert_array_equal(a[:, [0, 2]], b[:, [0, 2]])
    # with distinct distances the identities map through the permutation
    distinct = a[:, 0] != a[:, 2]
    np.testing.assert_array_equal(perm[b[distinct, 1]], a[distinct, 1])


def test_two_nn_duplicates():
    """Duplicated nearest keypoint => i1 < i2 and d1 == d2 (reading R2)."""
    R = np.zeros((4, 128), np.uint8)
    R[1, :] = 10
    R[3, :] = 10
    R[0, :] = 200
    R[2, :] = 200
    q = np.full(128, 11, np.uint8)
    d1, i1, d2, i2 = oracle.two_nn(q, R)
    assert (i1, i2) == (1, 3) and d1 == d2 == 128


def test_two_nn_degenerate_m():
    q = np.zeros(128, np.uint8)
    R = np.ones((1, 128), np.uint8)
    assert oracle.two_nn(q, R) == (128, 0, I64MAX, -1)
    assert oracle.two_nn(q, R, m_r=0) == (I64MAX, -1, I64MAX, -1)


# --------------------------------------------------------------------------- ratio test
def _golden_ratio_cases():
    rows = []
    with open(os.path.join(GOLDEN, "ratio_cases.txt")) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            c = [x.strip() for x in line.split("|")]
            rows.append(([int(v) for v in c[0].split(",")], [int(v) for v in c[1].split(",")],
                         int(c[2]), int(c[3]), int(c[4])))
    return rows


@pytest.mark.parametrize("r1,r2,d1,d2,ok", _golden_ratio_cases())
def test_ratio_golden(r1, r2, d1, d2, ok):
    """Worked cases (tests/golden/ratio_cases.txt, reading R1)."""
    R = np.zeros((2, 128), np.uint8)
    R[0, : len(r1)] = r1
    R[1, : len(r2)] = r2
    q = np.zeros((1, 128), np.uint8)
    c, nn = oracle.match_count(q, R, want_nn=True)
    assert (nn[0, 0], nn[0, 2]) == (d1, d2)
    assert c == ok
    assert oracle.ratio_pass(d1, d2) == bool(ok)


def test_ratio_float_crosscheck(rng):
    """Away from the boundary the integer test equals sqrt(d1) < 0.8 sqrt(d2) in float64."""
    d1 = rng.integers(0, 8_323_200, 20000)
    d2 = rng.integers(0, 8_323_200, 20000)
    d1, d2 = np.minimum(d1, d2), np.maximum(d1, d2)
    f = np.sqrt(d1) < 0.8 * np.sqrt(d2)
    away = np.abs(np.sqrt(d1) - 0.8 * np.sqrt(d2)) > 1e-6
    got = np.array([oracle.ratio_pass(int(a), int(b)) for a, b in zip(d1[away], d2[away])])
    np.testing.assert_array_equal(got, f[away])


def test_ratio_other_thresholds():
    # ratio 0.6 = 3/5 -> 25 d1 < 9 d2 ; ratio 1 -> d1 < d2
    assert oracle.ratio_pass(9, 26, num=3, den=5) and not oracle.ratio_pass(9, 25, num=3, den=5)
    assert oracle.ratio_pass(4, 5, num=1, den=1) and not oracle.ratio_pass(5, 5, num=1, den=1)
    assert not oracle.ratio_pass(0, 100, m_r=1)  # reading R3


# --------------------------------------------------------------------------- count
def test_count_onehot_closed_form():
    """Closed form: n orthogonal one-hot query descriptors (value v at a
    distinct dim); the reference is their first m rows => exactly m good matches."""
    v = 100
    for n, m in [(128, 128), (100, 37), (10, 2)]:
        Q = np.zeros((n, 128), np.uint8)
        Q[np.arange(n), np.arange(n)] = v
        R = Q[:m].copy()
        assert oracle.match_count(Q, R) == m
        assert oracle.np_match_count(Q, R) == m


def test_count_all_zero_reference(rng):
    """All-identical reference keypoints => d1 == d2 for every query row => count 0."""
    Q = rand_u8(rng, 64, 128)
    R = np.zeros((16, 128), np.uint8)
    assert oracle.match_count(Q, R) == 0


def test_count_query_order_invariance(rng):
    Q, R = rand_u8(rng, 64, 128, hi=64), rand_u8(rng, 20, 128, hi=64)
    R[:5] = Q[:5]  # some exact matches
    assert oracle.match_count(Q, R) == oracle.match_count(Q[rng.permutation(64)], R) > 0


def test_count_masks_padding(rng):
    """n_q / m_r exclude padded rows (reading R5): equal to slicing them away."""
    Q, R = rand_u8(rng, 30, 128), rand_u8(rng, 20, 128)
    R[:6] = Q[:6]
    assert oracle.match_count(Q, R, n_q=17, m_r=11) == oracle.match_count(Q[:17], R[:11])
    c, _ = oracle.verify(Q[None], R[None], n_q=[17], m_r=[11])
    assert c[0] == oracle.match_count(Q[:17], R[:11])


# --------------------------------------------------------------------------- search / top-k
def test_planted_target_ranks_first():
    """Generator plants 200 noisy copies of the target: the target must
    rank first for every query (top-1 identification)."""
    R_total, m, n = 48, 128, 300
    Rs, kp = tidgen.refs(0, R_total, m)
    Qs, tg = tidgen.queries(0, 4, n, R_total=R_total, m=m, n_planted=100)
    ids, cn, counts = oracle.search(Qs, Rs, k=5)
    np.testing.assert_array_equal(ids[:, 0], tg)
    assert (cn[:, 0] > 2 * cn[:, 1]).all()


def test_topk_vs_lexsort(rng):
    counts = rng.integers(0, 6, size=(7, 50)).astype(np.int32)  # many ties
    ids, cn = oracle.topk(counts, 9, id_base=1000)
    ei, ec = oracle.np_rank(counts, 9, id_base=1000)
    np.testing.assert_array_equal(ids, ei)
    np.testing.assert_array_equal(cn, ec)


def test_topk_identical_copies_ascending_ids(rng):
    """Identical reference copies => equal counts => ascending ids (reading R4)."""
    Q = rand_u8(rng, 2, 40, 128)
    R1 = rand_u8(rng, 1, 16, 128)
    R1[0, :8] = Q[0, :8]
    Rs = np.concatenate([rand_u8(rng, 3, 16, 128), R1, R1, R1], 0)
    ids, cn, _ = oracle.search(Q, Rs, k=3)
    assert list(ids[0]) == [3, 4, 5] and cn[0, 0] == cn[0, 1] == cn[0, 2] > 0


def test_search_reference_permutation(rng):
    """Permuting reference ids permutes the count matrix consistently."""
    Rs, _ = tidgen.refs(0, 20, 64)
    Qs, _ = tidgen.queries(0, 3, 100, R_total=20, m=64, n_planted=40)
    perm = rng.permutation(20)
    a = oracle.search_counts(Qs, Rs)
    b = oracle.search_counts(Qs, Rs[perm])
    np.testing.assert_array_equal(a[:, perm], b)


def test_search_counts_equal_verify(rng):
    """search_counts[b][r] == verify(pair (b, r)) — the one-by-one definition."""
    Rs, kp = tidgen.refs(0, 6, 64, kp_min=1, pad_byte=255)
    Qs, _ = tidgen.queries(0, 2, 70, R_total=6, m=64, kp_min=1, n_planted=30)
    c = oracle.search_counts(Qs, Rs, kp=kp)
    for b in range(2):
        for r in range(6):
            assert c[b, r] == oracle.np_match_count(Qs[b], Rs[r, : kp[r]]) if kp[r] >= 2 else c[b, r] == 0


def test_shard_merge_equals_global(rng):
    """merging per-shard top-k in the same total order == global top-k."""
    counts = rng.integers(0, 5, size=(5, 64)).astype(np.int32)
    gi, gc = oracle.topk(counts, 6)
    for G in (2, 4, 8):
        S = 64 // G
        li = np.empty((G, 5, 6), np.int64)
        lc = np.empty((G, 5, 6), np.int32)
        for g in range(G):
            li[g], lc[g] = oracle.topk(counts[:, g * S:(g + 1) * S], 6, id_base=g * S)
        mi, mc = oracle.merge_topk(li, lc)
        np.testing.assert_array_equal(mi, gi)
        np.testing.assert_array_equal(mc, gc)


def test_verify_multi_pair_strides(rng):
    """oracle_verify over P = 4 pairs with n != m and per-pair n_q[p], m_r[p] (P:31-35,
    P:284-288): every pair's count and (d1, i1, d2, i2) rows equal the NumPy brute force of
    that pair alone, and rows j >= n_q[p] stay untouched (-1).  A pair-stride bug (p*m vs
    p*n, or a shared n_q) puts another pair's keypoints under pair p and fails here."""
    P, n, m = 4, 37, 23
    Q = rand_u8(rng, P, n, 128, hi=48)
    R = rand_u8(rng, P, m, 128, hi=48)
    for p in range(P):  # distinct planted matches per pair so the pairs' counts differ
        R[p, : 3 + 4 * p] = Q[p, : 3 + 4 * p]
    n_q = np.array([37, 20, 5, 31], np.int32)
    m_r = np.array([23, 2, 17, 9], np.int32)
    counts, nn = oracle.verify(Q, R, n_q=n_q, m_r=m_r)
    assert len(set(counts.tolist())) > 2
    for p in range(P):
        e = oracle.np_two_nn(Q[p, : n_q[p]], R[p, : m_r[p]])
        np.testing.assert_array_equal(nn[p, : n_q[p]], e)
        assert (nn[p, n_q[p]:] == -1).all()
        assert counts[p] == oracle.np_match_count(Q[p, : n_q[p]], R[p, : m_r[p]])
    # without n_q / m_r every stored row takes part
    c2, nn2 = oracle.verify(Q, R)
    for p in range(P):
        np.testing.assert_array_equal(nn2[p], oracle.np_two_nn(Q[p], R[p]))
        assert c2[p] == oracle.np_match_count(Q[p], R[p])
