"""GPU parity of SURVEY §8 row f1 (float-descriptor path): RootSIFT / scaled SIFT in fp16 on
tcgen05.mma.kind::f16 with fp32 accumulation, vs the float64 oracle on the same fp16 values.

Acceptance: match counts within +-1 for >= 99.9% of (query, reference) pairs;
bit-exact where the fp16 values make every fp32 step exact (u8 SIFT x 2^-7)."""
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


def test_prepare_scaled_sift_exact(tid):
    """x * 2^-7 of u8 values is exact in fp16: bit-identical to the oracle's conversion."""
    R, _ = tidgen.refs(3, 20, 256)
    with tid.Index() as idx:
        got = idx.f16_prepare(R, rootsift=False, scale=2.0 ** -7)
    np.testing.assert_array_equal(got.view(np.uint16), oracle.to_fp16(R, 2.0 ** -7).view(np.uint16))


def test_prepare_rootsift_within_one_ulp(tid):
    """RootSIFT computed in fp32 then rounded to fp16: equal to the float64 oracle's
    rounding for >= 99.9% of elements, never more than one fp16 ulp away."""
    R, _ = tidgen.refs(4, 30, 256)
    R[0, :5] = 0  # all-zero rows stay zero
    with tid.Index() as idx:
        got = idx.f16_prepare(R, rootsift=True, scale=1.0)
    want = oracle.to_fp16(oracle.rootsift(R), 1.0)
    g, w = got.view(np.uint16).astype(np.int64), want.view(np.uint16).astype(np.int64)
    assert np.abs(g - w).max() <= 1
    assert np.mean(g == w) >= 0.999
    assert np.all(got[0, :5] == 0)


def test_f16_counts_exact_on_scaled_integer_sift(tid):
    """u8 SIFT x 2^-7 in fp16: products and fp32 sums are exact, so the float path must equal
    both the float64 oracle and the exact integer oracle (ragged n, m < 256)."""
    Rr, _ = tidgen.refs(5, 24, 200)
    Q, _ = tidgen.queries(5, 3, 300, R_total=24, m=200, n_planted=60)
    s = 2.0 ** -7
    with tid.Index(query_kp_max=1024) as idx:
        q16, r16 = idx.f16_prepare(Q, False, s), idx.f16_prepare(Rr, False, s)
        got = idx.f16_search_counts(q16, r16).astype(np.int64)
    np.testing.assert_array_equal(got, oracle.search_counts(Q, Rr))
    # the oracle end to end: its own conversion of the same u8 inputs, its own float64 counts
    np.testing.assert_array_equal(got, oracle.f16_search_counts(oracle.to_fp16(Q, s), oracle.to_fp16(Rr, s)))


def test_f16_rootsift_counts_within_one(tid):
    """RootSIFT fp16 (the paper's final configuration, §5.1): |GPU - oracle| <= 1 for >= 99.9% of
    pairs (and never more than 2), the planted reference ranks first for every query."""
    Rr, _ = tidgen.refs(0, 48, 256)  # reference i has global id i (planted targets are global ids)
    Q, tg = tidgen.queries(6, 4, 400, R_total=48, m=256, n_planted=80)
    with tid.Index(query_kp_max=1024) as idx:
        q16, r16 = idx.f16_prepare(Q, True, 1.0), idx.f16_prepare(Rr, True, 1.0)
        got = idx.f16_search_counts(q16, r16).astype(np.int64)
    # oracle end to end on the same u8 inputs (its own RootSIFT -> fp16 conversion; the GPU's agrees
    # to within one fp16 ulp, test_prepare_rootsift_within_one_ulp)
    want = oracle.f16_search_counts(oracle.to_fp16(oracle.rootsift(Q)), oracle.to_fp16(oracle.rootsift(Rr)))
    want = want.astype(np.int64)
    diff = np.abs(got - want)
    assert diff.max() <= 2
    assert np.mean(diff <= 1) >= 0.999
    assert np.all(np.argmax(got, axis=1) == tg)


def test_f16_ratio_boundary(tid):
    """d1 = 16 s^2, d2 = 25 s^2 (ratio exactly 0.8) fails, d2 + 1 passes, as in the integer path."""
    m = 64
    R = np.zeros((2, m, 128), np.float16)
    R[:, 2:, :] = 2.0                       # far keypoints
    R[0, 0, 0], R[0, 1, 0] = 4.0, 5.0       # d1 = 16, d2 = 25 -> fail
    R[1, 0, 0], R[1, 1, 0], R[1, 1, 1] = 4.0, 5.0, 1.0  # d2 = 26 -> pass
    q = np.zeros((1, 5, 128), np.float16)
    with tid.Index(query_kp_max=1024) as idx:
        got = idx.f16_search_counts(q, R)
    assert got.tolist() == [[0, 5]]
    np.testing.assert_array_equal(got.astype(np.int64), oracle.f16_search_counts(q, R))


def test_f16_rootsift_parity_at_scale(tid):
    """f1 acceptance at the verdict's scale: 64 RootSIFT queries (1000 keypoints) x 2,000 references
    (256 keypoints) in fp16 — 128,000 pairs — vs the C float64 oracle end to end on the same u8 inputs:
    |count difference| <= 1 for >= 99.9 % of pairs, and the planted target ranks first."""
    B, n, R, m = 64, 1000, 2000, 256
    Rr, _ = tidgen.refs(0, R, m, seed=2021)
    Q, tg = tidgen.queries(0, B, n, R_total=R, m=m, seed=2021)
    with tid.Index(query_kp_max=1024) as idx:
        q16, r16 = idx.f16_prepare(Q, True, 1.0), idx.f16_prepare(Rr, True, 1.0)
        got = idx.f16_search_counts(q16, r16).astype(np.int64)
    want = oracle.f16_search_counts_c(oracle.to_fp16(oracle.rootsift(Q)), oracle.to_fp16(oracle.rootsift(Rr)))
    want = want.astype(np.int64)
    diff = np.abs(got - want)
    assert diff.max() <= 2, diff.max()
    assert np.mean(diff <= 1) >= 0.999, np.mean(diff <= 1)
    np.testing.assert_array_equal(np.argmax(got, 1), tg)


def test_f16_counts_two_chunk_references(tid):
    """tid_f16_search_counts with m in (256, 512]: references of two 256-row chunks (exact on u8 SIFT
    x 2^-7, ragged n)."""
    Rr, _ = tidgen.refs(7, 9, 384)
    Q, _ = tidgen.queries(7, 2, 333, R_total=9, m=384, n_planted=80)
    s = 2.0 ** -7
    with tid.Index(query_kp_max=1024) as idx:
        q16, r16 = idx.f16_prepare(Q, False, s), idx.f16_prepare(Rr, False, s)
        got = idx.f16_search_counts(q16, r16).astype(np.int64)
    np.testing.assert_array_equal(got, oracle.search_counts(Q, Rr))
