"""Pins for the f1 float path of the oracle (RootSIFT + FP16, §4.2, §5.1, Alg. 2)."""
import numpy as np

import oracle
import tidgen


def test_rootsift_unit_norm_and_hellinger(rng):
    """||RootSIFT(x)||_2 = 1 and d^2 = 2 - 2 H(x, y) with the Hellinger kernel
    H(x,y) = sum sqrt(x_i y_i) of the L1-normalised histograms."""
    X = rng.integers(0, 256, (20, 128)).astype(np.float64)
    Y = rng.integers(0, 256, (30, 128)).astype(np.float64)
    rx, ry = oracle.rootsift(X), oracle.rootsift(Y)
    np.testing.assert_allclose(np.linalg.norm(rx, axis=1), 1.0, rtol=1e-12)
    xn, yn = X / X.sum(1, keepdims=True), Y / Y.sum(1, keepdims=True)
    H = np.sqrt(xn[:, None, :] * yn[None, :, :]).sum(-1)
    d2 = ((rx[:, None, :] - ry[None, :, :]) ** 2).sum(-1)
    np.testing.assert_allclose(d2, 2 - 2 * H, atol=1e-12)
    assert np.all(oracle.rootsift(np.zeros((1, 128))) == 0)


def test_table2_fp16_overflow_boundary():
    """Table 2: OpenCV-style SIFT has ||x||_2 = 512, so ||x s||^2 = 262144 s^2 against
    the fp16 maximum 65504: an fp16-accumulated similarity overflows for s = 1 and s = 2^-1 and
    not for 2^-2 ... 2^-16.  x below has ||x||^2 = 4*255^2 + 44^2 + 10^2 + 2^2 + 2^2 = 262144."""
    x = np.zeros(128)
    x[:8] = [255, 255, 255, 255, 44, 10, 2, 2]
    assert (x ** 2).sum() == 262144
    for s, overflow in [(1.0, True), (2.0 ** -1, True), (2.0 ** -2, False), (2.0 ** -7, False),
                        (2.0 ** -12, False), (2.0 ** -16, False)]:
        acc = oracle.fp16_accumulate_sq_norm(oracle.to_fp16(x, s))
        assert bool(np.isinf(acc)) == overflow, (s, acc)
    # exact-arithmetic form of the same boundary
    assert 262144 * 2.0 ** -2 > 65504 > 262144 * 2.0 ** -4


def test_f16_exact_on_integer_sift_matches_exact_oracle(rng):
    """u8 SIFT values (optionally scaled by 2^-7) are exact in fp16, so the float-path oracle
    must reproduce the exact integer oracle's counts."""
    R, _ = tidgen.refs(0, 6, 64)
    Q, _ = tidgen.queries(0, 2, 50, R_total=6, m=64, n_planted=20)
    exact = oracle.search_counts(Q, R)
    for s in (1.0, 2.0 ** -7):
        got = oracle.f16_search_counts(oracle.to_fp16(Q, s), oracle.to_fp16(R, s))
        np.testing.assert_array_equal(got, exact)


def test_f16_ratio_boundary():
    """d1 = 16, d2 = 25 (ratio exactly 0.8) fails (strict), d2 = 26 passes, as in the integer path."""
    R = np.zeros((2, 128), np.float16)
    R[0, 0] = 4
    R[1, 0] = 5
    q = np.zeros((1, 128), np.float16)
    assert oracle.f16_match_count(q, R) == 0
    R[1, 1] = 1
    assert oracle.f16_match_count(q, R) == 1


def test_compression_error_eq2(rng):
    """Eq. 2: zero for exactly representable data, small and positive for RootSIFT
    in fp16 (the paper reports ~0.1% on its data)."""
    R, _ = tidgen.refs(0, 1, 64)
    Q, _ = tidgen.queries(0, 1, 40, R_total=1, m=64, n_planted=10)
    assert oracle.compression_error(Q[0], R[0], oracle.to_fp16(Q[0]), oracle.to_fp16(R[0])) == 0.0
    rq, rr = oracle.rootsift(Q[0]), oracle.rootsift(R[0])
    e = oracle.compression_error(rq, rr, oracle.to_fp16(rq), oracle.to_fp16(rr))
    assert 0 < e < 5e-3


def test_compression_error_eq2_closed_form():
    """Eq. 2 on a 2 x 2 case known in closed form.  Queries q1 = 0, q2 = e1;
    references r1 = 0.1 e1, r2 = 3 e2.  fp16(0.1) = 1638 / 2^14 = 0.1 - 2^-15 * 0.8 =: 0.1 - u
    (u = 2.44140625e-5); every other value is exact in fp16.  The four distances:
    rho(r1,q1) = 0.1 (fp16: 0.1 - u), rho(r1,q2) = 0.9 (fp16: 0.9 + u), rho(r2,q*) exact
    (3, sqrt 10).  Eq. 2 = (u/0.1 + u/0.9 + 0 + 0) / (m*n = 4) = u * 25/9.
    Mistakes this catches: rho^2 instead of rho (about 2x), dividing by rho_FP16 (relative
    2.4e-4), averaging over the two non-zero terms only (1.8x), a dropped |.|."""
    u = 2.0 ** -15 * 0.8
    Qf = np.zeros((2, 128))
    Qf[1, 0] = 1.0
    Rf = np.zeros((2, 128))
    Rf[0, 0] = 0.1
    Rf[1, 1] = 3.0
    Q16 = oracle.to_fp16(Qf).astype(np.float64)
    R16 = oracle.to_fp16(Rf).astype(np.float64)
    assert R16[0, 0] == 1638 / 2 ** 14 == 0.1 - u
    e = oracle.compression_error(Qf, Rf, Q16, R16)
    np.testing.assert_allclose(e, u * 25 / 9, rtol=1e-12)
    # transposing the roles (m x n vs n x m) leaves the mean unchanged
    np.testing.assert_allclose(oracle.compression_error(Rf, Qf, R16, Q16), u * 25 / 9, rtol=1e-12)


def test_compression_error_zero_distance_pairs_excluded():
    """Reading (R12): Eq. 2 divides by rho, undefined (0/0) for identical descriptors;
    those pairs are left out of the mean.  q = r = 0.1 e1 (rho = rho_FP16 = 0) plus
    q2 = 0 (rho = 0.1, rho_FP16 = 0.1 - u): the mean is over the one defined pair, u / 0.1."""
    u = 2.0 ** -15 * 0.8
    Qf = np.zeros((2, 128))
    Qf[0, 0] = 0.1
    Rf = np.zeros((1, 128))
    Rf[0, 0] = 0.1
    e = oracle.compression_error(Qf, Rf, oracle.to_fp16(Qf).astype(np.float64), oracle.to_fp16(Rf).astype(np.float64))
    np.testing.assert_allclose(e, u / 0.1, rtol=1e-12)


def test_f16_c_oracle_equals_numpy_and_exact(rng):
    """The C float64 oracle (oracle_f64_search_counts) against two independent references:
    (i) the NumPy float formulation on RootSIFT fp16 data with ragged n_q / kp (distances from a
    broadcast matrix + partition, a different summation order); (ii) the exact integer oracle
    on u8 SIFT x 2^-7 (exact in fp16)."""
    R, _ = tidgen.refs(11, 7, 96)
    Q, _ = tidgen.queries(11, 3, 120, R_total=7, m=96, n_planted=40)
    q16 = oracle.to_fp16(oracle.rootsift(Q))
    r16 = oracle.to_fp16(oracle.rootsift(R))
    n_q = np.array([120, 77, 5], np.int32)
    kp = np.array([96, 1, 2, 50, 96, 0, 33], np.int32)
    got = oracle.f16_search_counts_c(q16, r16, n_q=n_q, kp=kp)
    want = np.zeros_like(got)
    for b in range(3):
        for r in range(7):
            want[b, r] = oracle.f16_match_count(q16[b], r16[r], n_q=int(n_q[b]), m_r=int(kp[r]))
    np.testing.assert_array_equal(got, want)
    assert got[:, 1].sum() == 0 and got[:, 5].sum() == 0 and got.max() > 0
    s = 2.0 ** -7
    np.testing.assert_array_equal(oracle.f16_search_counts_c(oracle.to_fp16(Q, s), oracle.to_fp16(R, s)),
                                  oracle.search_counts(Q, R))
