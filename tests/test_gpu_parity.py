"""GPU parity: the CUDA path (through the C ABI) vs the CPU oracle, element by element.

Bit-exact is the bar for everything (all arithmetic is integer): (d1, i1, d2, i2),
good-match counts, the full count matrix and the top-k ids/counts.  Inputs come from
tidgen (shared seeded generator) or are built here; expected values come only from
oracle/.  Sizes span several tiles and ragged tails (n not a multiple of 128, m not a
multiple of 256, partial reference groups).
"""
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


def nn_from_oracle(onn):
    """oracle int64 nn (INT64_MAX / -1 for a missing neighbour) -> the ABI's int32 convention (-1, -1)."""
    o = onn.copy()
    big = np.iinfo(np.int64).max
    o[..., 0][o[..., 0] == big] = -1
    o[..., 2][o[..., 2] == big] = -1
    return o.astype(np.int64)


# ------------------------------------------------------------------------------ search (C1)
def test_c1_search_bitexact(tid):
    """Config 1: 1 query x 64 references x 256 keypoints, ratio 0.8, top-5."""
    R, m, n, k = 64, 256, 256, 5
    refs, _ = tidgen.refs(0, R, m)
    qs, tg = tidgen.queries(0, 1, n, R_total=R, m=m)
    with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
        idx.add_references(refs)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, k)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, k)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)
    assert ids[0, 0] == tg[0]


@pytest.mark.parametrize("n,R,m,B", [(1000, 37, 256, 3), (130, 9, 200, 5), (1, 6, 2, 2), (383, 150, 256, 2)])
def test_search_shapes_bitexact(tid, n, R, m, B):
    """Ragged n (tile tails), m < 256, odd reference counts (partial groups), B > 1."""
    refs, _ = tidgen.refs(100, R, m)
    qs, _ = tidgen.queries(7, B, n, R_total=R, m=m, n_planted=min(50, n, m))
    with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
        idx.add_references(refs)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, min(5, R))
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, min(5, R))
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


def test_search_variable_kp_and_nq(tid):
    """Per-reference keypoint counts (padding rows hold garbage 0xFF) and per-query n_q."""
    R, m, n, B = 40, 256, 700, 3
    refs, kp = tidgen.refs(0, R, m, kp_min=0, pad_byte=255)
    kp[:3] = [0, 1, 2]  # degenerate references: never / never / can match
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, kp_min=0, n_planted=60)
    n_q = np.array([700, 513, 129], np.int32)
    with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
        idx.add_references(refs, kp)
        counts = idx.search_counts(qs, n_q=n_q)
        ids, cnt = idx.search(qs, 7, n_q=n_q)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, 7, n_q=n_q, kp=kp)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)
    assert (counts[:, :2] == 0).all()


# ------------------------------------------------------------------------------ verify
@pytest.mark.parametrize("n,m,P", [(300, 600, 6), (1000, 1000, 5), (128, 256, 4), (129, 257, 3), (5, 2, 3)])
def test_verify_bitexact(tid, n, m, P):
    """(d1, i1, d2, i2) per query row and counts; m > 256 exercises the cross-chunk merge."""
    Q, Rr, _ = tidgen.pairs(P, n, m, n_planted=min(200, n, m))
    with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
        c, nn = idx.verify(Q, Rr)
    ec, enn = oracle.verify(Q, Rr)
    np.testing.assert_array_equal(c.astype(np.int64), ec)
    np.testing.assert_array_equal(nn.astype(np.int64), nn_from_oracle(enn))


def test_verify_masks(tid):
    Q, Rr, _ = tidgen.pairs(4, 400, 500, n_planted=100)
    n_q = np.array([400, 1, 255, 129], np.int32)
    m_r = np.array([500, 2, 1, 256], np.int32)
    with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
        c, nn = idx.verify(Q, Rr, n_q=n_q, m_r=m_r)
    ec, enn = oracle.verify(Q, Rr, n_q=n_q, m_r=m_r)
    np.testing.assert_array_equal(c.astype(np.int64), ec)
    for p in range(4):
        np.testing.assert_array_equal(nn[p, :n_q[p]].astype(np.int64), nn_from_oracle(enn[p, :n_q[p]]))
        assert (nn[p, n_q[p]:] == -1).all()


def test_verify_adversarial(tid, rng):
    """all-255 vs all-0, duplicates, heavy ties (values in {0,1,2}), exact copies."""
    P, n, m = 6, 200, 300
    Q = np.zeros((P, n, 128), np.uint8)
    Rr = np.zeros((P, m, 128), np.uint8)
    Q[0] = 255                                   # max distance 8,323,200 everywhere
    Q[1] = rng.integers(0, 3, (n, 128)); Rr[1] = rng.integers(0, 3, (m, 128))    # ties
    Rr[2, :] = 7; Q[2] = rng.integers(0, 256, (n, 128))                          # all-identical reference
    Q[3] = rng.integers(0, 256, (n, 128)); Rr[3, :n] = Q[3]; Rr[3, n:] = Q[3, :m - n]  # duplicates of every row
    Q[4] = rng.integers(0, 256, (n, 128)); Rr[4] = rng.integers(0, 256, (m, 128)); Rr[4, 5:100] = Q[4, 5:100]
    Q[5] = 255; Rr[5] = 255
    with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
        c, nn = idx.verify(Q, Rr)
    ec, enn = oracle.verify(Q, Rr)
    np.testing.assert_array_equal(c.astype(np.int64), ec)
    np.testing.assert_array_equal(nn.astype(np.int64), nn_from_oracle(enn))
    assert nn[0, 0, 0] == 8_323_200


# ------------------------------------------------------------------------------ decompositions
def test_host_tier_equals_hbm(tid):
    """Host-streamed references (hbm_budget forces the level-2 tier) == HBM-resident."""
    R, m, n, B = 300, 256, 400, 2
    refs, kp = tidgen.refs(0, R, m, kp_min=100, pad_byte=9)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, kp_min=100)
    rb = m * 128
    with tid.Index(ref_kp=m) as a:
        a.add_references(refs, kp)
        ca = a.search_counts(qs)
        ia, na = a.search(qs, 10)
    with tid.Index(ref_kp=m, hbm_budget_bytes=100 * rb, host_budget_bytes=1000 * rb) as b:
        b.set_tuning(host_chunk_refs=64)
        b.add_references(refs[:150], kp[:150])
        b.add_references(refs[150:], kp[150:])
        info = b.info()
        cb = b.search_counts(qs)
        ib, nb = b.search(qs, 10)
    assert info["hbm_references"] == 100 and info["host_references"] == 200
    np.testing.assert_array_equal(ca, cb)
    np.testing.assert_array_equal(ia, ib)
    np.testing.assert_array_equal(na, nb)
    np.testing.assert_array_equal(ca.astype(np.int64), oracle.search_counts(qs, refs, kp=kp))


def test_host_tier_multichunk_references(tid):
    """Host tier with the paper's m = 384 (two 256-column chunks per reference, Table 7) and ragged
    kp: streamed chunks of references == the oracle."""
    R, m, n, B = 90, 384, 500, 2
    refs, kp = tidgen.refs(3, R, m, kp_min=150, pad_byte=5)
    qs, _ = tidgen.queries(3, B, n, R_total=R, m=m, kp_min=150)
    rb = m * 128
    with tid.Index(ref_kp=m, hbm_budget_bytes=30 * rb, host_budget_bytes=200 * rb) as b:
        b.set_tuning(host_chunk_refs=16)
        b.add_references(refs, kp)
        info = b.info()
        cb = b.search_counts(qs)
        ib, nb = b.search(qs, 6)
    assert info["hbm_references"] == 30 and info["host_references"] == 60
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, 6, kp=kp)
    np.testing.assert_array_equal(cb.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ib, e_ids)
    np.testing.assert_array_equal(nb, e_cnt)


def test_host_tier_map_zero_copy(tid):
    """tid_host_tier_map: references written in place into the pinned tier search like added ones;
    unwritten (zero) references match nothing; FIFO indexes refuse it."""
    R, m, n, B = 40, 256, 300, 2
    refs, _ = tidgen.refs(8, R, m)
    qs, _ = tidgen.queries(8, B, n, R_total=R, m=m, n_planted=80)
    rb = m * 128
    with tid.Index(ref_kp=m, hbm_budget_bytes=10 * rb, host_budget_bytes=64 * rb) as idx:
        idx.add_references(refs[:10])                 # HBM
        first, view = idx.host_tier_map(R - 10 + 4)   # pinned tier, filled in place (+4 left zero)
        assert first == 10 and view.shape == (R - 6, m, 128) and not view.any()
        view[:R - 10] = refs[10:]
        info = idx.info()
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, 5)
    assert info["hbm_references"] == 10 and info["host_references"] == R - 6
    want = oracle.search_counts(qs, refs)
    np.testing.assert_array_equal(counts[:, :R].astype(np.int64), want)
    assert (counts[:, R:] == 0).all()
    e_ids, e_cnt = oracle.topk(np.concatenate([want, np.zeros((B, 4), np.int64)], axis=1), 5)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)
    with tid.Index(ref_kp=m, hbm_budget_bytes=10 * rb, host_budget_bytes=64 * rb, cache_policy="fifo") as idx:
        with pytest.raises(tid.TidError) as e:
            idx.host_tier_map(4)
        assert e.value.status == tid.TID_ESTATE


def test_virtual_shards_merge_equals_single(tid):
    """G shards run one after another on one GPU, merged by the shard-merge kernel == the
    oracle's global top-k (and the 1-GPU search)."""
    R, m, n, B, k = 96, 256, 300, 3, 6
    refs, _ = tidgen.refs(0, R, m, K=16)        # K=16 clusters: many equal counts -> id tie-breaks
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, K=16, n_planted=30)
    e_ids, e_cnt, _ = oracle.search(qs, refs, k)
    with tid.Index(ref_kp=m) as one:
        one.add_references(refs)
        gi, gc = one.search(qs, k)
    for G in (2, 3, 8):
        li, lc = [], []
        for r in range(G):
            s, e = tid.shard_plan(R, G, r)
            with tid.Index(ref_kp=m, id_base=s) as sh:
                sh.add_references(refs[s:e])
                i, c = sh.search(qs, min(k, e - s))
                if e - s < k:  # pad short lists
                    i = np.concatenate([i, np.full((B, k - (e - s)), -1)], 1)
                    c = np.concatenate([c, np.zeros((B, k - (e - s)), np.int32)], 1)
                li.append(i); lc.append(c)
        with tid.Index(ref_kp=m) as mg:
            mi, mc = mg.merge_topk(np.stack(li), np.stack(lc))
        np.testing.assert_array_equal(mi, e_ids)
        np.testing.assert_array_equal(mc, e_cnt)
    np.testing.assert_array_equal(gi, e_ids)
    np.testing.assert_array_equal(gc, e_cnt)


def test_device_tensors_and_stream(tid):
    """Torch CUDA tensors in, device outputs; same answer as host buffers."""
    import torch
    R, m, n, B, k = 50, 256, 500, 4, 5
    refs, _ = tidgen.refs(0, R, m)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m)
    with tid.Index(ref_kp=m) as idx:
        idx.add_references(torch.from_numpy(refs).cuda())
        dq = torch.from_numpy(qs).cuda()
        ids = torch.empty((B, k), dtype=torch.int64, device="cuda")
        cnt = torch.empty((B, k), dtype=torch.int32, device="cuda")
        idx.search(dq, k, out=(ids, cnt))
        torch.cuda.synchronize()
        hi, hc = idx.search(qs, k)
    np.testing.assert_array_equal(ids.cpu().numpy(), hi)
    np.testing.assert_array_equal(cnt.cpu().numpy(), hc)
    e_ids, e_cnt, _ = oracle.search(qs, refs, k)
    np.testing.assert_array_equal(hi, e_ids)


@pytest.mark.parametrize("hi", [3, 24, 256])
def test_search_fast_path_fallback(tid, rng, hi):
    """Search path (folded norms: d known to +-1 from the MMA, exact global-memory recompute of
    the rows whose ratio decision that leaves open): low-range data makes many rows undecided,
    full-range data almost none; both must equal the oracle bit for bit (count matrix and
    top-k)."""
    R, m, n, B = 24, 256, 300, 2
    refs = rng.integers(0, hi, (R, m, 128), dtype=np.uint8)
    qs = rng.integers(0, hi, (B, n, 128), dtype=np.uint8)
    qs[0, :100] = refs[5, :100]                      # exact copies -> d1 = 0 rows
    qs[1, :50] = np.minimum(refs[7, :50].astype(int) + 1, 255)
    with tid.Index(ref_kp=m) as idx:
        idx.add_references(refs)
        fast = idx.search_counts(qs)
        ids, cnt = idx.search(qs, 5)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, 5)
    np.testing.assert_array_equal(fast.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


def test_search_boundary_ratios(tid):
    """Rows whose ratio sits exactly on / next to the 0.8 boundary at large distances (the
    folded +-1 bounds straddle it, forcing the exact recompute): q = 0, two reference keypoints
    with ||r||^2 = 16 s^2 and 25 s^2 (+/- 1)."""
    m, n = 256, 8
    R = np.zeros((1, m, 128), np.uint8)
    # d1 = 16*s^2 via sixteen entries of s; d2 = 25*s^2 via twenty-five entries of s (+ tweak)
    s = 40
    R[0, 0, :16] = s
    R[0, 1, :25] = s
    R[0, 2:, :] = 250                                 # far keypoints
    R2 = R.copy(); R2[0, 1, 25] = 1                    # d2 = 25 s^2 + 1 -> pass
    R3 = R.copy(); R3[0, 0, 16] = 1                    # d1 = 16 s^2 + 1 -> fail
    refs = np.concatenate([R, R2, R3], 0)
    qs = np.zeros((1, n, 128), np.uint8)
    with tid.Index(ref_kp=m) as idx:
        idx.add_references(refs)
        got = idx.search_counts(qs)
    np.testing.assert_array_equal(got.astype(np.int64), oracle.search_counts(qs, refs))
    assert got[0].tolist() == [0, n, 0]


def test_nccl_collective_path_single_rank(tid):
    """The multi-GPU path (collective reference count, local top-k -> ncclAllGather -> merge
    kernel) on a one-rank NCCL communicator must return exactly the oracle's top-k, with one
    count window and with several (running top-k), host and device buffers."""
    import torch  # loads PyTorch's NCCL first; libtid resolves the already-loaded library
    R, m, n, B, k = 80, 256, 300, 4, 7
    refs, _ = tidgen.refs(0, R, m, K=16)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, K=16, n_planted=40)
    gi, gc, _ = oracle.search(qs, refs, k)
    with tid.Index(ref_kp=m, rank=0, world_size=1, nccl_id=tid.nccl_unique_id()) as col:
        col.add_references(refs)
        ci, cc = col.search(qs, k)
        dq = torch.from_numpy(qs).cuda()
        di, dc = col.search(dq, k, out=(torch.empty((B, k), dtype=torch.int64, device="cuda"),
                                       torch.empty((B, k), dtype=torch.int32, device="cuda")))
        torch.cuda.synchronize()
        col.set_tuning(window_refs=13)
        wi, wc = col.search(qs, k)
        with pytest.raises(tid.TidError) as e:
            col.search(qs, R + 1)  # k > total references: refused on every rank alike
        assert e.value.status == tid.TID_EINVAL
    np.testing.assert_array_equal(ci, gi)
    np.testing.assert_array_equal(cc, gc)
    np.testing.assert_array_equal(di.cpu().numpy(), gi)
    np.testing.assert_array_equal(dc.cpu().numpy(), gc)
    np.testing.assert_array_equal(wi, gi)
    np.testing.assert_array_equal(wc, gc)


def test_nccl_empty_shard(tid):
    """A rank whose shard is empty still joins the collective (it used to return
    TID_ESTATE before the all-gather and hang the other ranks).  On a one-rank communicator the
    total is then 0: TID_ESTATE, raised after the collective count, consistently; once a
    reference exists the same index searches normally."""
    R, m, n, B = 5, 256, 200, 2
    refs, _ = tidgen.refs(0, R, m)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, n_planted=40)
    with tid.Index(ref_kp=m, rank=0, world_size=1, nccl_id=tid.nccl_unique_id()) as col:
        with pytest.raises(tid.TidError) as e:
            col.search(qs, 1)
        assert e.value.status == tid.TID_ESTATE
        col.add_references(refs)
        ids, cnt = col.search(qs, R)
    e_ids, e_cnt, _ = oracle.search(qs, refs, R)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


@pytest.mark.parametrize("W", [1, 7, 64, 4096])
def test_search_count_windows(tid, W):
    """tid_search over several count windows (window_refs = W): each window's counts are reduced
    into a running top-k (so the workspace does not grow with R); the ranking must equal the
    oracle's over the whole set, incl. heavy id tie-breaks (K = 16), deleted references, ragged
    kp and a host tier whose staging chunks straddle window boundaries."""
    R, m, n, B, k = 150, 256, 260, 3, 9
    refs, kp = tidgen.refs(0, R, m, K=16, kp_min=100, pad_byte=9)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, K=16, n_planted=40)
    dead = [3, 64, 65, 149]
    keep = np.setdiff1d(np.arange(R), dead)
    c = oracle.search_counts(qs, refs, kp=kp)
    e_ids, e_cnt = oracle.np_rank(c[:, keep], k)
    e_ids = keep[e_ids]
    rb = m * 128
    for host in (False, True):
        kw = dict(hbm_budget_bytes=40 * rb, host_budget_bytes=200 * rb) if host else {}
        with tid.Index(ref_kp=m, **kw) as idx:
            idx.add_references(refs, kp)
            idx.set_tuning(window_refs=W, host_chunk_refs=11)
            idx.delete(dead)
            ids, cnt = idx.search(qs, k)
            if host:
                assert idx.info()["host_references"] == R - 40
        np.testing.assert_array_equal(ids, e_ids, err_msg=f"host={host}")
        np.testing.assert_array_equal(cnt, e_cnt, err_msg=f"host={host}")


def test_add_all_or_nothing(tid, monkeypatch):
    """tid_add_references is all-or-nothing: an allocation failure in
    the middle of an add (injected with TID_FAULT_ALLOC: here the host-tier segment, after a new
    HBM segment was already allocated and filled) leaves the index exactly as before — same
    counts per tier, same ids, same search results — and the next add succeeds."""
    m, n, B, k = 256, 300, 2, 5
    rb = m * 128
    refs, _ = tidgen.refs(0, 30, m)
    qs, _ = tidgen.queries(0, B, n, R_total=30, m=m, n_planted=40)
    with tid.Index(ref_kp=m, hbm_budget_bytes=10 * rb, host_budget_bytes=100 * rb) as idx:
        assert idx.add_references(refs[:5]) == 0
        before = idx.info()
        monkeypatch.setenv("TID_FAULT_ALLOC", "2")  # 1st alloc: new HBM segment; 2nd: host tier
        with pytest.raises(tid.TidError) as e:
            idx.add_references(refs[5:25])
        assert e.value.status == tid.TID_ENOMEM
        monkeypatch.delenv("TID_FAULT_ALLOC")
        assert idx.info() == before
        ids, cnt = idx.search(qs, k)
        e_ids, e_cnt, _ = oracle.search(qs, refs[:5], k)
        np.testing.assert_array_equal(ids, e_ids)
        np.testing.assert_array_equal(cnt, e_cnt)
        idx.delete([1])  # dead flags sized to the committed references only
        assert idx.add_references(refs[5:30]) == 5
        info = idx.info()
        assert (info["hbm_references"], info["host_references"]) == (10, 20)
        ids, cnt = idx.search(qs, k)
    c = oracle.search_counts(qs, refs)
    c[:, 1] = -1
    e_ids, e_cnt = oracle.np_rank(c, k)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


def test_calls_on_different_streams(tid):
    """One index driven from two non-blocking torch streams back to back, device outputs, no host
    synchronisation in between: each call's work is ordered after the previous call's (the
    index's end-of-call event), so reused workspaces are never overwritten in flight."""
    import torch
    R, m, n, B, k = 200, 256, 1000, 8, 5
    refs, _ = tidgen.refs(0, R, m)
    qa, _ = tidgen.queries(0, B, n, R_total=R, m=m)
    qb, _ = tidgen.queries(50, B, 700, R_total=R, m=m)
    with tid.Index(ref_kp=m) as idx:
        idx.add_references(refs)
        s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
        da, db = torch.from_numpy(qa).cuda(), torch.from_numpy(qb).cuda()
        torch.cuda.synchronize()
        outs = []
        for i in range(4):
            st = s1 if i % 2 == 0 else s2
            with torch.cuda.stream(st):
                o = (torch.empty((B, k), dtype=torch.int64, device="cuda"),
                     torch.empty((B, k), dtype=torch.int32, device="cuda"))
                idx.search(da if i % 2 == 0 else db, k, out=o)
                outs.append(o)
        torch.cuda.synchronize()
    ea, eac, _ = oracle.search(qa, refs, k)
    eb, ebc, _ = oracle.search(qb, refs, k)
    for i, (ids, cnt) in enumerate(outs):
        np.testing.assert_array_equal(ids.cpu().numpy(), ea if i % 2 == 0 else eb)
        np.testing.assert_array_equal(cnt.cpu().numpy(), eac if i % 2 == 0 else ebc)


@pytest.mark.parametrize("m,n,kp_min", [(384, 768, 384), (384, 768, 100), (1024, 300, 500)])
def test_search_m_above_256(tid, m, n, kp_min):
    """The paper's operating point m = 384, n = 768 (Table 7) and m up to 1024:
    references span several 256-column chunks, merged per query row in index order."""
    R, B, k = 23, 2, 5
    refs, kp = tidgen.refs(0, R, m, kp_min=kp_min, pad_byte=77)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, kp_min=kp_min, n_planted=150)
    with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
        idx.add_references(refs, kp)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, k)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, k, kp=kp)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


# ------------------------------------------------------------------------------ index lifecycle (f3)
def _search_all(idx, qs, k):
    return idx.search_counts(qs), idx.search(qs, k)


def test_fifo_policy_swaps_oldest_batches(tid):
    """Paper §6.1: new batches enter HBM, the oldest are swapped to the host tier
    when HBM is full; results equal the all-HBM index."""
    R, m, n, B, k = 120, 256, 300, 3, 6
    refs, kp = tidgen.refs(0, R, m, kp_min=60, pad_byte=5)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, kp_min=60, n_planted=50)
    rb = m * 128
    with tid.Index(ref_kp=m) as a:
        a.add_references(refs, kp)
        ca, (ia, na) = _search_all(a, qs, k)
    with tid.Index(ref_kp=m, hbm_budget_bytes=50 * rb, host_budget_bytes=200 * rb, cache_policy="fifo") as b:
        b.set_tuning(host_chunk_refs=17)
        for s in range(0, R, 30):
            b.add_references(refs[s:s + 30], kp[s:s + 30])
        info = b.info()
        cb, (ib, nb) = _search_all(b, qs, k)
    assert info["hbm_references"] == 30 and info["host_references"] == 90  # newest batch in HBM
    np.testing.assert_array_equal(ca, cb)
    np.testing.assert_array_equal(ia, ib)
    np.testing.assert_array_equal(na, nb)


def test_delete_update_save_load(tid, tmp_path):
    R, m, n, B, k = 60, 256, 300, 3, 8
    refs, kp = tidgen.refs(0, R, m, kp_min=80, pad_byte=7)
    qs, tg = tidgen.queries(0, B, n, R_total=R, m=m, kp_min=80, n_planted=60)
    new_refs, new_kp = tidgen.refs(1000, 4, m, kp_min=80)
    upd_ids = np.array([3, 17, 41, 59])
    rb = m * 128
    with tid.Index(ref_kp=m, hbm_budget_bytes=35 * rb, host_budget_bytes=100 * rb) as idx:  # spans both tiers
        idx.add_references(refs, kp)
        idx.delete([int(tg[0]), 5, 50])
        idx.update(upd_ids, new_refs, new_kp)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, k)
        path = str(tmp_path / "index.tid")
        idx.save(path)
    # expected: the same edits applied to plain arrays, then the oracle
    e_refs, e_kp = refs.copy(), kp.copy()
    e_refs[upd_ids], e_kp[upd_ids] = new_refs, new_kp
    dead = {int(tg[0]), 5, 50}
    for d in dead:
        e_kp[d] = 0
    e_counts = oracle.search_counts(qs, e_refs, kp=e_kp)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    live = np.array([i for i in range(R) if i not in dead])
    li, lc = oracle.topk(e_counts[:, live], k)
    np.testing.assert_array_equal(ids, live[li])
    np.testing.assert_array_equal(cnt, lc)
    assert not np.isin(ids, list(dead)).any()
    with tid.Index(ref_kp=m, cache_policy="fifo", hbm_budget_bytes=40 * rb, host_budget_bytes=100 * rb) as idx2:
        assert idx2.load(path) == 0
        c2 = idx2.search_counts(qs)
        i2, n2 = idx2.search(qs, k)
    np.testing.assert_array_equal(c2, counts)
    np.testing.assert_array_equal(i2, ids)
    np.testing.assert_array_equal(n2, cnt)


# ------------------------------------------------------------------------------ ABI error behaviour
def test_abi_errors_and_empty_queries(tid):
    """include/tid.h conventions on a GPU: invalid arguments return TID_EINVAL (raised as TidError
    with the status) and leave the index usable; an empty query (n_q = 0) matches nothing."""
    R, m, n = 10, 256, 300
    refs, _ = tidgen.refs(0, R, m)
    qs, _ = tidgen.queries(0, 3, n, R_total=R, m=m, n_planted=50)
    with pytest.raises(tid.TidError) as e:
        tid.Index(ref_kp=1)  # ref_kp < 2
    assert e.value.status == tid.TID_EINVAL
    with tid.Index(ref_kp=m, query_kp_max=512) as idx:
        idx.add_references(refs)
        with pytest.raises(tid.TidError) as e:
            idx.search(qs, R + 1)  # k > number of references
        assert e.value.status == tid.TID_EINVAL
        big, _ = tidgen.queries(0, 1, 600, R_total=R, m=m)
        with pytest.raises(tid.TidError) as e:
            idx.search(big, 3)  # n > query_kp_max
        assert e.value.status == tid.TID_EINVAL
        n_q = np.array([0, n, 7], np.int32)  # still usable after the errors
        counts = idx.search_counts(qs, n_q=n_q)
        ids, cnt = idx.search(qs, 3, n_q=n_q)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, 3, n_q=n_q)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)
    assert (counts[0] == 0).all()


def test_search_massive_ties_stress(tid):
    """SURVEY §8(d) stress variant: K = 16 clusters (non-target counts ~ 0, massive ties) plus exact
    duplicate references: the (count desc, id asc) ranking must match the oracle element by element."""
    R, m, n, B, k = 120, 256, 600, 4, 20
    refs, _ = tidgen.refs(11, R, m, K=16)
    refs[60:90] = refs[30:60]  # identical copies -> identical counts -> ascending ids
    qs, _ = tidgen.queries(11, B, n, R_total=R, m=m, K=16, n_planted=40)
    with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
        idx.add_references(refs)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, k)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, k)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(counts[:, 30:60], counts[:, 60:90])
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


def test_plain_c_example_runs(tid, tmp_path):
    """The C ABI used from plain C (examples/search_example.c, host buffers): planted references rank
    first; exit status 0."""
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    lib_dir = os.path.join(root, "paper_conf_icpp_wangzll21_b200")
    exe = tmp_path / "search_example"
    subprocess.check_call(["gcc", "-O2", "-I", os.path.join(root, "include"),
                           os.path.join(root, "examples", "search_example.c"), "-L", lib_dir, "-ltid",
                           f"-Wl,-rpath,{lib_dir}", "-o", str(exe)])
    out = subprocess.run([str(exe)], capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stdout + out.stderr
    assert "verify(query 0, reference 3): 200 good matches" in out.stdout


def test_hbm_capacity_per_reference(tid):
    """HBM capacity (the paper's second headline metric): a resident
    m = 256 reference costs its 32,768 descriptor bytes plus 1 KiB of column terms W (the
    fifth MMA K-step's norm digits are expanded on chip from W, not stored), so the automatic
    budget of a 180 GB B200 holds >= 5 M references; m = 384 costs 49,152 + 2 KiB."""
    import torch
    free, total = torch.cuda.mem_get_info()
    with tid.Index(ref_kp=256) as idx:
        info = idx.info()
    assert info["hbm_bytes_per_reference"] == 256 * 128 + 1024
    cap = info["hbm_capacity_references"]
    assert cap * 256 * 128 <= free
    if total > 170e9:
        assert cap >= 4_900_000, cap
    with tid.Index(ref_kp=384) as idx:
        assert idx.info()["hbm_bytes_per_reference"] == 384 * 128 + 2048


def test_search_graph_replay_tracks_index_changes(tid):
    """Repeated device-buffer searches are replayed from a captured CUDA graph (second occurrence of
    a call shape); any change of the index (add, delete, tuning) must invalidate it: every result
    equals the oracle on the index as it is at that call."""
    import torch
    R, m, n, B, k = 40, 256, 300, 2, 4
    refs, _ = tidgen.refs(0, R + 10, m)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, n_planted=60)
    dq = torch.from_numpy(qs).cuda()
    ids = torch.empty((B, k), dtype=torch.int64, device="cuda")
    cnt = torch.empty((B, k), dtype=torch.int32, device="cuda")

    def check(nref, dead=()):
        c = oracle.search_counts(qs, refs[:nref])
        for d in dead:
            c[:, d] = -1
        e_ids, e_cnt = oracle.np_rank(c, k)
        np.testing.assert_array_equal(ids.cpu().numpy(), e_ids)
        np.testing.assert_array_equal(cnt.cpu().numpy(), e_cnt)

    with tid.Index(ref_kp=m) as idx:
        idx.add_references(refs[:R])
        for _ in range(4):  # direct, capture, replay, replay
            ids.fill_(-7)
            idx.search(dq, k, out=(ids, cnt))
            torch.cuda.synchronize()
            check(R)
        idx.add_references(refs[R:])
        for _ in range(3):
            idx.search(dq, k, out=(ids, cnt))
            torch.cuda.synchronize()
            check(R + 10)
        idx.delete([0, 7])
        for _ in range(3):
            idx.search(dq, k, out=(ids, cnt))
            torch.cuda.synchronize()
            check(R + 10, dead=(0, 7))
        idx.set_tuning(window_refs=9)
        for _ in range(3):
            idx.search(dq, k, out=(ids, cnt))
            torch.cuda.synchronize()
            check(R + 10, dead=(0, 7))


@pytest.mark.parametrize("n,m", [(2000, 700), (4100, 256)])
def test_large_query_budgets(tid, n, m):
    """Query keypoint budgets beyond the paper's (n = 2000, 4100: 16 / 33 query tiles) against
    references of 3 chunks (m = 700) and 1 chunk: search counts, top-k and verify (d1, i1, d2, i2)
    equal the oracle bit for bit."""
    R, B, k = 7, 2, 3
    refs, _ = tidgen.refs(0, R, m)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, n_planted=min(200, m))
    with tid.Index(ref_kp=m, query_kp_max=8192) as idx:
        idx.add_references(refs)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, k)
        vc, nn = idx.verify(qs, refs[:B])
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, k)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)
    ec, enn = oracle.verify(qs, refs[:B])
    np.testing.assert_array_equal(vc.astype(np.int64), ec)
    np.testing.assert_array_equal(nn.astype(np.int64), nn_from_oracle(enn))


@pytest.mark.parametrize("n,m,P", [(1000, 1000, 6), (300, 600, 5), (129, 257, 3), (200, 256, 4), (5, 2, 3)])
def test_verify_counts_only_folded(tid, rng, n, m, P):
    """Counts-only verification runs the folded kernel (s8 x u8 + norm K-step, column terms computed
    on chip, the +-1-undecided rows recomputed exactly): counts equal the oracle bit for bit, also
    with ragged n_q / m_r and adversarial pairs (ties in {0, 1, 2}, duplicates, identical rows)."""
    Q, Rr, _ = tidgen.pairs(P, n, m, n_planted=min(200, n, m))
    Q[1 % P, : n // 2] = rng.integers(0, 3, (n // 2, 128))
    Rr[1 % P] = rng.integers(0, 3, (m, 128))
    Rr[2 % P, : m // 2] = Rr[2 % P, m // 2: 2 * (m // 2)]
    n_q = rng.integers(1, n + 1, P).astype(np.int32)
    m_r = rng.integers(1, m + 1, P).astype(np.int32)
    with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
        c_full, _ = idx.verify(Q, Rr, want_nn=False)
        c_mask, _ = idx.verify(Q, Rr, n_q=n_q, m_r=m_r, want_nn=False)
    np.testing.assert_array_equal(c_full.astype(np.int64), oracle.verify(Q, Rr, want_nn=False)[0])
    np.testing.assert_array_equal(c_mask.astype(np.int64), oracle.verify(Q, Rr, n_q=n_q, m_r=m_r, want_nn=False)[0])


@pytest.mark.parametrize("n,m,grid", [(1000, 1000, 3), (300, 600, 2), (129, 257, 5), (100, 2, 4), (250, 384, 1),
                                      (700, 900, 7), (500, 2, 3), (384, 1024, 2), (1024, 256, 2), (257, 64, 1)])
def test_verify_streamed_pairs(tid, rng, n, m, grid):
    """Many pairs per CTA (a forced small grid): the pair-streaming verification kernel refills each
    reference slot as soon as the previous pair's tiles have left it, runs tile gt of its pair sequence
    on group gt % 3 and double-buffers the column terms by pair parity.  Every T (1 .. 8 query tiles),
    chunk count (1 .. 4), last-chunk piece skip and ragged n_q / m_r, with (d1, i1, d2, i2) and with the
    counts-only folded variant, equal the oracle."""
    P = 3 * grid + 4  # several pairs per CTA, uneven
    Q, Rr, _ = tidgen.pairs(P, n, m, n_planted=min(200, n, m))
    Q[1, : n // 2] = rng.integers(0, 3, (n // 2, 128))
    Rr[1] = rng.integers(0, 3, (m, 128))
    n_q = rng.integers(1, n + 1, P).astype(np.int32)
    m_r = rng.integers(1, m + 1, P).astype(np.int32)
    n_q[0], m_r[0] = n, m
    with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
        idx.set_tuning(grid=grid)
        c, nn = idx.verify(Q, Rr, n_q=n_q, m_r=m_r)
        c_fold, _ = idx.verify(Q, Rr, n_q=n_q, m_r=m_r, want_nn=False)
        c_full, _ = idx.verify(Q, Rr, want_nn=False)
    ec, enn = oracle.verify(Q, Rr, n_q=n_q, m_r=m_r)
    np.testing.assert_array_equal(c.astype(np.int64), ec)
    np.testing.assert_array_equal(c_fold.astype(np.int64), ec)
    np.testing.assert_array_equal(c_full.astype(np.int64), oracle.verify(Q, Rr, want_nn=False)[0])
    for p in range(P):
        np.testing.assert_array_equal(nn[p, :n_q[p]].astype(np.int64), nn_from_oracle(enn[p, :n_q[p]]))
        assert (nn[p, n_q[p]:] == -1).all()


@pytest.mark.parametrize("B,n,grid", [(1, 1000, 2), (2, 1000, 3), (3, 600, 1), (16, 100, 4)])
def test_search_small_batch_slot_banks(tid, B, n, grid):
    """Small batches (B * T <= 16 query tiles) alternate two banks of reference slots, and the producer
    warp expands the next job's norm digits while the current job runs; a forced small grid makes each
    CTA run many such jobs back to back (ragged last group, planted targets), bit-exact vs the oracle."""
    R, m = 301, 256
    refs, kp = tidgen.refs(11, R, m, kp_min=180)
    qs, tg = tidgen.queries(12, B, n, R_total=R, m=m, n_planted=min(120, n))
    with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
        idx.add_references(refs, kp)
        idx.set_tuning(grid=grid)
        counts = idx.search_counts(qs)
        ids, cnt = idx.search(qs, 5)
    e_ids, e_cnt, e_counts = oracle.search(qs, refs, 5, kp=kp)
    np.testing.assert_array_equal(counts.astype(np.int64), e_counts)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)
