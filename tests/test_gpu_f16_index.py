"""GPU parity of the float path stored in the index (descriptor "f16"): u8 SIFT
converted on the GPU to RootSIFT (or scaled SIFT) fp16 at ingest and per search, matched on
tcgen05.mma.kind::f16 through the same windows / top-k / host tier / merge machinery as the
integer path.  Expected values come from the float64 oracle on the same fp16 values (and, where
the fp16 values make every fp32 step exact, from the exact integer oracle)."""
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


def host_rank(counts, k, id_base=0):
    """(count desc, id asc) ranking of a count matrix the GPU produced, in plain NumPy (a property
    check of the top-k kernel against its own counts; the oracle never sees GPU output)."""
    counts = np.asarray(counts, np.int64)
    ids = np.arange(counts.shape[1]) + id_base
    order = np.lexsort((np.broadcast_to(ids, counts.shape), -counts), axis=1)[:, :k]
    return ids[order], np.take_along_axis(counts, order, 1).astype(np.int32)


def test_f16_index_rootsift_parity(tid):
    """RootSIFT fp16 index, 64 queries x 2,000 references: every count within +-1 of the float64
    oracle on the same fp16 values for >= 99.9 % of pairs; the planted target ranks first; the
    returned top-k is the (count desc, id asc) ranking of the index's own count matrix."""
    B, n, R, m, k = 64, 1000, 2000, 256, 5
    refs, _ = tidgen.refs(0, R, m)
    qs, tg = tidgen.queries(0, B, n, R_total=R, m=m)
    with tid.Index(ref_kp=m, query_kp_max=1024, descriptor="f16") as idx:
        idx.add_references(refs)
        counts = idx.search_counts(qs).astype(np.int64)
        ids, cnt = idx.search(qs, k)
        info = idx.info()
    assert info["hbm_bytes_per_reference"] == m * 128 * 2 + 256 * 16 * 2
    # the oracle end to end on the same u8 inputs: its own RootSIFT -> fp16, its own float64 counts
    want = oracle.f16_search_counts_c(oracle.to_fp16(oracle.rootsift(qs)), oracle.to_fp16(oracle.rootsift(refs)))
    want = want.astype(np.int64)
    d = np.abs(counts - want)
    assert np.mean(d <= 1) >= 0.999 and d.max() <= 2, (np.mean(d <= 1), d.max())
    np.testing.assert_array_equal(ids[:, 0], tg)
    e_ids, e_cnt = host_rank(counts, k)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


@pytest.mark.parametrize("host,m", [(False, 200), (True, 200), (False, 384), (True, 500)])
def test_f16_index_scaled_sift_exact(tid, host, m):
    """Raw SIFT x 2^-7 in fp16 is exact and so is every fp32 step of the kind::f16 path: the float
    index must reproduce the exact integer oracle bit for bit — with ragged kp and n_q, deleted
    references, several count windows, (host=True) a streamed pinned host tier, and references of
    two 256-row chunks (m = 384, the paper's operating point, Table 7; m = 500)."""
    R, n, B, k = 70, 300, 3, 6
    refs, kp = tidgen.refs(0, R, m, kp_min=60, pad_byte=31)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, kp_min=60, n_planted=50)
    n_q = np.array([300, 131, 7], np.int32)
    rb = m * 128 * 2
    kw = dict(hbm_budget_bytes=20 * rb, host_budget_bytes=100 * rb) if host else {}
    with tid.Index(ref_kp=m, query_kp_max=512, descriptor="f16", f16_rootsift=False, f16_scale=2.0 ** -7,
                   **kw) as idx:
        idx.add_references(refs, kp)
        if host:
            assert idx.info()["host_references"] == R - 20
        idx.set_tuning(window_refs=17, host_chunk_refs=9)
        idx.delete([4, 33])
        counts = idx.search_counts(qs, n_q=n_q).astype(np.int64)
        ids, cnt = idx.search(qs, k, n_q=n_q)
    want = oracle.search_counts(qs, refs, n_q=n_q, kp=kp)
    want[:, [4, 33]] = 0
    np.testing.assert_array_equal(counts, want)
    c = want.copy()
    c[:, [4, 33]] = -1
    e_ids, e_cnt = oracle.np_rank(c, k)
    np.testing.assert_array_equal(ids, e_ids)
    np.testing.assert_array_equal(cnt, e_cnt)


def test_f16_index_host_tier_map_and_equals_resident(tid):
    """A float index's host tier filled in place (fp16 values) searches exactly like the same
    references resident in HBM (same kernel, same fp16 values)."""
    R, m, n, B = 40, 256, 400, 2
    refs, _ = tidgen.refs(5, R, m)
    qs, _ = tidgen.queries(5, B, n, R_total=R, m=m)
    with tid.Index(ref_kp=m, descriptor="f16") as res:
        res.add_references(refs)
        c_res = res.search_counts(qs)
        r16 = res.f16_prepare(refs, True, 1.0)
    with tid.Index(ref_kp=m, descriptor="f16", host_budget_bytes=R * m * 256) as idx:
        first, view = idx.host_tier_map(R)
        view[:] = r16
        idx.set_tuning(host_chunk_refs=16)
        c_host = idx.search_counts(qs)
    np.testing.assert_array_equal(c_host, c_res)


def test_f16_index_m384_rootsift_parity(tid):
    """The paper's final configuration (RootSIFT + FP16, m = 384 reference keypoints, n = 768 query
    keypoints; §5.1, Table 7): counts within +-1 of the float64 oracle for >= 99.9 % of pairs and
    the planted target first."""
    B, n, R, m = 16, 768, 300, 384
    refs, _ = tidgen.refs(0, R, m)
    qs, tg = tidgen.queries(0, B, n, R_total=R, m=m)
    with tid.Index(ref_kp=m, query_kp_max=1024, descriptor="f16") as idx:
        idx.add_references(refs)
        counts = idx.search_counts(qs).astype(np.int64)
        ids, _ = idx.search(qs, 3)
    want = oracle.f16_search_counts_c(oracle.to_fp16(oracle.rootsift(qs)), oracle.to_fp16(oracle.rootsift(refs)))
    want = want.astype(np.int64)
    d = np.abs(counts - want)
    assert np.mean(d <= 1) >= 0.999 and d.max() <= 2
    np.testing.assert_array_equal(ids[:, 0], tg)


def test_f16_index_graph_replay(tid):
    """Repeated device-buffer searches of a float index replay a captured graph: the same answer as
    the first (direct) call, and as the index's own count matrix ranked on the host."""
    import torch
    R, m, n, B, k = 30, 256, 300, 2, 4
    refs, _ = tidgen.refs(3, R, m)
    qs, _ = tidgen.queries(3, B, n, R_total=R, m=m)
    dq = torch.from_numpy(qs).cuda()
    with tid.Index(ref_kp=m, descriptor="f16") as idx:
        idx.add_references(refs)
        c = idx.search_counts(qs).astype(np.int64)
        outs = []
        ids = torch.empty((B, k), dtype=torch.int64, device="cuda")
        cnt = torch.empty((B, k), dtype=torch.int32, device="cuda")
        for _ in range(4):  # same buffers: direct, capture, replay, replay
            ids.fill_(-5)
            idx.search(dq, k, out=(ids, cnt))
            torch.cuda.synchronize()
            outs.append((ids.cpu().numpy(), cnt.cpu().numpy()))
    e_ids, e_cnt = host_rank(c, k)
    for ids, cnt in outs:
        np.testing.assert_array_equal(ids, e_ids)
        np.testing.assert_array_equal(cnt, e_cnt)


def test_f16_index_lifecycle(tid, tmp_path):
    """Float index lifecycle: delete / update in place and the FIFO hybrid cache behave like the u8
    index (exact on u8 x 2^-7); save / load are refused (TID_EUNSUPPORTED: the persisted format is
    the u8 one)."""
    R, m, n, B, k = 24, 256, 200, 2, 5
    s = 2.0 ** -7
    refs, _ = tidgen.refs(0, R + 4, m)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, n_planted=50)
    rb = m * 256
    with tid.Index(ref_kp=m, descriptor="f16", f16_rootsift=False, f16_scale=s, hbm_budget_bytes=8 * rb,
                   host_budget_bytes=64 * rb, cache_policy="fifo") as idx:
        for b0 in range(0, R, 6):  # FIFO: every batch enters HBM, the oldest move to the host tier
            idx.add_references(refs[b0:b0 + 6])
        info = idx.info()
        assert info["hbm_references"] <= 8 and info["host_references"] >= R - 8
        idx.delete([3])
        idx.update([5, 20], refs[R:R + 2])  # one in the host tier, one in HBM
        counts = idx.search_counts(qs).astype(np.int64)
        with pytest.raises(tid.TidError) as e:
            idx.save(str(tmp_path / "f.tidx"))
        assert e.value.status == tid.TID_EUNSUPPORTED
    cur = refs[:R].copy()
    cur[5], cur[20] = refs[R], refs[R + 1]
    want = oracle.search_counts(qs, cur)
    want[:, 3] = 0
    np.testing.assert_array_equal(counts, want)
