"""Small search / verify / host-tier invocations for compute-sanitizer (memcheck, racecheck,
synccheck).  Checks results against the oracle too, so a silent corruption also fails."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
import tidgen  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402

refs, kp = tidgen.refs(0, 13, 256, kp_min=50, pad_byte=3)
qs, _ = tidgen.queries(0, 3, 300, R_total=13, m=256, kp_min=50, n_planted=40)
with tid.Index(ref_kp=256, query_kp_max=1024, hbm_budget_bytes=8 * 256 * 128, host_budget_bytes=64 * 256 * 128) as idx:
    idx.set_tuning(host_chunk_refs=3)
    idx.add_references(refs, kp)
    c = idx.search_counts(qs)
    ids, cn = idx.search(qs, 4)
e_ids, e_cn, e_c = oracle.search(qs, refs, 4, kp=kp)
assert np.array_equal(c.astype(np.int64), e_c) and np.array_equal(ids, e_ids)
Q, R, _ = tidgen.pairs(3, 200, 300)
with tid.Index(ref_kp=256) as idx:
    vc, nn = idx.verify(Q, R)
ec, _ = oracle.verify(Q, R)
assert np.array_equal(vc.astype(np.int64), ec)
# f1 float path (kind::f16, folded norms): u8 x 2^-7 is exact, so counts equal the integer oracle
Rr, _ = tidgen.refs(5, 5, 200)
Qf, _ = tidgen.queries(5, 2, 300, R_total=5, m=200, n_planted=60)
with tid.Index(query_kp_max=1024) as idx:
    q16, r16 = idx.f16_prepare(Qf, False, 2.0 ** -7), idx.f16_prepare(Rr, False, 2.0 ** -7)
    fc = idx.f16_search_counts(q16, r16)
assert np.array_equal(fc.astype(np.int64), oracle.search_counts(Qf, Rr))
# round 2: several count windows + deletes, verify with ragged m_r (rows masked in the kernel),
# the float index (fp16 storage + host tier), post-match verification (f4)
with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
    idx.add_references(refs, kp)
    idx.set_tuning(window_refs=4)
    idx.delete([2])
    ids, cn = idx.search(qs, 4)
c2 = oracle.search_counts(qs, refs, kp=kp)
c2[:, 2] = -1
assert np.array_equal(ids, oracle.np_rank(c2, 4)[0])
m_r = np.array([300, 17, 2], np.int32)
with tid.Index(ref_kp=256) as idx:
    vc, nn = idx.verify(Q, R, m_r=m_r)
assert np.array_equal(vc.astype(np.int64), oracle.verify(Q, R, m_r=m_r)[0])
with tid.Index(ref_kp=200, descriptor="f16", f16_rootsift=False, f16_scale=2.0 ** -7,
               hbm_budget_bytes=2 * 200 * 256, host_budget_bytes=8 * 200 * 256) as idx:
    idx.set_tuning(host_chunk_refs=2)
    idx.add_references(Rr)
    fc2 = idx.search_counts(Qf)
assert np.array_equal(fc2.astype(np.int64), oracle.search_counts(Qf, Rr))
rng = np.random.default_rng(1)
qxy = (rng.random((3, 200, 2)) * 100).astype(np.float32)
rxy = (rng.random((3, 300, 2)) * 100).astype(np.float32)
with tid.Index(ref_kp=256) as idx:
    _, g, inl, mdl = idx.verify_geometric(Q, R, qxy, rxy, iterations=64, inlier_px=5.0)
_, onn = oracle.verify(Q, R)
eg, ei, em = oracle.geometric(onn, qxy, rxy, iterations=64, inlier_px=5.0)
assert np.array_equal(g.astype(np.int64), eg) and np.array_equal(inl.astype(np.int64), ei)
# graph replay (device buffers, repeated shape) and a small batch (two slot banks)
import torch  # noqa: E402
with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
    idx.add_references(refs, kp)
    dq = torch.from_numpy(qs).cuda()
    did = torch.empty((3, 4), dtype=torch.int64, device="cuda")
    dcn = torch.empty((3, 4), dtype=torch.int32, device="cuda")
    for _ in range(3):
        idx.search(dq, 4, out=(did, dcn))
    torch.cuda.synchronize()
assert np.array_equal(did.cpu().numpy(), e_ids)
print("sanitize run ok")
# streamed verification (n > 256): several pairs per CTA (grid 2), ragged n_q / m_r, nn and counts-only
Qs, Rs, _ = tidgen.pairs(7, 500, 600, n_planted=150)
n_q = np.array([500, 3, 257, 400, 129, 500, 1], np.int32)
m_r = np.array([600, 2, 300, 599, 256, 257, 600], np.int32)
with tid.Index(ref_kp=256, query_kp_max=1024) as idx:
    idx.set_tuning(grid=2)
    vc, nn = idx.verify(Qs, Rs, n_q=n_q, m_r=m_r)
    vf, _ = idx.verify(Qs, Rs, n_q=n_q, m_r=m_r, want_nn=False)
ec, _ = oracle.verify(Qs, Rs, n_q=n_q, m_r=m_r)
assert np.array_equal(vc.astype(np.int64), ec) and np.array_equal(vf.astype(np.int64), ec)
print("streamed verification ok")
