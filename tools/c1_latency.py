import sys, time, statistics
sys.path.insert(0, '.')
import numpy as np, torch
import tidgen, paper_conf_icpp_wangzll21_b200 as tid
R, m, n, k = 64, 256, 256, 5
refs, _ = tidgen.refs(0, R, m)
qs, tg = tidgen.queries(0, 1, n, R_total=R, m=m)
dq = torch.from_numpy(qs).cuda()
ids = torch.empty((1, k), dtype=torch.int64, device='cuda'); cnt = torch.empty((1, k), dtype=torch.int32, device='cuda')
with tid.Index(ref_kp=m, query_kp_max=1024) as idx:
    idx.add_references(refs)
    for _ in range(20): idx.search(dq, k, out=(ids, cnt))
    torch.cuda.synchronize()
    hs = []
    for _ in range(200):
        t0 = time.perf_counter(); idx.search(dq, k, out=(ids, cnt)); hs.append(time.perf_counter() - t0)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ds = []
    for _ in range(200):
        e0.record(); idx.search(dq, k, out=(ids, cnt)); e1.record(); e1.synchronize(); ds.append(e0.elapsed_time(e1))
    print("host call p50 us", 1e6 * statistics.median(hs), "device p50 us", 1e3 * statistics.median(ds))
