"""One warm-up + N timed searches of B queries against R references (device-resident queries);
prints match-kernel ms and comparisons/s.  Used under ncu / for A-B experiments with TID_LIB.
usage: python tools/run_search.py [R=20000] [B=256] [N=3]"""
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tidgen  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402

R = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
B = int(sys.argv[2]) if len(sys.argv) > 2 else 256
N = int(sys.argv[3]) if len(sys.argv) > 3 else 3
n, m, k = 1000, 256, 5
refs, _ = tidgen.refs(0, R, m)
qs, tg = tidgen.queries(0, B, n, R_total=R, m=m)
import torch  # noqa: E402
dq = torch.from_numpy(qs).cuda()
with tid.Index(ref_kp=m) as idx:
    idx.add_references(refs)
    ids, cnt = idx.search(dq, k)
    torch.cuda.synchronize()
    idx.profile(True)
    t0 = time.perf_counter()
    for _ in range(N):
        ids, cnt = idx.search(dq, k)
    torch.cuda.synchronize()
    dt = (time.perf_counter() - t0) / N
    st = idx.stats()
    ids = ids.cpu().numpy() if hasattr(ids, "cpu") else ids
    top1 = float(np.mean(ids[:, 0] == tg))
    ms = st["match_ms"] / max(1, st["match_launches"])
    print(f"R={R} B={B} wall {dt * 1e3:.2f} ms/search; match kernel {ms:.3f} ms/launch "
          f"-> {B * R / (ms / 1e3) / 1e6:.2f} M comparisons/s (kernel), {B * R / dt / 1e6:.2f} M/s (wall); "
          f"planted top1 {top1:.3f}")
