"""Row f4 timing: tid_verify_geometric on C2-shaped pairs (4,096 x 1,000 x 1,000) with planted coordinates,
vs tid_verify alone (the difference is the edge-removal + RANSAC kernel).  python tools/geom_bench.py [iters]"""
import json
import os
import statistics
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tidgen  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402

iters = int(sys.argv[1]) if len(sys.argv) > 1 else 256
P, n, m = 4096, 1000, 1000
Q, R, pos = tidgen.pairs(P, n, m)
rng = np.random.default_rng(3)
qxy = (rng.random((P, n, 2)) * 640).astype(np.float32)
rxy = (rng.random((P, m, 2)) * 640).astype(np.float32)
import torch  # noqa: E402
dq, dr = torch.from_numpy(Q).cuda(), torch.from_numpy(R).cuda()
with tid.Index(ref_kp=256, query_kp_max=n) as idx:
    for _ in range(2):
        idx.verify_geometric(dq, dr, qxy, rxy, iterations=iters, inlier_px=3.0)
        idx.verify(dq, dr, want_nn=True)
    tg, tv = [], []
    for _ in range(5):
        torch.cuda.synchronize(); t = time.perf_counter()
        idx.verify_geometric(dq, dr, qxy, rxy, iterations=iters, inlier_px=3.0)
        torch.cuda.synchronize(); tg.append(1e3 * (time.perf_counter() - t))
        t = time.perf_counter()
        idx.verify(dq, dr, want_nn=True)
        torch.cuda.synchronize(); tv.append(1e3 * (time.perf_counter() - t))
print(json.dumps({"case": "f4 verify_geometric (C2 shape, host coordinates)", "pairs": P, "iterations": iters,
                  "geometric_ms_p50": statistics.median(tg), "verify_nn_ms_p50": statistics.median(tv)}))
