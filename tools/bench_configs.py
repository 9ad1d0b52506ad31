#!/usr/bin/env python
"""Secondary measurements (one B200): C1 latency, C2 verification, C3 throughput, the batch
sweep (B200 analogue of the paper's Fig. 4) and host-tier streaming (C5 analogue,
§6).  Prints one JSON object per measurement; DESIGN.md §8 quotes them.

    python tools/bench_configs.py [c1] [c2] [c3] [sweep] [host]
"""
from __future__ import annotations

import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import tidgen  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402
from bench import ClockSampler  # noqa: E402  (nvidia-smi clocks during each timed region)


def log(*a):
    print(*a, file=sys.stderr, flush=True)


LAST_CLOCKS = {}


def timed(fn, reps, warm=3):
    """CUDA-event times (ms) of `reps` calls after `warm` untimed ones; nvidia-smi clocks sampled
    during the timed calls land in LAST_CLOCKS (added to every JSON record)."""
    import torch
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    ts = []
    with ClockSampler(torch.cuda.current_device()) as clk:
        t_start = time.perf_counter()
        # at least `reps` calls and at least 1.5 s, so that nvidia-smi (200 ms period, slow to start)
        # samples the clocks during timed calls even for sub-millisecond ones (C1, C2)
        while len(ts) < reps or (time.perf_counter() - t_start < 1.5 and len(ts) < 100000):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            fn()
            e1.record()
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
    LAST_CLOCKS.clear()
    LAST_CLOCKS.update(clk.summary())
    return ts


def search_case(name, B, n, R, m, k, reps, hbm_budget=0, host_budget=0, chunk=0):
    import torch
    t0 = time.perf_counter()
    idx = tid.Index(ref_kp=m, query_kp_max=max(n, 1), hbm_budget_bytes=hbm_budget, host_budget_bytes=host_budget)
    if chunk:
        idx.set_tuning(host_chunk_refs=chunk)
    step = 100_000
    for s in range(0, R, step):
        refs, _ = tidgen.refs(s, min(step, R - s), m)
        idx.add_references(refs)
    qs, tg = tidgen.queries(0, B, n, R_total=R, m=m)
    log(f"{name}: setup {time.perf_counter() - t0:.1f}s info {idx.info()}")
    dq = torch.from_numpy(qs).cuda()
    ids = torch.empty((B, k), dtype=torch.int64, device="cuda")
    cnt = torch.empty((B, k), dtype=torch.int32, device="cuda")
    for _ in range(3):
        idx.search(dq, k, out=(ids, cnt))
    idx.profile(True)
    ts = timed(lambda: idx.search(dq, k, out=(ids, cnt)), reps, warm=0)
    st = idx.stats()
    hq = torch.from_numpy(qs).pin_memory()
    ts_e2e = []
    for _ in range(min(reps, 5)):
        t = time.perf_counter()
        idx.search(hq, k)
        ts_e2e.append(1e3 * (time.perf_counter() - t))
    top1 = float(np.mean(ids[:, 0].cpu().numpy() == tg))
    p50 = statistics.median(ts)
    out = {"case": name, "queries": B, "query_kp": n, "refs": R, "ref_kp": m, "top_k": k,
           "p50_ms": p50, "p99_ms": float(np.percentile(ts, 99)), "comparisons_per_s": B * R / (p50 / 1e3),
           "e2e_p50_ms": statistics.median(ts_e2e), "e2e_comparisons_per_s": B * R / (statistics.median(ts_e2e) / 1e3),
           "match_kernel_ms_per_search": st["match_ms"] / len(ts) if st["match_launches"] else None,
           "h2d_GBps": (st["h2d_bytes"] / (sum(ts) / 1e3) / 1e9) if st["h2d_bytes"] else 0.0,
           "planted_top1": top1, "info": idx.info(), "clocks": dict(LAST_CLOCKS),
           "tensor_tops_int8": 2.0 * B * R * n * m * 128 / (p50 / 1e3) / 1e12}
    idx.close()
    print(json.dumps(out), flush=True)
    return out


def verify_case(P=4096, n=1000, m=1000, reps=10):
    import torch
    Q, Rr, pos = tidgen.pairs(P, n, m)
    idx = tid.Index(ref_kp=256, query_kp_max=max(n, 1))
    dq, dr = torch.from_numpy(Q).cuda(), torch.from_numpy(Rr).cuda()
    cnt = torch.empty(P, dtype=torch.int32, device="cuda")
    nn = torch.empty((P, n, 4), dtype=torch.int32, device="cuda")
    ts = timed(lambda: idx.verify(dq, dr, out=(cnt, None)), reps)
    ts_nn = timed(lambda: idx.verify(dq, dr, out=(cnt, nn)), reps)
    c = cnt.cpu().numpy()
    out = {"case": "C2 verify", "pairs": P, "query_kp": n, "ref_kp": m, "p50_ms": statistics.median(ts),
           "comparisons_per_s": P / (statistics.median(ts) / 1e3), "p50_ms_with_nn": statistics.median(ts_nn),
           "positives_mean_count": float(c[pos].mean()), "negatives_mean_count": float(c[~pos].mean()),
           "tensor_tops_int8": 2.0 * P * n * m * 128 / (statistics.median(ts) / 1e3) / 1e12, "clocks": dict(LAST_CLOCKS)}
    idx.close()
    print(json.dumps(out), flush=True)


def f16_case(B=64, n=1000, R=20000, m=256, reps=5):
    """Row f1: RootSIFT fp16 search counts (tcgen05 kind::f16) vs the integer path on the same
    workload; Eq. 2 compression error of RootSIFT in fp16 on a small sample (oracle)."""
    import torch
    import oracle
    refs, _ = tidgen.refs(0, R, m)
    qs, tg = tidgen.queries(0, B, n, R_total=R, m=m)
    idx = tid.Index(ref_kp=m, query_kp_max=n)
    dq, dr = torch.from_numpy(qs).cuda(), torch.from_numpy(refs).cuda()
    q16 = torch.empty(qs.shape, dtype=torch.float16, device="cuda")
    r16 = torch.empty(refs.shape, dtype=torch.float16, device="cuda")
    idx.f16_prepare(dq, True, 1.0, out=q16)
    idx.f16_prepare(dr, True, 1.0, out=r16)
    out = torch.empty((B, R), dtype=torch.int32, device="cuda")
    ts = timed(lambda: idx.f16_search_counts(q16, r16, out=out), reps)
    top1 = float(np.mean(out.argmax(1).cpu().numpy() == tg))
    rq, rr = oracle.rootsift(qs[0, :200]), oracle.rootsift(refs[0])
    err = oracle.compression_error(rq, rr, oracle.to_fp16(rq), oracle.to_fp16(rr))
    res = {"case": "f1 RootSIFT fp16", "queries": B, "query_kp": n, "refs": R, "ref_kp": m,
           "p50_ms": statistics.median(ts), "comparisons_per_s": B * R / (statistics.median(ts) / 1e3),
           "planted_top1": top1, "eq2_compression_error_sample": err}
    idx.close()
    print(json.dumps(res), flush=True)


def main():
    what = sys.argv[1:] or ["c1", "c3", "c2", "sweep", "f16"]
    if "f16" in what:
        f16_case()
    if "c1" in what:
        search_case("C1", 1, 256, 64, 256, 5, reps=100)
    if "c3" in what:
        search_case("C3", 64, 1000, 100_000, 256, 5, reps=5)
    if "c2" in what:
        verify_case()
    if "sweep" in what:
        for B in (1, 8, 64, 256):
            search_case(f"sweep B={B}", B, 1000, 100_000, 256, 5, reps=5 if B >= 64 else 20)
    if "table7" in what:
        # B200 analogue of the speed half of Table 7: reference budget m
        # and query budget n at B = 256
        for m, n in ((768, 768), (512, 768), (384, 768), (256, 768), (384, 1024), (384, 512), (384, 384)):
            R = int(os.environ.get("T7_REFS", "30000"))
            search_case(f"table7 m={m} n={n}", 256, n, R, m, 5, reps=3)
    if "host" in what:
        R = int(os.environ.get("HOST_REFS", "1000000"))
        rb = 256 * 128
        for B in (8, 64):
            search_case(f"host-tier B={B}", B, 1000, R, 256, 5, reps=3, hbm_budget=rb, host_budget=(R + 1) * rb,
                        chunk=32768)


if __name__ == "__main__":
    main()
