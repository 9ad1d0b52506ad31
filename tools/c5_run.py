#!/usr/bin/env python
"""C5 (BASELINE configs[4], hybrid host cache; §6.1, Table 6) at the
box's real scale on one B200: fill the HBM tier (automatic budget) plus a pinned host tier filled
in place through tid_host_tier_map, then
  * time tid_search at B in {8, 64, 256} (comparisons/s, host-tier H2D GB/s, clocks);
  * check parity on samples the oracle can compute: every query's planted target ranks first,
    and the counts of sampled (query, reference) pairs from both tiers equal the oracle's;
  * check streamed == resident on a subset (the same 2,048 references searched from HBM).
Writes one JSON object (profiles/r2_c5.json when run under gpurun).

    python tools/c5_run.py [--refs 10000000] [--host-frac 0.6] [--steps 2]
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import tidgen  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402
from bench import ClockSampler, mem_available  # noqa: E402

SEED = 2021


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--refs", type=int, default=10_000_000)
    ap.add_argument("--host-frac", type=float, default=0.6)
    ap.add_argument("--steps", type=int, default=2)
    ap.add_argument("--batches", default="8,64,256")
    args = ap.parse_args()
    import torch
    m, n, k = 256, 1000, 5
    rb = m * 128
    avail = mem_available()
    probe = tid.Index(ref_kp=m)
    cap = probe.info()["hbm_capacity_references"]
    probe.close()
    n_hbm = min(args.refs, cap)
    n_host = min(args.refs - n_hbm, int(args.host_frac * avail) // rb)
    R = n_hbm + n_host
    log(f"host MemAvailable {avail / 1e9:.1f} GB; HBM capacity {cap} refs -> {n_hbm} HBM + {n_host} host")
    idx = tid.Index(ref_kp=m, query_kp_max=1024, host_budget_bytes=n_host * rb)
    t0 = time.perf_counter()
    step = 65536
    for off in range(0, n_hbm, step):
        r, _ = tidgen.refs(off, min(step, n_hbm - off), m, seed=SEED)
        idx.add_references(r)
    t_hbm = time.perf_counter() - t0
    t0 = time.perf_counter()
    if n_host:
        first, view = idx.host_tier_map(n_host)
        for off in range(0, n_host, step):
            c = min(step, n_host - off)
            tidgen.refs(n_hbm + off, c, m, seed=SEED, out=view[off:off + c])
    t_host = time.perf_counter() - t0
    info = idx.info()
    log(f"filled in {t_hbm:.0f}s + {t_host:.0f}s: {info}")
    out = {"case": "C5 hybrid host cache, 1 B200", "refs": R, "hbm_refs": n_hbm, "host_refs": n_host,
           "host_tier_GB": n_host * rb / 1e9, "host_mem_available_GB": avail / 1e9, "info": info,
           "fill_s": {"hbm": t_hbm, "host_in_place": t_host}, "runs": []}
    Bmax = max(int(b) for b in args.batches.split(","))
    qs, tg = tidgen.queries(0, Bmax, n, R_total=R, m=m, seed=SEED)
    dq_all = torch.from_numpy(qs).cuda()
    for B in (int(b) for b in args.batches.split(",")):
        dq = dq_all[:B].contiguous()
        ids = torch.empty((B, k), dtype=torch.int64, device="cuda")
        cnt = torch.empty((B, k), dtype=torch.int32, device="cuda")
        idx.search(dq, k, out=(ids, cnt))  # warm-up (also the first host-tier pass)
        torch.cuda.synchronize()
        idx.profile(True)
        ts = []
        with ClockSampler(0) as clk:
            for _ in range(args.steps):
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                idx.search(dq, k, out=(ids, cnt))
                e1.record()
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
        st = idx.stats()
        idx.profile(False)
        p50 = statistics.median(ts)
        top1 = float(np.mean(ids[:, 0].cpu().numpy() == tg[:B]))
        run = {"queries": B, "p50_ms": p50, "comparisons_per_s": B * R / (p50 / 1e3),
               "match_kernel_ms_per_search": st["match_ms"] / args.steps,
               "h2d_GB_per_search": st["h2d_bytes"] / args.steps / 1e9,
               "h2d_GBps_over_search": st["h2d_bytes"] / (sum(ts) / 1e3) / 1e9,
               "compute_share": st["match_ms"] / sum(ts), "planted_top1": top1, "clocks": clk.summary()}
        out["runs"].append(run)
        log(json.dumps(run))
    # ---- sampled parity vs the oracle (both tiers) + every planted target ranks first
    rng = np.random.default_rng(SEED)
    qsel = [0, 1]
    rsel = np.unique(np.concatenate([rng.choice(n_hbm, 600, replace=False),
                                     n_hbm + rng.choice(max(n_host, 1), 600 if n_host else 0, replace=False),
                                     tg[qsel]]))
    # the library's counts for these pairs: search_counts over a 2-query batch is the full R-long row
    got = idx.search_counts(qs[qsel])
    sub_counts = got[:, rsel].astype(np.int64)
    refs_sel = np.stack([tidgen.refs(int(r), 1, m, seed=SEED)[0][0] for r in rsel])
    want = oracle.search_counts(qs[qsel], refs_sel)
    out["parity"] = {"pairs_checked": int(sub_counts.size), "hbm_pairs": int(len(qsel) * np.sum(rsel < n_hbm)),
                     "host_pairs": int(len(qsel) * np.sum(rsel >= n_hbm)),
                     "exact": bool(np.array_equal(sub_counts, want)),
                     "planted_top1_all_batches": all(r["planted_top1"] == 1.0 for r in out["runs"])}
    # ---- streamed == resident on a subset: the first 2,048 host-tier references, searched from HBM
    if n_host:
        sub = 2048
        refs_h, _ = tidgen.refs(n_hbm, sub, m, seed=SEED)
        with tid.Index(ref_kp=m, query_kp_max=1024) as res:
            res.add_references(refs_h)
            rc = res.search_counts(qs[:8])
        sc8 = idx.search_counts(qs[:8])
        out["streamed_equals_resident"] = {"queries": 8, "refs": sub,
                                           "equal": bool(np.array_equal(sc8[:, n_hbm:n_hbm + sub], rc))}
    idx.close()
    print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
