"""Run one search (or, with `verify` as the first argument, one C2 verification of 4,096 pairs
n = m = 1000) with a -DTID_PROF build of libtid (TID_LIB=...) and print the per-role cycle buckets."""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tidgen  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402

if len(sys.argv) > 1 and sys.argv[1] == "verify":
    Q, Rr, _ = tidgen.pairs(4096, 1000, 1000)
    idx = tid.Index(ref_kp=256, query_kp_max=1000)
    idx.verify(Q, Rr, want_nn=False)
    idx.profile(True)
    idx.verify(Q, Rr, want_nn=False)
else:
    R, B, n, m = int(sys.argv[1]) if len(sys.argv) > 1 else 20000, 256, 1000, 256
    refs, _ = tidgen.refs(0, R, m)
    qs, _ = tidgen.queries(0, B, n, R_total=R, m=m)
    idx = tid.Index(ref_kp=m)
    idx.add_references(refs)
    idx.search(qs, 5)
    idx.profile(True)
    idx.search(qs, 5)
st = idx.stats()
lib = tid.load_library()
buf = np.zeros(148 * 32 * 8, np.uint64)
lib.tid_debug_read_prof(buf.ctypes.data, ctypes.c_size_t(buf.nbytes))
buf = buf.reshape(148, 32, 8).astype(np.float64)
nw = (tid.load_library() and 0) or None
print("match kernel ms", st["match_ms"], "launches", st["match_launches"])
names = {0: "producer", 1: "mma", 2: "mma", 3: "mma"}
for w in range(0, 32):
    if buf[:, w, 7].sum() == 0:
        continue
    tot = buf[:, w, 7].mean()
    parts = " ".join(f"{k}:{100 * buf[:, w, k].mean() / tot:5.1f}%" for k in range(7) if buf[:, w, k].sum() > 0)
    parts += f" other:{100 * (1 - buf[:, w, :7].sum(1).mean() / tot):5.1f}%"
    print(f"warp {w:2d} ({names.get(w, 'epilogue')}): total {tot / 1e6:8.2f} Mcyc  {parts}")
