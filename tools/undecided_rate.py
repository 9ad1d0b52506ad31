"""Rate of rows the folded search leaves undecided (ratio within the +-1 bound -> exact global
recompute), from a -DTID_PROF build: python tools/undecided_rate.py [R]"""
import ctypes
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import tidgen  # noqa: E402
import paper_conf_icpp_wangzll21_b200 as tid  # noqa: E402

R, B, n, m = int(sys.argv[1]) if len(sys.argv) > 1 else 20000, 256, 1000, 256
refs, _ = tidgen.refs(0, R, m)
qs, _ = tidgen.queries(0, B, n, R_total=R, m=m)
with tid.Index(ref_kp=m) as idx:
    idx.add_references(refs)
    idx.search(qs, 5)
lib = tid.load_library()
buf = np.zeros(148 * 32 * 8, np.uint64)
lib.tid_debug_read_prof(buf.ctypes.data, ctypes.c_size_t(buf.nbytes))
rows = B * 1024 * R  # padded rows x references, one search
units = B * 8 * R * 4  # warp-units (4 lane-quarter warps per 128-row unit)
print(f"undecided rows {int(buf[-2])} of {rows} ({buf[-2] / rows:.2e}); warp-units with any: {int(buf[-1])} "
      f"of {units} ({buf[-1] / units:.2e})")
