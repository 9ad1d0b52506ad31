"""Three C2 verifications with (d1, i1, d2, i2) output (for ncu captures of the packed-key streamed kernel)."""
import sys, os
sys.path.insert(0, os.getcwd())
import torch, tidgen, paper_conf_icpp_wangzll21_b200 as tid
Q, Rr, pos = tidgen.pairs(4096, 1000, 1000)
idx = tid.Index(ref_kp=256, query_kp_max=1000)
dq, dr = torch.from_numpy(Q).cuda(), torch.from_numpy(Rr).cuda()
cnt = torch.empty(4096, dtype=torch.int32, device="cuda")
nn = torch.empty((4096, 1000, 4), dtype=torch.int32, device="cuda")
for _ in range(3): idx.verify(dq, dr, out=(cnt, nn))
torch.cuda.synchronize()
