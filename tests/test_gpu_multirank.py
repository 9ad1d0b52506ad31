"""Multi-GPU sharded search through libtid's own NCCL path: one process per
GPU, contiguous reference-id shards (dist.shard_plan), ncclUniqueId broadcast over the torch
process group, collective tid_search (all-reduced reference total, local top-k, ncclAllGather,
identical GPU merge on every rank).  Every rank's result must equal the oracle's global top-k,
including a layout where one rank's shard is empty.  Needs >= 2 GPUs: skipped (with the reason)
on a one-GPU box; the host logic is covered on CPU by tests/test_distributed.py and
tests/test_bench_multirank.py."""
import os
import socket
import sys

import numpy as np
import pytest

import oracle
import tidgen

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, R, B, k, out_dir):
    sys.path.insert(0, ROOT)
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_wangzll21_b200 as tid
    from paper_conf_icpp_wangzll21_b200.dist import create_sharded_index
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        m, n = 256, 300
        idx, (start, end) = create_sharded_index(R, ref_kp=m, device=rank)
        with idx:
            if end > start:
                refs, _ = tidgen.refs(start, end - start, m, K=16)
                idx.add_references(refs)
            qs, _ = tidgen.queries(0, B, n, R_total=R, m=m, K=16, n_planted=min(40, n))
            ids, cnt = idx.search(qs, k)
            info = idx.info()
        np.save(os.path.join(out_dir, f"r{rank}.npy"), np.concatenate([ids, cnt.astype(np.int64)], 1))
        assert info["world_size"] == world
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("R,k", [(97, 6), (1, 1)])
def test_two_rank_nccl_search_equals_oracle(tmp_path, R, k):
    import torch
    import torch.multiprocessing as mp
    if torch.cuda.device_count() < 2:
        pytest.skip(f"needs 2 GPUs, {torch.cuda.device_count()} visible (NCCL refuses two ranks on one GPU)")
    world, B = 2, 3
    mp.start_processes(_worker, args=(world, _free_port(), R, B, k, str(tmp_path)), nprocs=world, join=True,
                       start_method="spawn")
    refs, _ = tidgen.refs(0, R, 256, K=16)
    qs, _ = tidgen.queries(0, B, 300, R_total=R, m=256, K=16, n_planted=40)
    ei, ec, _ = oracle.search(qs, refs, k)
    want = np.concatenate([ei, ec.astype(np.int64)], 1)
    for r in range(world):
        np.testing.assert_array_equal(np.load(tmp_path / f"r{r}.npy"), want)
