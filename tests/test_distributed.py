"""Multi-process (gloo, world_size 2, CPU) checks of the sharded-search host logic
(SURVEY.md §8(e)): contiguous id shards, ncclUniqueId broadcast plumbing, and that merging the
per-rank top-k lists in the shared total order reproduces the single-process top-k.  The
per-rank lists come from the oracle (test infrastructure); the GPU merge kernel itself is
covered by tests/test_gpu_parity.py::test_virtual_shards_merge_equals_single."""
import os
import socket
import sys

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, R, B, k, result_dir):
    sys.path.insert(0, ROOT)
    import oracle
    import tidgen
    from paper_conf_icpp_wangzll21_b200.dist import exchange_nccl_id, shard_plan
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import torch
        uid = exchange_nccl_id(lambda: bytes(range(128)))
        assert uid == bytes(range(128))
        start, end = shard_plan(R, world, rank)
        refs, _ = tidgen.refs(start, end - start, 64, K=16)
        qs, _ = tidgen.queries(0, B, 80, R_total=R, m=64, K=16, n_planted=20)
        c = oracle.search_counts(qs, refs)
        ids, cnt = oracle.topk(c, k, id_base=start)
        gi = [torch.zeros((B, k), dtype=torch.int64) for _ in range(world)]
        gc = [torch.zeros((B, k), dtype=torch.int32) for _ in range(world)]
        dist.all_gather(gi, torch.from_numpy(ids))
        dist.all_gather(gc, torch.from_numpy(cnt))
        mi, mc = oracle.merge_topk(np.stack([t.numpy() for t in gi]), np.stack([t.numpy() for t in gc]))
        np.save(os.path.join(result_dir, f"r{rank}.npy"), np.concatenate([mi, mc.astype(np.int64)], 1))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_gloo_sharded_topk_equals_single(tmp_path, world):
    import oracle
    import tidgen
    R, B, k = 37, 3, 6
    mp.start_processes(_worker, args=(world, _free_port(), R, B, k, str(tmp_path)), nprocs=world,
                       join=True, start_method="spawn")
    refs, _ = tidgen.refs(0, R, 64, K=16)
    qs, _ = tidgen.queries(0, B, 80, R_total=R, m=64, K=16, n_planted=20)
    ei, ec, _ = oracle.search(qs, refs, k)
    expect = np.concatenate([ei, ec.astype(np.int64)], 1)
    for r in range(world):
        np.testing.assert_array_equal(np.load(tmp_path / f"r{r}.npy"), expect)


def test_shard_plan_properties():
    from paper_conf_icpp_wangzll21_b200.dist import shard_plan
    for R, G in [(1_000_000, 8), (10, 3), (7, 8), (100_000, 1), (5, 5)]:
        spans = [shard_plan(R, G, r) for r in range(G)]
        assert spans[0][0] == 0 and spans[-1][1] == R
        assert all(spans[i][1] == spans[i + 1][0] for i in range(G - 1))
        assert max(e - s for s, e in spans) - min(e - s for s, e in spans) <= 1
    with pytest.raises(ValueError):
        shard_plan(10, 2, 2)
