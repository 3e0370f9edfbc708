"""Multi-process host logic of the weak-scaling path (§8(e)) on CPU with gloo, world
size 2: the per-checkpoint 32-byte records are all-gathered, each rank's file offset is
the exclusive prefix of diff bytes over ranks, and the box time is the max over ranks."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, out):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    import bench
    # rank r's diffs: k-th checkpoint has 1000*(r+1) + k bytes
    recs = [[1000 * (rank + 1) + k, 64 * (k + 1), 1000 * (rank + 1) + k - 64 * (k + 1), 10 + rank] for k in range(3)]
    g = bench.allgather_sizes(recs, ws)
    offs = bench.file_offsets(g)
    mx = bench.max_over_ranks(1.5 + rank, ws)
    sm = bench.sum_over_ranks(100.0 * (rank + 1), ws)
    out[rank] = (g, offs, mx, sm)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.timeout(120)
def test_allgather_offsets_and_max_gloo():
    ws = 2
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(ws, _free_port(), out), nprocs=ws, join=True)
    for r in range(ws):
        g, offs, mx, sm = out[r]
        assert len(g) == ws
        assert g[0][1][0] == 1001 and g[1][2][0] == 2002
        # rank 0 writes first; rank 1 starts after rank 0's diff of the same checkpoint
        assert offs[0] == [0, 0, 0]
        assert offs[1] == [1000, 1001, 1002]
        assert mx == 2.5 and sm == 300.0


def test_file_offsets_single_rank():
    import bench
    g = [[[10, 1, 9, 0], [20, 1, 19, 0]]]
    assert bench.file_offsets(g) == [[0, 0]]
