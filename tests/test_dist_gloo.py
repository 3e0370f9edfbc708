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


@pytest.mark.timeout(300)
def test_bench_self_launches_ranks():
    """`bench.py --gpus 2` without torchrun's environment re-runs itself under
    torch.distributed.run with 2 processes; the ranks rendezvous on 127.0.0.1 and rank 0
    prints one line with n_gpus = 2, the max-over-ranks time and the all-gathered offsets
    (the multi-rank plumbing of run_ours, over gloo here)."""
    import json
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR",
                                                            "MASTER_PORT")}
    out = subprocess.run([sys.executable, os.path.join(root, "bench.py"), "--gpus", "2", "--steps", "3",
                          "--bytes", "1000000000", "--dist-selftest"], cwd=root, capture_output=True, text=True,
                         timeout=280, env=env)
    assert out.returncode == 0, out.stderr[-2000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["ms"] == 11.0
    assert abs(d["value"] - 2 * 3 * 1e9 / 0.011 / 1e9) < 1e-6
    assert d["file_offsets"] == [0, 1000]
