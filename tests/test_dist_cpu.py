"""The multi-GPU plumbing of bench.py on CPU (gloo, world size 2): the path does
not shard (replicas only), so the only collective steps are the
barrier around the timed region and the max over ranks of its duration."""
import os
import socket
import sys

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world),
                      LOCAL_RANK=str(rank))
    import bench
    w, r, local = bench.dist_init(None)
    assert (w, r, local) == (world, rank, rank)
    bench.barrier(w)
    m = bench.allmax(w, 10.0 + rank)            # rank 1 is the slowest
    v = bench.aggregate(w, 5, m)
    # C5: each rank's C2 pair (its best sequential time, co-run makespan, STP) gathered
    g = bench.gather(w, {"t_seq_ms": 30.0 + rank, "makespan_ms": 24.0 + 2 * rank, "stp": 1.2 + 0.1 * rank})
    out[rank] = (m, v, bench.c5_aggregate(g))
    bench.barrier(w)
    dist.destroy_process_group()


def test_gloo_world2_barrier_and_max():
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(2, port, out), nprocs=2, join=True)
    assert out[0] == out[1]
    m, v, c5 = out[0]
    assert m == 11.0
    assert v == pytest.approx(2 * 5 / 0.011)
    # G_agg = max_g T_seq / max_g makespan = 31 / 26; per-GPU gains 30/24, 31/26; STP summed
    assert c5["g_agg"] == pytest.approx(31 / 26, abs=1e-4) and c5["stp_sum"] == pytest.approx(2.5)
    assert c5["per_gpu_gain"] == [pytest.approx(1.25), pytest.approx(31 / 26, abs=1e-4)]
    assert c5["gpus"] == 2 and c5["clients"] == 4


def test_reference_arm_only_rank0_prints(capsys):
    sys.path.insert(0, ROOT)
    import bench

    class A:
        warmup, steps, cpu_sample_s, gpus = 0, 1, 0.1, 2
    bench.run_reference(A, 2, 1)                 # rank 1: no work, no output
    assert capsys.readouterr().out == ""
