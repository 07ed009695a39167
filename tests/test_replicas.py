"""Replica harness on CPU with the gloo backend, world size 2 (the N>1 path of
bench.py: independent replicas, max-over-ranks time, summed work)."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_jungkl23_b200.replicas import aggregate, replica_seed


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import workloads as wl
    seed = replica_seed(1, rank)
    tr = wl.make_T(seed=seed)
    # each replica: its own trace; local "time" and work
    t_ms, recs = 10.0 + 5 * rank, tr.n_fault
    mx, tot = aggregate(t_ms, recs)
    dist.barrier()
    q.put((rank, seed, mx, tot, int(tr.launch_hash.sum() % (1 << 61))))
    dist.destroy_process_group()


def test_two_replicas_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(120)
        assert p.exitcode == 0
    res = sorted(q.get() for _ in range(2))
    assert [r[1] for r in res] == [1, 1001]                    # seed 3 + 1000 r pattern (T base 1)
    assert all(r[2] == 15.0 for r in res)                      # max over ranks
    assert all(r[3] == 2 * 2576 for r in res)                  # summed work
    assert res[0][4] == res[1][4]                              # T has no jitter: same kernels per replica


def test_single_process_aggregate_is_identity():
    assert aggregate(3.5, 7) == (3.5, 7.0)
