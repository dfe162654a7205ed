"""Multi-rank host logic on CPU: world_size-2 process groups over gloo.

Covers the partition rule of the library [A21], the NCCL unique-id bootstrap
through torch.distributed, the max-over-ranks timing reduction, and the
sharding semantics of the step itself (each rank's owned targets and update,
assembled by an all-gather, equal the single-process step) using the oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_casselldahg24_b200 import dist as D

        # 1. the partition tiles [0, N) with 256-aligned slices [A21]
        for n in (1, 31, 32, 33, 1000, 4097, 10_000_000, 100_000_000):
            mine = D.owned_range(n, rank, world)
            ranges = [None] * world
            dist.all_gather_object(ranges, mine)
            assert ranges[0][0] == 0 and ranges[-1][1] == n
            for (b0, e0), (b1, e1) in zip(ranges, ranges[1:]):
                assert e0 == b1 and b0 <= e0
            assert all(b % 256 == 0 and (e - b) % 256 == 0 for b, e in ranges[:-1] if e < n)

        # 2. every rank gets rank 0's NCCL unique id
        uid = D.broadcast_unique_id(rank)
        ids = [None] * world
        dist.all_gather_object(ids, uid)
        assert len(uid) == 128 and all(i == ids[0] for i in ids)

        # 3. timing is reported as the max over ranks
        assert D.max_over_ranks(float(rank + 1)) == float(world)

        # 4. sharded step == single-process step (oracle semantics)
        from oracle import oracle as O
        from workloads import generate
        n = 3001
        pos, vel, mass = generate("plummer", n, 31)
        full = O.step(pos, vel, mass, theta=0.5, eps=1e-3, dt=1e-3, key_bits=16)
        b, e = D.owned_range(n, rank, world)
        part = O.step(pos, vel, mass, theta=0.5, eps=1e-3, dt=1e-3, key_bits=16, integrate=False,
                      targets=np.arange(b, e))
        # the owned update, as K7 does it (fp64 kick-drift stored in fp32)
        v_new = part.vel[b:e].astype(np.float64) + part.acc * 1e-3
        x_new = part.pos[b:e].astype(np.float64) + v_new * 1e-3
        mine = (part.acc, part.count, x_new.astype(np.float32), v_new.astype(np.float32))
        got = [None] * world
        dist.all_gather_object(got, mine)
        acc = np.concatenate([g[0] for g in got])
        cnt = np.concatenate([g[1] for g in got])
        x = np.concatenate([g[2] for g in got])
        v = np.concatenate([g[3] for g in got])
        assert (acc == full.acc).all() and (cnt == full.count).all()
        assert (x == full.pos).all() and (v == full.vel).all()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_two_rank_gloo(world):
    mp.spawn(_worker, args=(world, _free_port()), nprocs=world, join=True)
