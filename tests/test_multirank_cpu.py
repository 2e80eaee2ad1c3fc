"""N > 1 host logic on CPU with the gloo backend (world_size 2): client sharding is
disjoint and covering, and the per-tick result gather to the map-owning rank 0 delivers
every rank's packed per-frame results intact (bench.py)."""
import os
import socket

import numpy as np
import torch
import torch.distributed as dist
import torch.multiprocessing as tmp

import bench


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    clients = bench.client_ids(rank, world, 4)
    kps = torch.full((4, 7, 20), rank + 1, dtype=torch.uint8)
    desc = torch.tensor(clients, dtype=torch.uint8).reshape(4, 1, 1).repeat(1, 7, 32)
    counts = torch.tensor([[0, 3, 7]] * 4, dtype=torch.int32) * (rank + 1)
    out = torch.arange(12, dtype=torch.int32).reshape(4, 3) + 100 * rank
    send = bench.pack_results([kps, desc, counts, out])
    got = bench.gather_to_owner(send, rank, world)
    if rank == 0:
        q.put([g.numpy().copy() for g in got])
    dist.barrier()
    dist.destroy_process_group()


def test_client_sharding():
    for world in (1, 2, 4, 8):
        all_c = [c for r in range(world) for c in bench.client_ids(r, world, 8)]
        assert sorted(all_c) == list(range(8 * world))


def test_gather_to_owner_gloo_world2():
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert len(got) == 2
    for rank, slot in enumerate(got):
        n_kps = 4 * 7 * 20
        assert (slot[:n_kps] == rank + 1).all()
        desc = slot[n_kps:n_kps + 4 * 7 * 32].reshape(4, 7, 32)
        assert (desc[:, 0, 0] == np.array(bench.client_ids(rank, 2, 4))).all()
        tail = slot[-48:].view(np.int32).reshape(4, 3)
        assert (tail == np.arange(12).reshape(4, 3) + 100 * rank).all()
