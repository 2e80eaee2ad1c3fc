"""N > 1 host logic on CPU with the gloo backend (world_size 2): client sharding is
disjoint and covering, and the per-tick result gather to the map-owning rank 0 delivers
every rank's packed per-frame results intact (bench.py)."""
import os
import socket

import numpy as np
import pytest
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


def _np_shard_top2(desc, counts, shard, offset):
    """Definition of one shard's top-2 (test-local brute force): per keypoint the two smallest
    (distance << 32 | global index) over the shard rows, UINT64_MAX = none."""
    F, cap = desc.shape[:2]
    L = counts.shape[1] - 1
    out = np.full((F, cap, 2), np.iinfo(np.uint64).max, np.uint64)
    if len(shard) == 0:
        return out
    mb = np.unpackbits(shard, axis=-1)
    for f in range(F):
        n = int(counts[f, L])
        if n == 0:
            continue
        qb = np.unpackbits(desc[f, :n], axis=-1)
        d = (qb[:, None, :] != mb[None, :, :]).sum(-1).astype(np.uint64)
        key = (d << np.uint64(32)) | (np.arange(len(shard), dtype=np.uint64) + np.uint64(offset))[None, :]
        key.sort(axis=1)
        out[f, :n, 0] = key[:, 0]
        if key.shape[1] > 1:
            out[f, :n, 1] = key[:, 1]
    return out


def _np_merge(parts, counts, th=50, num=3, den=4):
    """O10's accept rule on the merged top-2 of the parts [R, F, cap, 2]."""
    R, F, cap = parts.shape[:3]
    L = counts.shape[1] - 1
    out = np.zeros((F, cap), np.dtype([("idx", "<i4"), ("dist", "<i4"), ("dist2", "<i4")]))
    out["idx"], out["dist"], out["dist2"] = -1, 256, 256
    NONE = np.iinfo(np.uint64).max
    for f in range(F):
        for k in range(int(counts[f, L])):
            keys = sorted(int(x) for x in parts[:, f, k, :].ravel() if x != NONE)
            d1 = keys[0] >> 32 if keys else 256
            d2 = keys[1] >> 32 if len(keys) > 1 else 256
            out[f, k] = (keys[0] & 0xFFFFFFFF if keys and d1 <= th and den * d1 < num * d2 else -1, d1, d2)
    return out


def _shard_worker(rank, world, port, n_map, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    rng = np.random.default_rng(7)  # same map on every rank; per-rank frames below
    base = rng.integers(0, 256, (40, 32), dtype=np.uint8)
    full_map = np.concatenate([base ^ (rng.random((40, 32)) < 0.02).astype(np.uint8) * 1,
                               rng.integers(0, 256, (n_map - 40, 32), dtype=np.uint8)])
    B, cap, L = 3, 12, 2
    fr = np.random.default_rng(100 + rank)
    desc = fr.integers(0, 256, (B, cap, 32), dtype=np.uint8)
    desc[:, :4] = base[fr.integers(0, 40, (B, 4))]          # some true matches
    counts = np.zeros((B, L + 1), np.int32)
    counts[:, 1] = fr.integers(0, 6, B)
    counts[:, 2] = counts[:, 1] + fr.integers(0, cap - 5, B)
    lo, hi = bench.shard_range(n_map, rank, world)
    qd, qc = bench.allgather_queries(torch.from_numpy(desc), torch.from_numpy(counts), world)
    top2 = _np_shard_top2(qd.numpy(), qc.numpy(), full_map[lo:hi], lo)
    parts = bench.exchange_partials(torch.from_numpy(top2.view(np.int64)), world).numpy().view(np.uint64)
    got = _np_merge(parts, counts)
    q.put((rank, got, desc, counts, full_map))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,n_map", [(2, 301), (3, 100)])
def test_sharded_brute_exchange_gloo(ref, world, n_map):
    """F4 host logic: all-gather of the queries, per-shard top-2 with global indices, all-to-all
    of the partials back to the frames' owner, merge -- equals the oracle's O10 over the whole
    map for every rank's frames (shards of uneven size)."""
    ctx = tmp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, world, port, n_map, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=180) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert sorted(r[0] for r in res) == list(range(world))
    for rank, got, desc, counts, full_map in res:
        p = ref.params(752, 480, 1000)
        cap = desc.shape[1]
        # the oracle's O10 on the same keypoints (padded to its own kp_capacity)
        d_pad = np.zeros((len(desc), p.kp_capacity, 32), np.uint8)
        d_pad[:, :cap] = desc
        c_pad = np.zeros((len(desc), p.n_levels + 1), np.int32)
        c_pad[:, 1:] = counts[:, -1:]
        want = ref.match_brute(p, d_pad, c_pad, full_map)[:, :cap]
        for f in range(len(desc)):
            n = int(counts[f, -1])
            assert (got[f, :n] == want[f, :n]).all(), (rank, f)
        assert (got["idx"] >= 0).sum() > 0
