"""World-size-2 CPU test (gloo) of the multi-GPU host logic: rank 0's
weights/params reach every rank through the one broadcast, each rank computes its
contiguous batch shard, and the concatenated shards equal the single-process
result byte for byte.  The per-shard compute here is the oracle (no GPU)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from bench import broadcast_params, shard_bounds
from workloads import ConvShape, make_layer_inputs, make_layer_params

CS = ConvShape("mg", 5, 10, 10, 32, 24, 3, 3, 1, 1)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    li = make_layer_inputs(CS, 4, seed=9)                      # same activations everywhere
    if rank == 0:
        lp = make_layer_params(CS, 4, seed=77)
        m, n = oracle.requant_params(lp.s_x, lp.s_w, lp.s_y)
        w = torch.from_numpy(lp.w_bytes.reshape(-1).copy())
        p = torch.from_numpy(np.stack([lp.bias, m, n]).astype(np.int32))
    else:
        w = torch.zeros(CS.k * CS.r * CS.s * CS.c // 2, dtype=torch.uint8)
        p = torch.zeros((3, CS.k), dtype=torch.int32)
    broadcast_params(dist, (w, p))
    start, count = shard_bounds(rank, world, CS.n)
    li.w_bytes = w.numpy().reshape(CS.k, CS.r, CS.s, CS.c // 2)
    li.bias = p[0].numpy()
    y = oracle.conv2d_layer(li, mult=p[1].numpy(), shift=p[2].numpy(),
                            n_slice=slice(start, start + count))
    counts = [shard_bounds(r, world, CS.n)[1] for r in range(world)]
    gathered = [torch.zeros((c,) + y.shape[1:], dtype=torch.uint8) for c in counts]
    dist.all_gather(gathered, torch.from_numpy(y)) if len(set(counts)) == 1 else None
    if len(set(counts)) != 1:
        # uneven shards: gather through rank-0 point-to-point
        if rank == 0:
            gathered[0] = torch.from_numpy(y)
            for r in range(1, world):
                dist.recv(gathered[r], src=r)
        else:
            dist.send(torch.from_numpy(y), dst=0)
    if rank == 0:
        q.put(torch.cat(gathered).numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_shard_bounds_cover_batch():
    for world in (1, 2, 3, 4, 8):
        for gb in (1, 7, 32, 256, 257):
            spans = [shard_bounds(r, world, gb) for r in range(world)]
            assert sum(c for _, c in spans) == gb
            assert all(spans[r][0] + spans[r][1] == spans[r + 1][0] for r in range(world - 1))


def test_two_rank_gloo_shards_equal_single_process():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    li = make_layer_inputs(CS, 4, seed=9)
    lp = make_layer_params(CS, 4, seed=77)
    li.w_bytes, li.bias = lp.w_bytes, lp.bias
    m, n = oracle.requant_params(lp.s_x, lp.s_w, lp.s_y)
    ref = oracle.conv2d_layer(li, mult=m, shift=n)
    np.testing.assert_array_equal(got, ref)
