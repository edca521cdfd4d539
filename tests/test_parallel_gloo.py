"""Multi-GPU host logic on CPU: row-band partition, halo plan, halo exchange and result
merge over torch.distributed with the gloo backend (world size 2 and 3).

The spectra slots of each rank are emulated by a CPU tensor laid out like the library's
resident store ([resident tiles][bytes per tile]); each slot is filled with its global tile
index, so after the exchange every received halo slot must hold exactly the index of the
tile it stands for (the sender owns and transformed that tile).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_icpp_blattnerkcsbz14_b200 import PAIR_DTYPE
from paper_conf_icpp_blattnerkcsbz14_b200.parallel import (band, exchange_feasible, exchange_halo,
                                                           gather_translations, halo_plan)


@pytest.mark.parametrize("n,m,world", [(42, 59, 1), (42, 59, 2), (42, 59, 8), (3, 3, 2),
                                       (18, 22, 4), (100, 100, 8), (5, 7, 3), (2, 9, 4)])
def test_band_partition_and_plan(n, m, world):
    nt = n * m
    bands = [band(k, world, n, m) for k in range(world)]
    assert bands[0].t_begin == 0 and bands[-1].t_end == nt
    for a, b in zip(bands, bands[1:]):
        assert a.t_end == b.t_begin
    for bd in bands:
        assert bd.halo_begin == max(0, bd.t_begin - m)
        assert bd.row_begin * m <= bd.halo_begin and bd.row_end * m >= bd.t_end
    plans = [halo_plan(k, world, n, m) for k in range(world)]
    for k in range(world - 1):
        assert plans[k].send == plans[k + 1].recv
    if exchange_feasible(world, n, m):
        for k in range(1, world):
            first, cnt = plans[k].recv
            assert bands[k - 1].t_begin <= first and first + cnt == bands[k - 1].t_end


def _worker(rank, world, port, n, m, per_tile, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        bd = band(rank, world, n, m)
        plan = halo_plan(rank, world, n, m)
        nres = bd.t_end - bd.halo_begin
        store = torch.full((nres, per_tile), -1, dtype=torch.int32)
        for t in range(bd.t_begin, bd.t_end):             # owned tiles "transformed" here
            store[t - bd.halo_begin] = t

        def view(rng):
            first, cnt = rng
            return store[first - bd.halo_begin: first - bd.halo_begin + cnt]
        send = view(plan.send).contiguous() if plan.send else None
        recv = view(plan.recv) if plan.recv else None
        exchange_halo(send, recv, rank, world)
        ok = all(int(store[t - bd.halo_begin].min()) == t == int(store[t - bd.halo_begin].max())
                 for t in range(bd.halo_begin, bd.t_end))
        west = np.zeros(n * m, PAIR_DTYPE)
        north = np.zeros(n * m, PAIR_DTYPE)
        west["dx"][bd.t_begin:bd.t_end] = np.arange(bd.t_begin, bd.t_end)
        north["dy"][bd.t_begin:bd.t_end] = -np.arange(bd.t_begin, bd.t_end)
        w, nn = gather_translations(west, north, bd)
        merged = (np.array_equal(w["dx"], np.arange(n * m)) and
                  np.array_equal(nn["dy"], -np.arange(n * m)))
        q.put((rank, ok, merged))
    finally:
        dist.destroy_process_group()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("n,m,world", [(6, 7, 2), (9, 4, 3)])
def test_gloo_halo_exchange_and_gather(n, m, world):
    assert exchange_feasible(world, n, m)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(k, world, port, n, m, 16, q)) for k in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert sorted(r[0] for r in res) == list(range(world))
    assert all(r[1] for r in res), res
    assert all(r[2] for r in res), res
