"""World-size-2 CPU tests (gloo) of the multi-process host logic.

* element split (C5 mode): every rank computes G for the cells landau_partition gives it, places it
  in its chunk of the [world][5][Nc] exchange buffer and all-gathers; the gathered buffer, read with
  the library's chunked layout, must equal the single-process G -- here with the oracle standing in
  for the GPU kernels (this box has no GPU), including a cell count that does not divide evenly;
* the NCCL id broadcast of make_dist; the contiguous batch sharding of C4 (each vertex exactly once).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_adamsbkw22_b200 import inputs
from paper_conf_ipps_adamsbkw22_b200 import landau as L

WORLD = 2


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _five_cell_problem():
    R = inputs.R_E
    cells = inputs.refine_uniform([(0.0, -R, R)], 1) + [(0.0, 0.0, R)]   # 4 + 1 cells, 2:1 balanced
    return inputs.Problem("odd", 2, [(R, cells)], [inputs.Species("e", 1.0, -1.0, 0)], fmix=[[(1.0, 1.0, 0.0)]],
                          seed=7)


def _worker(rank, port, name, out_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        from oracle.oracle import Oracle
        prob = _five_cell_problem() if name == "odd" else inputs.CONFIGS[name]()
        o = Oracle(prob)
        f = o.coefficients()
        ncell = int(prob.ncells.sum())
        nqp = (prob.order + 1) ** 2
        e0, e1 = L.landau_partition(ncell, WORLD, rank)
        Nc = L.chunk_points(ncell, nqp, WORLD)
        targets = np.arange(e0 * nqp, e1 * nqp)
        chunk = torch.zeros((5, Nc), dtype=torch.float64)
        if targets.size:
            G, _ = o.point_coeffs(f, targets)
            chunk[:, :targets.size] = torch.from_numpy(G)
        gathered = [torch.zeros_like(chunk) for _ in range(WORLD)]
        dist.all_gather(gathered, chunk)
        buf = torch.stack(gathered).numpy()                      # [world][5][Nc]
        i = np.arange(o.npoints)
        Gfull = buf[i // Nc, :, i % Nc].T                         # the library's chunked read
        # NCCL id broadcast and batch sharding
        d = L.make_dist(L.LANDAU_DIST_ELEMENTS)
        ids = [None] * WORLD
        dist.all_gather_object(ids, d["nccl_unique_id"])
        lo, hi = L.batch_range(1024, WORLD, rank)
        ranges = [None] * WORLD
        dist.all_gather_object(ranges, (lo, hi))
        if rank == 0:
            Gref, _ = o.point_coeffs(f)
            out_q.put((name, np.array_equal(Gfull, Gref), ids[0] == ids[1] and len(ids[0]) == 128, ranges))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", ["odd", "C1", "C3"])
def test_element_split_and_sharding_gloo(name):
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    mp.start_processes(_worker, args=(_free_port(), name, q), nprocs=WORLD, join=True, start_method="spawn")
    got_name, same_G, same_id, ranges = q.get()
    assert got_name == name
    assert same_G, "gathered chunked G differs from the single-process G"
    assert same_id
    cover = np.zeros(1024, dtype=int)
    for lo, hi in ranges:
        cover[lo:hi] += 1
    assert np.all(cover == 1)
