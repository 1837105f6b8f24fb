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


# ---------------------------------------------------------------------------------------------------
# Pair split (LANDAU_DIST_ELEMENTS on a z-mirror mesh, the C5 path): rank r runs the slot kernel's items
# (tile pairs a <= b of the upper half, U and V tensors, both directions) in its landau_pair_partition
# range and reduces a partial G over ALL points; one all-reduce (sum) gives every rank the full G.
# Here the oracle stands in for the kernels: a rank's partial G at a target t sums the sources in the
# tiles its items pair with t's tile (upper points and their mirrors), and the gloo all-reduce of the
# [5][N] partials must reproduce the oracle's full G.
# ---------------------------------------------------------------------------------------------------
def _mirror_tiles(r, z, grid_of_point):
    """The library's upper-half ordering (landau_create / detect_mirror): per grid, the points with z > 0
    sorted by (r, z), grids concatenated; tile = position // 32.  Returns the tile of every point (a
    mirror point takes its partner's tile)."""
    tile = np.full(r.size, -1)
    pos = 0
    for g in np.unique(grid_of_point):
        up = [i for i in np.nonzero(grid_of_point == g)[0] if z[i] > 0]
        up.sort(key=lambda i: (r[i], z[i]))
        lo = {(r[i], z[i]): i for i in np.nonzero(grid_of_point == g)[0] if z[i] < 0}
        for i in up:
            tile[i] = pos // 32
            tile[lo[(r[i], -z[i])]] = pos // 32
            pos += 1
    return tile, (pos + 31) // 32


def _pair_split_worker(rank, port, out_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        from oracle.oracle import Oracle, inner
        prob = inputs.config3()
        o = Oracle(prob)
        f = o.coefficients()
        r, z, w = o.points()
        TD, TKr, TKz = o.point_fields(f)
        gop = np.repeat(np.arange(len(prob.grids)), [o.npoints // len(prob.grids)] * len(prob.grids))
        tile, T = _mirror_tiles(r, z, gop)
        q0, q1 = L.landau_pair_partition(T, WORLD, rank)
        items = [(a, b) for b in range(T) for a in range(b + 1)][q0:q1]
        partner = [set() for _ in range(T)]
        for a, b in items:
            partner[a].add(b)
            partner[b].add(a)
        part = np.zeros((5, o.npoints))
        for A in range(T):
            if not partner[A]:
                continue
            tg = np.nonzero(tile == A)[0]
            src = np.isin(tile, sorted(partner[A]))
            part[:, tg] = inner(r, z, w * src, TD, TKr, TKz, targets=tg)
        t = torch.from_numpy(part)
        dist.all_reduce(t)                      # the exchange step: sum of the ranks' partial G
        counts = [None] * WORLD
        dist.all_gather_object(counts, (q1 - q0, sum(1 if a == b else 2 for a, b in items)))
        if rank == 0:
            G, Ga = o.point_coeffs(f)
            out_q.put((float(np.max(np.abs(t.numpy() - G) / Ga)), counts, T))
    finally:
        dist.destroy_process_group()


def test_pair_split_partials_allreduce_gloo():
    ctx = mp.get_context("spawn")
    q = ctx.SimpleQueue()
    mp.start_processes(_pair_split_worker, args=(_free_port(), q), nprocs=WORLD, join=True, start_method="spawn")
    err, counts, T = q.get()
    assert sum(c for c, _ in counts) == T * (T + 1) // 2          # every tile pair exactly once
    assert all(abs(wt - T * T / WORLD) <= 2 for _, wt in counts)   # balanced work (pair 2, diagonal 1)
    assert err <= 1e-13, err
