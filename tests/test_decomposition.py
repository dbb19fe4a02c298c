"""Host logic of the multi-GPU decomposition (-m "not gpu"): block extents and
neighbour ranks come from the C library (pf_query_layout /
pf_query_neighbors, host-only), and the ghost-exchange protocol of pf_api.cu
(ordered x -> y -> z stages; per dimension send hi, send lo, receive lo,
receive hi; the k-th message of a rank pair matches the k-th receive, as in
NCCL) is replayed with world-size-2 and -4 gloo process groups on CPU and
checked against the periodic / Neumann images of the global field."""
import itertools
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_sc_0003hehshhkwnr19_b200 import pf


@pytest.fixture(scope="module", autouse=True)
def lib():
    from paper_conf_sc_0003hehshhkwnr19_b200 import build
    build.build()
    pf.load_library()


@pytest.mark.parametrize("shape,procs", [((16, 12, 20), (2, 1, 1)), ((9, 7, 11), (2, 2, 1)),
                                         ((10, 10, 10), (2, 2, 2)), ((8, 6, 33), (4, 1, 2))])
def test_blocks_tile_the_domain(shape, procs):
    world = procs[0] * procs[1] * procs[2]
    cover = np.zeros(shape, dtype=int)
    for r in range(world):
        L = pf.query_layout(shape, procs, r, world)
        nx, ny, nz = L.local
        ox, oy, oz = L.offset
        cover[oz:oz + nz, oy:oy + ny, ox:ox + nx] += 1
        assert L.pitch % 16 == 0 and L.x_off == 16
        # structure of arrays [c][z][y][x] (default); PF_LAYOUT=il:
        # plane-interleaved [z][c][y][x], component stride = one padded x-y
        # plane, z stride = 4 of them
        pxy = L.pitch * (ny + 4)
        assert (L.field, L.plane) in ((pxy, 4 * pxy), (pxy * (nz + 4), pxy))
    assert np.all(cover == 1)


@pytest.mark.parametrize("periodic", [True, False])
def test_neighbours_are_symmetric(periodic):
    shape, procs = (8, 8, 8), (2, 3, 2)
    world = 12
    bc = None if periodic else {"lo": ("neumann",) * 3, "hi": ("neumann",) * 3}
    nb = [pf.query_neighbors(shape, procs, r, world, bc) for r in range(world)]
    for r in range(world):
        lo, hi = nb[r]
        for d in range(3):
            if hi[d] >= 0:
                assert nb[hi[d]][0][d] == r
            if lo[d] >= 0:
                assert nb[lo[d]][1][d] == r
            if not periodic:
                coord = [r % 2, (r // 2) % 3, r // 6][d]
                assert (lo[d] < 0) == (coord == 0) and (hi[d] < 0) == (coord == procs[d] - 1)


# --------------------------------------------------------------------------
# replay of the exchange protocol with gloo
# --------------------------------------------------------------------------
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _slab(arr, d, idx):
    """The slab of dimension d (array axes: 0=z,1=y,2=x; d: 0=x,1=y,2=z) at
    index idx, with the ghosted range of the dimensions before d and the
    interior range of the dimensions after d (ghost layer of width 1)."""
    sl = [slice(None)] * 3
    for e in range(3):
        ax = 2 - e
        if e == d:
            sl[ax] = idx + 1
        elif e < d:
            sl[ax] = slice(None)           # ghosts included
        else:
            sl[ax] = slice(1, -1)          # interior only
    return tuple(sl)


def _worker(rank, world, port, shape, procs, bc_kind, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        bc = None if bc_kind == "periodic" else {"lo": ("periodic", "periodic", "neumann"),
                                                 "hi": ("periodic", "periodic", "neumann")}
        L = pf.query_layout(shape, procs, rank, world, bc)
        lo, hi = pf.query_neighbors(shape, procs, rank, world, bc)
        rng = np.random.default_rng(7)
        glob = rng.standard_normal(shape)
        nx, ny, nz = L.local
        ox, oy, oz = L.offset
        loc = np.full((nz + 2, ny + 2, nx + 2), np.nan)
        loc[1:-1, 1:-1, 1:-1] = glob[oz:oz + nz, oy:oy + ny, ox:ox + nx]
        n = (nx, ny, nz)
        for d in range(3):
            if procs[d] == 1:  # local: periodic wrap or Neumann copy inside the block
                per = d < 2 or bc_kind == "periodic"
                loc[_slab(loc, d, -1)] = loc[_slab(loc, d, n[d] - 1 if per else 0)]
                loc[_slab(loc, d, n[d])] = loc[_slab(loc, d, 0 if per else n[d] - 1)]
                continue
            sends = []  # (peer, payload) in issue order: hi face, then lo face
            if hi[d] >= 0:
                sends.append((hi[d], loc[_slab(loc, d, n[d] - 1)].copy()))
            if lo[d] >= 0:
                sends.append((lo[d], loc[_slab(loc, d, 0)].copy()))
            recvs = []  # (peer, ghost index) in issue order: lo ghost, then hi ghost
            if lo[d] >= 0:
                recvs.append((lo[d], -1))
            if hi[d] >= 0:
                recvs.append((hi[d], n[d]))
            reqs, bufs, seq = [], [], {}
            for peer, payload in sends:
                k = seq.get(("s", peer), 0)
                seq[("s", peer)] = k + 1
                reqs.append(dist.isend(torch.from_numpy(payload), dst=peer, tag=100 * d + k))
            for peer, gi in recvs:
                k = seq.get(("r", peer), 0)
                seq[("r", peer)] = k + 1
                buf = torch.empty(loc[_slab(loc, d, gi)].shape, dtype=torch.float64)
                reqs.append(dist.irecv(buf, src=peer, tag=100 * d + k))
                bufs.append((gi, buf))
            for q in reqs:
                q.wait()
            for gi, buf in bufs:
                loc[_slab(loc, d, gi)] = buf.numpy()
            for side, nbr in ((-1, lo[d]), (n[d], hi[d])):  # physical boundary of a split dim
                if nbr < 0:
                    loc[_slab(loc, d, side)] = loc[_slab(loc, d, 0 if side < 0 else n[d] - 1)]
        # reference: per-axis images of the global field (periodic x, y; z per bc)
        ref = np.empty_like(loc)
        for k, j, i in itertools.product(range(nz + 2), range(ny + 2), range(nx + 2)):
            gz, gy, gx = oz + k - 1, oy + j - 1, ox + i - 1
            gx %= shape[2]
            gy %= shape[1]
            gz = gz % shape[0] if bc_kind == "periodic" else min(max(gz, 0), shape[0] - 1)
            ref[k, j, i] = glob[gz, gy, gx]
        # corners (all three coordinates ghosts) are never read by the stencils
        mask = np.ones_like(loc, dtype=bool)
        for k in (0, nz + 1):
            for j in (0, ny + 1):
                for i in (0, nx + 1):
                    mask[k, j, i] = False
        out[rank] = bool(np.array_equal(loc[mask], ref[mask]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("procs,bc_kind", [((2, 1, 1), "periodic"), ((1, 2, 1), "periodic"),
                                           ((1, 1, 2), "periodic"), ((2, 2, 1), "periodic"),
                                           ((1, 1, 2), "ds"), ((2, 1, 2), "ds")])
def test_gloo_exchange_protocol(procs, bc_kind):
    world = procs[0] * procs[1] * procs[2]
    shape = (6, 7, 9)  # (nz, ny, nx), uneven splits
    mgr = mp.Manager()
    out = mgr.dict()
    mp.start_processes(_worker, args=(world, _free_port(), shape, procs, bc_kind, out), nprocs=world,
                       join=True, start_method="spawn")
    assert dict(out) == {r: True for r in range(world)}
