"""Multi-GPU halo sum of shared-node partial residuals.

Column partition: rank r owns footprint columns [ranges[r], ranges[r+1]) and
all their cells; nodes on inter-partition node-columns are shared.  After the
local evaluation each rank holds partial sums on shared nodes; one grouped
send/recv per neighbour (NCCL over NVLink via torch.distributed.batch_isend_irecv)
carries the packed partial sums, then every rank adds what it received, so
each rank ends with the full sum on all of its local nodes.  Pack everything
before any unpack (corner nodes shared by 3+ ranks stay correct).

torch.distributed is plumbing here; pack/unpack run in libstokesfo's kernels
on GPU (stokesfo_halo_pack / _unpack_add).  For CPU (gloo) tests the same
schedule runs with index_select / index_add_.
"""
from __future__ import annotations

import numpy as np

from . import stokesfo as S


class LocalPart:
    """This rank's share of an extruded mesh (host arrays)."""

    def __init__(self, conn_global, L: int, nf: int, rank: int, world: int):
        self.ranges = S.mesh_partition_columns(nf, world)
        self.rank, self.world, self.L = rank, world, L
        lo, hi = int(self.ranges[rank]), int(self.ranges[rank + 1])
        self.cell_lo, self.cell_hi = lo * L, hi * L
        self.conn, self.gids = S.mesh_localize(conn_global[self.cell_lo:self.cell_hi])
        # every rank derives every part's node set (deterministic) -> halo lists
        self.neighbors = {}
        for r in range(world):
            if r == rank:
                continue
            a, b = int(self.ranges[r]) * L, int(self.ranges[r + 1]) * L
            if b <= a:
                continue
            g_other = np.unique(conn_global[a:b])
            idx = S.mesh_halo_list(self.gids, g_other)
            if idx.size:
                self.neighbors[r] = idx


class Halo:
    """Grouped halo exchange; `pack(R, idx, buf)` / `unpack_add(buf, idx, R)`."""

    def __init__(self, neighbors: dict, device, pack=None, unpack_add=None, group=None, host_staging=False):
        import torch
        self.group = group
        self.host_staging = host_staging  # gloo debug runs: send/recv host copies of the buffers
        self.idx = {r: torch.from_numpy(np.ascontiguousarray(v, dtype=np.int32)).to(device)
                    for r, v in sorted(neighbors.items())}
        self.send = {r: torch.empty((v.numel(), 2), dtype=torch.float64, device=device) for r, v in self.idx.items()}
        self.recv = {r: torch.empty_like(b) for r, b in self.send.items()}
        self.pack = pack or (lambda R, idx, buf: buf.copy_(R.index_select(0, idx.long())))
        self.unpack_add = unpack_add or (lambda buf, idx, R: R.index_add_(0, idx.long(), buf))

    @property
    def launches_per_exchange(self) -> int:
        return 2 * len(self.idx)

    def exchange(self, R):
        import torch.distributed as dist
        if not self.idx:
            return
        for r, idx in self.idx.items():          # pack everything first
            self.pack(R, idx, self.send[r])
        send, recv = self.send, self.recv
        if self.host_staging:
            send = {r: b.cpu() for r, b in self.send.items()}
            recv = {r: b.cpu() for r, b in self.recv.items()}
        ops = []
        for r in self.idx:
            ops.append(dist.P2POp(dist.isend, send[r], r, group=self.group))
            ops.append(dist.P2POp(dist.irecv, recv[r], r, group=self.group))
        for req in dist.batch_isend_irecv(ops):
            req.wait()
        if self.host_staging:
            for r in self.idx:
                self.recv[r].copy_(recv[r])
        for r, idx in self.idx.items():          # then unpack-add
            self.unpack_add(self.recv[r], idx, R)
