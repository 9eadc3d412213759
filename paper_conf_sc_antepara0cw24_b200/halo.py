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

import contextlib
import os

import numpy as np

from . import stokesfo as S

_PROFILE = os.environ.get("STOKESFO_PROFILE") == "1"


@contextlib.contextmanager
def nvtx(name: str):
    """NVTX range (torch.cuda.nvtx) when STOKESFO_PROFILE=1, as the C ABI's entry points."""
    if not _PROFILE:
        yield
        return
    import torch
    torch.cuda.nvtx.range_push(name)
    try:
        yield
    finally:
        torch.cuda.nvtx.range_pop()


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
        self.remote_index = {}   # r -> local ids ON RANK r of the nodes in neighbors[r] (same gid order)
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
                self.remote_index[r] = S.mesh_halo_list(g_other, self.gids)

    def remote_table(self, rem_max: int = 7):
        """(rem [num_local_nodes] int32, remtab [rows][1+2*rem_max] int32) for
        stokesfo_set_remote: row of a boundary node = {count, peer, index on peer, ...}."""
        per_node = {}
        for r in sorted(self.neighbors):
            for m, t in zip(self.neighbors[r].tolist(), self.remote_index[r].tolist()):
                per_node.setdefault(m, []).append((r, t))
        rem = np.full(self.gids.size, -1, dtype=np.int32)
        remtab = np.zeros((max(len(per_node), 1), 1 + 2 * rem_max), dtype=np.int32)
        for row, m in enumerate(sorted(per_node)):
            lst = per_node[m]
            if len(lst) > rem_max:
                raise ValueError(f"node shared by {len(lst) + 1} parts > {rem_max + 1}")
            rem[m] = row
            remtab[row, 0] = len(lst)
            for k, (r, t) in enumerate(lst):
                remtab[row, 1 + 2 * k] = r
                remtab[row, 2 + 2 * k] = t
        return rem, remtab


class P2PHalo:
    """Fused halo sum over peer memory: the evaluation kernels add boundary-node
    contributions straight into the peers' R (CUDA IPC-mapped, NVLink), so a
    step is  zero(R_next) -> evaluate(R_cur) -> one stream-ordered barrier.
    R is double-buffered (step t writes R[t % 2]; R[(t+1) % 2] is zeroed before
    the barrier of step t, so no peer can write it before it is clear).
    fields = 2 adds the J.v output Y under the same protocol (stokesfo_jvp).

    Use: h = P2PHalo(ctx, part, device); for each step: R = h.begin();
    ctx.jacobian(U, J, R=R); h.end()  (R now holds the full sum).  With
    fields = 2, begin() returns (R, Y)."""

    def __init__(self, ctx, part: LocalPart, device, gloo_debug: bool = False, fields: int = 1):
        import torch
        import torch.distributed as dist
        self.ctx, self.device, self.gloo = ctx, device, gloo_debug
        self.rank, self.world = part.rank, part.world
        self.fields = fields
        nn = part.gids.size
        # one allocation per buffer parity holding every field: [fields][nn][2]
        self.buf = [torch.zeros((fields, nn, 2), dtype=torch.float64, device=device) for _ in range(2)]
        rem, remtab = part.remote_table()
        self.rem = torch.from_numpy(rem).to(device)
        self.remtab = torch.from_numpy(remtab).to(device)
        # an allocation CUDA IPC cannot export (e.g. torch expandable segments) -> every rank falls back
        try:
            handles = [S.ipc_get_handle(b) for b in self.buf]
        except Exception:
            handles = None
        allh = [None] * self.world
        dist.all_gather_object(allh, handles)
        nns = [None] * self.world      # node counts: the field stride of each peer's buffer
        dist.all_gather_object(nns, int(nn))
        self.opened = []
        ok = 1 if all(h is not None for h in allh) else 0
        ptrs = [[[0] * self.world for _ in range(fields)] for _ in range(2)]
        bases = {}   # one mapping per distinct peer allocation (handles may repeat)
        try:
            if not ok:
                raise RuntimeError("a rank could not export its buffers")
            for b in range(2):
                for f in range(fields):
                    ptrs[b][f][self.rank] = self.buf[b].data_ptr() + f * nn * 16
                for r in part.neighbors:
                    raw, off = allh[r][b]
                    if raw not in bases:
                        bases[raw] = S.ipc_open_handle((raw, 0))
                        self.opened.append(bases[raw])
                    for f in range(fields):
                        ptrs[b][f][r] = bases[raw] + off + f * nns[r] * 16
        except Exception:
            ok = 0
        flag = torch.tensor([ok], dtype=torch.int32, device="cpu" if gloo_debug else device)
        dist.all_reduce(flag, op=dist.ReduceOp.MIN)
        self.ok = bool(flag.item())
        self.peers = [[torch.tensor(ptrs[b][f], dtype=torch.int64, device=device) for f in range(fields)]
                      for b in range(2)]
        self.token = torch.zeros(1, dtype=torch.float32, device=device)
        self.t = 0
        self.launches_per_step = 1  # the buffer clear; the halo itself rides the evaluation kernel

    def begin(self):
        """Returns this step's R (or (R, Y)), already zero; zeroes the next step's buffers."""
        with nvtx("halo.p2p.begin"):
            return self._begin()

    def _begin(self):
        b = self.t % 2
        self.buf[(self.t + 1) % 2].zero_()
        self.ctx.set_remote(self.rem, self.remtab, self.peers[b][0])
        if self.fields > 1:
            self.ctx.set_remote_jvp(self.peers[b][1])
        cur = self.buf[b]
        return cur[0] if self.fields == 1 else tuple(cur[f] for f in range(self.fields))

    def end(self):
        """Stream-ordered barrier: after it, every rank's kernel of this step is complete."""
        import torch
        import torch.distributed as dist
        with nvtx("halo.p2p.barrier"):
            if self.gloo:
                torch.cuda.synchronize(self.device)
                dist.barrier()
            else:
                dist.all_reduce(self.token)
        self.t += 1
        cur = self.buf[(self.t - 1) % 2]
        return cur[0] if self.fields == 1 else tuple(cur[f] for f in range(self.fields))

    def close(self):
        self.ctx.set_remote(None, None, None)
        for p in self.opened:
            S.ipc_close(p)
        self.opened = []


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
        with nvtx("halo.nccl.exchange"):
            self._exchange(R)

    def _exchange(self, R):
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
