"""Device-side (torch CUDA) version of synth.RandomWalk for the update-heavy C4 sweep.

Same process as RandomWalk (SURVEY §8(d) 'Updates'): each tick every object advances
U[10,30] length units along its arc, turning onto a random non-U-turn out-arc at each vertex
(U-turn only at dead ends), and reports once, in a random order; t = tick*1000 + U[0,999].
Only the random stream differs (torch's Philox generator on the device instead of numpy's
PCG64), so its batches are distributed like RandomWalk's but not equal to them.  It exists
because C4 needs up to 10^9 updates per step, which the numpy walk produces in minutes.
Input generator only: holds none of the method's arithmetic.
"""
import numpy as np
import torch

from . import SEED_OBJECTS, SEED_UPDATES, out_csr, random_locations


class DeviceRandomWalk:
    def __init__(self, graph, n_objects: int, seed_objects: int = SEED_OBJECTS,
                 seed_updates: int = SEED_UPDATES, speed=(10, 30), device="cuda"):
        self.n = int(n_objects)
        self.dev = torch.device(device)
        ptr, order = out_csr(graph)
        self.w = torch.from_numpy(graph["w"].astype(np.int64)).to(self.dev)
        self.dst = torch.from_numpy(graph["dst"].astype(np.int64)).to(self.dev)
        self.ptr = torch.from_numpy(ptr).to(self.dev)
        self.order = torch.from_numpy(order).to(self.dev)
        rng0 = np.random.default_rng(seed_objects)
        arc, off = random_locations(graph, self.n, rng0)
        self.arc = torch.from_numpy(arc.astype(np.int64)).to(self.dev)
        self.off = torch.from_numpy(off.astype(np.int64)).to(self.dev)
        self.gen = torch.Generator(device=self.dev)
        self.gen.manual_seed(seed_updates)
        self.speed = speed
        self.tick_no = 0
        self.obj_ids = torch.arange(self.n, dtype=torch.int64, device=self.dev)

    def _advance(self):
        g = self.gen
        self.off += torch.randint(self.speed[0], self.speed[1] + 1, (self.n,), generator=g, device=self.dev)
        over = torch.nonzero(self.off >= self.w[self.arc]).flatten()
        while over.numel():
            a = self.arc[over]
            self.off[over] -= self.w[a]
            v = self.dst[a]
            p0 = self.ptr[v]
            deg = self.ptr[v + 1] - p0
            twin = a ^ 1
            j = (torch.rand(over.numel(), generator=g, device=self.dev) * torch.clamp(deg - 1, min=1)).long()
            j = torch.minimum(j, torch.clamp(deg - 2, min=0))
            cand = self.order[p0 + j]
            last = self.order[p0 + deg - 1]
            cand = torch.where((deg > 1) & (cand == twin), last, cand)
            cand = torch.where(deg == 1, self.order[p0], cand)
            self.arc[over] = cand
            over = over[self.off[over] >= self.w[self.arc[over]]]

    def ticks_into(self, out: torch.Tensor, n_ticks: int) -> torch.Tensor:
        """Write n_ticks ticks into out[: n_ticks*n] (int32 (m, 4) CUDA tensor: obj, edge,
        offset, t in arrival order) and return that slice."""
        n = self.n
        for i in range(n_ticks):
            self._advance()
            t = self.tick_no * 1000 + torch.randint(0, 1000, (n,), generator=self.gen, device=self.dev)
            perm = torch.randperm(n, generator=self.gen, device=self.dev)
            blk = out[i * n:(i + 1) * n]
            blk[:, 0] = self.obj_ids[perm].to(torch.int32)
            blk[:, 1] = self.arc[perm].to(torch.int32)
            blk[:, 2] = self.off[perm].to(torch.int32)
            blk[:, 3] = t[perm].to(torch.int64).to(torch.int32)  # t < 2^31 for < 2.1M ticks
            self.tick_no += 1
        return out[: n_ticks * n]

    def ticks(self, n_ticks: int) -> torch.Tensor:
        out = torch.empty((n_ticks * self.n, 4), dtype=torch.int32, device=self.dev)
        return self.ticks_into(out, n_ticks)
