"""Multi-GPU partitioning of the map index space (BASELINE.json north_star:
"work is partitioned ... by splitting the map's output index space per GPU").

One process per GPU; torch.distributed (NCCL over NVLink on the box) is the plumbing:
  * N-Body (config 5): contiguous equal target shards; each step all-gathers positions
    (`all_gather_into_tensor`, the one real exchange step of the path), runs the force map on
    the local targets against all sources, then the local integrator. Forces are bit-identical
    to the single-GPU run because the per-target summation order depends on n_src only.
  * Black-Scholes fused sums (config 2): contiguous option shards, one `all_reduce` (sum) of the
    per-GPU fp64 partials (`blackscholes_total` on a rank's own options = weak scaling;
    `blackscholes_shard_total` on a shard of one global array = strong scaling).
  * Mandelbrot (config 3): cyclic rows (row r -> rank r mod P; `mandelbrot_cyclic`), no collective;
    `gather_cyclic_rows` reassembles the frame for validation only.
  * Matmul (config 4): contiguous row blocks of C against a replicated Bt (`matmul_row_block`), no
    collective; `gather_row_blocks` reassembles C for validation only.

The step functions take the map/integrator callables as parameters so the partition and
exchange logic can be exercised on CPU (gloo) in tests; the product binds them to the CUDA ABI.
"""
from __future__ import annotations

from typing import Callable

import torch
import torch.distributed as dist


def shard_range(n: int, rank: int, world: int) -> tuple[int, int]:
    """Contiguous block shard [begin, begin + count) of n elements (balanced to +-1)."""
    base, rem = divmod(n, world)
    begin = rank * base + min(rank, rem)
    return begin, base + (1 if rank < rem else 0)


def shard_range_aligned(n: int, rank: int, world: int, align: int) -> tuple[int, int]:
    """Contiguous shard whose begin is a multiple of `align` elements (the 128-bit loads of the
    streaming maps need 16-byte aligned operands: align = 4 fp32); the tail goes to the last rank."""
    units = n // align
    b, c = shard_range(units, rank, world)
    begin, count = b * align, c * align
    if rank == world - 1:
        count += n - units * align
    return begin, count


def cyclic_rows(height: int, rank: int, world: int) -> tuple[int, int, int]:
    """Cyclic row shard for Mandelbrot: (row_first, row_stride, row_count)."""
    return rank, world, len(range(rank, height, world))


class NBodySim:
    """Sharded N-Body simulation state (positions+mass and velocities of the local shard).

    force_fn(pos_full, tgt_begin, tgt_count, eps2, out) fills out[tgt_count][4];
    integrate_fn(pos, vel, accel, dt) updates pos/vel in place.
    """

    def __init__(self, bodies_full: torch.Tensor, eps2: float, dt: float, device,
                 force_fn: Callable | None = None, integrate_fn: Callable | None = None,
                 group=None):
        self.group = group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        n = bodies_full.shape[0]
        if n % self.world:
            raise ValueError("n must be divisible by the number of ranks (equal all-gather shards)")
        self.n = n
        self.count = n // self.world
        self.begin = self.rank * self.count
        self.eps2, self.dt = eps2, dt
        self.device = torch.device(device)
        self.pos = bodies_full[self.begin:self.begin + self.count].to(self.device).contiguous()
        self.vel = torch.zeros_like(self.pos)
        # one rank: the force map reads the shard itself (the integrator updates it in place only
        # after the map has run), so there is no exchange and no copy
        self.pos_full = self.pos if self.world == 1 else torch.empty((n, 4), dtype=torch.float32, device=self.device)
        self.accel = torch.empty_like(self.pos)
        # the CUDA path fuses the integrator into the force map (lime_map_nbody_step): one launch per
        # step at n <= 8192, no accelerations in memory. It writes the new shard positions out of
        # place: into pos_alt (then swapped) at one rank, where the map reads the shard itself.
        self.fused = force_fn is None and integrate_fn is None
        if force_fn is None or integrate_fn is None:
            import paper_conf_pldi_dubachcrbf12_b200 as lime
            force_fn = force_fn or (lambda p, b, c, e, out: lime.map_nbody(p, e, b, c, out=out))
            integrate_fn = integrate_fn or lime.map_nbody_integrate
            self._step_fn = lime.map_nbody_step
        self.force_fn, self.integrate_fn = force_fn, integrate_fn
        self.pos_alt = torch.empty_like(self.pos) if (self.fused and self.world == 1) else None

    def gather(self):
        if self.world > 1:
            dist.all_gather_into_tensor(self.pos_full, self.pos, group=self.group)

    def step(self):
        """One task-graph pass: exchange, force map, integrate."""
        self.gather()
        if self.fused:
            if self.world == 1:
                self._step_fn(self.pos, self.eps2, self.dt, self.vel, 0, self.count, out=self.pos_alt)
                self.pos, self.pos_alt = self.pos_alt, self.pos
                self.pos_full = self.pos
            else:
                self._step_fn(self.pos_full, self.eps2, self.dt, self.vel, self.begin, self.count, out=self.pos)
            return
        self.force_fn(self.pos_full, self.begin, self.count, self.eps2, self.accel)
        self.integrate_fn(self.pos, self.vel, self.accel, self.dt)

    def step_host(self, h_pos: torch.Tensor, h_vel: torch.Tensor):
        """End-to-end step from host (pinned) shard state: H2D, step, D2H."""
        self.pos.copy_(h_pos, non_blocking=True)
        self.vel.copy_(h_vel, non_blocking=True)
        self.step()
        h_pos.copy_(self.pos, non_blocking=True)
        h_vel.copy_(self.vel, non_blocking=True)

    def capture(self, steps: int) -> "torch.cuda.CUDAGraph":
        """Capture `steps` simulation steps into one CUDA graph (single rank only). The kernels take
        no host decisions and their workspaces self-reset, so a replay runs the steps back to back
        without launch gaps -- the paper's repeated task-graph passes (L113-114) as one launch."""
        if self.world != 1:
            raise RuntimeError("graph capture of the multi-rank step (NCCL inside the graph) is not supported")
        if self.fused and steps % 2:
            raise ValueError("capture an even number of steps (the fused step ping-pongs two position buffers)")
        s = torch.cuda.Stream(self.device)
        s.wait_stream(torch.cuda.current_stream(self.device))
        with torch.cuda.stream(s):
            self.step()                      # warm-up on the capture stream (workspace, lazy init)
        torch.cuda.current_stream(self.device).wait_stream(s)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(steps):
                self.step()
        return g

    def momentum(self) -> torch.Tensor:
        """Global sum of m v over all ranks (all_reduce), float64 [3]."""
        m = self.pos[:, 3:4].double()
        p = (m * self.vel[:, :3].double()).sum(0)
        if self.world > 1:
            dist.all_reduce(p, group=self.group)
        return p


def blackscholes_total(S, X, T, r: float, sigma: float, fused_fn: Callable | None = None, group=None):
    """Global (sum call, sum put) over the option shards of all ranks: local fused map+reduce,
    then one all_reduce of the two fp64 partials."""
    if fused_fn is None:
        import paper_conf_pldi_dubachcrbf12_b200 as lime
        fused_fn = lime.map_reduce_blackscholes_sum
    sums = fused_fn(S, X, T, r, sigma)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(sums, group=group)
    return sums


def _rank_world(group=None) -> tuple[int, int]:
    if dist.is_initialized():
        return dist.get_rank(group), dist.get_world_size(group)
    return 0, 1


def blackscholes_shard_total(S, X, T, r: float, sigma: float, fused_fn: Callable | None = None, group=None):
    """Strong-scaled fused Black-Scholes (config 2): every rank holds (or views) the full option
    arrays, sums its contiguous shard [begin, begin+count) and all-reduces the two fp64 partials."""
    rank, world = _rank_world(group)
    b, c = shard_range_aligned(S.numel(), rank, world, 4)
    return blackscholes_total(S[b:b + c], X[b:b + c], T[b:b + c], r, sigma, fused_fn=fused_fn, group=group)


def mandelbrot_cyclic(width: int, height: int, x0: float, y0: float, dx: float, dy: float, max_iter: int,
                      device="cuda", out=None, map_fn: Callable | None = None, group=None) -> torch.Tensor:
    """This rank's cyclic rows of the Mandelbrot frame (config 3; rows rank, rank+P, ...): int32
    [row_count][width]. No collective: the output stays sharded."""
    rank, world = _rank_world(group)
    first, stride, count = cyclic_rows(height, rank, world)
    if map_fn is None:
        import paper_conf_pldi_dubachcrbf12_b200 as lime
        map_fn = lime.map_mandelbrot
    return map_fn(width, height, x0, y0, dx, dy, max_iter, row_first=first, row_stride=stride, row_count=count,
                  device=device, out=out)


def gather_cyclic_rows(local: torch.Tensor, height: int, group=None) -> torch.Tensor:
    """Reassemble the full [height][width] frame from every rank's cyclic rows (validation only):
    shards are padded to ceil(height/P) rows for one all_gather_into_tensor, then interleaved."""
    rank, world = _rank_world(group)
    if world == 1:
        return local
    width = local.shape[1]
    rows = -(-height // world)
    pad = torch.zeros((rows, width), dtype=local.dtype, device=local.device)
    pad[:local.shape[0]] = local
    allp = torch.empty((world * rows, width), dtype=local.dtype, device=local.device)
    dist.all_gather_into_tensor(allp, pad, group=group)
    allp = allp.view(world, rows, width)
    full = torch.empty((height, width), dtype=local.dtype, device=local.device)
    for k in range(world):
        cnt = len(range(k, height, world))
        full[k::world] = allp[k, :cnt]
    return full


def matmul_row_block(A: torch.Tensor, Bt: torch.Tensor, out=None, mm_fn: Callable | None = None, group=None):
    """This rank's contiguous row block of C = A . Bt^T (config 4): rows [begin, begin+count) of A
    against the replicated Bt; no per-call collective."""
    rank, world = _rank_world(group)
    b, c = shard_range(A.shape[0], rank, world)
    if mm_fn is None:
        import paper_conf_pldi_dubachcrbf12_b200 as lime
        mm_fn = lime.map_matmul_bf16
    if c == 0:
        return torch.empty((0, Bt.shape[0]), dtype=torch.float32, device=A.device)
    return mm_fn(A[b:b + c], Bt, out)


def gather_row_blocks(local: torch.Tensor, M: int, group=None) -> torch.Tensor:
    """Reassemble C [M][N] from every rank's contiguous row block (validation only)."""
    rank, world = _rank_world(group)
    if world == 1:
        return local
    rows = -(-M // world)
    pad = torch.zeros((rows,) + tuple(local.shape[1:]), dtype=local.dtype, device=local.device)
    pad[:local.shape[0]] = local
    allp = torch.empty((world * rows,) + tuple(pad.shape[1:]), dtype=local.dtype, device=local.device)
    dist.all_gather_into_tensor(allp, pad, group=group)
    allp = allp.view((world,) + tuple(pad.shape))
    return torch.cat([allp[k, :shard_range(M, k, world)[1]] for k in range(world)])
