"""Multi-GPU partitioning of the local-operator path (BASELINE configs 4 and 5).

One process per GPU (torchrun), torch.distributed for the plumbing:

* frame parallelism (config 4): frames are independent units -> each rank
  takes a contiguous frame range and runs one batched launch; no data-path
  collective (only the barrier / MAX of the timings in bench.py).
* row bands (config 5): one large image is cut into P row bands; rank r owns
  rows [floor(rH/P), floor((r+1)H/P)) stored with `halo` rows above and
  below.  Before filtering, every rank sends its first `halo` owned rows to
  rank r-1 and its last `halo` rows to rank r+1 (NCCL send/recv over NVLink,
  batched in one group).  At the global top/bottom the boundary modes resolve
  locally, except REPEAT, whose halo closes the ring (rank 0 <-> rank P-1).
  The interior rows of the band are filtered while the halo messages are in
  flight; the 2*halo edge rows after they land.  The band view
  (lop_image.halo_*/global_*) makes every output pixel's arithmetic
  identical to the single-GPU call, so the result is bit-identical.

The exchange itself is device-agnostic (it works on CPU tensors with gloo,
which is how tests/test_dist.py exercises it without a GPU).
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def frame_range(n_frames: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous frame range [lo, hi) of `rank` (config 4)."""
    return n_frames * rank // world, n_frames * (rank + 1) // world


def band_range(height: int, world: int, rank: int) -> tuple[int, int]:
    """Owned global rows [y0, y1) of `rank` (config 5)."""
    return height * rank // world, height * (rank + 1) // world


class Bands:
    """Row band of a (height x width) image owned by `rank`, with halo rows."""

    def __init__(self, height: int, width: int, world: int, rank: int, halo: int,
                 device="cpu", mode: str = "clamp", dtype=torch.float32, group=None):
        self.H, self.W = int(height), int(width)
        self.world, self.rank, self.halo = int(world), int(rank), int(halo)
        self.mode = mode
        self.group = group
        self.y0, self.y1 = band_range(self.H, self.world, self.rank)
        self.rows = self.y1 - self.y0
        if self.rows < self.halo and self.world > 1:
            raise ValueError("band of %d rows is thinner than the halo (%d)" % (self.rows, halo))
        ring = mode == "repeat"
        self.up = self.rank - 1 if self.rank > 0 else (self.world - 1 if ring else None)
        self.down = self.rank + 1 if self.rank < self.world - 1 else (0 if ring else None)
        self.halo_top = self.halo if self.up is not None else 0
        self.halo_bottom = self.halo if self.down is not None else 0
        self.buf = torch.empty((self.rows + 2 * self.halo, self.W), dtype=dtype, device=device)
        self.owned = self.buf[self.halo:self.halo + self.rows]
        self.top = self.buf[:self.halo]
        self.bottom = self.buf[self.halo + self.rows:]

    def fill(self, make_rows):
        """owned <- make_rows(y0, y1) (e.g. synthetic.angio(..., row_range=...))."""
        self.owned.copy_(make_rows(self.y0, self.y1))

    def band_args(self):
        """(halo_top, halo_bottom, global_y0, global_height) for lop.* band views."""
        return (self.halo_top, self.halo_bottom, self.y0, self.H)

    def exchange_ops(self):
        """P2P ops of the halo exchange, in a fixed order so that two messages
        between the same pair of ranks (REPEAT ring with P = 2) match."""
        h = self.halo
        ops = []
        if h == 0:
            return ops
        # phase 1: last owned rows travel down, top halo arrives from up
        if self.down is not None:
            ops.append(dist.P2POp(dist.isend, self.owned[self.rows - h:].contiguous(),
                                  self.down, self.group))
        if self.up is not None:
            ops.append(dist.P2POp(dist.irecv, self.top, self.up, self.group))
        # phase 2: first owned rows travel up, bottom halo arrives from down
        if self.up is not None:
            ops.append(dist.P2POp(dist.isend, self.owned[:h].contiguous(), self.up, self.group))
        if self.down is not None:
            ops.append(dist.P2POp(dist.irecv, self.bottom, self.down, self.group))
        return ops

    def exchange_start(self):
        """Post the halo exchange; returns the requests (wait() to complete)."""
        if self.world == 1:
            if self.halo and self.mode == "repeat":       # ring with itself
                self.top.copy_(self.owned[self.rows - self.halo:])
                self.bottom.copy_(self.owned[:self.halo])
            return []
        ops = self.exchange_ops()
        return dist.batch_isend_irecv(ops) if ops else []

    def exchange(self):
        for req in self.exchange_start():
            req.wait()


def bilateral_bands(lop, band: Bands, sigma_d, sigma_r, mode="clamp", constant=0.0, size=None,
                    out=None, stream=None):
    """Config 5 step: halo exchange overlapped with the interior rows, then the
    edge rows; bit-identical to the single-GPU call on the whole image."""
    if out is None:
        out = torch.empty_like(band.owned)
    if size is None:
        size = int(round(4 * sigma_d)) + 1
    ry = (size if isinstance(size, int) else size[1]) // 2
    reqs = band.exchange_start()
    args = band.band_args()
    rows, W = band.rows, band.W
    inner = (0, ry, W, rows - 2 * ry) if rows > 2 * ry else None
    if inner is not None:
        # interior rows need no halo: run them while the messages are in flight
        lop.bilateral(band.owned, sigma_d, sigma_r, mode, constant, size=size, out=out,
                      roi=inner, stream=stream, band=args)
    for r in reqs:
        r.wait()
    if inner is None:
        lop.bilateral(band.owned, sigma_d, sigma_r, mode, constant, size=size, out=out,
                      stream=stream, band=args)
    else:
        for roi in ((0, 0, W, ry), (0, rows - ry, W, ry)):
            lop.bilateral(band.owned, sigma_d, sigma_r, mode, constant, size=size, out=out,
                          roi=roi, stream=stream, band=args)
    return out
