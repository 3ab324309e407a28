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

Transports: NCCL (CUDA tensors; the production path), or gloo.  gloo moves
CPU tensors only, so with CUDA band buffers on a gloo group the exchange is
host-staged (edge rows copied to host, exchanged, copied back; blocking) --
how tests run the CUDA kernels on several ranks of ONE GPU, where NCCL
refuses two ranks on the same device.

Streams: the exchange and the launches of `bilateral_bands` run under
`torch.cuda.stream(stream)`, so NCCL's internal stream waits for the owned
rows written on `stream` before sending, and `Work.wait()` makes `stream`
(not just torch's default stream) wait for the received halo rows.
"""
from __future__ import annotations

import contextlib

import torch
import torch.distributed as dist


def default_window(sigma_d: float) -> int:
    """Window when only sigma_d is given: 2*round(2 sigma_d) + 1 -- the paper's
    4 sigma_d + 1 (Alg. 1 l.6-7) for integer sigma_d, and
    always odd (reading c1)."""
    return 2 * int(round(2.0 * float(sigma_d))) + 1


def frame_range(n_frames: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous frame range [lo, hi) of `rank` (config 4)."""
    return n_frames * rank // world, n_frames * (rank + 1) // world


def band_range(height: int, world: int, rank: int) -> tuple[int, int]:
    """Owned global rows [y0, y1) of `rank` (config 5)."""
    return height * rank // world, height * (rank + 1) // world


def _backend(group) -> str | None:
    if not dist.is_available() or not dist.is_initialized():
        return None
    return dist.get_backend(group)


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

    @property
    def halo_bytes(self) -> int:
        """Bytes this rank receives per exchange."""
        n = (self.halo_top + self.halo_bottom) if self.world > 1 else 0
        return n * self.W * self.buf.element_size()

    def fill(self, make_rows):
        """owned <- make_rows(y0, y1) (e.g. synthetic.angio(..., row_range=...))."""
        self.owned.copy_(make_rows(self.y0, self.y1))

    def band_args(self):
        """(halo_top, halo_bottom, global_y0, global_height) for lop.* band views."""
        return (self.halo_top, self.halo_bottom, self.y0, self.H)

    def staged(self) -> bool:
        """gloo group with CUDA buffers: exchange through host memory."""
        return self.buf.is_cuda and _backend(self.group) == "gloo"

    def exchange_ops(self, send_last=None, send_first=None, recv_top=None, recv_bottom=None):
        """P2P ops of the halo exchange, in a fixed order so that two messages
        between the same pair of ranks (REPEAT ring with P = 2) match."""
        h = self.halo
        ops = []
        if h == 0:
            return ops
        send_last = self.owned[self.rows - h:] if send_last is None else send_last
        send_first = self.owned[:h] if send_first is None else send_first
        recv_top = self.top if recv_top is None else recv_top
        recv_bottom = self.bottom if recv_bottom is None else recv_bottom
        # phase 1: last owned rows travel down, top halo arrives from up
        if self.down is not None:
            ops.append(dist.P2POp(dist.isend, send_last.contiguous(), self.down, self.group))
        if self.up is not None:
            ops.append(dist.P2POp(dist.irecv, recv_top, self.up, self.group))
        # phase 2: first owned rows travel up, bottom halo arrives from down
        if self.up is not None:
            ops.append(dist.P2POp(dist.isend, send_first.contiguous(), self.up, self.group))
        if self.down is not None:
            ops.append(dist.P2POp(dist.irecv, recv_bottom, self.down, self.group))
        return ops

    def _exchange_staged(self):
        h = self.halo
        host = lambda t: t.detach().to("cpu", copy=True)            # noqa: E731 (synchronous)
        top = torch.empty((h, self.W), dtype=self.buf.dtype)
        bot = torch.empty((h, self.W), dtype=self.buf.dtype)
        ops = self.exchange_ops(host(self.owned[self.rows - h:]), host(self.owned[:h]), top, bot)
        for req in (dist.batch_isend_irecv(ops) if ops else []):
            req.wait()
        if self.up is not None:
            self.top.copy_(top)
        if self.down is not None:
            self.bottom.copy_(bot)

    def exchange_start(self):
        """Post the halo exchange on the current stream; returns the requests
        (wait() to complete).  The host-staged transport completes before
        returning."""
        if self.world == 1:
            if self.halo and self.mode == "repeat":       # ring with itself
                self.top.copy_(self.owned[self.rows - self.halo:])
                self.bottom.copy_(self.owned[:self.halo])
            return []
        if self.staged():
            self._exchange_staged()
            return []
        ops = self.exchange_ops()
        return dist.batch_isend_irecv(ops) if ops else []

    def exchange(self, stream=None):
        with _on_stream(self.buf, stream):
            for req in self.exchange_start():
                req.wait()


def _on_stream(t: torch.Tensor, stream):
    if t.is_cuda and stream is not None:
        return torch.cuda.stream(stream)
    return contextlib.nullcontext()


def bilateral_bands(lop, band: Bands, sigma_d, sigma_r, mode="clamp", constant=0.0, size=None,
                    out=None, stream=None):
    """Config 5 step: halo exchange overlapped with the interior rows, then the
    edge rows; bit-identical to the single-GPU call on the whole image.
    Everything (exchange, waits, launches) is ordered on `stream` (default:
    the current stream)."""
    if out is None:
        out = torch.empty_like(band.owned)
    if size is None:
        size = default_window(sigma_d)
    if stream is None and band.buf.is_cuda:
        stream = torch.cuda.current_stream(band.buf.device)
    ry = (size if isinstance(size, int) else size[1]) // 2
    args = band.band_args()
    rows, W = band.rows, band.W
    inner = (0, ry, W, rows - 2 * ry) if rows > 2 * ry else None
    with _on_stream(band.buf, stream):
        reqs = band.exchange_start()
        if inner is not None:
            # interior rows need no halo: run them while the messages are in flight
            lop.bilateral(band.owned, sigma_d, sigma_r, mode, constant, size=size, out=out,
                          roi=inner, stream=stream, band=args)
        for r in reqs:
            r.wait()                     # the current stream (= stream) waits for the halos
        if inner is None:
            lop.bilateral(band.owned, sigma_d, sigma_r, mode, constant, size=size, out=out,
                          stream=stream, band=args)
        else:
            for roi in ((0, 0, W, ry), (0, rows - ry, W, ry)):
                lop.bilateral(band.owned, sigma_d, sigma_r, mode, constant, size=size, out=out,
                              roi=roi, stream=stream, band=args)
    return out


def launches_per_band_step(band: Bands, size: int) -> int:
    """Kernel launches of one bilateral_bands call (interior + 2 edge ROIs, or
    one launch when the band is no taller than the two edges)."""
    ry = size // 2
    return 3 if band.rows > 2 * ry else 1
