"""Multi-GPU frames: horizontal bands, one per rank, assembled with one all-gather.

The paper is single-GPU and names multi-GPU scaling as future work (Sec. V).  Here the image is split
into G horizontal bands of whole 64-row tiles; every rank renders its band with ``starsim_render_band`` (stars are
routed to a band iff their ROI rows intersect it: ``band_star_mask`` selects a rank's catalogue, and the library's
binning pass clips every star to the band), and ``torch.distributed.all_gather_into_tensor`` concatenates the bands: row-major band
concatenation *is* the frame, so there is no re-layout.  With tile-aligned band edges the assembled frame is bitwise
equal to the single-GPU render (same per-pixel star order).

torch.distributed (NCCL on GPUs, gloo in the CPU tests) is plumbing only; the render runs in libstarsim.so.
"""
from __future__ import annotations

TILE_H = 64   # must equal the library tile height (csrc/common.cuh) for bitwise band equality


def band_rows(height: int, world: int, rank: int, align: int = TILE_H) -> tuple[int, int]:
    """Rows [row0, row0 + rows) of rank's band: equal bands of whole `align`-row tiles when height allows, the last
    band taking the remainder.  Every row is in exactly one band."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError("bad world/rank")
    tiles = -(-height // align)
    per = -(-tiles // world)                      # tiles per band (ceil); trailing ranks may get fewer / none
    t0 = min(tiles, rank * per)
    t1 = min(tiles, (rank + 1) * per)
    row0 = min(height, t0 * align)
    row1 = min(height, t1 * align)
    return row0, row1 - row0


def band_star_mask(y, row0: int, rows: int, roi: int):
    """The stars routed to band [row0, row0 + rows): those whose ROI rows meet it, as a boolean
    mask over the catalogue (host, numpy).  The ROI's first row is the exact rule of reading R7 (the R rows nearest
    y, ties at k + 1/2 upward), evaluated exactly in fp64 on the fp32 coordinate; stars with a non-finite y are left
    out (they contribute nothing).  Keeping the catalogue order, a band rendered from ``catalogue[mask]`` has the same
    tile lists, in the same relative order, as the band rendered from the whole catalogue: the same image bit for bit.
    This is the per-band catalogue query of a distributed render (the catalogue retrieval itself is out of scope,
    SURVEY.md §8f); bench.py applies it before the timed region, so no rank bins stars of other bands."""
    import numpy as np
    y64 = np.asarray(y, dtype=np.float32).astype(np.float64)
    fin = np.isfinite(y64)
    yc = np.where(fin, y64, 0.0)
    fy = np.floor(yc)
    ly = (fy + (yc >= fy + 0.5) - (roi - 1) // 2) if roi % 2 else (fy + 1 - roi // 2)
    return fin & (ly <= row0 + rows - 1) & (ly + roi - 1 >= row0)


def padded_band_rows(height: int, world: int, align: int = TILE_H) -> int:
    """Rows of the equal-size band buffers used by the all-gather (all_gather_into_tensor needs equal chunks)."""
    tiles = -(-height // align)
    return -(-tiles // world) * align


def render_frame(render_band, x, y, mag, width: int, height: int, sigma: float, roi: int, gain: float,
                 group=None, full_out=None, band_out=None):
    """Render this rank's band and all-gather the frame.

    ``render_band(x, y, mag, width, height, row0, rows, sigma, roi, gain, out)`` renders rows [row0, row0+rows) into
    ``out`` (rows x width); for the product it is ``Context.render_band``.  Returns (full_frame, band_view).
    The gathered tensor has world * padded rows; the frame is its first ``height`` rows.
    """
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    prow = padded_band_rows(height, world)
    dev = x.device
    if band_out is None:
        band_out = torch.zeros((prow, width), dtype=torch.float32, device=dev)
    row0, rows = band_rows(height, world, rank)
    if rows > 0:
        render_band(x, y, mag, width, height, row0, rows, sigma, roi, gain, band_out[:rows])
    if rows < prow:
        band_out[rows:].zero_()
    if world == 1:
        return band_out[:height], band_out
    if full_out is None:
        full_out = torch.empty((world * prow, width), dtype=torch.float32, device=dev)
    dist.all_gather_into_tensor(full_out, band_out, group=group)
    return full_out[:height], band_out


class FusedFrame:
    """The fused band exchange (north star: bands assembled over NVLink).

    The frame lives in torch symmetric memory: every rank maps every other rank's frame into its address space, and
    ``starsim_render_band_to`` makes the tile kernel's epilogue store each pixel of this rank's band into all of them
    over NVLink / NVSwitch while the rest of the band is still being rendered.  A device-side barrier on the render
    stream (the symmetric-memory handle's signal pads) then orders every rank's stores before any rank reads its
    frame.  There is no all-gather pass: the exchange overlaps the render.  Needs CUDA peer access between the ranks'
    GPUs (one node); ``available()`` says whether this process can use it, otherwise ``render_frame`` (NCCL
    all-gather) is the path.
    """

    def __init__(self, height: int, width: int, device, group=None):
        import torch
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem

        self.height, self.width = height, width
        self.group = group if group is not None else dist.group.WORLD
        self.world = dist.get_world_size(self.group)
        self.rank = dist.get_rank(self.group)
        self.frame = symm_mem.empty((height, width), dtype=torch.float32, device=device)
        self.handle = symm_mem.rendezvous(self.frame, self.group.group_name)
        self.ptrs = [int(p) for p in self.handle.buffer_ptrs]
        if len(self.ptrs) != self.world:
            raise RuntimeError("symmetric-memory rendezvous returned a wrong number of peer buffers")

    @staticmethod
    def available() -> bool:
        try:
            import torch
            import torch.distributed as dist
            import torch.distributed._symmetric_memory  # noqa: F401
        except Exception:
            return False
        return torch.cuda.is_available() and dist.is_initialized() and dist.get_backend() == "nccl"

    def render(self, ctx, x, y, mag, sigma: float, roi: int, gain: float, stream=None):
        """This rank's band into every rank's frame, then the cross-GPU barrier (all on `stream`); returns the local
        frame, complete once the stream reaches the barrier."""
        import torch

        row0, rows = band_rows(self.height, self.world, self.rank)
        st = stream if stream is not None else torch.cuda.current_stream()
        with torch.cuda.stream(st):
            if rows > 0:
                ctx.render_band_to(x, y, mag, self.width, self.height, row0, rows, sigma, roi, gain, self.ptrs,
                                   stream=st)
            self.handle.barrier(channel=0)
        return self.frame
