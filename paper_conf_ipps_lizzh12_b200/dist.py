"""Multi-GPU frames: horizontal bands, one per rank, assembled with one all-gather.

The paper is single-GPU and names multi-GPU scaling as future work (Sec. V).  Here the image is split
into G horizontal bands of whole 64-row tiles.  Every rank holds the replicated catalogue and, each frame, routes it
to its band on the device (``starsim_route_band``: the stars whose ROI rows meet the band, compacted in catalogue
order, the count left in device memory) and renders the band from the routed stars (``starsim_set_star_count`` +
``starsim_render_band``; ``Context.render_band_routed`` does both) -- there is no ROI arithmetic in this module.
``torch.distributed.all_gather_into_tensor`` then concatenates the bands (row-major band concatenation *is* the frame,
no re-layout), or ``FusedFrame`` stores every band pixel straight into every rank's frame from the tile kernel.  With
tile-aligned band edges the assembled frame is bitwise equal to the single-GPU render (same per-pixel star order).

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


def padded_band_rows(height: int, world: int, align: int = TILE_H) -> int:
    """Rows of the equal-size band buffers used by the all-gather (all_gather_into_tensor needs equal chunks)."""
    tiles = -(-height // align)
    return -(-tiles // world) * align


def render_frame(render_band, x, y, mag, width: int, height: int, sigma: float, roi: int, gain: float,
                 group=None, full_out=None, band_out=None):
    """Render this rank's band and all-gather the frame.

    ``render_band(x, y, mag, width, height, row0, rows, sigma, roi, gain, out)`` renders rows [row0, row0+rows) of the
    frame of the whole catalogue (x, y, mag) into ``out`` (rows x width); for the product it is
    ``Context.render_band_routed`` (device routing + band render), in the CPU tests the oracle.  Returns (full_frame, band_view).
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


def frames_agree(frame, ref, group=None) -> bool:
    """True iff this rank's assembled frame equals ``ref`` bitwise on EVERY rank of the group (one MIN all-reduce):
    the validation of a multi-GPU frame against the single-GPU (or oracle) frame, used by bench.py's strong_C5 record
    and the gloo tests."""
    import torch
    import torch.distributed as dist
    ok = torch.tensor([1 if (frame.shape == ref.shape and bool(torch.equal(frame, ref))) else 0], dtype=torch.int32,
                      device=frame.device)
    if dist.is_initialized():
        dist.all_reduce(ok, op=dist.ReduceOp.MIN, group=group)
    return bool(ok.item())


class FusedFrame:
    """The fused band exchange (north star: bands assembled over NVLink).

    The frame lives in torch symmetric memory: every rank maps every other rank's frame into its address space, and
    ``starsim_render_band_to`` makes the tile kernel's epilogue store each pixel of this rank's band into all of them
    over NVLink / NVSwitch while the rest of the band is still being rendered.  Two device-side barriers on the render
    stream (the symmetric-memory handle's signal pads) bracket the stores: the one before keeps a rank from writing
    frame k+1 into a peer's frame while that peer's stream may still be reading frame k, the one after orders every
    rank's stores before any rank reads its frame.  There is no all-gather pass: the exchange overlaps the render.  Needs CUDA peer access between the ranks'
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
        """Barrier, this rank's band (device-routed from the whole catalogue x, y, mag) into every rank's frame,
        barrier -- all on `stream`.  Returns the local frame, complete once the stream passes the second barrier and
        valid until the next ``render`` (readers on other streams must be ordered before it)."""
        import torch

        row0, rows = band_rows(self.height, self.world, self.rank)
        st = stream if stream is not None else torch.cuda.current_stream()
        with torch.cuda.stream(st):
            self.handle.barrier(channel=0)  # every peer is done with the previous frame before anyone overwrites it
            if rows > 0:
                ctx.render_band_routed(x, y, mag, self.width, self.height, row0, rows, sigma, roi, gain,
                                       frames=self.ptrs, stream=st)
            self.handle.barrier(channel=0)
        return self.frame
