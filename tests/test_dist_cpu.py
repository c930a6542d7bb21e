"""Multi-GPU band decomposition, host logic on CPU: world_size-2 (and 3) gloo process groups render bands with the fp64
oracle standing in for the per-rank renderer and assemble them with all_gather_into_tensor; the result must equal the
single-process frame bitwise."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_lizzh12_b200 import dist as sdist


def test_band_rows_partition_every_row():
    for H in [1, 63, 64, 65, 512, 1000, 4096]:
        for G in [1, 2, 3, 4, 8]:
            rows = []
            for r in range(G):
                r0, n = sdist.band_rows(H, G, r)
                assert n >= 0 and r0 % sdist.TILE_H == 0 or n == 0
                assert n <= sdist.padded_band_rows(H, G)
                rows.extend(range(r0, r0 + n))
                if n:
                    assert r0 == r * sdist.padded_band_rows(H, G)
            assert rows == list(range(H))


@pytest.mark.parametrize("R", [1, 4, 9, 15])
def test_band_star_mask_routes_exactly_the_stars_whose_roi_meets_the_band(R):
    """band_star_mask against the oracle's clipped ROI rows (reading R7, exact) on adversarial coordinates: a star is
    routed to a band iff its clipped ROI rows meet it; every contributing star reaches at least one band."""
    import oracle
    import synth
    W, H, G = 70, 256, 4
    f = synth.adversarial_field(3000, W, H, R, seed=7)
    masks = [sdist.band_star_mask(f.y, *sdist.band_rows(H, G, g), R) for g in range(G)]
    for i in range(f.n):
        roi = oracle.star_roi(float(f.x[i]), float(f.y[i]), float(f.mag[i]), W, H, R)
        if roi is None:
            continue
        y0, y1 = roi[2], roi[3]
        for g in range(G):
            r0, n = sdist.band_rows(H, G, g)
            assert bool(masks[g][i]) == (y0 <= r0 + n - 1 and y1 >= r0), (i, g)
        assert any(m[i] for m in masks)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, W, H, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import synth
    f = synth.uniform_field(600, W, H, seed=3)

    def render_band(x, y, mag, width, height, row0, rows, sigma, roi, gain, out):
        # the rank's own catalogue: the stars routed to its band (bench.py does the same before its timed region)
        sel = sdist.band_star_mask(f.y, row0, rows, roi)
        img = oracle.render_band(f.x[sel], f.y[sel], f.mag[sel], width, height, row0, rows, sigma, roi, gain)
        out.copy_(torch.from_numpy(img.astype(np.float32)))

    x = torch.zeros(1)
    frame, band = sdist.render_frame(render_band, x, x, x, W, H, 1.7, 9, 1.0)
    if rank == 0:
        q.put(frame.numpy().copy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_bands_assemble_the_frame(world):
    import oracle
    import synth
    W, H = 96, 200
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, W, H, q)) for r in range(world)]
    for p in procs:
        p.start()
    frame = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    f = synth.uniform_field(600, W, H, seed=3)
    ref = oracle.render(f.x, f.y, f.mag, W, H, 1.7, 9, 1.0).astype(np.float32)
    assert frame.shape == (H, W)
    assert np.array_equal(frame, ref)
