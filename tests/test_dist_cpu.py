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
        img = oracle.render_band(f.x, f.y, f.mag, width, height, row0, rows, sigma, roi, gain)
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
