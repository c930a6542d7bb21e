"""Multi-GPU band decomposition, host logic on CPU: world_size-2 (and 3) gloo process groups render bands with the fp64
oracle standing in for the per-rank renderer and assemble them with all_gather_into_tensor; the result must equal the
single-process frame bitwise.  Band routing: oracle.route_band, the definition the library's
starsim_route_band is compared with on the GPU (tests/test_gpu_parity.py), pinned here against exact arithmetic."""
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
def test_oracle_route_band_is_the_exact_roi_row_rule(R):
    """oracle.route_band (the definition starsim_route_band computes) pinned against exact rational arithmetic: a star
    is routed to a band iff y is finite and its ROI rows [lo, lo + R - 1], lo = floor(y + 1 - R/2) in exact arithmetic
    (reading R7: the R rows nearest y, ties upward), meet the band; indices ascending.  Adversarial coordinates
    (half-integers and their fp32 neighbours, band edges, non-finite values, far-off stars); every star whose clipped
    ROI is non-empty reaches the band(s) its clipped rows meet."""
    import math
    from fractions import Fraction
    import oracle
    import synth
    W, H, G = 70, 256, 4
    f = synth.adversarial_field(3000, W, H, R, seed=7)
    for g in range(G):
        r0, n = sdist.band_rows(H, G, g)
        got = oracle.route_band(f.y, R, r0, n)
        want = []
        for i, yv in enumerate(f.y.tolist()):
            if not math.isfinite(yv):
                continue
            lo = math.floor(Fraction(yv) + 1 - Fraction(R, 2))
            if lo <= r0 + n - 1 and lo + R - 1 >= r0:
                want.append(i)
        assert got.tolist() == want, g
    sel = [set(oracle.route_band(f.y, R, *sdist.band_rows(H, G, g)).tolist()) for g in range(G)]
    for i in range(f.n):
        roi = oracle.star_roi(float(f.x[i]), float(f.y[i]), float(f.mag[i]), W, H, R)
        if roi is None:
            continue
        for g in range(G):
            r0, n = sdist.band_rows(H, G, g)
            if roi[2] <= r0 + n - 1 and roi[3] >= r0:
                assert i in sel[g], (i, g)


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
        # stand-in for Context.render_band_routed on CPU: route the whole catalogue to the band (the oracle's
        # definition of starsim_route_band), render the band from the routed stars
        sel = oracle.route_band(y.numpy(), roi, row0, rows)
        xs, ys, ms = (t.numpy()[sel] for t in (x, y, mag))
        img = oracle.render_band(xs, ys, ms, width, height, row0, rows, sigma, roi, gain)
        out.copy_(torch.from_numpy(img.astype(np.float32)))

    # back-to-back frames through the same band buffer (different catalogues): each assembled frame checked
    band_out = None
    ok = True
    for k, seed in enumerate((11, 12, 13)):
        fk = synth.uniform_field(400 + 50 * k, W, H, seed=seed)
        xk, yk, mk = (torch.from_numpy(a) for a in (fk.x, fk.y, fk.mag))
        fr, band_out = sdist.render_frame(render_band, xk, yk, mk, W, H, 1.7, 9, 1.0, band_out=band_out)
        refk = torch.from_numpy(oracle.render(fk.x, fk.y, fk.mag, W, H, 1.7, 9, 1.0).astype(np.float32))
        ok = ok and sdist.frames_agree(fr, refk)
    x, y, m = (torch.from_numpy(a) for a in (f.x, f.y, f.mag))
    frame, band = sdist.render_frame(render_band, x, y, m, W, H, 1.7, 9, 1.0)
    # the bench's validation (dist.frames_agree): every rank compares its assembled frame with the single-process
    # frame; a corrupted frame on any one rank must make it fail on all ranks
    ref = torch.from_numpy(oracle.render(f.x, f.y, f.mag, W, H, 1.7, 9, 1.0).astype(np.float32))
    ok = ok and sdist.frames_agree(frame, ref)
    bad = frame.clone()
    if rank == world - 1:
        bad[H - 1, W - 1] += 1.0
    ok_bad = sdist.frames_agree(bad, ref)
    if rank == 0:
        q.put((frame.numpy().copy(), ok, ok_bad))
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
    frame, ok, ok_bad = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    f = synth.uniform_field(600, W, H, seed=3)
    ref = oracle.render(f.x, f.y, f.mag, W, H, 1.7, 9, 1.0).astype(np.float32)
    assert frame.shape == (H, W)
    assert np.array_equal(frame, ref)
    assert ok and not ok_bad
