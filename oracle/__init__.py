"""TEST INFRASTRUCTURE ONLY -- the fp64 CPU oracle of the star intensity model (Sec. II, Eqs. 1-3, Fig. 5).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may
import this package.  It shares no code with ``paper_conf_ipps_lizzh12_b200`` and imports nothing from it; the CUDA
path never imports it.  The C source ``starsim_oracle.c`` is compiled on first use with
``gcc -O2 -fno-fast-math -ffp-contract=off`` into ``liboracle.so`` next to it (``build()`` also does this).

Every function here only marshals numpy arrays into the C routines; each C routine cites the paper passage it follows.
Pins: tests/test_oracle_pins.py.  Parity status of each function: DESIGN.md §Oracle.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "starsim_oracle.c")
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

CFLAGS = ["-O2", "-fno-fast-math", "-ffp-contract=off", "-fPIC", "-shared", "-std=c11", "-D_GNU_SOURCE"]


def build(force: bool = False) -> str:
    """Compile starsim_oracle.c -> liboracle.so (skipped when the .so is newer than the source)."""
    if (not force and os.path.exists(_LIB_PATH)
            and os.path.getmtime(_LIB_PATH) >= os.path.getmtime(_SRC)):
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    subprocess.run(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm", "-lpthread"], check=True)
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        lib = ctypes.CDLL(build())
        f32p = ctypes.POINTER(ctypes.c_float)
        f64p = ctypes.POINTER(ctypes.c_double)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        i64p = ctypes.POINTER(ctypes.c_int64)
        i32, i64, f64 = ctypes.c_int32, ctypes.c_int64, ctypes.c_double
        lib.oracle_brightness.argtypes = [f64, f64]
        lib.oracle_brightness.restype = f64
        lib.oracle_psf.argtypes = [f64, f64, f64, f64, f64]
        lib.oracle_psf.restype = f64
        lib.oracle_psf_integrated.argtypes = [f64, f64, f64, f64, f64]
        lib.oracle_psf_integrated.restype = f64
        lib.oracle_roi_lo.argtypes = [ctypes.c_float, i32]
        lib.oracle_roi_lo.restype = i64
        lib.oracle_star_roi.argtypes = [ctypes.c_float, ctypes.c_float, ctypes.c_float, i32, i32, i32, i64p]
        lib.oracle_in_circle.argtypes = [ctypes.c_int64, ctypes.c_int64, i32]
        lib.oracle_in_circle.restype = ctypes.c_int
        lib.oracle_star_roi.restype = ctypes.c_int
        lib.oracle_render.argtypes = [f32p, f32p, f32p, i64, i32, i32, f64, i32, f64, i32, f64p]
        lib.oracle_render.restype = i64
        lib.oracle_render_band.argtypes = [f32p, f32p, f32p, i64, i32, i32, i32, i32, f64, i32, f64, i32, f64p]
        lib.oracle_render_band.restype = None
        lib.oracle_render_mt.argtypes = [f32p, f32p, f32p, i64, i32, i32, f64, i32, f64, i32, f64p, i32]
        lib.oracle_render_mt.restype = ctypes.c_int
        lib.oracle_render_full.argtypes = [f32p, f32p, f32p, i64, i32, i32, f64, f64, i32, f64p]
        lib.oracle_render_full.restype = None
        lib.oracle_bins.argtypes = [f32p, f32p, f32p, i64, i32, i32, i32, i32, i32, u32p, u32p, i64]
        lib.oracle_bins.restype = i64
        lib.oracle_route_band.argtypes = [f32p, i64, i32, i32, i32, i64p]
        lib.oracle_route_band.restype = i64
        lib.oracle_quantize.argtypes = [f64p, i64, i32, ctypes.c_void_p]
        lib.oracle_quantize.restype = None
        _lib = lib
        return lib


def _f32(a):
    a = np.ascontiguousarray(a, dtype=np.float32)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_float))


def _stars(x, y, mag):
    (x, px), (y, py), (mag, pm) = _f32(x), _f32(y), _f32(mag)
    if not (x.shape == y.shape == mag.shape and x.ndim == 1):
        raise ValueError("x, y, mag must be 1-D arrays of equal length")
    return (x, y, mag), (px, py, pm), x.shape[0]


def brightness(m: float, A: float) -> float:
    """Eq. 1: g(m) = A * 2.512^-m."""
    return _load().oracle_brightness(float(m), float(A))


PSF_MODES = {"point": 0, "integrated": 1}
ROI_SHAPES = {"square": 0, "circle": 2}  # NEXT-3 (reading R21): the paper's "pixel circle", mode bit 1


def _mode(psf_mode, roi="square"):
    if psf_mode not in PSF_MODES:
        raise ValueError(f"psf must be one of {sorted(PSF_MODES)}")
    if roi not in ROI_SHAPES:
        raise ValueError(f"roi must be one of {sorted(ROI_SHAPES)}")
    return PSF_MODES[psf_mode] | ROI_SHAPES[roi]


def in_circle(i: int, j: int, R: int) -> bool:
    """NEXT-3 (reading R21): is ROI pixel (row offset i, column offset j) inside the circle inscribed in the R x R
    square ROI?"""
    return bool(_load().oracle_in_circle(int(i), int(j), int(R)))


def psf(px: float, py: float, X: float, Y: float, sigma: float, mode: str = "point") -> float:
    """Eq. 2 at pixel (px, py) for a star at (X, Y); mode "integrated": Eq. 2 integrated over the pixel
    square (NEXT-2)."""
    f = _load().oracle_psf_integrated if _mode(mode) else _load().oracle_psf
    return f(float(px), float(py), float(X), float(Y), float(sigma))


def roi_lo(c: float, R: int) -> int:
    """First ROI column/row: the R integers nearest to fp32 c (reading R7)."""
    return int(_load().oracle_roi_lo(ctypes.c_float(c), int(R)))


def star_roi(x: float, y: float, m: float, W: int, H: int, R: int):
    """Clipped ROI (x0, x1, y0, y1) inclusive, or None if the star is skipped (readings R10, R11)."""
    out = (ctypes.c_int64 * 4)()
    ok = _load().oracle_star_roi(ctypes.c_float(x), ctypes.c_float(y), ctypes.c_float(m), int(W), int(H), int(R), out)
    return tuple(out) if ok else None


def render(x, y, mag, W: int, H: int, sigma: float, R: int, A: float, threads: int = 1, return_units: bool = False,
           psf: str = "point", roi: str = "square"):
    """The oracle image, fp64 (H, W), row-major with y = row: Eqs. 1-3 over square ROIs in star order (Fig. 5).

    ``threads > 1`` splits rows over pthreads; the result is bitwise identical (same per-pixel order).
    ``psf="integrated"``: the pixel-integrated variant of Eq. 2 (NEXT-2); ``roi="circle"``: the pixel circle
    inscribed in the square ROI (NEXT-3, reading R21); U then counts the circle's pixels."""
    mode = _mode(psf, roi)
    _, (px, py, pm), n = _stars(x, y, mag)
    img = np.empty((int(H), int(W)), dtype=np.float64)
    pimg = img.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
    lib = _load()
    if threads <= 1:
        U = lib.oracle_render(px, py, pm, n, int(W), int(H), float(sigma), int(R), float(A), mode, pimg)
    else:
        if lib.oracle_render_mt(px, py, pm, n, int(W), int(H), float(sigma), int(R), float(A), mode, pimg,
                                int(threads)):
            raise MemoryError("oracle_render_mt")
        U = None
    return (img, U) if return_units else img


def lut_positions(x, y, R: int):
    """Reading R20 (the adaptive simulator): every star taken at the centre of its ROI, i.e. at
    roi_lo(c, R) + (R - 1) / 2 on each axis (exact in fp32); non-finite coordinates are kept (the star is skipped)."""
    def snap(c):
        c64 = np.asarray(c, dtype=np.float32).astype(np.float64)
        fin = np.isfinite(c64)
        c0 = np.where(fin, c64, 0.0)
        fl = np.floor(c0)
        lo = (fl + (c0 >= fl + 0.5) - (R - 1) // 2) if R % 2 else (fl + 1 - R // 2)  # reading R7, exact in fp64
        return np.where(fin, lo + 0.5 * (R - 1), c64).astype(np.float32)
    return snap(x), snap(y)


def render_lut(x, y, mag, W: int, H: int, sigma: float, R: int, A: float, threads: int = 1, psf: str = "point",
               roi: str = "square"):
    """The adaptive simulator's image (NEXT-4): ``render`` with every star at its ROI centre."""
    sx, sy = lut_positions(x, y, R)
    return render(sx, sy, mag, W, H, sigma, R, A, threads=threads, psf=psf, roi=roi)


def render_band(x, y, mag, W: int, H: int, row0: int, rows: int, sigma: float, R: int, A: float,
                psf: str = "point"):
    """Rows [row0, row0+rows) of the oracle image, fp64 (rows, W)."""
    _, (px, py, pm), n = _stars(x, y, mag)
    img = np.empty((int(rows), int(W)), dtype=np.float64)
    _load().oracle_render_band(px, py, pm, n, int(W), int(H), int(row0), int(rows), float(sigma), int(R), float(A),
                               _mode(psf), img.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    return img


def render_full(x, y, mag, W: int, H: int, sigma: float, A: float, psf: str = "point"):
    """No ROI cut-off (Fig. 1 left): every star at every pixel.  Tiny inputs only."""
    _, (px, py, pm), n = _stars(x, y, mag)
    img = np.empty((int(H), int(W)), dtype=np.float64)
    _load().oracle_render_full(px, py, pm, n, int(W), int(H), float(sigma), float(A), _mode(psf),
                               img.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    return img


def units(x, y, mag, W: int, H: int, R: int):
    """(U, E, n_live): U = sum of clipped ROI areas (star-pixel updates), E = sum of clipped (w + h) (exps)."""
    lib = _load()
    xs, ys, ms = (np.ascontiguousarray(a, dtype=np.float32) for a in (x, y, mag))
    out = (ctypes.c_int64 * 4)()
    U = E = live = 0
    for i in range(xs.shape[0]):
        if lib.oracle_star_roi(ctypes.c_float(xs[i]), ctypes.c_float(ys[i]), ctypes.c_float(ms[i]),
                               int(W), int(H), int(R), out):
            w, h = out[1] - out[0] + 1, out[3] - out[2] + 1
            U += w * h
            E += w + h
            live += 1
    return U, E, live


def bins(x, y, mag, W: int, H: int, R: int, tile_w: int, tile_h: int):
    """Binning CSR (tile_off[ntiles+1] uint32, ids[P] uint32): stars by tile key ty*ntx+tx, star order inside."""
    _, (px, py, pm), n = _stars(x, y, mag)
    ntiles = ((W + tile_w - 1) // tile_w) * ((H + tile_h - 1) // tile_h)
    off = np.zeros(ntiles + 1, dtype=np.uint32)
    cap = max(1, n * (((R - 1) // tile_w) + 2) * (((R - 1) // tile_h) + 2))
    ids = np.zeros(cap, dtype=np.uint32)
    P = _load().oracle_bins(px, py, pm, n, int(W), int(H), int(R), int(tile_w), int(tile_h),
                            off.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)),
                            ids.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), cap)
    if P < 0:
        raise RuntimeError(f"oracle_bins failed ({P})")
    return off, ids[:P].copy()


def route_band(y, R: int, row0: int, rows: int):
    """Indices (int64, catalogue order) of the stars routed to rows [row0, row0+rows): ROI rows (reading R7) meet the
    band, y finite -- the definition of starsim_route_band."""
    ys = np.ascontiguousarray(y, dtype=np.float32)
    idx = np.empty(max(1, ys.shape[0]), dtype=np.int64)
    k = _load().oracle_route_band(ys.ctypes.data_as(ctypes.POINTER(ctypes.c_float)), ys.shape[0], int(R), int(row0),
                                  int(rows), idx.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)))
    return idx[:k].copy()


def quantize(v, bits: int):
    """Output stage: q = min(2^bits-1, floor(v+1/2)), v<=0 or NaN -> 0; uint8 or uint16."""
    if bits not in (8, 16):
        raise ValueError("bits must be 8 or 16")
    v = np.ascontiguousarray(v, dtype=np.float64)
    out = np.empty(v.shape, dtype=np.uint8 if bits == 8 else np.uint16)
    _load().oracle_quantize(v.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), v.size, int(bits),
                            out.ctypes.data_as(ctypes.c_void_p))
    return out
