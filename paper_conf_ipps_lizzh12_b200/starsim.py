"""Thin ctypes binding of libstarsim.so (include/starsim.h) -- argument marshalling only.

Every step of the render runs in the library's sm_100a kernels; this module only converts torch CUDA tensors to
device pointers and the current torch stream to a ``cudaStream_t``.  There is no CPU fallback: if the library is not
built, or the device is not an sm_100 GPU, the calls raise.  torch is used for device memory and streams only.

Names mirror the C ABI (one Python function per entry point of include/starsim.h, same name and argument order,
``n`` taken from the tensors): ``starsim_create``, ``starsim_render``, ``starsim_render_band``,
``starsim_render_band_to``, ``starsim_render_gray``, ``starsim_render_atomic``, ``starsim_render_lut``,
``starsim_route_band``, ``starsim_set_star_count``, ``starsim_set_psf``, ``starsim_set_roi``, ``starsim_set_binning``,
``starsim_set_tile_kernel``, ``starsim_upload_aos``, ``starsim_quantize``, ``starsim_get_bins``, ``starsim_profile``,
``starsim_kernel_times``, ``starsim_destroy``; :class:`Context` wraps a handle with the same methods.  Output
tensors are checked for dtype, contiguity and size here, so a too-small buffer raises instead of being overrun.
"""
from __future__ import annotations

import ctypes
import os
import threading

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("STARSIM_LIB") or os.path.join(_PKG, "libstarsim.so")  # override: A/B tooling only

STARSIM_OK, STARSIM_EINVAL, STARSIM_ENOMEM, STARSIM_ECUDA, STARSIM_ENODEV = 0, -1, -2, -3, -4
KCLASSES = ("prep", "sort", "csr", "tile", "atomic", "memset", "quantize", "aos", "route")
NUM_KCLASS = len(KCLASSES)

_lock = threading.Lock()
_lib = None


class StarsimError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"starsim error {code}: {msg}")
        self.code = code


class StarsimSizeError(StarsimError, ValueError):
    """A buffer smaller than the call would access: rejected by the binding (EINVAL) before the library runs."""

    def __init__(self, msg: str):
        super().__init__(STARSIM_EINVAL, msg)


def lib():
    """Load libstarsim.so (fails loudly if it has not been built)."""
    global _lib
    with _lock:
        if _lib is not None:
            return _lib
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is not built; run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        vp, i32, i64, f32 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64, ctypes.c_float
        L.starsim_create.argtypes = [ctypes.POINTER(vp), ctypes.c_int]
        L.starsim_create.restype = ctypes.c_int
        L.starsim_destroy.argtypes = [vp]
        L.starsim_destroy.restype = None
        L.starsim_last_error.argtypes = [vp]
        L.starsim_last_error.restype = ctypes.c_char_p
        L.starsim_render.argtypes = [vp, vp, vp, vp, i64, i32, i32, f32, i32, f32, vp, vp]
        L.starsim_render.restype = ctypes.c_int
        L.starsim_render_band.argtypes = [vp, vp, vp, vp, i64, i32, i32, i32, i32, f32, i32, f32, vp, vp]
        L.starsim_render_band_to.argtypes = [vp, vp, vp, vp, i64, i32, i32, i32, i32, f32, i32, f32,
                                             ctypes.POINTER(vp), i32, vp]
        L.starsim_render_band_to.restype = ctypes.c_int
        L.starsim_render_band.restype = ctypes.c_int
        L.starsim_render_gray.argtypes = [vp, vp, vp, vp, i64, i32, i32, f32, i32, f32, i32, vp, vp]
        L.starsim_render_gray.restype = ctypes.c_int
        L.starsim_set_psf.argtypes = [vp, i32]
        L.starsim_set_psf.restype = ctypes.c_int
        L.starsim_set_roi.argtypes = [vp, i32]
        L.starsim_set_roi.restype = ctypes.c_int
        L.starsim_set_binning.argtypes = [vp, i32]
        L.starsim_set_binning.restype = ctypes.c_int
        L.starsim_set_tile_kernel.argtypes = [vp, i32]
        L.starsim_set_tile_kernel.restype = ctypes.c_int
        L.starsim_route_band.argtypes = [vp, vp, vp, vp, i64, i32, i32, i32, i32, vp, vp, vp, vp, vp]
        L.starsim_route_band.restype = ctypes.c_int
        L.starsim_set_star_count.argtypes = [vp, vp]
        L.starsim_set_star_count.restype = ctypes.c_int
        L.starsim_render_atomic.argtypes = [vp, vp, vp, vp, i64, i32, i32, f32, i32, f32, vp, vp]
        L.starsim_render_atomic.restype = ctypes.c_int
        L.starsim_render_lut.argtypes = [vp, vp, vp, vp, i64, i32, i32, f32, i32, f32, vp, vp]
        L.starsim_render_lut.restype = ctypes.c_int
        L.starsim_upload_aos.argtypes = [vp, vp, i64, vp, vp, vp, vp]
        L.starsim_upload_aos.restype = ctypes.c_int
        L.starsim_quantize.argtypes = [vp, vp, i64, i32, vp, vp]
        L.starsim_quantize.restype = ctypes.c_int
        L.starsim_get_bins.argtypes = [vp, ctypes.POINTER(i32), ctypes.POINTER(i32), vp, i64, vp, i64,
                                       ctypes.POINTER(i64)]
        L.starsim_get_bins.restype = ctypes.c_int
        L.starsim_profile.argtypes = [vp, ctypes.c_int]
        L.starsim_profile.restype = ctypes.c_int
        L.starsim_kernel_times.argtypes = [vp, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(i64)]
        L.starsim_kernel_times.restype = ctypes.c_int
        _lib = L
        return L


def _check(ctx, rc: int):
    if rc != STARSIM_OK:
        raise StarsimError(rc, lib().starsim_last_error(ctx).decode(errors="replace"))


def _stream(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


def _ptr(t, dtype=None, name="tensor", numel=None):
    """Device pointer of a contiguous CUDA tensor; numel: the elements the library will access (checked >=)."""
    if t is None:
        if numel:
            raise ValueError(f"{name} is None")
        return None
    if not t.is_cuda:
        raise ValueError(f"{name} must be a CUDA tensor")
    if not t.is_contiguous():
        raise ValueError(f"{name} must be contiguous")
    if dtype is not None and t.dtype != dtype:
        raise ValueError(f"{name} must be {dtype}, got {t.dtype}")
    if numel is not None and t.numel() < numel:
        raise StarsimSizeError(f"{name} has {t.numel()} elements, the call writes / reads {numel}")
    return ctypes.c_void_p(t.data_ptr())


def _cat(x, y, mag):
    """Pointers and n of a SoA catalogue (x, y, mag float32, same length; None for an empty catalogue)."""
    import torch
    n = int(x.numel()) if x is not None else 0
    for t, nm in ((y, "y"), (mag, "mag")):
        if (t.numel() if t is not None else 0) != n:
            raise ValueError(f"{nm} has a different length than x")
    return (_ptr(x, torch.float32, "x"), _ptr(y, torch.float32, "y"), _ptr(mag, torch.float32, "mag"), n)


# ------------------------------------------------------------------ C-named functions

def starsim_create(device: int = 0):
    h = ctypes.c_void_p()
    rc = lib().starsim_create(ctypes.byref(h), int(device))
    if rc != STARSIM_OK:
        raise StarsimError(rc, lib().starsim_last_error(None).decode(errors="replace"))
    return h


def starsim_last_error(h=None) -> str:
    """Text of the last error on context h (or of the last create failure when h is None)."""
    return lib().starsim_last_error(h).decode(errors="replace")


def starsim_destroy(h) -> None:
    if h:
        lib().starsim_destroy(h)


def starsim_render(h, x, y, mag, width, height, sigma, roi, gain, out, stream=None) -> None:
    import torch
    px, py, pm, n = _cat(x, y, mag)
    _check(h, lib().starsim_render(h, px, py, pm, n, int(width), int(height), float(sigma), int(roi), float(gain),
                                   _ptr(out, torch.float32, "out", int(width) * int(height)), _stream(stream)))


def starsim_render_band_to(h, x, y, mag, width, height, row0, rows, sigma, roi, gain, dst_ptrs, stream=None) -> None:
    """dst_ptrs: device addresses (ints) of ndst full float32 frames (height x width), local or peer-mapped."""
    px, py, pm, n = _cat(x, y, mag)
    arr = (ctypes.c_void_p * max(1, len(dst_ptrs)))(*[ctypes.c_void_p(int(p)) for p in dst_ptrs])
    _check(h, lib().starsim_render_band_to(h, px, py, pm, n, int(width), int(height), int(row0),
                                           int(rows), float(sigma), int(roi), float(gain), arr, len(dst_ptrs),
                                           _stream(stream)))


def starsim_render_gray(h, x, y, mag, width, height, sigma, roi, gain, bits, out, stream=None) -> None:
    import torch
    px, py, pm, n = _cat(x, y, mag)
    dt = torch.uint8 if int(bits) == 8 else torch.uint16
    _check(h, lib().starsim_render_gray(h, px, py, pm, n, int(width), int(height), float(sigma), int(roi),
                                        float(gain), int(bits), _ptr(out, dt, "out", int(width) * int(height)),
                                        _stream(stream)))


PSF_MODES = {"point": 0, "integrated": 1}


def starsim_set_psf(h, mode) -> None:
    _check(h, lib().starsim_set_psf(h, PSF_MODES.get(mode, mode) if isinstance(mode, str) else int(mode)))


ROI_SHAPES = {"square": 0, "circle": 1}


def starsim_set_roi(h, shape) -> None:
    _check(h, lib().starsim_set_roi(h, ROI_SHAPES.get(shape, shape) if isinstance(shape, str) else int(shape)))


BINNINGS = {"auto": 0, "atomic": 1}


def starsim_set_binning(h, mode) -> None:
    _check(h, lib().starsim_set_binning(h, BINNINGS.get(mode, mode) if isinstance(mode, str) else int(mode)))


TILE_KERNELS = {"auto": 0, "lists": 1, "sb": 2, "ws": 3, "t8": 4}


def starsim_set_tile_kernel(h, mode) -> None:
    _check(h, lib().starsim_set_tile_kernel(h, TILE_KERNELS.get(mode, mode) if isinstance(mode, str) else int(mode)))


def starsim_render_band(h, x, y, mag, width, height, row0, rows, sigma, roi, gain, out_band, stream=None) -> None:
    import torch
    px, py, pm, n = _cat(x, y, mag)
    _check(h, lib().starsim_render_band(h, px, py, pm, n, int(width), int(height), int(row0), int(rows), float(sigma),
                                        int(roi), float(gain),
                                        _ptr(out_band, torch.float32, "out_band", int(rows) * int(width)),
                                        _stream(stream)))


def starsim_route_band(h, x, y, mag, height, row0, rows, roi, x_out, y_out, mag_out, n_out, stream=None) -> None:
    """The stars of (x, y, mag) routed to rows [row0, row0+rows) -> (x_out, y_out, mag_out)[:*n_out] (device)."""
    import torch
    px, py, pm, n = _cat(x, y, mag)
    _check(h, lib().starsim_route_band(h, px, py, pm, n, int(height), int(row0), int(rows), int(roi),
                                       _ptr(x_out, torch.float32, "x_out", n), _ptr(y_out, torch.float32, "y_out", n),
                                       _ptr(mag_out, torch.float32, "mag_out", n),
                                       _ptr(n_out, torch.int32, "n_out", 1), _stream(stream)))


def starsim_set_star_count(h, n_dev) -> None:
    """n_dev: a CUDA int32 tensor holding the star count (read as uint32 by the kernels), or None to clear."""
    import torch
    _check(h, lib().starsim_set_star_count(h, None if n_dev is None else _ptr(n_dev, torch.int32, "n_dev", 1)))


def starsim_render_atomic(h, x, y, mag, width, height, sigma, roi, gain, out, stream=None) -> None:
    import torch
    px, py, pm, n = _cat(x, y, mag)
    _check(h, lib().starsim_render_atomic(h, px, py, pm, n, int(width), int(height), float(sigma), int(roi),
                                          float(gain), _ptr(out, torch.float32, "out", int(width) * int(height)),
                                          _stream(stream)))


def starsim_render_lut(h, x, y, mag, width, height, sigma, roi, gain, out, stream=None) -> None:
    import torch
    px, py, pm, n = _cat(x, y, mag)
    _check(h, lib().starsim_render_lut(h, px, py, pm, n, int(width), int(height), float(sigma), int(roi),
                                       float(gain), _ptr(out, torch.float32, "out", int(width) * int(height)),
                                       _stream(stream)))


def starsim_upload_aos(h, host_aos: np.ndarray, x, y, mag, stream=None) -> None:
    import torch
    a = np.ascontiguousarray(host_aos, dtype=np.float32)
    if a.ndim != 2 or a.shape[1] != 3:
        raise ValueError("host_aos must be (n, 3) float32 {mag, posX, posY}")
    n = a.shape[0]
    _check(h, lib().starsim_upload_aos(h, a.ctypes.data_as(ctypes.c_void_p), n,
                                       _ptr(x, torch.float32, "x", n), _ptr(y, torch.float32, "y", n),
                                       _ptr(mag, torch.float32, "mag", n), _stream(stream)))


def starsim_quantize(h, img, bits, out, stream=None) -> None:
    import torch
    want = torch.uint8 if bits == 8 else torch.uint16 if bits == 16 else None
    npix = int(img.numel())
    _check(h, lib().starsim_quantize(h, _ptr(img, torch.float32, "img"), npix, int(bits),
                                     _ptr(out, want, "out", npix) if want is not None else ctypes.c_void_p(out.data_ptr()),
                                     _stream(stream)))


def starsim_get_bins(h, max_pairs: int | None = None):
    """(tile_w, tile_h, tile_off uint32[ntiles+1], ids uint32[P]) of the last tiled render (synchronises)."""
    tw, th, P = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int64()
    rc = lib().starsim_get_bins(h, ctypes.byref(tw), ctypes.byref(th), None, 0, None, 0, ctypes.byref(P))
    if rc not in (STARSIM_OK, STARSIM_EINVAL) or P.value < 0:
        _check(h, rc)
    # ask again with buffers sized from the reply; ntiles is unknown here so grow until accepted
    cap_off = 1 << 12
    while True:
        off = np.zeros(cap_off, dtype=np.uint32)
        ids = np.zeros(max(1, P.value), dtype=np.uint32)
        rc = lib().starsim_get_bins(h, ctypes.byref(tw), ctypes.byref(th), off.ctypes.data_as(ctypes.c_void_p),
                                    cap_off, ids.ctypes.data_as(ctypes.c_void_p), ids.size, ctypes.byref(P))
        if rc == STARSIM_OK:
            break
        if rc != STARSIM_EINVAL or cap_off > (1 << 26):
            _check(h, rc)
        cap_off *= 4
    return tw.value, th.value, off, ids[:P.value]


def starsim_profile(h, enable: bool) -> None:
    _check(h, lib().starsim_profile(h, 1 if enable else 0))


def starsim_kernel_times(h) -> dict:
    ms = (ctypes.c_double * NUM_KCLASS)()
    ln = (ctypes.c_int64 * NUM_KCLASS)()
    _check(h, lib().starsim_kernel_times(h, ms, ln))
    return {k: (ms[i], ln[i]) for i, k in enumerate(KCLASSES)}


# ------------------------------------------------------------------ convenience handle

class Context:
    """One libstarsim context bound to one CUDA device (not thread-safe)."""

    def __init__(self, device: int | None = None):
        import torch
        self.device = torch.cuda.current_device() if device is None else int(device)
        self.h = starsim_create(self.device)

    def close(self):
        if self.h:
            starsim_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def _out(self, rows, width, out):
        import torch
        if out is None:
            out = torch.empty((rows, width), dtype=torch.float32, device=f"cuda:{self.device}")
        return out

    def render(self, x, y, mag, width, height, sigma, roi, gain, out=None, stream=None):
        out = self._out(height, width, out)
        starsim_render(self.h, x, y, mag, width, height, sigma, roi, gain, out, stream)
        return out

    def render_gray(self, x, y, mag, width, height, sigma, roi, gain, bits=8, out=None, stream=None):
        import torch
        if out is None:
            out = torch.empty((height, width), dtype=torch.uint8 if bits == 8 else torch.uint16, device=x.device)
        starsim_render_gray(self.h, x, y, mag, width, height, sigma, roi, gain, bits, out, stream)
        return out

    def set_psf(self, mode="point"):
        """"point" (Eq. 2 sampled at the pixel, the paper) or "integrated" (Eq. 2 integrated over the pixel)."""
        starsim_set_psf(self.h, mode)

    def set_roi(self, shape="square"):
        """"square" (the R x R ROI, reading R5) or "circle" (the pixel circle inscribed in it, NEXT-3, reading R21: every
        render; the tiled ones mask it in the tile kernel's walk: k_tile_sb for R <= 17, k_tile_wide for 27 <= R <= 65,
        k_tile otherwise)."""
        starsim_set_roi(self.h, shape)

    def set_binning(self, mode="auto"):
        """"auto" (deterministic counting sort when the frame has <= 2048 tiles and R <= 65) or "atomic"."""
        starsim_set_binning(self.h, mode)

    def set_tile_kernel(self, mode="auto"):
        """"auto" (R <= 17: "ws" on dense frames, else "sb"; 27 <= R <= 65: k_tile_wide; else "lists"), "lists" (k_tile,
        any R), "sb" (k_tile_sb; k_tile_wide for 27 <= R <= 65), "ws" (k_tile_ws; k_tile_wws) or "t8" (k_t8sort + k_tile8;
        k_tile_wws); include/starsim.h, starsim_set_tile_kernel."""
        starsim_set_tile_kernel(self.h, mode)

    def render_band(self, x, y, mag, width, height, row0, rows, sigma, roi, gain, out=None, stream=None):
        out = self._out(rows, width, out)
        starsim_render_band(self.h, x, y, mag, width, height, row0, rows, sigma, roi, gain, out, stream)
        return out

    def render_band_to(self, x, y, mag, width, height, row0, rows, sigma, roi, gain, frames, stream=None):
        """Render rows [row0, row0+rows) into every frame of `frames` (full height x width float32 frames: CUDA
        tensors, or raw device addresses of peer-mapped frames) -- the fused band exchange."""
        ptrs = [f if isinstance(f, int) else f.data_ptr() for f in frames]
        for f in frames:
            if not isinstance(f, int) and (f.dtype.itemsize != 4 or not f.is_contiguous() or
                                           f.numel() != width * height):
                raise ValueError("frames must be contiguous float32 tensors of height x width")
        starsim_render_band_to(self.h, x, y, mag, width, height, row0, rows, sigma, roi, gain, ptrs, stream)

    def route_band(self, x, y, mag, height, row0, rows, roi, out=None, stream=None):
        """Device band routing (starsim_route_band): returns (x_r, y_r, mag_r, n_dev) -- capacity len(x) arrays whose
        first n_dev[0] entries are the stars routed to rows [row0, row0+rows), in catalogue order, and the count as a
        one-element int32 CUDA tensor (not read back)."""
        import torch
        n = int(x.numel())
        if out is None:
            out = tuple(torch.empty(max(n, 1), dtype=torch.float32, device=x.device) for _ in range(3)) + (
                torch.empty(1, dtype=torch.int32, device=x.device),)
        xo, yo, mo, nd = out
        starsim_route_band(self.h, x, y, mag, height, row0, rows, roi, xo, yo, mo, nd, stream)
        return xo, yo, mo, nd

    def set_star_count(self, n_dev=None):
        """Tiled renders take the first n_dev[0] stars (device int32 tensor) of their catalogue; None clears."""
        starsim_set_star_count(self.h, n_dev)
        self._n_dev = n_dev  # the library keeps the pointer: hold the tensor

    def render_band_routed(self, x, y, mag, width, height, row0, rows, sigma, roi, gain, out=None, frames=None,
                           stream=None):
        """Route the catalogue to the band on the device, then render the band from the routed stars (the device
        count is read by the kernels: no host round trip).  Into `out` (rows x width), or -- with `frames` -- into
        every full frame of `frames` (the fused exchange, as render_band_to).  Bitwise the band of render_band on the
        whole catalogue.  The routed buffers are cached per capacity so repeated calls replay one CUDA graph."""
        import torch
        n = int(x.numel())
        key = (n, x.device)
        if getattr(self, "_route_key", None) != key:
            self._route_buf = tuple(torch.empty(max(n, 1), dtype=torch.float32, device=x.device) for _ in range(3)) + (
                torch.empty(1, dtype=torch.int32, device=x.device),)
            self._route_key = key
        xo, yo, mo, nd = self.route_band(x, y, mag, height, row0, rows, roi, out=self._route_buf, stream=stream)
        xo, yo, mo = xo[:n], yo[:n], mo[:n]
        self.set_star_count(nd)
        try:
            if frames is not None:
                self.render_band_to(xo, yo, mo, width, height, row0, rows, sigma, roi, gain, frames, stream)
                return None
            return self.render_band(xo, yo, mo, width, height, row0, rows, sigma, roi, gain, out, stream)
        finally:
            self.set_star_count(None)

    def render_atomic(self, x, y, mag, width, height, sigma, roi, gain, out=None, stream=None):
        out = self._out(height, width, out)
        starsim_render_atomic(self.h, x, y, mag, width, height, sigma, roi, gain, out, stream)
        return out

    def render_lut(self, x, y, mag, width, height, sigma, roi, gain, out=None, stream=None):
        out = self._out(height, width, out)
        starsim_render_lut(self.h, x, y, mag, width, height, sigma, roi, gain, out, stream)
        return out

    def upload_aos(self, host_aos, stream=None):
        import torch
        n = int(np.asarray(host_aos).shape[0])
        dev = f"cuda:{self.device}"
        x, y, m = (torch.empty(n, dtype=torch.float32, device=dev) for _ in range(3))
        starsim_upload_aos(self.h, host_aos, x, y, m, stream)
        return x, y, m

    def quantize(self, img, bits=8, out=None, stream=None):
        import torch
        if out is None:
            out = torch.empty(img.shape, dtype=torch.uint8 if bits == 8 else torch.uint16, device=img.device)
        starsim_quantize(self.h, img, bits, out, stream)
        return out

    def get_bins(self):
        return starsim_get_bins(self.h)

    def profile(self, enable=True):
        starsim_profile(self.h, enable)

    def kernel_times(self):
        return starsim_kernel_times(self.h)
