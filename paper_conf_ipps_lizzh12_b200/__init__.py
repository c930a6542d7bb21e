"""B200-native (sm_100a) star-image renderer: the star intensity model with Gaussian blur of Li et al. (IPDPS-W 2012).

The product is ``libstarsim.so`` (C ABI in ``include/starsim.h``; kernels in ``csrc/``); :mod:`.starsim` is its thin
ctypes binding.  :mod:`.dist` renders horizontal bands per GPU (device-routed catalogue) and assembles them with an
NCCL all-gather or the fused peer-memory exchange.
"""
from .starsim import (Context, StarsimError, starsim_create, starsim_destroy, starsim_last_error, starsim_render,
                      starsim_render_band, starsim_render_band_to, starsim_render_gray, starsim_render_atomic,
                      starsim_render_lut, starsim_route_band, starsim_set_star_count, starsim_set_psf,
                      starsim_set_roi, starsim_set_binning, starsim_set_tile_kernel, starsim_upload_aos,
                      starsim_quantize, starsim_get_bins, starsim_profile, starsim_kernel_times, LIB_PATH, KCLASSES)

__all__ = ["Context", "StarsimError", "starsim_create", "starsim_destroy", "starsim_last_error", "starsim_render",
           "starsim_render_band", "starsim_render_band_to", "starsim_render_gray", "starsim_render_atomic",
           "starsim_render_lut", "starsim_route_band", "starsim_set_star_count", "starsim_set_psf", "starsim_set_roi",
           "starsim_set_binning", "starsim_set_tile_kernel", "starsim_upload_aos", "starsim_quantize",
           "starsim_get_bins", "starsim_profile", "starsim_kernel_times", "LIB_PATH", "KCLASSES"]
