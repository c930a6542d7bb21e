"""B200-native (sm_100a) star-image renderer: the star intensity model with Gaussian blur of Li et al. (IPDPS-W 2012).

The product is ``libstarsim.so`` (C ABI in ``include/starsim.h``; kernels in ``csrc/``); :mod:`.starsim` is its thin
ctypes binding.  :mod:`.dist` renders horizontal bands per GPU and assembles them with an NCCL all-gather.
"""
from .starsim import (Context, StarsimError, starsim_create, starsim_destroy, starsim_render, starsim_render_band,
                      starsim_render_gray, starsim_render_atomic, starsim_upload_aos, starsim_quantize,
                      starsim_get_bins, starsim_profile, starsim_kernel_times, starsim_set_psf, LIB_PATH, KCLASSES)

__all__ = ["Context", "StarsimError", "starsim_create", "starsim_destroy", "starsim_render", "starsim_render_band",
           "starsim_render_gray", "starsim_render_atomic", "starsim_upload_aos", "starsim_quantize", "starsim_get_bins",
           "starsim_profile", "starsim_kernel_times", "starsim_set_psf", "LIB_PATH", "KCLASSES"]
