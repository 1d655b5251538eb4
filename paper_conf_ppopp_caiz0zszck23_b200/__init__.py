"""DSP's collective sampling primitive (CSP) + feature gather on B200.

The product is ``libdsp.so`` (CUDA C++ for sm_100a behind the C ABI of
``include/dsp.h``); this package is its thin ctypes binding (``dsp``).  It
never imports ``oracle/`` and has no CPU fallback.
"""
from .dsp import (  # noqa: F401
    ABI_SYMBOLS, Block, DSPError, LocalGroup, Sampler, dsp_abi_version, dsp_create, dsp_destroy,
    dsp_export_handle, dsp_gather_features, dsp_import_handles, dsp_last_error, dsp_load_partition,
    dsp_load_weights, dsp_random_walk, dsp_set_option, dsp_set_persistent_blocks, dsp_load_features_tiered,
    dsp_pipeline_flush, dsp_reserve, dsp_reserve_layerwise, dsp_sample, dsp_sample_bounds, dsp_sample_bounds_layerwise, dsp_sample_gather, dsp_sample_group, dsp_status_str, dsp_sync, lib,
    torch_exchange)
from . import dsp  # noqa: F401
