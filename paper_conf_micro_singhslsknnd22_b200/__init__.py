"""B200-native (sm_100a) Skipper SNN training hot path.

The compute lives in libskipper.so (C ABI: include/skipper.h); `skipper` is a
thin ctypes binding.  Importing this package fails loudly if the library has
not been built (no CPU fallback).
"""
from .skipper import (  # noqa: F401
    SkipperNet, SkipperError, lib, sst_host, workspace_bytes, make_config, make_layers,
    k_fc_fwd, k_fc_wgrad, k_conv_fwd, k_conv_dgrad, k_conv_wgrad, k_conv_lif,
    PASS_FIRST, PASS_RECOMPUTE, PASS_RECORD,
)
