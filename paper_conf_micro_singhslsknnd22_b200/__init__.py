"""B200-native (sm_100a) Skipper SNN training hot path.

The compute lives in libskipper.so (C ABI: include/skipper.h); `skipper` is a
thin ctypes binding.  Using any name exported here loads the library and fails
loudly if it has not been built (no CPU fallback).  The names resolve lazily so
that `paper_conf_micro_singhslsknnd22_b200.build` can run before the library
exists.
"""
_EXPORTS = (
    "SkipperNet", "SkipperError", "lib", "sst_host", "workspace_bytes", "make_config", "make_layers",
    "k_fc_fwd", "k_fc_wgrad", "k_conv_fwd", "k_conv_dgrad", "k_conv_wgrad", "k_narrow_wgrad", "k_narrow_dgrad", "k_conv_lif", "k_conv_s", "encode_poisson",
    "PASS_FIRST", "PASS_RECOMPUTE", "PASS_RECORD",
)
__all__ = list(_EXPORTS)


def __getattr__(name):
    if name in _EXPORTS:
        from . import skipper
        return getattr(skipper, name)
    raise AttributeError(name)
