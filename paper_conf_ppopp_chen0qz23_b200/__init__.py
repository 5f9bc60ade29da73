"""B200-native elastic-averaging step of AvgPipe (PPoPP'23), behind a C ABI.

The compute path is ``libavgpipe_ea.so`` (hand-written sm_100a CUDA + NCCL,
declared in ``include/ea.h``); ``binding`` is a thin ctypes layer that only
marshals torch tensors / streams into that ABI.  There is no CPU fallback:
every entry point fails loudly if the library is missing.
"""
from .synth import CONFIGS, MODES, mode_coeffs, stage_split  # noqa: F401

__all__ = ["CONFIGS", "MODES", "mode_coeffs", "stage_split"]
