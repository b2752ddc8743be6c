"""B200-native TOAST pointing->map hot path (Demeure et al., SC-W 2023).

The compute lives in the C-ABI library ``libtoastb200.so`` (hand-written
sm_100a CUDA, declared in ``include/toast_b200.h``); ``binding`` is the thin
ctypes layer with the same entry-point names.  Import of the package itself is
cheap: the shared library loads on first use of ``binding``.
"""
__all__ = ["binding", "synth", "dist"]
