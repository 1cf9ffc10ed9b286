"""libctaclust -- locality-aware CTA clustering (Li et al., ASPLOS'17) for B200.

The compute path lives in the C-ABI shared library ``libctaclust.so`` (built
from ``csrc/`` for sm_100a); :mod:`.ctaclust` is a thin ctypes binding with the
same names.  The library is loaded lazily on first use and a missing library is
an error -- there is no CPU fallback.
"""
__all__ = ["synth"]


def __getattr__(name):
    if name in ("ctaclust", "lib"):
        from . import ctaclust
        return ctaclust
    raise AttributeError(name)
