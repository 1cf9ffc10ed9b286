"""libctaclust -- locality-aware CTA clustering (Li et al., ASPLOS'17) for B200.

The compute path lives in the C-ABI shared library ``libctaclust.so`` (built
from ``csrc/`` for sm_100a); :mod:`.ctaclust` is a thin ctypes binding with the
same names, :mod:`.ops` the tensor-level calls tests and bench use, and
:mod:`.synth` the seeded input generators.  The library is loaded lazily on
first use and a missing library is an error -- there is no CPU fallback.
"""
