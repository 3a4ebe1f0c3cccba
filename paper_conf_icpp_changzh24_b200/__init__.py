"""B200 (sm_100a) implementation of the hot path of GSAP's stochastic block
partitioning (Chang, Zhang & Huang, ICPP'24).

The product is libgsap.so (csrc/, C-ABI in include/gsap.h); ``gsap`` is its
thin ctypes binding.  No CPU fallback exists: calls raise if the library is
not built or no sm_100 device is present.
"""
from . import gsap  # noqa: F401
from .gsap import (GSAP_MERGE, GSAP_MOVE, Context, GsapError, gsap_default_params,  # noqa: F401
                   gsap_partition)
