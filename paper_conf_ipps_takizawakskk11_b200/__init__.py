"""B200-native CheCL device-state snapshot (Takizawa et al., IPDPS 2011).

libchecl.so (C ABI in include/checl.h) does the work; `checl` is its binding and
`coordination` the multi-rank commit barrier.
"""
from . import checl  # noqa: F401  (raises ImportError when libchecl.so is missing)
from .checl import CheclError, Context, Image, Report  # noqa: F401
