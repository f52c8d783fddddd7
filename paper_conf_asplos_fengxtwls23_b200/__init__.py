"""B200-native Mobius (Feng et al., ASPLOS '23) fine-tuning step.

Python side is a thin binding of libmobius.so (include/mobius.h); see
``api`` for the entry points with the same names as the C ABI.
"""
from . import _lib  # noqa: F401  (raises ImportError when the library is not built)
from .api import *  # noqa: F401,F403
