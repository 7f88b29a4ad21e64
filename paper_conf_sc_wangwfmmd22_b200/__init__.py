"""B200-native TT-EmbeddingBag hot path of EL-Rec (SC'22): forward, backward and
core update behind the C ABI of libttemb.so (include/ttemb.h).

Importing this package loads the in-tree CUDA library and fails loudly if it is
missing; there is no CPU fallback.
"""
from ._lib import TTEmbError, load as _load

_load()

from .binding import *  # noqa: E402,F401,F403
from .binding import TTEmbeddingBag  # noqa: E402,F401
