"""B200-native active-gradient-offloading AdamW step (Ratel, ICDE 2025).

The product is libratel.so (include/ratel.h); `ratel` is its ctypes binding
and `api` the PyTorch-facing wrappers named after the paper's user API
(Fig. 4).  Importing this package loads the CUDA
library and fails loudly if it is missing -- there is no CPU fallback.
"""
from . import ratel  # noqa: F401  (loads libratel.so)
from .ratel import *  # noqa: F401,F403
