"""B200-native cellular batching (BatchMaker, EuroSys'18): the C-ABI library libbm.so
(include/bm.h: C++ scheduler + sm_100a kernels) and its thin Python binding `bm`."""
from . import bm  # noqa: F401  (raises if libbm.so is missing: there is no fallback)

__all__ = ["bm"]
