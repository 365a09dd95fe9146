"""B200-native flat embedding cache (Fleche, EuroSys '22) — Python face of libfleche.so.

The product is the C-ABI library built from ``csrc/`` (``include/fleche.h``); this
package only marshals arguments to it (``binding``).  There is no CPU fallback.
"""
from .binding import FlatCache, FlecheError, LIB_PATH, STAT_FIELDS  # noqa: F401

__all__ = ["FlatCache", "FlecheError", "LIB_PATH", "STAT_FIELDS"]
