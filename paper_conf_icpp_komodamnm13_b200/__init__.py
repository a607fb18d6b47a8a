"""B200-native multi-GPU parallel-loop runtime (Komoda et al., ICPP'13 hot path).

The product is the C-ABI library libaccmg.so (include/accmg.h); `accmg` is its thin ctypes
binding. See DESIGN.md.
"""
from . import accmg  # noqa: F401  (fails loudly if libaccmg.so is missing)
