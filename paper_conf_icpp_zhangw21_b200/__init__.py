"""B200-native out-of-core recursive classical Gram-Schmidt QR (Zhang & Wu, ICPP'21).

The product is `librgsqr.so` (C ABI, include/rgsqr.h; CUDA sources in csrc/);
`rgsqr.py` is its ctypes binding.  Build with
``python -m paper_conf_icpp_zhangw21_b200.build``.
"""
from .rgsqr import Handle, RgsqrError, load_library, PRECISIONS, STORAGE, Stats  # noqa: F401

__all__ = ["Handle", "RgsqrError", "load_library", "PRECISIONS", "STORAGE", "Stats"]
