"""paper_conf_ipps_allenf019_b200 -- B200-native Slate slate-kernel path.

The product is the CUDA/C++ library ``libslate.so`` (C ABI in
``include/slate.h``); ``slate`` is its thin ctypes binding and ``inputs`` the
seeded synthetic input generator.  Import ``paper_conf_ipps_allenf019_b200.slate``
explicitly: it raises if the library has not been built (no CPU fallback).
"""
__all__ = ["slate", "inputs", "build"]
