"""B200-native LC-style lossless floating-point codecs (SPspeed, SPratio,
DPspeed, DPratio) after Azami, Fallin & Burtscher, ASPLOS '25.

The product is the C-ABI library `liblcf.so` (include/lcf.h) built from
`csrc/`; `lcf` is its thin ctypes binding. Submodules are imported lazily so
that `datagen` can be used without loading the CUDA library.
"""

__all__ = ["lcf", "datagen", "sharded"]


def __getattr__(name):
    if name in __all__:
        import importlib
        return importlib.import_module(f"{__name__}.{name}")
    raise AttributeError(name)
