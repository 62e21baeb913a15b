"""B200-native SPH time step (libsph) for the method measured in Simsek,
Piccinali and Ciorba, SC'24 workshops (SPH-EXA GPU frequency scaling).

Submodules:
  ics   seeded initial conditions and step parameters (no method arithmetic)
  sph   ctypes binding of include/sph.h (loads lib/libsph.so; no CPU fallback)

Nothing is imported eagerly so that ``ics`` can be used without a GPU.
"""

__all__ = ["ics", "sph"]


def __getattr__(name):
    if name in __all__:
        import importlib
        return importlib.import_module(f"{__name__}.{name}")
    raise AttributeError(name)
