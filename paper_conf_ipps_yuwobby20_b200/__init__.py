"""B200-native GDroid: worklist construction of the IDFG on sm_100a (C ABI + ctypes binding).

See DESIGN.md.  Public API: :func:`load` / :class:`App` (binding of include/gdroid.h).
"""
from ._binding import App, GdroidError, BuildStats, lib, load, make_desc  # noqa: F401

__all__ = ["App", "GdroidError", "load", "lib", "make_desc"]
