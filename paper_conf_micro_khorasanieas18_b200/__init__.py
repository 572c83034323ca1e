"""B200-native VPPS hot path (Khorasani et al., MICRO'18): persistent forward-backward training kernel
with register-resident weights, driven by per-batch host scripts.  See DESIGN.md and include/vpps.h.

The compute path lives in libvpps.so (csrc/); `vpps` is its ctypes binding.  Importing `vpps`
raises if the library has not been built — there is no CPU fallback.
"""
__all__ = ["vpps"]
