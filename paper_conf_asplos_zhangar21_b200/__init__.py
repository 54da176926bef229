"""B200-native GPU virtual-function dispatch after "Judging a Type by Its Pointer:
Optimizing GPU Virtual Functions" (Zhang, Alawneh, Rogers, ASPLOS'21).

The product is libvf.so (C ABI: include/vf.h), hand-written CUDA for sm_100a.
``vf`` is its ctypes binding and ``apps`` the workload drivers. Importing this
package does not load the library; ``vf.lib()`` / ``vf.Ctx()`` do, and fail
loudly when it is missing (there is no CPU fallback).
"""
__all__ = ["vf", "apps", "build"]
