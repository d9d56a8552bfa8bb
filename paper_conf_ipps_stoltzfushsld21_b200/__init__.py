"""rafd: B200-native room-acoustics FDTD step (Stoltzfus et al., IPDPS'21).

The product is the CUDA C-ABI library librafd.so (include/rafd.h); `rafd` is
its ctypes binding, `inputs` the seeded synthetic-input generators, `build`
the in-tree nvcc build.
"""
from .rafd import Room, RafdError, rafd_create, rafd_slab_plan, rafd_nccl_unique_id  # noqa: F401
