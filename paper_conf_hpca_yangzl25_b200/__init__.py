"""B200-native hot path of Buffalo (HPCA'25): C-ABI library libbuffalo.so + thin binding.

Modules: `buffalo` (ctypes binding of include/buffalo.h), `train` (epoch driver),
`build_lib` (nvcc build of the sm_100a library).  Importing the package does not load the
library; `buffalo.lib()` does, and fails loudly without it or without a GPU.
"""
__all__ = ["buffalo", "train", "build_lib"]
