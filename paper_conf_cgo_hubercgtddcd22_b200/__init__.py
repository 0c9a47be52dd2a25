"""gtr -- a B200-native GPU team runtime for CPU-style OpenMP offload regions.

After Huber et al., "Efficient Execution of OpenMP on GPUs" (CGO 2022).  The
compute path is libgtr.so (CUDA for sm_100a, C ABI in include/gtr.h); this
package is its thin Python binding (`gtr`), device-memory plumbing
(`problems`) and the build script (`build`).  Importing `gtr` fails if the
library has not been built: there is no CPU fallback.
"""
__all__ = ["gtr", "problems", "build"]
