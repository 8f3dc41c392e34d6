"""B200-native batched sparse iterative solver (Kashi et al., IPDPS 2022 hot path).

The product path is libbsolve.so (C ABI, include/bsolve.h) + this thin
binding.  It never imports the CPU oracle (oracle/) and has no CPU fallback.
"""
from .bsolve import (  # noqa: F401
    BsolveError, Solver, lib, probe_smem_bandwidth, probe_fp64, LIB_PATH, ell_layout, ell_values,
    SYS_CONVERGED, SYS_MAXITER, SYS_BREAKDOWN,
)

__all__ = ["Solver", "BsolveError", "lib", "probe_smem_bandwidth", "probe_fp64"]
