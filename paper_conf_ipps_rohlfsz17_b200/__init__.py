"""B200-native LOO cross-validation bandwidth grid search for univariate
Nadaraya-Watson regression (Rohlfs & Zahran, IPDPSW 2017).

The product is ``libkrcv.so`` (include/krcv.h): hand-written sm_100a CUDA
behind a C-ABI.  This package is its thin Python binding (``krcv``) and the
multi-GPU orchestration over ``torch.distributed`` (``api``).
"""
from .krcv import (  # noqa: F401
    EPANECHNIKOV, TRIANGULAR, UNIFORM, KERNELS, KrcvError,
    kr_cv_grid, kr_cv_shard_async, kr_default_grid, kr_finalize, kr_finalize_async,
    kr_strerror, kr_validate_grid, kr_version, kr_workspace_bytes,
    kr_cv_ci, kr_kde_ci, confidence_intervals,
)
from .api import CVResult, GridSearch, cv_grid  # noqa: F401

__version__ = "0.1.0"
