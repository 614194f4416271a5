"""paper_conf_cluster_sunlyjldlq21_b200 — B200-native complex-stencil sweep + csTuner.

The product is libcst.so (include/cst.h): hand-written sm_100a CUDA kernels for FP64
star / box / hypterm-like stencil sweeps, parameterised by the csTuner optimisation
space (Table I of Sun et al., CLUSTER'21), plus the host C++ tuner and the z-slab
distributed sweep.  This package is the thin ctypes binding (cst.py) and a small
torch-tensor convenience layer (stencil.py).
"""
from .cst import (CST_BOX, CST_HYPTERM, CST_RHS4, CST_STAR, CstError, cst_grid, cst_setting,  # noqa: F401
                  make_grid, version)
from .stencil import Stencil  # noqa: F401
