"""Seeded counter-based input generator shared by the oracle side and the CUDA side
(it holds no stencil arithmetic).  See cst_gen.h for the C/CUDA twin."""
from .gen import Layout, at, fill, index, key, make_layout, splitmix64, value  # noqa: F401
