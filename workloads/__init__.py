"""Seeded synthetic inputs shared by the oracle and the CUDA path.

This package holds ONLY input generation (random numbers, sparsity patterns,
shapes).  It contains none of DySel's arithmetic (no SpMV, no GEMM, no format
conversion, no slice planning), so that `oracle/` and the product path can both
import it without sharing any code of the method (task rule ③).
"""
from .generators import *  # noqa: F401,F403
