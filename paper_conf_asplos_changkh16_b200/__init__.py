"""DySel on B200: micro-profiled dynamic selection among SpMV / SGEMM variants.

The product is libdysel.so (C ABI: include/dysel.h; kernels: csrc/).  This
package is its thin Python binding (`dysel.py`) plus the in-tree build
(`build.py`).  Importing `paper_conf_asplos_changkh16_b200.dysel` loads the
library and fails loudly when it is missing.
"""
import os

LIB_PATH = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libdysel.so")


def load():
    from . import dysel
    return dysel
