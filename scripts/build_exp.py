"""Build an experimental copy of libdysel.so with extra -D flags (scratch, not
the product): python scripts/build_exp.py NAME -DFOO=1 ...  ->  exp_libs/NAME/libdysel.so
Load it with DYSEL_LIB=exp_libs/NAME/libdysel.so (scripts only)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_changkh16_b200 import build as B
name, extra = sys.argv[1], sys.argv[2:]
out = os.path.join(B.ROOT, "exp_libs", name)   # git-ignored, not gpurun-ignored
B.OBJ = os.path.join(out, "obj")
B.LIB = os.path.join(out, "libdysel.so")
B.FLAGS = B.FLAGS + extra
print(B.build())
