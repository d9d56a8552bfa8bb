"""Build librafd.so from another csrc directory (same-session A/B of kernel
variants; the binding loads it with RAFD_LIB=<path>).

    python tools/build_variant.py <csrc_dir> <out.so>
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_stoltzfushsld21_b200 import build as b  # noqa: E402

src, out = os.path.abspath(sys.argv[1]), os.path.abspath(sys.argv[2])
b.CSRC = src
b.LIB = out
b.OBJ = out + ".objs"
b.build(force=True)
print(out)
