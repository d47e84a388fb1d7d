"""Build an A/B variant of libhydro_b200.so with extra nvcc defines, as a separate file.

    python tools/build_variant.py NAME -DFOO=1 ...   ->  paper_conf_icppw_pearce18_b200/libhydro_NAME.so
Select it at run time with HYDRO_LIB=<path> (hydro.py).  The default library is rebuilt after.
"""
import os
import shutil
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_icppw_pearce18_b200 import _build as b  # noqa: E402

name, flags = sys.argv[1], sys.argv[2:]
os.environ["HYDRO_NVCC_FLAGS"] = " ".join(flags)
lib = b.build(force=True)
dst = os.path.join(os.path.dirname(lib), f"libhydro_{name}.so")
shutil.copy(lib, dst)
os.environ["HYDRO_NVCC_FLAGS"] = ""
b.build(force=True)
print(dst)
