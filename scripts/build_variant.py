"""Build liblf.so with extra compile flags into another path (A/B experiments):
python scripts/build_variant.py OUT.so -DLF_ROWS_T=128 -DLF_ROWS_BUD=1024 ...
then run with LF_LIB_PATH=OUT.so."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_0002s22_b200 import _build  # noqa: E402

out = os.path.abspath(sys.argv[1])
_build.FLAGS = [*sys.argv[2:], *_build.FLAGS]
_build.LIB = out
_build.OBJ = out + ".objs"
_build.build(force=True, verbose=True)
