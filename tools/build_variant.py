"""Build an experimental variant of libgfsl.so (extra nvcc -D flags) next to the real one.
python tools/build_variant.py OUT.so -DGFSL_SEARCH_MIN_BLOCKS=6 ...; then run with GFSL_LIB=OUT.so"""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ppopp_moscovicicp17_b200 import build as B  # noqa: E402

out, extra = sys.argv[1], sys.argv[2:]
cmd = [B.NVCC, *B.ARCH, *B.FLAGS, *extra, "-o", out, *[os.path.join(B.CSRC, f) for f in B.SOURCES]]
r = subprocess.run(cmd, capture_output=True, text=True)
if r.returncode:
    sys.stderr.write(r.stdout + r.stderr)
    sys.exit(1)
print(out)
