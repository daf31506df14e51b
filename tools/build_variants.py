"""Build experiment variants of libspcg (compile-time knobs) next to the default one.
Each variant is loaded with SPCG_LIB=<path> (tools/exp_iter.py).  Not part of the product."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_maacsh25_b200 import _build as b  # noqa: E402

VARIANTS = {a.split(":")[0]: a.split(":")[1].split(",") for a in sys.argv[1:]}
b.build()
for tag, d in VARIANTS.items():
    print(b.build(defines=d, out=b.LIB.replace("libspcg.so", f"libspcg_{tag}.so")))
