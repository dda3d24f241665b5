"""Build an experimental libsam variant with -D overrides (developer tool).
    python tools/build_variant.py NAME -DSAM_LAG_SMALL=20 ...   -> paper_conf_pldi_malekiyb16_b200/lib/var/libsam_NAME.so
Run with SAM_LIB_PATH=<that path> to use it."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_pldi_malekiyb16_b200 import _build as B
name, flags = sys.argv[1], sys.argv[2:]
B.BUILD = os.path.join(B.PKG, "build", "var_" + name)
B.LIBDIR = os.path.join(B.PKG, "lib", "var")
B.LIB = os.path.join(B.LIBDIR, f"libsam_{name}.so")
print(B.build(force=True, extra=flags))
