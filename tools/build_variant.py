"""Build a diagnostic variant of the library: only the tile-kernel units are
recompiled with extra -D flags, the rest is linked from the shipped build.
  python tools/build_variant.py NAME -DFLAG1 -DFLAG2 ...  ->  paper_conf_sc_asahilbpbgo24_b200/libsb_NAME.so"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_sc_asahilbpbgo24_b200 import build as b  # noqa: E402

name, flags = sys.argv[1], tuple(sys.argv[2:])
print(b.build(extra_flags=flags, lib=os.path.join(b.HERE, f"libsb_{name}.so"),
              build_dir=os.path.join(b.HERE, f"_build_{name}"), only=("tile_f64.cu", "tile_f32.cu")))
