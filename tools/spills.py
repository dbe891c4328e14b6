"""Print stack/spill info of the tile kernels from the ptxas logs."""
import re
import sys

ROOT = "/root/repo/paper_conf_sc_asahilbpbgo24_b200/_build/"
pat = sys.argv[1] if len(sys.argv) > 1 else "Li1EEEv"
for f in ("tile_f64", "tile_f32", "warp_f64", "warp_f32"):
    cur = None
    for line in open(ROOT + f + ".cu.o.ptxas.txt"):
        m = re.search(r"Compiling entry function '(\S+)'", line)
        if m:
            cur = m.group(1)
        m2 = re.search(r"(\d+) bytes stack frame, (\d+) bytes spill stores", line)
        if m2 and cur and pat in cur:
            print(re.sub(r"_ZN2sb\d+", "", cur)[:48], m2.group(0))
