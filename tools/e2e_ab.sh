#!/bin/bash
# PCIe ceiling (tools/pcie_probe.py) and the e2e line of the default bench for
# several host pipeline chunk sizes (SB_HOST_CHUNK_MB)
O=gpurun_out/${O:-e2e}
mkdir -p $O
timeout 120 python tools/pcie_probe.py > $O/pcie_probe.txt 2>&1
cat $O/pcie_probe.txt
for mb in ${MBS:-16 32 64 128}; do
  SB_HOST_CHUNK_MB=$mb timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --extra none --e2e-steps 5 > $O/bench_mb$mb.json 2> $O/bench_mb$mb.err
  python -c "import json; d=json.load(open('$O/bench_mb$mb.json')); print('chunk $mb MB', d['e2e'])" 2>/dev/null || echo "chunk $mb failed"
done
