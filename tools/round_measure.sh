#!/bin/bash
# Full measurement session: bench lines of every workload, reference arm, ncu
# launch list of the default bench command, ncu --set full of the tile-kernel
# workloads.  Output under gpurun_out/${O:-measure}.
O=gpurun_out/${O:-measure}
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.limit --format=csv > $O/gpu.txt
cp MEASURED_PEAKS.json $O/ 2>/dev/null
python bench.py > $O/bench_C2.json 2> $O/bench_C2.err
for w in ${WL:-C1 C3G C3H C4 C4F32 C4M ADV ADVNU C6 C6NU C5}; do
  python bench.py --workload $w --no-cpu-baseline > $O/bench_$w.json 2> $O/bench_$w.err
done
python bench.py --impl reference --steps 3 --warmup 1 > $O/reference_C2.json 2> $O/reference_C2.err
# launch list of the bench command (cold-cache, serialised: shares, not absolutes)
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 30 --csv \
    --log-file $O/ncu_launches_C2.csv python bench.py --steps 6 --warmup 2 --no-cpu-baseline --no-e2e > $O/ncu_launches_C2.log 2>&1
for w in ${PROF:-C2 C3G C3H}; do
  ncu --set full --clock-control none --import-source on -k regex:sb_ -s 2 -c 1 -o $O/prof_$w -f \
      python tools/prof_run.py --workload $w --n 3 > $O/prof_$w.log 2>&1
done
ls -la $O
