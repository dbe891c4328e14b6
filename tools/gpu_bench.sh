#!/bin/bash
# one GPU session: bench lines + ncu launch list + one ncu --set full capture
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err
for w in ${EXTRA:-C3G C3H C4 C4F32}; do
  python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 12 --csv \
    --log-file gpurun_out/launches_C2.csv python bench.py --steps 4 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/b_ncu.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:sb_ -s 2 -c 1 -o gpurun_out/prof_${TAG:-C2} -f \
    python tools/prof_run.py --workload ${PROFW:-C2} --n 3 > gpurun_out/prof.log 2>&1
