#!/bin/bash
# Round-end style check: pytest -m gpu, smoke, default bench, reference arm, torchrun line
# through the NCCL path (SB_BENCH_FORCE_DIST=1), ncu launch list and one ncu --set full of C2
O=gpurun_out/fin
mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.limit --format=csv > $O/gpu.txt 2>&1
cp MEASURED_PEAKS.json $O/ 2>/dev/null
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $O/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log
timeout 600 python bench.py > $O/bench_C2.json 2> $O/bench_C2.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $O/reference_C2.json 2> $O/reference_C2.err
SB_BENCH_FORCE_DIST=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 20 --warmup 3 --no-cpu-baseline > $O/bench_torchrun_n1.json 2> $O/bench_torchrun_n1.err
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 30 --csv --log-file $O/ncu_launches_C2.csv python bench.py --steps 6 --warmup 3 --no-cpu-baseline --no-e2e > $O/ncu_launches_C2.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:sb_ -s 2 -c 1 -o $O/prof_C2 -f python tools/prof_run.py --workload C2 --n 3 > $O/prof_C2.log 2>&1
tail -3 $O/pytest_gpu.log; tail -5 $O/smoke.log; tail -c 400 $O/bench_C2.json; tail -c 300 $O/bench_torchrun_n1.json
