#!/bin/bash
# Evidence for profiles/: full bench line, launch list (ncu, cold/serialised), one full ncu capture.
mkdir -p gpurun_out
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_full.log 2>&1; echo "rc=$?" >> gpurun_out/bench_full.log
for c in c3 c5; do timeout 900 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
timeout 900 python bench.py --config c4 --K 8192 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c4.log 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_ref.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 3 -c 1 -o gpurun_out/prof_eval python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
tail -c 2500 gpurun_out/bench_full.log
for f in gpurun_out/bench_c*.log gpurun_out/bench_ref.log; do echo $f; grep -o '"value": [0-9.e+]*, "unit"[^,]*' $f | head -1; grep -o '"frac": [0-9.]*' $f; done
timeout 600 python bench.py --windows --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_windows.log 2>&1
grep -o '"value": [0-9.e+]*' gpurun_out/bench_windows.log | head -1
