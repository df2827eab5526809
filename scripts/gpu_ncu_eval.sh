#!/bin/bash
# ncu --set full of one eval2 launch on config $1 (K $2) with line / stall / phase summaries
mkdir -p gpurun_out
c=${1:-c3}; K=${2:-65536}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 3 -c 1 -o gpurun_out/full_$c python bench.py --config $c --K $K --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_$c.log 2>&1
python scripts/ncu_summary.py gpurun_out/full_$c.ncu-rep 30 > gpurun_out/ncu_full_eval2_$c.txt 2>&1
python scripts/ncu_phases.py gpurun_out/full_$c.ncu-rep $K > gpurun_out/ncu_phases_eval2_$c.txt 2>&1
python scripts/ncu_lines.py gpurun_out/full_$c.ncu-rep $K 60 > gpurun_out/ncu_lines_eval2_$c.txt 2>&1
python scripts/ncu_stalls.py gpurun_out/full_$c.ncu-rep 40 > gpurun_out/ncu_stalls_eval2_$c.txt 2>&1
