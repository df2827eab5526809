#!/bin/bash
# Round-2 evidence for profiles/r02: GPU suite, smoke, bench lines for every
# config and mode (cpu_baseline with parity on the oracle's sample), the
# oracle arm, the ncu launch list of the default bench, ncu --set full of the
# eval kernel on C3 (default, tier 1), C2 (tier 0) and C4 (tier 2) with
# per-line / stall / phase summaries and the DRAM traffic record.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvidia-smi --query-gpu=index,name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -2 gpurun_out/smoke.log
run() { name=$1; shift; timeout 900 python bench.py "$@" > gpurun_out/bench_$name.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$name.log
  grep '^{' gpurun_out/bench_$name.log > gpurun_out/bench_$name.json; echo -n "$name: "; python scripts/jq_line.py < gpurun_out/bench_$name.log; }
run c3 --steps 10 --warmup 3
run c1 --config c1 --steps 20 --warmup 3
run c2 --config c2 --steps 10 --warmup 3
run c4 --config c4 --steps 5 --warmup 3
run c5 --config c5 --steps 10 --warmup 3
run c3f --config c3f --steps 5 --warmup 3
run windows --windows --steps 10 --warmup 3 --no-cpu-baseline
run ghash_c2 --ghash --config c2 --steps 10 --warmup 3
run ghash_c4 --ghash --config c4 --steps 5 --warmup 3 --no-cpu-baseline
run ref --impl reference --steps 3 --warmup 1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c3.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
python scripts/launch_summary.py gpurun_out/launches_c3.csv "ncu --metrics gpu__time_duration.sum --clock-control none python bench.py --steps 3 --warmup 3 (c3, K=262144)" > gpurun_out/launches_summary.txt 2>&1
cat gpurun_out/launches_summary.txt
for ck in c3:262144 c2:65536 c4:16384; do c=${ck%%:*}; K=${ck#*:}
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 3 -c 1 -o gpurun_out/full_$c python bench.py --config $c --K $K --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_$c.log 2>&1
  python scripts/ncu_summary.py gpurun_out/full_$c.ncu-rep 30 > gpurun_out/ncu_full_eval2_$c.txt 2>&1
  python scripts/ncu_phases.py gpurun_out/full_$c.ncu-rep $K > gpurun_out/ncu_phases_eval2_$c.txt 2>&1
  python scripts/ncu_lines.py gpurun_out/full_$c.ncu-rep $K 60 > gpurun_out/ncu_lines_eval2_$c.txt 2>&1
  python scripts/ncu_stalls.py gpurun_out/full_$c.ncu-rep 40 > gpurun_out/ncu_stalls_eval2_$c.txt 2>&1
  python scripts/ncu_traffic_update.py gpurun_out/full_$c.ncu-rep $c $K gpurun_out/ncu_traffic.json
  rm -f gpurun_out/full_$c.ncu-rep
done
du -sh gpurun_out
