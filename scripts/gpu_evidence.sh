#!/bin/bash
# Round-end evidence for profiles/: GPU suite, smoke, bench lines for every
# config and mode, the oracle arm, the ncu launch list, ncu --set full of the
# eval kernel on C2 (tier 0), C3 (tier 1) and C4 (tier 2).
mkdir -p gpurun_out
nvidia-smi --query-gpu=index,name,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv > gpurun_out/smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -2 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -2 gpurun_out/smoke.log
run() { name=$1; shift; timeout 900 python bench.py "$@" > gpurun_out/bench_$name.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$name.log
  python - gpurun_out/bench_$name.log <<'PY'
import json,sys
for line in open(sys.argv[1]):
    if line.startswith('{'):
        d=json.loads(line); r=d.get('roofline') or {}
        print(' %-28s %.4g %s kern %s ms frac %s e2e %s cpu %s' % (sys.argv[1][11:], d['value'], d['unit'], r.get('kernel_ms_avg'), r.get('frac'), (d.get('e2e') or {}).get('value'), (d.get('cpu_baseline') or {}).get('value')))
PY
}
run full --steps 10 --warmup 3
run c3 --config c3 --steps 5 --warmup 3 --no-cpu-baseline
run c4 --config c4 --steps 5 --warmup 3 --no-cpu-baseline
run c5 --config c5 --steps 10 --warmup 3 --no-cpu-baseline
run windows --windows --steps 10 --warmup 3 --no-cpu-baseline
run c3f --config c3f --steps 5 --warmup 3 --no-cpu-baseline
run ghash_c2 --ghash --config c2 --steps 10 --warmup 3
run ghash_c4 --ghash --config c4 --steps 5 --warmup 3 --no-cpu-baseline
run ref --impl reference --steps 3 --warmup 1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 3 -c 1 -o gpurun_out/prof_eval python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 3 -c 1 -o gpurun_out/prof_eval_c3 python bench.py --config c3 --K 65536 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_c3.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:eval2_kernel -s 3 -c 1 -o gpurun_out/prof_eval_c4 python bench.py --config c4 --K 8192 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_c4.log 2>&1
# summaries on the box (gpurun_out/ must stay < 64 MiB: only the C2 report comes back)
for rk in prof_eval:65536 prof_eval_c3:65536 prof_eval_c4:8192; do r=${rk%%:*}
  python scripts/ncu_summary.py gpurun_out/$r.ncu-rep 30 > gpurun_out/$r.summary.txt 2>&1
  python scripts/ncu_phases.py gpurun_out/$r.ncu-rep ${rk#*:} > gpurun_out/$r.phases.txt 2>&1
done
rm -f gpurun_out/prof_eval_c3.ncu-rep gpurun_out/prof_eval_c4.ncu-rep
du -sh gpurun_out
