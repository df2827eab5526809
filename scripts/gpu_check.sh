#!/bin/bash
# One GPU round-trip: parity tests, smoke, bench lines for each kernel variant.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 900 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for v in ${BENCH_VARIANTS:-auto}; do
  case $v in
    auto) env="";; v1) env="MAGIS_VARIANT=1";; p1) env="MAGIS_P=1";; p2) env="MAGIS_P=2";; p4) env="MAGIS_P=4";;
  esac
  env $env timeout 600 python bench.py --steps 10 --warmup 3 ${BENCH_ARGS} > gpurun_out/bench_$v.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench_$v.log
done
tail -3 gpurun_out/pytest_gpu.log; tail -2 gpurun_out/smoke.log
for f in gpurun_out/bench_*.log; do echo $f; python - "$f" <<'PY'
import json,sys
for line in open(sys.argv[1]):
    if line.startswith('{'):
        d=json.loads(line); r=d['roofline']
        print(' value %.4g cand/s  op-steps %.4g  kern %.3f ms  frac %.4f  e2e %s  setup %s' % (d['value'], d['op_steps_per_s'], r['kernel_ms_avg'], r['frac'], (d.get('e2e') or {}).get('value'), d['setup']))
    elif 'rc=' in line or 'Error' in line or 'error' in line: print(' ', line.strip()[:300])
PY
done
