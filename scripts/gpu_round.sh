#!/bin/bash
# Full GPU round trip: every GPU test, smoke, bench lines (default + extra configs/modes).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q ${PYTEST_ARGS} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -2 gpurun_out/smoke.log
for spec in ${BENCHES:-"full:"}; do
  name=${spec%%:*}; args=${spec#*:}; args=${args//,/ }
  timeout 900 python bench.py --steps 10 --warmup 3 $args > gpurun_out/bench_$name.log 2>&1; echo "rc=$?" >> gpurun_out/bench_$name.log
  python - gpurun_out/bench_$name.log <<'PY'
import json,sys
for line in open(sys.argv[1]):
    if line.startswith('{'):
        d=json.loads(line); r=d.get('roofline') or {}
        print(' %s value %.4g %s kern %s ms frac %s e2e %s cpu %s' % (sys.argv[1], d['value'], d['unit'], r.get('kernel_ms_avg'), r.get('frac'), (d.get('e2e') or {}).get('value'), (d.get('cpu_baseline') or {}).get('value')))
    elif 'Error' in line or 'error' in line or 'rc=' in line: print(' ', line.strip()[:300])
PY
done
