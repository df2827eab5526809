#!/bin/bash
# Quick GPU iteration: eval parity tests + bench lines for c2 / c5 / c3 (+ c4 small K), no CPU baseline / e2e.
mkdir -p gpurun_out
timeout 900 python -m pytest ${QUICK_TESTS:-tests/test_parity_gpu.py tests/test_windows_gpu.py} -x -q > gpurun_out/pytest_quick.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_quick.log
tail -4 gpurun_out/pytest_quick.log
for c in ${QUICK_CFGS:-c2 c5 c3}; do
  extra=""; [ $c = c4 ] && extra="--K 8192"
  timeout 600 python bench.py --config $c $extra --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bq_$c.log 2>&1
  python - gpurun_out/bq_$c.log <<'PY'
import json,sys
for line in open(sys.argv[1]):
    if line.startswith('{'):
        d=json.loads(line); r=d['roofline']
        print(' %s value %.4g cand/s kern %.3f ms frac %.4f clocks %s' % (sys.argv[1], d['value'], r['kernel_ms_avg'], r['frac'], d.get('clocks',{}).get('sm_mhz')))
    elif 'Error' in line or 'error' in line: print(' ', line.strip()[:300])
PY
done
[ -n "$QUICK_PROF" ] && bash scripts/prof_quick.sh
exit 0
