#!/bin/bash
# interleaved A/B over (lib, env) pairs: AB_RUNS="a:abtest/lib_a.so: f:abtest/lib_f.so: fnoga:abtest/lib_f.so:MAGIS_NOGA=1"
for rep in 1 2; do
for c in ${AB_CFGS:-c3}; do
for run in $AB_RUNS; do
  IFS=: read -r name lib envs <<< "$run"
  v=$(env MAGIS_LIB=$lib $envs timeout 300 python bench.py --config $c --steps ${AB_STEPS:-10} --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'): d=json.loads(l); print('%.4g cand/s  %.4f ms  smem %s block %s' % (d['value'], d['roofline']['kernel_ms_avg'], d['setup']['smem_bytes'], d['setup']['block']))")
  echo "$c $name $v"
done; done; done
