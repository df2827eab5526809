#!/bin/bash
# A/B timing of alternative builds (abtest/lib_*.so via MAGIS_LIB), interleaved, same box.
mkdir -p gpurun_out
for rep in 1 2; do
for c in ${AB_CFGS:-c2 c5}; do
for lib in ${AB_LIBS:-abtest/lib_*.so}; do
  v=$(MAGIS_LIB=$lib timeout 300 python bench.py --config $c --steps ${AB_STEPS:-10} --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'): d=json.loads(l); print('%.4g cand/s  %.4f ms' % (d['value'], d['roofline']['kernel_ms_avg']))")
  echo "$c $lib $v"
done; done; done
