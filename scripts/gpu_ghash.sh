#!/bin/bash
# NEXT-2 round trip: GraphHash parity tests, bench lines per config, one ncu capture.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_graphhash_gpu.py -x -q > gpurun_out/pytest_ghash.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_ghash.log
tail -15 gpurun_out/pytest_ghash.log
for c in c2 c5 c3 c4; do for C in level topo; do
  MAGIS_GH_ORDER=$C MAGIS_DEBUG=1 timeout 600 python bench.py --ghash --config $c --K 65536 --steps 10 --warmup 3 ${GH_ARGS} > gpurun_out/bench_ghash_${c}_C$C.log 2>&1
  grep "ghash NT" gpurun_out/bench_ghash_${c}_C$C.log | head -1
  python - gpurun_out/bench_ghash_${c}_C$C.log <<"PY"
import json,sys
for line in open(sys.argv[1]):
    if line.startswith('{'):
        d=json.loads(line); r=d['roofline']
        print(' %s value %.4g cand/s kern %.3f ms frac %.4f e2e %s cpu %s' % (sys.argv[1], d['value'], r['kernel_ms_avg'], r['frac'], d['e2e']['value'], (d.get('cpu_baseline') or {}).get('value')))
    elif 'Error' in line or 'error' in line: print(' ', line.strip()[:300])
PY
done; done
if [ -n "$GH_NCU" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ghash_kernel -s 2 -c 1 -o gpurun_out/prof_ghash python bench.py --ghash --config c2 --K 65536 --steps 2 --warmup 2 --no-cpu-baseline > gpurun_out/ncu_ghash.log 2>&1
fi
