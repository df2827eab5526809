#!/bin/bash
# A/B + source-level ncu of C3 and C2 (text summaries made on the box)
mkdir -p gpurun_out
AB_STEPS=10 AB_CFGS="${AB_CFGS:-c3 c2}" bash scripts/ab.sh
for c in ${PROF_CFGS:-c3 c2}; do
  NCU_NAME=p_$c NCU_CFG=$c bash scripts/ncu_one.sh > /dev/null 2>&1
  python scripts/ncu_lines.py gpurun_out/p_$c.ncu-rep 16384 70 > gpurun_out/p_$c.lines.txt 2>&1
  python scripts/ncu_stalls.py gpurun_out/p_$c.ncu-rep 40 > gpurun_out/p_$c.stalls.txt 2>&1
  python scripts/ncu_summary.py gpurun_out/p_$c.ncu-rep 20 > gpurun_out/p_$c.summary.txt 2>&1
  rm -f gpurun_out/p_$c.ncu-rep
done
