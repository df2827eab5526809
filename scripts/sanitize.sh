#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck of the eval path on every
# plan tier (C2 / C5, and C4 on tier 2) -- summary in gpurun_out/sanitizer.txt
mkdir -p gpurun_out
out=gpurun_out/sanitizer.txt
: > $out
run() {  # tool cfg K env...
  tool=$1; cfg=$2; K=$3; shift 3
  res=$(env "$@" timeout 1200 compute-sanitizer --tool $tool --racecheck-report hazard python scripts/dbg_small.py $cfg $K 2>&1 | grep -E "mismatches|SUMMARY|Error|error" | tr '\n' ' ')
  echo "$tool $cfg K=$K ${*:-auto} :: $res" | tee -a $out
}
for cfg in c2 c5; do
  run memcheck $cfg 2048 MAGIS_TEAMS=1
  run synccheck $cfg 2048 MAGIS_TEAMS=1
  run racecheck $cfg 512 MAGIS_TEAMS=1
  for tv in "MAGIS_TIER=1 MAGIS_P=4" "MAGIS_TIER=2 MAGIS_P=1" "MAGIS_TIER=3 MAGIS_P=2" "MAGIS_P=2 MAGIS_TEAMS=2"; do
    run synccheck $cfg 1024 MAGIS_TEAMS=1 $tv
    run racecheck $cfg 512 MAGIS_TEAMS=1 $tv
  done
done
# tier 1 with the staged row tables (rows_sm) and the device generator (a1)
run synccheck c3 512 MAGIS_TIER=1
run racecheck c3 256 MAGIS_TIER=1
gen() {  # tool cfg K
  res=$(timeout 1200 compute-sanitizer --tool $1 python scripts/dbg_gen.py $2 $3 2>&1 | grep -E "mismatches|SUMMARY|Error|error" | tr '\n' ' ')
  echo "$1 generator $2 K=$3 :: $res" | tee -a $out
}
gen memcheck c2 1024
gen racecheck c2 512
gen memcheck c4 128
run memcheck c4 256
run synccheck c4 256
run racecheck c4 160
