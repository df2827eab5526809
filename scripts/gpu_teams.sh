mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_parity_gpu.py -x -q > gpurun_out/pytest_teams.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_teams.log
tail -4 gpurun_out/pytest_teams.log
for c in c2 c5; do for t in 2 1; do
  MAGIS_DEBUG=1 MAGIS_TEAMS=$t timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_teams_${c}_$t.log 2>&1
  echo "$c teams=$t: $(grep -o '"value": [0-9.e+]*' gpurun_out/bench_teams_${c}_$t.log | head -1) $(grep -o '"kernel_ms_avg": [0-9.]*' gpurun_out/bench_teams_${c}_$t.log) $(grep 'eval2 P=' gpurun_out/bench_teams_${c}_$t.log | tail -1)"
done; done
