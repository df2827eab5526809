#!/bin/bash
# round-2 first GPU pass: new parity tests, the full GPU suite, default bench (C3) and C1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_parity_bench_sizes.py tests/test_nccl_gpu.py -q -x --durations=15 > gpurun_out/pytest_new.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_new.log
tail -25 gpurun_out/pytest_new.log
timeout 900 python -m pytest tests -m gpu -q -x --ignore=tests/test_parity_bench_sizes.py > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/bench_c3.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c3.log
tail -c 3000 gpurun_out/bench_c3.log
timeout 300 python bench.py --config c1 --steps 20 --warmup 3 > gpurun_out/bench_c1.log 2>&1; echo "rc=$?" >> gpurun_out/bench_c1.log
tail -c 3000 gpurun_out/bench_c1.log
