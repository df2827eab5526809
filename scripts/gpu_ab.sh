#!/bin/bash
# parity subset on the in-tree lib, then interleaved A/B of abtest/lib_*.so
mkdir -p gpurun_out
timeout 900 python -m pytest ${AB_TESTS:-tests/test_parity_gpu.py tests/test_parity_bench_sizes.py} -x -q > gpurun_out/ab_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/ab_pytest.log
tail -4 gpurun_out/ab_pytest.log
AB_CFGS="${AB_CFGS:-c3 c2 c5}" bash scripts/ab.sh
