#!/bin/bash
# Device generator (a1): byte-identity tests against the CPU generator, then
# the time per 65,536 candidates on every config.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_parity_gpu.py -k generator -x -q > gpurun_out/pytest_gen.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gen.log
tail -3 gpurun_out/pytest_gen.log
timeout 900 python scripts/gen_time.py c2 c5 c3 c4 2>&1 | tee gpurun_out/gen_time.log
