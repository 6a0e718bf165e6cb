#!/bin/bash
timeout 1200 python -m pytest tests/test_gpu_tgcn.py -m gpu -x -q > gpurun_out/pytest_tgcn.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tgcn.log
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_default.log 2>&1
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_default2.log 2>&1
