#!/bin/bash
# TGCN parity tests + default bench + dL A/B
timeout 1200 python -m pytest tests/test_gpu_tgcn.py tests/test_gpu_peer.py tests/test_gpu_tc.py -m gpu -x -q > gpurun_out/pytest_tgcn.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_tgcn.log
timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_default.log 2>&1
STG_DL3=0 timeout 900 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench_dl_old.log 2>&1
timeout 900 python bench.py --mode peer --no-e2e --no-cpu-baseline > gpurun_out/bench_peer_n1.log 2>&1
