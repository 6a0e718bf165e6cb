timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:k_tc_atb2" -s 2 -c 2 -o gpurun_out/ncu_atb2_lo python scripts/profile_seq.py --S 4 --seqs 1 > gpurun_out/ncu_atb2_lo.log 2>&1
tail -2 gpurun_out/ncu_atb2_lo.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -3 gpurun_out/pytest_gpu.log
