#!/bin/bash
# ncu --set full of the original T-GCN's tcgen05 [A1|A2]·W kernel (NEXT-2), summarised on the box
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:k_tc_catmm_pipe" -s 3 -c 3 -o gpurun_out/ncu_k_tc_catmm_pipe python scripts/tgcn2_probe.py --config C5 \
  --epochs 0 > gpurun_out/ncu_k_tc_catmm_pipe.log 2>&1
python scripts/ncu_extract.py "gpurun_out/ncu_k_tc_catmm_pipe.ncu-rep" > gpurun_out/ncu_catmm.json 2>&1
rm -f gpurun_out/*.ncu-rep
