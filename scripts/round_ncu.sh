#!/bin/bash
# ncu --set full of the hot kernels (scripts/ncu_capture.sh), summarised on the box
# (ncu_extract.py, SASS stall tops); the reports themselves are deleted (gpurun_out <= 64 MiB)
bash scripts/ncu_capture.sh
python scripts/ncu_extract.py > gpurun_out/ncu_full.json 2>&1
for r in gpurun_out/ncu_k_*.ncu-rep; do
  k=$(basename $r .ncu-rep)
  python scripts/ncu_src_top.py $r sass 25 > gpurun_out/src_$k.txt 2>&1
done
rm -f gpurun_out/*.ncu-rep
