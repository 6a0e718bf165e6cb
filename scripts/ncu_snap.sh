#!/bin/bash
# ncu --set full of the snapshot-step kernels (one C5 delta step each) + source-level stall tops
set -u
for k in k_merge4 k_touch3 k_rowscan k_ids_scatter k_items2; do
  PROBE_NCU=1 timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 2 -c 1 -o gpurun_out/ncu_$k python scripts/snapshot_probe2.py > gpurun_out/ncu_$k.log 2>&1
  python scripts/ncu_src_top.py gpurun_out/ncu_$k.ncu-rep sass 30 > gpurun_out/src_$k.txt 2>&1
done
python scripts/ncu_extract.py "gpurun_out/ncu_k_*.ncu-rep" > gpurun_out/ncu_snap_full.json 2>&1
