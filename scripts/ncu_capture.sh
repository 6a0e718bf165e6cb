#!/bin/bash
# One `ncu --set full` capture per hot kernel (1 GPU): the TGCN kernels of a steady-state
# C5 sequence (scripts/profile_seq.py), the snapshot kernels of a C5 delta step
# (scripts/snapshot_probe2.py) and the original T-GCN's tcgen05 kernels (scripts/tgcn2_probe.py).
# Reports land in gpurun_out/ncu_<name>.ncu-rep; scripts/ncu_extract.py summarises them.
set -u
for k in k_agg_stream k_tc_gru_bwd2 k_tc_dl3 k_tc_atb2 k_tc_gru_fwd2 k_tc_xw_pipe; do
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 2 -c 2 -o gpurun_out/ncu_$k python scripts/profile_seq.py --S 4 --seqs 1 \
    > gpurun_out/ncu_$k.log 2>&1
done
for k in k_merge4 k_touch3 k_rowscan k_ids_scatter k_ids_finish k_items2; do
  PROBE_NCU=1 timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 2 -c 1 -o gpurun_out/ncu_$k python scripts/snapshot_probe2.py > gpurun_out/ncu_$k.log 2>&1
done
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
  -k "regex:k_tc_catmm_pipe" -s 3 -c 3 -o gpurun_out/ncu_k_tc_catmm_pipe python scripts/tgcn2_probe.py --config C5 \
  --epochs 0 > gpurun_out/ncu_k_tc_catmm_pipe.log 2>&1
