#!/bin/bash
# One `ncu --set full` capture per hot kernel of a steady-state C5 sequence (1 GPU).
# Reports land in gpurun_out/ncu_<name>.ncu-rep; scripts/ncu_extract.py summarises them.
set -u
for k in k_agg_stream k_tc_gru_bwd2 k_tc_atb2 k_tc_gru_fwd2 k_tc_xw_pipe k_merge_old; do
  timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 2 -c 1 -o gpurun_out/ncu_$k python scripts/profile_seq.py --S 4 --seqs 1 \
    > gpurun_out/ncu_$k.log 2>&1
done
