# source-level ncu captures of the GRU tcgen05 kernels (steady-state C5 sequence)
for k in k_tc_gru_fwd2 k_tc_gru_bwd2; do
timeout 600 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$k" -s 2 -c 1 -o gpurun_out/ncu_src_$k python scripts/profile_seq.py --S 4 --seqs 1 > gpurun_out/ncu_src_$k.log 2>&1
tail -1 gpurun_out/ncu_src_$k.log
done
