#!/bin/bash
# per-kernel launch list of ONE steady-state C5 sequence (S=4) -> gpurun_out/launches_seq.csv + ncu10.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_seq.csv \
  python scripts/profile_seq.py --S 4 --seqs 1 > gpurun_out/ncu10.log 2>&1
