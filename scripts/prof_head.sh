#!/bin/bash
# ncu --set full of the u8 head conv (first k_conv_roll launch of an inference call) + its per-line stall table
ncu --set full --clock-control none --import-source on -k "regex:k_conv_roll" -s 3 -c 1 -o gpurun_out/r02_ncu_head \
  python scripts/infer_profile.py > /dev/null 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_head.ncu-rep > gpurun_out/r02_ncu_head.txt
python scripts/ncu_lines.py gpurun_out/r02_ncu_head.ncu-rep 40 > gpurun_out/r02_ncu_head_lines.txt
