#!/bin/bash
# ncu --set full of the inference residual block, the training data-gradient rolling conv and the batched weight
# gradient, then their per-source-line stall tables (scripts/ncu_lines.py)
ncu --set full --clock-control none --import-source on -k "regex:k_resblock" -s 10 -c 1 -o gpurun_out/r02_ncu_resblock48b \
  python scripts/infer_profile.py > /dev/null 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_resblock48b.ncu-rep > gpurun_out/r02_ncu_resblock48b.txt
python scripts/ncu_lines.py gpurun_out/r02_ncu_resblock48b.ncu-rep 40 > gpurun_out/r02_ncu_resblock48b_lines.txt
ncu --set full --clock-control none --import-source on -k "regex:k_conv_roll" -s 40 -c 1 -o gpurun_out/r02_ncu_train_dgradb \
  python scripts/train_eager.py 3 > /dev/null 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_train_dgradb.ncu-rep > gpurun_out/r02_ncu_train_dgradb.txt
python scripts/ncu_lines.py gpurun_out/r02_ncu_train_dgradb.ncu-rep 40 > gpurun_out/r02_ncu_train_dgradb_lines.txt
ncu --set full --clock-control none --import-source on -k "regex:k_wgrad_multi" -s 1 -c 1 -o gpurun_out/r02_ncu_train_wgradb \
  python scripts/train_eager.py 3 > /dev/null 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_train_wgradb.ncu-rep > gpurun_out/r02_ncu_train_wgradb.txt
python scripts/ncu_lines.py gpurun_out/r02_ncu_train_wgradb.ncu-rep 40 > gpurun_out/r02_ncu_train_wgradb_lines.txt
