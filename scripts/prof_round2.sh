#!/bin/bash
# Round-2 measurement evidence (run under gpurun; everything lands in gpurun_out/):
#  1. live CUDA-event GB/s of the memory-bound kernels, then their ncu DRAM bytes per launch;
#  2. ncu --set full of one k_resblock<32> launch (config 2) and of the training kernels (one dgrad k_conv_roll, one
#     fused training k_resblock, the batched k_wgrad_multi);
#  3. the launch list of one bench step (gpu__time_duration per kernel, cold + serialised).
set -x
python scripts/hbm_kernels.py > gpurun_out/r02_hbm_events.json 2> gpurun_out/r02_hbm_events.err
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k "regex:k_adam|k_sample_gather|k_sse_u8|k_conv_roll|k_pack_weights" -c 60 --csv \
  --log-file gpurun_out/r02_ncu_hbm.csv python scripts/hbm_kernels.py > gpurun_out/r02_ncu_hbm.log 2>&1
ncu --set full --clock-control none --import-source on -k "regex:k_resblock" -s 2 -c 1 -o gpurun_out/r02_ncu_resblock32 \
  python scripts/cfg2_profile.py > gpurun_out/r02_ncu_resblock32.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_resblock32.ncu-rep > gpurun_out/r02_ncu_resblock32.txt
# training: iteration 2 (after one warm iteration): 1 head + 8 blocks + body + tail + 18 dgrad rolls + wgrad
ncu --set full --clock-control none --import-source on -k "regex:k_conv_roll" -s 40 -c 1 -o gpurun_out/r02_ncu_train_dgrad \
  python scripts/train_eager.py 3 > gpurun_out/r02_ncu_train_dgrad.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_train_dgrad.ncu-rep > gpurun_out/r02_ncu_train_dgrad.txt
ncu --set full --clock-control none --import-source on -k "regex:k_wgrad_multi" -s 1 -c 1 -o gpurun_out/r02_ncu_train_wgrad \
  python scripts/train_eager.py 3 > gpurun_out/r02_ncu_train_wgrad.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_train_wgrad.ncu-rep > gpurun_out/r02_ncu_train_wgrad.txt
ncu --set full --clock-control none --import-source on -k "regex:k_resblock" -s 8 -c 1 -o gpurun_out/r02_ncu_train_resblock \
  python scripts/train_eager.py 3 > gpurun_out/r02_ncu_train_resblock.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_train_resblock.ncu-rep > gpurun_out/r02_ncu_train_resblock.txt
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_train.csv \
  python scripts/train_eager.py 3 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/r02_launches_train.csv > gpurun_out/r02_launches_train_summary.txt
