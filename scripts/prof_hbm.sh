#!/bin/bash
# ncu DRAM bytes + duration per launch of the memory-bound kernels, one clean capture per kernel/shape
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
run() {  # name, kernel regex, skip, --only
  ncu --metrics $M --clock-control none -k "regex:$2" -s $3 -c 3 --csv --log-file gpurun_out/r02_ncu_hbm_$1.csv \
    python scripts/hbm_kernels.py --only $4 > /dev/null 2>&1
}
run adam_small k_adam 20 adam_small
run adam64m k_adam 20 adam64m
run gather k_sample_gather 10 gather
run sse4k k_sse_u8 10 sse4k
run sseval k_sse_u8 10 sseval
run head "k_conv_roll" 5 infer
run bodytail "k_bodytail" 5 infer
run resblock "k_resblock" 40 infer
python scripts/ncu_hbm_summary.py gpurun_out/r02_ncu_hbm_*.csv > gpurun_out/r02_ncu_hbm_summary.txt
