#!/bin/bash
# Round profile: launch list of one bench step + full ncu captures of the inference kernels (one launch each).
set -x
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bench.csv \
  python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/launches_bench.log 2>&1
python scripts/launch_summary.py gpurun_out/launches_bench.csv > gpurun_out/launches_bench_summary.txt
for k in k_resblock k_bodytail "k_conv_roll"; do
  n=$(echo $k | tr -cd 'a-z_')
  ncu --set full --clock-control none --import-source on -k "regex:$k" -s 0 -c 1 -o gpurun_out/ncu_$n \
    python scripts/infer_profile.py > gpurun_out/ncu_$n.log 2>&1
  python scripts/ncu_summary.py gpurun_out/ncu_$n.ncu-rep > gpurun_out/ncu_$n.txt
done
