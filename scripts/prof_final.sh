#!/bin/bash
# Final round-2 evidence for the bench line: launch list of one bench step (cold, serialised), and one
# `ncu --set full` capture of the dominant kernel in the bench's configuration (30 x 720p, k_resblock<48>) whose DRAM
# bytes are the roofline's `traffic`.
# (ncu cannot profile kernels launched on green-context streams -- "Failed to prepare kernel for profiling" -- so the
# launch list is of the sequential step, --partition 0: the same kernels and shapes on whole-GPU grids)
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_launches_bench.csv \
  python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-cfg2 --partition 0 > gpurun_out/r02_launches_bench.log 2>&1
python scripts/launch_summary.py gpurun_out/r02_launches_bench.csv > gpurun_out/r02_launches_bench_summary.txt
ncu --set full --clock-control none --import-source on -k "regex:k_resblock" -s 10 -c 1 -o gpurun_out/r02_ncu_resblock48 \
  python scripts/infer_profile.py > gpurun_out/r02_ncu_resblock48.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_resblock48.ncu-rep > gpurun_out/r02_ncu_resblock48.txt
ncu --set full --clock-control none --import-source on -k "regex:k_resblock2" -s 10 -c 1 -o gpurun_out/r02_ncu_resblock2_32 \
  python scripts/cfg2_timing.py > gpurun_out/r02_ncu_resblock2_32.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_resblock2_32.ncu-rep > gpurun_out/r02_ncu_resblock2_32.txt
