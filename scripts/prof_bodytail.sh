set -x
ncu --set full --clock-control none --import-source on -k "regex:k_bodytail" -s 2 -c 1 -o gpurun_out/r02_ncu_bodytail48 \
  python scripts/infer_profile.py > gpurun_out/r02_ncu_bodytail48.log 2>&1
python scripts/ncu_summary.py gpurun_out/r02_ncu_bodytail48.ncu-rep > gpurun_out/r02_ncu_bodytail48.txt
python scripts/bodytail_timeline.py 3 > gpurun_out/bt_timeline.txt 2>&1
python scripts/infer_profile.py > gpurun_out/infer_profile.txt 2>&1
