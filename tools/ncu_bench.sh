#!/bin/bash
# Profiles for the bench workload (run under gpurun, 1 GPU):
#   1. launch list with per-launch device time (cold-cache, serialized) of a short bench run
#   2. one `ncu --set full` capture of the encode kernel inside the bench workload
set -x
R=${1:-r01}
# the kernel-source hash of this capture (bench.py drops profile-derived keys of other builds)
python -c "from paper_conf_pact_map17_b200._build import source_hash; print(source_hash())" > gpurun_out/build_$R.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_$R.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu \
  > gpurun_out/ncu_launch_stdout.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:lzr_encode -s 3 -c 1 \
  -f -o gpurun_out/encode_full_$R python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu \
  > gpurun_out/ncu_full_stdout.log 2>&1
