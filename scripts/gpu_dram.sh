#!/bin/bash
# DRAM bytes + duration of the v8 launches at config 3 (ncu, two metrics only) and a short bench
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-d}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:ntt_v8 -s 2 -c 2 \
  python scripts/one_step.py 128 auto 2>&1 | grep -E "ntt_v8|gpu__time|dram__" > gpurun_out/dram_$TAG.txt
cat gpurun_out/dram_$TAG.txt
