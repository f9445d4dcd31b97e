#!/bin/bash
# ncu --set full of one kernel generation at config 3: gpu_ncu.sh TAG VER KERNEL_REGEX
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; VER=$2; KRE=$3
mkdir -p gpurun_out
export WD_NTT_KERNEL=$VER
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$KRE" -s 2 -c 2 -o gpurun_out/prof_${TAG} \
  python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu > gpurun_out/ncu_${TAG}.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv \
  python bench.py --steps 2 --warmup 1 --e2e-steps 0 --no-cpu > /dev/null 2>&1
echo done
