#!/bin/bash
# ncu --set full of the tc4 kernel (one launch after a warm-up) + summaries; report deleted after
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-n1}; B=${2:-32}; DIR=${3:-fwd}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tc4 -s 1 -c 1 \
   -o gpurun_out/prof_$TAG python scripts/tc4_one.py $B tc4 $DIR > gpurun_out/ncu_run_$TAG.log 2>&1
echo "ncu exit $?"
python scripts/ncu_summary.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/ncu_$TAG.txt 2>&1
python scripts/ncu_hot.py gpurun_out/prof_$TAG.ncu-rep 40 > gpurun_out/hot_$TAG.txt 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/raw_$TAG.csv 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page source --csv --print-source sass > gpurun_out/src_$TAG.csv 2>&1
rm -f gpurun_out/prof_$TAG.ncu-rep
head -60 gpurun_out/ncu_$TAG.txt
