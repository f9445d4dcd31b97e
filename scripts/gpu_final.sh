#!/bin/bash
# end-of-round pass: full GPU pass (gpu_full.sh), ncu summaries (reports deleted afterwards to
# stay under gpurun's 64 MiB copy-back), modes sweep, small-config cluster sweep
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
bash scripts/gpu_full.sh $TAG
python scripts/ncu_summary.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/ncu_$TAG.txt 2>&1
python scripts/ncu_hot.py gpurun_out/prof_$TAG.ncu-rep 25 > gpurun_out/hot_$TAG.txt 2>&1
python scripts/sass_mix.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/sass_$TAG.txt 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/raw_$TAG.csv 2>&1
rm -f gpurun_out/prof_$TAG.ncu-rep
bash scripts/gpu_modes.sh m$TAG
for r in tc fu; do
  python scripts/ncu_summary.py gpurun_out/prof_m${TAG}_$r.ncu-rep > gpurun_out/ncu_m${TAG}_$r.txt 2>&1
  rm -f gpurun_out/prof_m${TAG}_$r.ncu-rep
done
bash scripts/gpu_ab.sh cl$TAG 30 "c2:v8:4:2 c2:v8:4:4 c2:v8:4:8" 1
python scripts/ab_table.py cl$TAG > gpurun_out/ab_cl$TAG.txt
bash scripts/gpu_dram.sh $TAG > gpurun_out/dram_$TAG.txt 2>&1
du -sh gpurun_out
