#!/bin/bash
# profiles of the default path: ncu launch list of a short bench run, one --set full capture of the
# v8 forward + inverse at config 3 with source, and the summaries (scripts/ncu_summary.py, ncu_hot.py,
# sass_mix.py).  gpu_prof.sh TAG
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-p}
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"ntt|rns|tc4" -c 400 --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu --e2e-steps 0 > gpurun_out/launches_${TAG}_bench.txt 2>&1
echo "launch list rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"ntt_v8|ntt_tmr" -s 4 -c 4 -o gpurun_out/prof_$TAG \
  python scripts/one_step.py 128 auto > gpurun_out/prof_${TAG}_run.txt 2>&1
echo "full rc=$?"
python scripts/ncu_summary.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/ncu_$TAG.txt 2>&1
python scripts/ncu_hot.py gpurun_out/prof_$TAG.ncu-rep 25 > gpurun_out/hot_$TAG.txt 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page source --csv --print-source cuda 2>&1 | head -60 > gpurun_out/srcraw_$TAG.txt
python scripts/ncu_hot_src.py gpurun_out/prof_$TAG.ncu-rep 30 > gpurun_out/hotsrc_$TAG.txt 2>&1
python scripts/sass_mix.py gpurun_out/prof_$TAG.ncu-rep $((4608 * 65536)) > gpurun_out/sass_$TAG.txt 2>&1
[ -n "$KEEP" ] || rm -f gpurun_out/prof_$TAG.ncu-rep
grep -E "==|time_dur|dram__bytes|issue_active|stalls" gpurun_out/ncu_$TAG.txt
head -3 gpurun_out/sass_$TAG.txt
python scripts/launch_summary.py gpurun_out/launches_$TAG.csv > gpurun_out/launch_summary_$TAG.txt 2>&1
