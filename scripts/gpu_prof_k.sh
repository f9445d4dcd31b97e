#!/bin/bash
# ncu --set full of one kernel family at config 3 (forward + inverse) with source + summaries.
# gpu_prof_k.sh TAG KERNEL_REGEX [env assignments...]   e.g. gpu_prof_k.sh tm1 ntt_tmr WD_NTT_KERNEL=tm
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; KRE=$2; shift 2
mkdir -p gpurun_out
env "$@" timeout 900 ncu --set full --import-source on --clock-control none -k regex:$KRE -s 2 -c 2 -o gpurun_out/prof_$TAG \
  python scripts/one_step.py 128 auto > gpurun_out/prof_${TAG}_run.txt 2>&1
echo "full rc=$?"
python scripts/ncu_summary.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/ncu_$TAG.txt 2>&1
python scripts/ncu_hot.py gpurun_out/prof_$TAG.ncu-rep 40 > gpurun_out/hot_$TAG.txt 2>&1
python scripts/ncu_hot_src.py gpurun_out/prof_$TAG.ncu-rep 40 > gpurun_out/hotsrc_$TAG.txt 2>&1
python scripts/sass_mix.py gpurun_out/prof_$TAG.ncu-rep $((4608 * 65536)) > gpurun_out/sass_$TAG.txt 2>&1
[ -n "$KEEP" ] || rm -f gpurun_out/prof_$TAG.ncu-rep
grep -E "==|time_dur|dram__bytes|issue_active|warps_active|stalls" gpurun_out/ncu_$TAG.txt
