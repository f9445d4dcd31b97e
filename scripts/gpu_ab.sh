#!/bin/bash
# A/B with repeats: gpu_ab.sh TAG STEPS "cfg:ver[:minb[:cl]] ..." REPEATS
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; STEPS=$2; PAIRS=$3; REP=${4:-1}
mkdir -p gpurun_out
for r in $(seq 1 $REP); do
for pv in $PAIRS; do
  IFS=: read cfg v mb cl <<< "$pv"
  unset WD_NTT_KERNEL WD_NTT_MINB WD_NTT_CL
  [ "$v" != auto ] && export WD_NTT_KERNEL=$v
  [ -n "$mb" ] && export WD_NTT_MINB=$mb
  [ -n "$cl" ] && export WD_NTT_CL=$cl
  key=$(echo $pv | tr ':' '-')
  timeout 300 python bench.py --steps $STEPS --warmup 5 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/ab_${TAG}_${key}_$r.json 2> gpurun_out/ab_${TAG}_${key}_$r.err
done; done
echo done
