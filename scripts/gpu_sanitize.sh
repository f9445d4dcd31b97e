#!/bin/bash
# compute-sanitizer memcheck / synccheck over every group, racecheck per group (profiles/r02/sanitizer/);
# SAN_GROUPS="tm v8" restricts the groups (bash reserves $GROUPS)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-s}
mkdir -p gpurun_out
SAN=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck; do
  timeout 1500 $SAN --tool $tool --print-limit 10 python scripts/sanitize_run.py $SAN_GROUPS > gpurun_out/san_${tool}_$TAG.log 2>&1
  echo "$tool exit $?"; grep -E "ERROR SUMMARY|sanitize group" gpurun_out/san_${tool}_$TAG.log | tr '\n' ' '; echo
done
for g in ${SAN_GROUPS:-v8 v8feeds tm cc cl small tensor fused ftc gemm tc4 rns host}; do
  timeout 900 $SAN --tool racecheck --racecheck-report hazard --print-limit 4 python scripts/sanitize_run.py $g > gpurun_out/san_racecheck_${g}_$TAG.log 2>&1
  echo "racecheck $g exit $? $(grep -E 'RACECHECK SUMMARY|sanitize group' gpurun_out/san_racecheck_${g}_$TAG.log | tr '\n' ' ')"
done
