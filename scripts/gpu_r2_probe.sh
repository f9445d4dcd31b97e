#!/bin/bash
# round-2 job: tc4 probes (int8 peak, SW64 TMA->UMMA layout) + compute-sanitizer over every launch path
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-p1}
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi_$TAG.txt 2>&1
timeout 300 python scripts/tc4_probe.py > gpurun_out/tc4_probe_$TAG.jsonl 2> gpurun_out/tc4_probe_$TAG.err
cat gpurun_out/tc4_probe_$TAG.jsonl
SAN=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck; do
  timeout 900 $SAN --tool $tool --print-limit 20 python scripts/sanitize_run.py ${SGROUPS:-} > gpurun_out/san_${tool}_$TAG.log 2>&1
  echo "$tool exit $?"; tail -3 gpurun_out/san_${tool}_$TAG.log
done
timeout 900 $SAN --tool racecheck --racecheck-report hazard --print-limit 20 python scripts/sanitize_run.py ${RGROUPS:-v8 cc cl small tensor gemm rns} > gpurun_out/san_racecheck_$TAG.log 2>&1
echo "racecheck exit $?"; tail -3 gpurun_out/san_racecheck_$TAG.log
