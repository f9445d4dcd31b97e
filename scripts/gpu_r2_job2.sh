#!/bin/bash
# round-2 job 2: probes, sanitizers per group, GPU tests + smoke on the refactored library
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-p2}
mkdir -p gpurun_out
timeout 300 python scripts/tc4_probe.py > gpurun_out/tc4_probe_$TAG.jsonl 2> gpurun_out/tc4_probe_$TAG.err
cat gpurun_out/tc4_probe_$TAG.jsonl | grep sw64
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -1 gpurun_out/smoke_$TAG.log
SAN=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck synccheck; do
  timeout 900 $SAN --tool $tool --print-limit 10 python scripts/sanitize_run.py > gpurun_out/san_${tool}_$TAG.log 2>&1
  echo "$tool exit $?"; grep -E "ERROR SUMMARY|sanitize group" gpurun_out/san_${tool}_$TAG.log | tr '\n' ' '; echo
done
for g in v8 cc cl small tensor fused ftc gemm rns host; do
  timeout 600 $SAN --tool racecheck --racecheck-report hazard --print-limit 4 python scripts/sanitize_run.py $g > gpurun_out/san_racecheck_${g}_$TAG.log 2>&1
  echo "racecheck $g exit $? $(grep -E 'RACECHECK SUMMARY' gpurun_out/san_racecheck_${g}_$TAG.log)"
done
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_$TAG.log 2>&1; tail -3 gpurun_out/pytest_$TAG.log
