#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 300 python scripts/tc4_trace.py ${1:-128} > gpurun_out/tc4_trace_${2:-x}.log 2>&1; echo "exit $?"; cat gpurun_out/tc4_trace_${2:-x}.log
