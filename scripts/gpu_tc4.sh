#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-t1}
mkdir -p gpurun_out
timeout 300 python scripts/tc4_try.py > gpurun_out/tc4_try_$TAG.log 2>&1
echo "exit $?"; cat gpurun_out/tc4_try_$TAG.log | tail -20
