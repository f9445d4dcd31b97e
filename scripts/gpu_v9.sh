#!/bin/bash
# v9 parity (generations + many-row tests for v8/v9) then A/B v8 vs v9
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "v9 or many_rows" > gpurun_out/pytest_v9.log 2>&1
tail -3 gpurun_out/pytest_v9.log
bash scripts/gpu_ab.sh $1 40 "c3:v8 c3:v9 c3:v9:4:1 s13:v8 s13:v9 s14:v8 s14:v9 s15:v8 s15:v9 c2:v8 c2:v9" 2
