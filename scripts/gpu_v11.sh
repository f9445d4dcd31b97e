#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "v11" > gpurun_out/pytest_v11.log 2>&1
tail -3 gpurun_out/pytest_v11.log
for tm in 1 3 6 7; do
WD_NTT_TMASK=$tm bash scripts/gpu_ab.sh $1_tm$tm 30 "c3:v11" 1 > /dev/null
done
bash scripts/gpu_ab.sh $1 30 "c3:v8" 1 > /dev/null
echo done
