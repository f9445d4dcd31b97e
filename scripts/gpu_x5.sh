#!/bin/bash
# v8 coalesced-store change: parity (v8 + RNS epilogues) and A/B against the old stores (v88)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
TAG=${1:-x5}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_rns.py -m gpu -x -q > gpurun_out/pytest_$TAG.log 2>&1
tail -3 gpurun_out/pytest_$TAG.log

bash scripts/gpu_ab.sh $TAG 30 "${2:-c3:auto c3:v89 c4:auto c2:auto}" 2
python scripts/ab_table.py $TAG
