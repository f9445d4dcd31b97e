#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "generations or many_rows or prime_sizes" > gpurun_out/pytest_z.log 2>&1
tail -2 gpurun_out/pytest_z.log
bash scripts/gpu_ab.sh $1 40 "c3:auto c4:auto s13:auto s14:auto s15:auto c2:auto" 2 > /dev/null
echo done
