#!/bin/bash
# v10 parity then A/B v8 vs v10 (config 3) + ncu of v10
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "v10 or prime_sizes" > gpurun_out/pytest_v10.log 2>&1
tail -3 gpurun_out/pytest_v10.log
bash scripts/gpu_ab.sh $1 40 "c3:v8 c3:v10 c3:v10:4:1" 2
export WD_NTT_KERNEL=v10
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"ntt_v10" -s 2 -c 2 -o gpurun_out/prof_$1 \
  python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/ncu_$1.log 2>&1
echo done
