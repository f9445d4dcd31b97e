#!/bin/bash
# v8 experiments: coalesced-store variants and grid stagger
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
export WD_NTT_PIPE_SOLO=1
bash scripts/gpu_ab.sh x4 30 "c3:v86 c3:v87" 1
unset WD_NTT_PIPE_SOLO
for st in 0 5000 10000 20000 40000; do
  WD_NTT_STAGGER=$st timeout 300 python bench.py --steps 30 --warmup 5 --e2e-steps 0 --no-cpu > gpurun_out/ab_x4_st${st}_1.json 2> gpurun_out/ab_x4_st${st}_1.err
done
python scripts/ab_table.py x4
