#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
export WD_NTT_KERNEL=v10
WD_NTT_DEBUG=1 timeout 120 python bench.py --steps 5 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/v10b_dbg.json 2> gpurun_out/v10b_dbg.err
for ncl in 148 222 296; do
WD_NTT_V10_CLUSTERS=$ncl timeout 120 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/v10b_$ncl.json 2> gpurun_out/v10b_$ncl.err
done
echo done
