#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
for so in 0 1 2; do
  WD_NTT_PIPE_SOLO=$so timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode fused > gpurun_out/bench_${TAG}_solo$so.json 2> gpurun_out/bench_${TAG}_solo$so.err
done
WD_NTT_KERNEL=v2 timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > gpurun_out/bench_${TAG}_cuda.json 2>&1
echo done
