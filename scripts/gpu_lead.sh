#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
for ld in 1 3 4; do for sh in 1.0 0.55; do
  WD_NTT_PIPE_LEAD=$ld timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode fused --share $sh > gpurun_out/bench_${TAG}_l${ld}_f$sh.json 2> gpurun_out/bench_${TAG}_l${ld}_f$sh.err
done; done
WD_NTT_PIPE_LEAD=1 timeout 600 ncu --set full --clock-control none -k regex:"ntt_fused" -s 1 -c 1 -o gpurun_out/prof_${TAG}_fu python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode fused --share 1.0 > /dev/null 2>&1
echo done
