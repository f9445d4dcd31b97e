#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "modes" > gpurun_out/pytest_$TAG.log 2>&1
for so in 1 2; do
  WD_NTT_PIPE_SOLO=$so timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode fused > gpurun_out/bench_${TAG}_solo$so.json 2> gpurun_out/bench_${TAG}_solo$so.err
done
for m in fused tensor; do
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode $m > gpurun_out/bench_${TAG}_$m.json 2> gpurun_out/bench_${TAG}_$m.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"ntt_fused" -s 1 -c 1 -o gpurun_out/prof_${TAG}_fu python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode fused > /dev/null 2>&1
echo done
