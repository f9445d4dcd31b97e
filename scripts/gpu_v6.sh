#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "generations and (v6 or v2) or config3 or in_place or pointwise" > gpurun_out/pytest_$TAG.log 2>&1
for v in v2 v6; do
  WD_NTT_KERNEL=$v timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > gpurun_out/bench_${TAG}_$v.json 2> gpurun_out/bench_${TAG}_$v.err
done
WD_NTT_KERNEL=v6 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"ntt_persist" -s 2 -c 1 -o gpurun_out/prof_${TAG}_v6 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > /dev/null 2>&1
WD_NTT_PIPE_SOLO=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"ntt_fused" -s 1 -c 1 -o gpurun_out/prof_${TAG}_solo1 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode fused > /dev/null 2>&1
echo done
