#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "generations or modes" > gpurun_out/pytest_$TAG.log 2>&1
for v in v2 v3 v5; do
  WD_NTT_KERNEL=$v timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > gpurun_out/bench_${TAG}_$v.json 2> gpurun_out/bench_${TAG}_$v.err
done
WD_NTT_KERNEL=v5 timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda --config c4 > gpurun_out/bench_${TAG}_v5_c4.json 2>&1
WD_NTT_KERNEL=v2 timeout 300 python bench.py --steps 10 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda --config c4 > gpurun_out/bench_${TAG}_v2_c4.json 2>&1
WD_NTT_KERNEL=v5 timeout 600 ncu --set full --clock-control none --import-source on -k regex:"ntt_.*_cl" -s 2 -c 2 -o gpurun_out/prof_${TAG}_v5 python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > /dev/null 2>&1
echo done
