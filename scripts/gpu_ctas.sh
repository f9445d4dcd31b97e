#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
for c in 2 3 4; do
  WD_NTT_CTAS=$c timeout 300 python bench.py --steps 30 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > gpurun_out/bench_${TAG}_c$c.json 2> gpurun_out/bench_${TAG}_c$c.err
done
for cfg in c1 c2 c4; do
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/bench_${TAG}_$cfg.json 2> gpurun_out/bench_${TAG}_$cfg.err
done
echo done
