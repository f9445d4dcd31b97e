#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
for cfg in c2 c3; do for v in auto; do
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/bench_${TAG}_${cfg}_$v.json 2> gpurun_out/bench_${TAG}_${cfg}_$v.err
done; done
echo done
timeout 900 python -m pytest tests -m gpu -q -k "config2 or config5 or generations" > gpurun_out/pytest_$TAG.log 2>&1
