#!/bin/bash
# FUSED split sweep (tensor share of the column phases) + CUDA-only and TENSOR-only references
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "modes" > gpurun_out/pytest_$TAG.log 2>&1
for sh in 1.0 0.85 0.7 0.55 0.4; do
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode fused --share $sh > gpurun_out/bench_${TAG}_f$sh.json 2> gpurun_out/bench_${TAG}_f$sh.err
done
timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > gpurun_out/bench_${TAG}_cuda.json 2>&1
timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode tensor > gpurun_out/bench_${TAG}_tensor.json 2>&1
echo done
