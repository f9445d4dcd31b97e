#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "wd_cuda_gemm" > gpurun_out/pytest_wdc.log 2>&1
tail -3 gpurun_out/pytest_wdc.log
for m in cuda cuda_gemm tensor fused; do
timeout 300 python bench.py --mode $m --steps 20 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/bench_mode_$m.json 2> gpurun_out/bench_mode_$m.err
done
echo done
