#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_rns.py -q -x > gpurun_out/pytest_rns.log 2>&1
tail -3 gpurun_out/pytest_rns.log
for op in rescale modup moddown; do
timeout 300 python bench.py --op $op --steps 20 --warmup 3 > gpurun_out/bench_$op.json 2> gpurun_out/bench_$op.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$op.csv python bench.py --op $op --steps 2 --warmup 1 > /dev/null 2>&1
done
echo done
