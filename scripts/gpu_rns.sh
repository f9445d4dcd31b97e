#!/bin/bash
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_rns.py -q -x > gpurun_out/pytest_rns.log 2>&1
tail -3 gpurun_out/pytest_rns.log
timeout 300 python bench.py --op rescale --steps 20 --warmup 3 > gpurun_out/bench_rescale.json 2> gpurun_out/bench_rescale.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_rescale.csv python bench.py --op rescale --steps 2 --warmup 1 > /dev/null 2>&1
echo done
