#!/bin/bash
# first GPU pass: build, smoke, parity tests, bench, launch list, one full ncu capture per direction
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/smi.txt 2>&1
nproc > gpurun_out/nproc.txt; lscpu | head -20 >> gpurun_out/nproc.txt
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 50 --warmup 5 --e2e-steps 2 --cpu-seconds 8 > gpurun_out/bench1.json 2> gpurun_out/bench1.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 40 --csv --log-file gpurun_out/launches1.csv python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ntt_fwd_cc -s 3 -c 1 -o gpurun_out/prof_fwd1 python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/ncu_fwd1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ntt_inv_cc -s 3 -c 1 -o gpurun_out/prof_inv1 python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/ncu_inv1.log 2>&1
echo done
