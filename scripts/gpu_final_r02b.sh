#!/bin/bash
# round-2 final pass after tm: GPU suite + smoke, default bench line, config-5 sweep, profiles
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-f2}
mkdir -p gpurun_out
bash scripts/gpu_validate.sh $TAG
timeout 400 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?"
timeout 600 python scripts/sweep_c5.py > gpurun_out/sweep_c5_$TAG.jsonl 2> gpurun_out/sweep_c5_$TAG.err; echo "sweep rc=$?"
KEEP=1 bash scripts/gpu_prof.sh $TAG
