#!/bin/bash
# usage: bash scripts/gpu_check.sh TAG [pytest-k-expr] [bench-args...]
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; shift
KEXPR=$1; shift
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
if [ "$KEXPR" != "none" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q -k "$KEXPR" > gpurun_out/pytest_$TAG.log 2>&1
  echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
fi
timeout 600 python bench.py --steps 50 --warmup 5 --e2e-steps 0 --no-cpu "$@" > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
if [ -n "$NCU" ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$NCU" -s 2 -c 1 -o gpurun_out/prof_$TAG python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu "$@" > gpurun_out/ncu_$TAG.log 2>&1
fi
echo done
