#!/bin/bash
# A/B bench of kernel generations: gpu_var.sh TAG "c4:v2 c4:v6 c3:auto" [pytest -k expr]
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; PAIRS=$2; KEXPR=$3
mkdir -p gpurun_out
for pv in $PAIRS; do
  cfg=${pv%%:*}; v=${pv##*:}
  if [ "$v" = auto ]; then unset WD_NTT_KERNEL; else export WD_NTT_KERNEL=$v; fi
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/var_${TAG}_${cfg}_$v.json 2> gpurun_out/var_${TAG}_${cfg}_$v.err
done
unset WD_NTT_KERNEL
if [ -n "$KEXPR" ]; then timeout 900 python -m pytest tests -m gpu -q -k "$KEXPR" > gpurun_out/pytest_$TAG.log 2>&1; fi
echo done
