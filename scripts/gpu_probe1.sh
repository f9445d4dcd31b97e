#!/bin/bash
# integer-pipe probes + v8 phase-only timings (config 3)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
timeout 120 python scripts/int_probe.py > gpurun_out/int_probe.jsonl 2>&1
for v in v8 v81 v82; do
  WD_NTT_PIPE_SOLO=1 WD_NTT_KERNEL=$v timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/phase_$v.json 2>&1
done
echo done
