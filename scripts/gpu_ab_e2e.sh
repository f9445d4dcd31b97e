#!/bin/bash
# e2e A/B of the host pipeline's chunk cap: gpu_ab_e2e.sh TAG "32 64 128" REPS
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; VALS=$2; REP=${3:-2}
mkdir -p gpurun_out
for r in $(seq 1 $REP); do for v in $VALS; do
  WD_HOST_MAXCH=$v timeout 600 python bench.py --steps 5 --warmup 3 --e2e-steps 5 --no-cpu > gpurun_out/e2e_${TAG}_${v}_$r.json 2> gpurun_out/e2e_${TAG}_${v}_$r.err
  python - "$v" gpurun_out/e2e_${TAG}_${v}_$r.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1]); e = d["e2e"]
    print("maxch=%-5s e2e=%.1f KOPS  pcie_bound=%.1f  frac=%.3f  value=%.0f" % (sys.argv[1], e["value"], e["pcie_bound"]["value"], e["frac_of_pcie_bound"], d["value"]))
except Exception as ex:
    print(sys.argv[1], "FAILED", ex)
PY
done; done
