#!/bin/bash
# A/B of an environment knob: gpu_ab_env.sh TAG VAR "v1 v2 ..." REPEATS "configs" [pytest-k]
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; VAR=$2; VALS=$3; REP=${4:-2}; CFGS=${5:-c3}; PK=$6
mkdir -p gpurun_out
if [ -n "$PK" ]; then
  for v in $VALS; do
    env $VAR=$v timeout 900 python -m pytest tests -m gpu -q -x -p no:cacheprovider -k "$PK" > gpurun_out/abe_${TAG}_pytest_$v.txt 2>&1
    echo "pytest $VAR=$v rc=$? $(tail -1 gpurun_out/abe_${TAG}_pytest_$v.txt)"
  done
fi
for r in $(seq 1 $REP); do
for cfg in $CFGS; do
for v in $VALS; do
  env $VAR=$v timeout 300 python bench.py --steps 30 --warmup 5 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/abe_${TAG}_${cfg}_${v}_$r.json 2> gpurun_out/abe_${TAG}_${cfg}_${v}_$r.err
  python - "$VAR=$v" "$cfg" gpurun_out/abe_${TAG}_${cfg}_${v}_$r.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[3]).read().strip().splitlines()[-1])
    print("%-16s %s value=%.1f fwd=%.4f inv=%.4f sm=%s" % (sys.argv[1], sys.argv[2], d["value"], d["fwd_ms"], d["inv_ms"], d.get("clocks", {}).get("sm_mhz")))
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", e)
PY
done; done; done
