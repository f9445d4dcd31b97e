#!/bin/bash
# A/B of library variants (scripts/build_variant.py): gpu_ab_lib.sh TAG "name1 name2 ..." REPEATS [CONFIGS]
# each variant's libwdntt_<name>.so is copied over libwdntt.so, then bench.py times it (no cpu / e2e legs)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1; VARS=$2; REP=${3:-2}; CFGS=${4:-c3}
D=paper_conf_hpca_fanzzfzdtksy25_b200
mkdir -p gpurun_out
cp $D/libwdntt.so /tmp/libwdntt_orig.so
for r in $(seq 1 $REP); do
for cfg in $CFGS; do
for v in $VARS; do
  cp $D/libwdntt_$v.so $D/libwdntt.so
  timeout 300 python bench.py --steps 30 --warmup 5 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/abl_${TAG}_${cfg}_${v}_$r.json 2> gpurun_out/abl_${TAG}_${cfg}_${v}_$r.err
  python - "$v" "$cfg" gpurun_out/abl_${TAG}_${cfg}_${v}_$r.json <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[3]).read().strip().splitlines()[-1])
    print("%-10s %s value=%.1f fwd=%s inv=%s sm=%s" % (sys.argv[1], sys.argv[2], d["value"], d.get("fwd_ms"), d.get("inv_ms"), d.get("clocks", {}).get("sm_mhz")))
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", e)
PY
done; done; done
cp /tmp/libwdntt_orig.so $D/libwdntt.so
