#!/bin/bash
# per-launch time + DRAM bytes of the default kernels (config 3 and 4): gpu_dram.sh TAG
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
for cfg in c3 c4; do
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"ntt_" -c 6 --csv --log-file gpurun_out/dram_${TAG}_$cfg.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu --config $cfg > /dev/null 2>&1
python - "$TAG" "$cfg" <<'PY'
import csv, sys
txt = open("gpurun_out/dram_%s_%s.csv" % (sys.argv[1], sys.argv[2])).read().splitlines()
rows = list(csv.reader([l for l in txt if l.startswith("\"")]))
h = rows[0]; ix = {k: i for i, k in enumerate(h)}
for r in rows[1:]:
    if len(r) < len(h): continue
    print(sys.argv[2], r[ix["Kernel Name"]][:40], r[ix["Metric Name"]], r[ix["Metric Value"]])
PY
done
