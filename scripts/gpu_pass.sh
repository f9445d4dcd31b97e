#!/bin/bash
# validation pass: smoke, all GPU tests, default bench (e2e + cpu baseline), reference arm, configs
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
tail -1 gpurun_out/smoke_$TAG.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_$TAG.log 2>&1
tail -1 gpurun_out/pytest_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_${TAG}_ref.json 2> gpurun_out/bench_${TAG}_ref.err
for cfg in c2 c4 c1; do
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/bench_${TAG}_$cfg.json 2> gpurun_out/bench_${TAG}_$cfg.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"ntt_|rns_|rs_" --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 3 --warmup 3 --e2e-steps 0 --no-cpu > /dev/null 2>&1
for f in bench_$TAG bench_${TAG}_ref bench_${TAG}_c2 bench_${TAG}_c4 bench_${TAG}_c1; do
  python -c "import json; d=json.loads(open('gpurun_out/$f.json').read().strip().splitlines()[-1]); print('$f', d.get('value'), d.get('fwd_ms'), d.get('inv_ms'), (d.get('roofline') or {}).get('frac'))"
done
