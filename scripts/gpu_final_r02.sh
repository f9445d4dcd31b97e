#!/bin/bash
# round-2 final measurements: default bench line (with e2e + cpu baseline), other configs, config-5 sweep
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-fin}
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_${TAG}_default.json 2> gpurun_out/bench_${TAG}_default.err
tail -c 300 gpurun_out/bench_${TAG}_default.json; echo
for c in c1 c2 c4; do
  timeout 600 python bench.py --config $c --steps 30 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/bench_${TAG}_$c.json 2> gpurun_out/bench_${TAG}_$c.err
  python -c "import json,sys; d=json.loads(open('gpurun_out/bench_${TAG}_$c.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), d['fwd_ms'], d['inv_ms'])"
done
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_${TAG}_reference.json 2> gpurun_out/bench_${TAG}_reference.err
tail -c 300 gpurun_out/bench_${TAG}_reference.json; echo
timeout 1500 python scripts/sweep_c5.py > gpurun_out/sweep_c5_${TAG}.jsonl 2> gpurun_out/sweep_c5_${TAG}.err
echo "sweep rc=$? lines=$(wc -l < gpurun_out/sweep_c5_${TAG}.jsonl)"
