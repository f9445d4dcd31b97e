#!/bin/bash
# round-2 bench checks: default line, tc4 line, limb-shard line (plain and torchrun 1 rank), ncu traffic
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=${1:-b1}
mkdir -p gpurun_out
timeout 600 python bench.py --steps 30 --warmup 3 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; tail -c 2500 gpurun_out/bench_$TAG.json; echo
timeout 300 python bench.py --mode tc4 --steps 10 --warmup 3 --e2e-steps 0 --no-cpu > gpurun_out/bench_${TAG}_tc4.json 2> gpurun_out/bench_${TAG}_tc4.err; tail -c 600 gpurun_out/bench_${TAG}_tc4.json; echo
timeout 300 python bench.py --shard limbs --config c4 --steps 10 --warmup 3 > gpurun_out/bench_${TAG}_shard.json 2> gpurun_out/bench_${TAG}_shard.err; tail -c 800 gpurun_out/bench_${TAG}_shard.json; tail -3 gpurun_out/bench_${TAG}_shard.err; echo
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --shard limbs --config c4 --steps 10 --warmup 3 > gpurun_out/bench_${TAG}_shard_tr.json 2> gpurun_out/bench_${TAG}_shard_tr.err; grep -c "NCCL INFO" gpurun_out/bench_${TAG}_shard_tr.json gpurun_out/bench_${TAG}_shard_tr.err; tail -1 gpurun_out/bench_${TAG}_shard_tr.json | head -c 400; echo
timeout 600 ncu --set full --clock-control none -k regex:ntt_v8 -s 2 -c 2 -o gpurun_out/prof_$TAG python scripts/one_step.py 128 auto > /dev/null 2>&1
ncu -i gpurun_out/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/raw_$TAG.csv 2>&1
python scripts/ncu_summary.py gpurun_out/prof_$TAG.ncu-rep > gpurun_out/ncu_$TAG.txt 2>&1; rm -f gpurun_out/prof_$TAG.ncu-rep
grep -E "==|time_dur|dram__bytes" gpurun_out/ncu_$TAG.txt
