#!/bin/bash
# bench lines of every BASELINE config with the final library, a 100-step headline run, and ncu captures
# of the tm kernels at N = 2^15 / 2^14 / 2^13 (config-5 shapes, 128 ciphertexts, L = 36)
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
mkdir -p gpurun_out
for c in c1 c2 c4; do
  timeout 400 python bench.py --config $c --no-cpu > gpurun_out/cfg_$c.json 2> gpurun_out/cfg_$c.err; echo "$c rc=$?"
done
timeout 600 python bench.py --steps 100 --warmup 5 --no-cpu --e2e-steps 0 > gpurun_out/cfg_c3_100.json 2> gpurun_out/cfg_c3_100.err; echo "c3x100 rc=$?"
timeout 400 python bench.py --shard limbs --config c4 --no-cpu > gpurun_out/cfg_shard_c4.json 2> gpurun_out/cfg_shard_c4.err; echo "shard rc=$?"
for ln in 15 14 13; do
  timeout 600 ncu --set full --clock-control none -k regex:"ntt_tm" -s 2 -c 2 -o gpurun_out/prof_tm$ln \
    python scripts/one_step.py 256 auto $ln 36 > gpurun_out/prof_tm${ln}_run.txt 2>&1; echo "ncu $ln rc=$?"
  python scripts/ncu_summary.py gpurun_out/prof_tm$ln.ncu-rep > gpurun_out/ncu_tm$ln.txt 2>&1
  rm -f gpurun_out/prof_tm$ln.ncu-rep
done
