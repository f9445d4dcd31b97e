#!/bin/bash
# modes run: tests for modes, benches for cuda(v2, v4) / tensor / fused, ncu of tensor + fused kernels
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
TAG=$1
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_$TAG.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -k "modes or config3 or all_sizes and 16" > gpurun_out/pytest_$TAG.log 2>&1
for m in cuda tensor fused; do :; done; for m in tensor fused; do
  SH=-1; MM=$m; if [ $m = fused2 ]; then SH=0.5; MM=fused; fi
  timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode $MM --share $SH > gpurun_out/bench_${TAG}_$m.json 2> gpurun_out/bench_${TAG}_$m.err
done
WD_NTT_KERNEL=v4 timeout 300 python bench.py --steps 20 --warmup 3 --e2e-steps 0 --no-cpu --mode cuda > gpurun_out/bench_${TAG}_cuda_v4.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"ntt_tcc16" -s 1 -c 1 -o gpurun_out/prof_${TAG}_tc python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode tensor > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"ntt_fused" -s 1 -c 1 -o gpurun_out/prof_${TAG}_fu python bench.py --steps 1 --warmup 3 --e2e-steps 0 --no-cpu --mode fused > /dev/null 2>&1
echo done
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 10 --warmup 3 --e2e-steps 1 --no-cpu > gpurun_out/bench_${TAG}_torchrun.json 2> gpurun_out/bench_${TAG}_torchrun.err
