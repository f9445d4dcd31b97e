#!/bin/bash
# limb-major row schedule A/B (WD_NTT_LM=1 default vs 0): config 3, config 4, and a 60-limb batch
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for r in 1 2; do for lm in 1 0; do for cfg in c3 c4; do
  WD_NTT_LM=$lm timeout 300 python bench.py --steps 30 --warmup 5 --e2e-steps 0 --no-cpu --config $cfg > gpurun_out/ab_lm_${cfg}-lm$lm\_$r.json 2> gpurun_out/ab_lm_${cfg}-lm$lm\_$r.err
done; done; done
python scripts/ab_table.py lm
for lm in 1 0; do
  WD_NTT_LM=$lm timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"ntt_v8" -c 4 --csv --log-file gpurun_out/dram_lm$lm.csv python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu > /dev/null 2>&1
  grep -h "dram__bytes\|gpu__time" gpurun_out/dram_lm$lm.csv | awk -F'","' '{print "lm'$lm'", $5, $(NF-2), $NF}' | cut -c1-140 | tail -6
done
