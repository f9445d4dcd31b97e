#!/bin/bash
# A/B of a library variant against libwdntt_base.so at N = 2^13..2^15 (tm forced), with tm_check's
# bit-exact / oracle checks of the variant first.  gpu_ab_var_sizes.sh VARIANT
cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
D=paper_conf_hpca_fanzzfzdtksy25_b200
V=${1:-var}
cp $D/libwdntt.so /tmp/orig.so
cp $D/libwdntt_$V.so $D/libwdntt.so
for ln in 13 14 15; do
  timeout 300 python scripts/tm_check.py 36 10 $ln > gpurun_out/ab_${V}_check$ln.txt 2>&1; echo "check $ln rc=$?"; tail -1 gpurun_out/ab_${V}_check$ln.txt
done
cp /tmp/orig.so $D/libwdntt.so
for ln in 13 14 15; do bash scripts/gpu_ab_kern.sh "base $V" "tm" 2 $ln 36 128; done > gpurun_out/ab_${V}_sizes.txt 2>&1
cat gpurun_out/ab_${V}_sizes.txt
