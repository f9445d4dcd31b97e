cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
D=paper_conf_hpca_fanzzfzdtksy25_b200
V=${1:-dst}
cp $D/libwdntt.so /tmp/orig.so
cp $D/libwdntt_$V.so $D/libwdntt.so
timeout 300 python scripts/tm_check.py 36 20 16 > gpurun_out/ab_${V}_check.txt 2>&1; echo check rc=$?; tail -3 gpurun_out/ab_${V}_check.txt
cp /tmp/orig.so $D/libwdntt.so
bash scripts/gpu_ab_kern.sh "base $V" "tm" 3 > gpurun_out/ab_$V.txt 2>&1; cat gpurun_out/ab_$V.txt
