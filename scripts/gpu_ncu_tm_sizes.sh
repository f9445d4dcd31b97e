cd "$GRAFT_REPO_ROOT" 2>/dev/null || cd /root/repo
for ln in 15 14 13; do
  timeout 600 ncu --set full --clock-control none -k regex:"ntt_tm" -s 2 -c 2 -o gpurun_out/prof_tm$ln \
    python scripts/one_step.py 256 auto $ln 36 > gpurun_out/prof_tm${ln}_run.txt 2>&1; echo "ncu $ln rc=$?"
  python scripts/ncu_summary.py gpurun_out/prof_tm$ln.ncu-rep > gpurun_out/ncu_tm$ln.txt 2>&1
  rm -f gpurun_out/prof_tm$ln.ncu-rep
done
