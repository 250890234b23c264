# usage: bash scripts/gpu_late.sh TAG N SKIP (GPU box): launch list + full capture of a late-step plain reverse sweep
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=$1; N=${2:-300}; S=${3:-150}
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${T}_late_launches_C4.csv python scripts/late_prof.py C4 $N > gpurun_out/${T}_late.log 2>&1
timeout 900 ncu --profile-from-start off --set full --clock-control none --import-source on -k regex:k_sweep_reverse -s $S -c 1 \
  -o gpurun_out/${T}_late_rev python scripts/late_prof.py C4 $N > gpurun_out/${T}_late_rev.log 2>&1
tail -2 gpurun_out/${T}_late.log
