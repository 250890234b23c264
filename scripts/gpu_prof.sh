# usage: bash scripts/gpu_prof.sh TAG CONFIG   (GPU box) -- ncu launch list + full captures
# of the sweep kernels: k_wspmv (a frozen sweep), k_sweep_reverse (launch SKIP_REV: a
# sweep before the seeds freeze on C4), k_sweep_forward (an early, busy sweep)
cd $GRAFT_REPO_ROOT
TAG=${1:-prof}; CFG=${2:-C4}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches_${CFG}.csv python scripts/prof_step.py $CFG 2 > gpurun_out/${TAG}_launches.log 2>&1
for KS in k_wspmv:${SKIP_W:-20} k_sweep_reverse:${SKIP_REV:-190} k_sweep_forward:3; do
  K=${KS%%:*}; S=${KS##*:}
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 \
    -o gpurun_out/${TAG}_${CFG}_${K} python scripts/prof_step.py $CFG 1 > gpurun_out/${TAG}_${K}.log 2>&1
done
ls -la gpurun_out | tail
