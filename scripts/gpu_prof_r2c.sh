# usage: bash scripts/gpu_prof_r2c.sh TAG   (GPU box) -- C4 launch list of bench.py's
# graph-replayed steps + the kernel captures of scripts/gpu_prof.sh
cd $GRAFT_REPO_ROOT
TAG=${1:-prof}
mkdir -p gpurun_out
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv -c 20000 \
  --log-file gpurun_out/${TAG}_bench_launches_C4.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e \
  --ttb-steps 0 --no-converge-leg --no-p1-leg > gpurun_out/${TAG}_bench_launches.log 2>&1
bash scripts/gpu_prof.sh $TAG C4
