# usage: bash scripts/ab_w2.sh TAG "CONFIGS"  (GPU box): bench with / without the W path + C4 launch list
cd $GRAFT_REPO_ROOT
TAG=${1:-abw}; CF=${2:-"C5 C4"}
mkdir -p gpurun_out
for C in $CF; do
  for W in 1 0; do
    SMOOTHE_REV_W=$W timeout 900 python bench.py --config $C --steps 10 --warmup 3 --no-cpu --no-e2e --ttb-steps 0 > gpurun_out/${TAG}_${C}_w$W.json 2> gpurun_out/${TAG}_${C}_w$W.err
  done
done
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launch_C4.csv python scripts/prof_step.py C4 2 > gpurun_out/${TAG}_launch.log 2>&1
