# usage: bash scripts/gpu_prof_mlp.sh TAG   (GPU box) -- C5 launch list + full captures of the MLP tensor-core kernels
cd $GRAFT_REPO_ROOT
TAG=${1:-prof}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches_C5.csv python scripts/prof_step.py C5 2 > gpurun_out/${TAG}_launches.log 2>&1
for K in k_mlp_l1_tc k_mlp_l1_back_tc k_sweep_reverse; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 \
    -o gpurun_out/${TAG}_C5_${K} python scripts/prof_step.py C5 1 > gpurun_out/${TAG}_${K}.log 2>&1
done
ls -la gpurun_out | tail
