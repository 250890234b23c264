# usage: bash scripts/gpu_prof_w.sh TAG [SKIP1 SKIP2]  (GPU box): C4 launch list + full captures of two k_wspmv launches
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-w}; S1=${2:-20}; S2=${3:-110}
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_launches_C4.csv python scripts/prof_step.py C4 1 > gpurun_out/${TAG}_launches.log 2>&1
for S in $S1 $S2; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_wspmv -s $S -c 1 \
    -o gpurun_out/${TAG}_C4_k_wspmv_$S python scripts/prof_step.py C4 1 > gpurun_out/${TAG}_w$S.log 2>&1
done
