# usage: bash scripts/gpu_prof_f.sh TAG  (GPU box): full captures of a peak forward sweep, k_wbuild and the final S pass
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
TAG=${1:-f}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sweep_forward -s 18 -c 1 \
  -o gpurun_out/${TAG}_C4_k_sweep_forward_18 python scripts/prof_step.py C4 1 > gpurun_out/${TAG}_f18.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_wbuild -c 1 \
  -o gpurun_out/${TAG}_C4_k_wbuild python scripts/prof_step.py C4 1 > gpurun_out/${TAG}_wb.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sweep_reverse -s 207 -c 1 \
  -o gpurun_out/${TAG}_C4_k_sweep_reverse_S python scripts/prof_step.py C4 1 > gpurun_out/${TAG}_rs.log 2>&1
ls gpurun_out | grep $TAG
