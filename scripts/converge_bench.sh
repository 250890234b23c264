# usage: bash scripts/converge_bench.sh TAG  (GPU box): bench C4 / C5 in converge mode (SMOOTHE_CONVERGE=1)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for C in ${CFGS:-C5 C4}; do
  timeout 900 python bench.py --converge --config $C --steps 10 --warmup 3 --no-cpu --no-e2e --ttb-steps 80 > gpurun_out/${1}_${C}_conv.json 2> gpurun_out/${1}_${C}_conv.err
done
