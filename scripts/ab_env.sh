# usage: VAR=SMOOTHE_X VALS="1 0" CFGS="C2 C5" bash scripts/ab_env.sh TAG   (GPU box)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for C in ${CFGS:-C4}; do
  for v in ${VALS:-1 0}; do
    env $VAR=$v timeout 900 python bench.py --config $C --steps ${STEPS:-10} --warmup 3 --no-cpu --no-e2e --ttb-steps 0 > gpurun_out/${1}_${C}_$v.json 2> gpurun_out/${1}_${C}_$v.err
  done
done
