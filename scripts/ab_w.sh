# usage: bash scripts/ab_w.sh TAG   (GPU box): GPU tests, then the bench with and
# without the frozen-sweep W path (SMOOTHE_REV_W=0) on C2-C5
cd $GRAFT_REPO_ROOT
TAG=${1:-abw}
mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > gpurun_out/${TAG}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${TAG}_tests.log
for C in C2 C3 C5 C4; do
  for W in 1 0; do
    SMOOTHE_REV_W=$W timeout 900 python bench.py --config $C --steps 10 --warmup 3 --no-cpu --no-e2e --ttb-steps 0 > gpurun_out/${TAG}_${C}_w$W.json 2> gpurun_out/${TAG}_${C}_w$W.err
  done
done
tail -n 3 gpurun_out/${TAG}_tests.log
