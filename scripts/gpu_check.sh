# usage: bash scripts/gpu_check.sh TAG [pytest-args...]   (runs on the GPU box)
cd $GRAFT_REPO_ROOT
TAG=${1:-run}; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/${TAG}_nvsmi.txt 2>&1
nproc >> gpurun_out/${TAG}_nvsmi.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${TAG}_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider "$@" > gpurun_out/${TAG}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${TAG}_tests.log
for C in C2 C3 C5; do
  timeout 600 python bench.py --config $C --steps 10 --warmup 3 --no-cpu --no-e2e --ttb-steps 0 --no-converge-leg > gpurun_out/${TAG}_bench_$C.json 2> gpurun_out/${TAG}_bench_$C.err
done
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench_C4.json 2> gpurun_out/${TAG}_bench_C4.err
tail -n 3 gpurun_out/${TAG}_smoke.log gpurun_out/${TAG}_tests.log
