# usage: bash scripts/gpu_final.sh TAG  (GPU box): smoke, GPU suite, bench lines C2-C5 (+ reference arm),
# ncu launch list of the C4 bench command
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=${1:-final}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/${T}_nvsmi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/${T}_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/${T}_tests.log
timeout 1200 python bench.py > gpurun_out/${T}_bench_C4.json 2> gpurun_out/${T}_bench_C4.err
for C in C2 C3 C5; do
  timeout 900 python bench.py --config $C > gpurun_out/${T}_bench_$C.json 2> gpurun_out/${T}_bench_$C.err
done
timeout 900 python bench.py --impl reference > gpurun_out/${T}_bench_reference.json 2> gpurun_out/${T}_bench_reference.err
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv -c 20000 \
  --log-file gpurun_out/${T}_bench_launches_C4.csv python bench.py --steps 2 --warmup 3 --no-cpu --no-e2e \
  --ttb-steps 0 --no-converge-leg --no-p1-leg > gpurun_out/${T}_bench_launches.log 2>&1
tail -n 2 gpurun_out/${T}_smoke.log gpurun_out/${T}_tests.log
