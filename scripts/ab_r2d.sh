# usage: bash scripts/ab_r2d.sh TAG   (GPU box): pipelined k_wspmv A/B + schedule identity tests
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=$1
timeout 600 python scripts/ab_graph.py C4 20 SMOOTHE_WFUSE=1 SMOOTHE_WFUSE=0 > gpurun_out/${T}_ab.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "schedule_variants or c4_graph_replay or dead_gradient or frozen_sweeps" > gpurun_out/${T}_tests.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${T}_launches_C4.csv python scripts/prof_step.py C4 1 > gpurun_out/${T}_launches.log 2>&1
tail -n 3 gpurun_out/${T}_ab.log gpurun_out/${T}_tests.log
