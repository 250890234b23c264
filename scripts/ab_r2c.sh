# usage: bash scripts/ab_r2c.sh TAG   (GPU box): persistent k_wspmv / forward skip A/B + parity subset
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=$1
B="timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --ttb-steps 0 --no-converge-leg --no-p1-leg"
$B > gpurun_out/${T}_C4_new.json 2> gpurun_out/${T}_C4_new.err
SMOOTHE_WSPMV_PERSIST=0 $B > gpurun_out/${T}_C4_p0.json 2> gpurun_out/${T}_C4_p0.err
SMOOTHE_FSKIP=0 $B > gpurun_out/${T}_C4_f0.json 2> gpurun_out/${T}_C4_f0.err
$B --config C5 > gpurun_out/${T}_C5_new.json 2> gpurun_out/${T}_C5_new.err
SMOOTHE_WSPMV_PERSIST=1 $B --config C5 > gpurun_out/${T}_C5_p1.json 2> gpurun_out/${T}_C5_p1.err
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "c4_graph_replay or dead_gradient or frozen_sweeps or debug_step_after_graph or change_propagation or seed_sharding or converge_mode" > gpurun_out/${T}_tests.log 2>&1
tail -3 gpurun_out/${T}_tests.log
