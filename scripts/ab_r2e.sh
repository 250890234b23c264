# usage: bash scripts/ab_r2e.sh TAG   (GPU box): switch-node A/B, schedule identity tests, long-run profile
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=$1
timeout 600 python scripts/ab_graph.py C4 20 SMOOTHE_RSWITCH=1 SMOOTHE_RSWITCH=0 > gpurun_out/${T}_ab.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "schedule_variants or c4_graph_replay or converge_mode" > gpurun_out/${T}_tests.log 2>&1
timeout 1500 python scripts/long_run_profile.py C4 500 5 > gpurun_out/${T}_long.log 2>&1
tail -n 3 gpurun_out/${T}_ab.log gpurun_out/${T}_tests.log
