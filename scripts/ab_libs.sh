# usage: bash scripts/ab_libs.sh TAG CFG lib1.so lib2.so ...  (GPU box): graph-step A/B of builds,
# each in its own process (SMOOTHE_LIB), alternated twice
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=$1; C=$2; shift 2
for r in 1 2; do
  for L in default "$@"; do
    if [ "$L" = default ]; then unset SMOOTHE_LIB; else export SMOOTHE_LIB=$PWD/$L; fi
    echo "== $L" >> gpurun_out/${T}_ab.log
    timeout 600 python scripts/ab_graph.py $C 20 SMOOTHE_X=1 2>&1 | tail -1 >> gpurun_out/${T}_ab.log
  done
done
cat gpurun_out/${T}_ab.log
