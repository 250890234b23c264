# usage: CFGS="C3 C5" bash scripts/ab_libs_multi.sh TAG lib1.so ...  (GPU box)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
T=$1; shift
for C in ${CFGS:-C3 C5}; do
for r in 1 2; do
  for L in default "$@"; do
    if [ "$L" = default ]; then unset SMOOTHE_LIB; else export SMOOTHE_LIB=$PWD/$L; fi
    echo "== $C $L $(timeout 600 python scripts/ab_graph.py $C 40 SMOOTHE_X=1 2>&1 | tail -1)" >> gpurun_out/${T}_ab.log
  done
done
done
cat gpurun_out/${T}_ab.log
