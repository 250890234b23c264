# compute-sanitizer passes over the library (GPU box): one summary line per tool.
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck initcheck synccheck; do
  for w in small frozen; do
    if [ $tool = initcheck ]; then export SAN_NODUMP=1; else unset SAN_NODUMP; fi
    timeout 900 $CS --tool $tool --error-exitcode 7 --print-limit 20 python scripts/sanitize_run.py $w \
      > gpurun_out/san_${tool}_$w.log 2>&1
    echo "$tool $w rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|hazard' gpurun_out/san_${tool}_$w.log | tail -2 | tr '\n' ' ')"
  done
done
timeout 900 $CS --tool memcheck --error-exitcode 7 python scripts/sanitize_run.py mlp > gpurun_out/san_memcheck_mlp.log 2>&1
echo "memcheck mlp rc=$? $(grep -E 'ERROR SUMMARY' gpurun_out/san_memcheck_mlp.log | tail -1)"
