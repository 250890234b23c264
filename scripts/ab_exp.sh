# A/B timing of alternative builds: bash scripts/ab_exp.sh lib1.so lib2.so ...  (GPU box)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
i=0
for L in default "$@"; do
  if [ "$L" = default ]; then unset SMOOTHE_LIB; else export SMOOTHE_LIB=$PWD/$L; fi
  timeout 600 python bench.py --steps 4 --warmup 3 --no-e2e --no-cpu > gpurun_out/ab_$i.json 2> gpurun_out/ab_$i.err
  python -c "
import json,sys; d=json.load(open('gpurun_out/ab_$i.json')); p=d['phases_ms_per_step']
print('$L', round(d['ms_per_step'],1), 'fwd/sweep', round(p['forward']/207,3), 'rev/sweep', round(p['reverse']/207,3), 'decode', round(p['decode'],1))" || tail -3 gpurun_out/ab_$i.err
  i=$((i+1))
done
