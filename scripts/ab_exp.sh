# A/B timing of alternative builds: CFGS="C4 C5" bash scripts/ab_exp.sh lib1.so lib2.so ...  (GPU box)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for C in ${CFGS:-C4}; do
i=0
for L in default "$@"; do
  if [ "$L" = default ]; then unset SMOOTHE_LIB; else export SMOOTHE_LIB=$PWD/$L; fi
  timeout 600 python bench.py --config $C --steps ${STEPS:-4} --warmup 3 --no-e2e --no-cpu --ttb-steps 0 > gpurun_out/ab_${C}_$i.json 2> gpurun_out/ab_${C}_$i.err
  python -c "
import json,sys; d=json.load(open('gpurun_out/ab_${C}_$i.json')); p=d['phases_ms_per_step']
k=d.get('sweep_kernel_ms_per_step',{})
print('$C', '$L', round(d['ms_per_step'],2), 'fwd', round(p['forward'],2), 'rev', round(p['reverse'],2), 'decode', round(p['decode'],2), 'kernels', {a: round(b,2) for a,b in k.items()})" || tail -3 gpurun_out/ab_${C}_$i.err
  i=$((i+1))
done
done
