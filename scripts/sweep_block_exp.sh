cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for B in 64 128 256; do
  SMOOTHE_SWEEP_BLOCK=$B timeout 600 python bench.py --steps 5 --warmup 3 --no-e2e --no-cpu > gpurun_out/blk_$B.json 2> gpurun_out/blk_$B.err
done
python - <<'PY'
import json
for B in (64,128,256):
    try:
        d=json.load(open(f"gpurun_out/blk_{B}.json"))
        print(B, round(d["ms_per_step"],1), {k: round(v,1) for k,v in d["phases_ms_per_step"].items()})
    except Exception as e: print(B, "ERR", e)
PY
