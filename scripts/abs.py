"""Summarise A/B bench lines: python scripts/abs.py gpurun_out/TAG_*.json"""
import json
import sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f, "ERR", e)
        continue
    sk = d.get("sweep_kernel_ms_per_step", {})
    r = d.get("roofline", {})
    print(f"{f.split('/')[-1]:28s} ms/step={d['ms_per_step']:8.3f} value={d['value']:.4g} "
          f"fwd={sk.get('forward', 0):6.2f} rev={sk.get('reverse', 0):6.2f} frozen={sk.get('frozen', 0):6.2f} "
          f"{r.get('kernel')} frac={r.get('frac', 0):.3f} avg_us={1e3 * r.get('avg_launch_ms', 0):.1f}")
