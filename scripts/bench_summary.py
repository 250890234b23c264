"""One line per bench JSON file: ms/step, value, sweep kernel ms, phases."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f.split("/")[-1], round(d["ms_per_step"], 2), "%.3g" % d["value"],
              {k: round(v, 2) for k, v in d["sweep_kernel_ms_per_step"].items()},
              {k: round(v, 2) for k, v in d["phases_ms_per_step"].items()})
    except Exception as e:  # noqa: BLE001
        print(f, "ERR", e)
