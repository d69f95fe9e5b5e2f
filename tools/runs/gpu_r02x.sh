#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python bench.py --config 3 > gpurun_out/b_x_c3.json 2>gpurun_out/b_x_c3.err
python - <<'PY'
import json
d = json.loads([l for l in open("gpurun_out/b_x_c3.json") if l.startswith("{")][-1])
print(round(d["ms_per_step"], 2), d.get("step_ms"), d.get("host_enqueue_ms_per_step"), d.get("e2e", {}).get("value"), d["clocks"])
PY
