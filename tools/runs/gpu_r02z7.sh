#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 900 python bench.py --encode --no-cpu-baseline --e2e-steps 2 > gpurun_out/b_z7.json 2>gpurun_out/b_z7.err
python - <<'PY'
import json
l = [x for x in open("gpurun_out/b_z7.json") if x.startswith("{")]
if not l: print(open("gpurun_out/b_z7.err").read()[-1500:])
else:
    d = json.loads(l[-1]); print(d["value"], d["e2e"]["value"], d.get("e2e_package"), d.get("hybrid_encode"))
PY
