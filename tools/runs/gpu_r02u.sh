#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for i in 1 2; do timeout 600 python bench.py --config 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_u_c3_$i.json 2>gpurun_out/b_u_c3_$i.err; done
timeout 600 python bench.py --config 3 --no-cpu-baseline --e2e-steps 0 --steps 20 > gpurun_out/b_u_c3_20.json 2>gpurun_out/b_u_c3_20.err
timeout 900 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_u_c4.json 2>gpurun_out/b_u_c4.err
for f in gpurun_out/b_u_*.json; do python - "$f" <<'PY'
import json, sys
d = json.loads([l for l in open(sys.argv[1]) if l.startswith("{")][-1])
print(sys.argv[1], round(d["value"]), round(d["ms_per_step"], 2), d["clocks"], d.get("host_enqueue_ms_per_step"))
PY
done
