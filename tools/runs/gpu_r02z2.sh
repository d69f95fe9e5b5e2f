#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_gpu_abi.py -q -x > gpurun_out/t_z2.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_z2.log; tail -2 gpurun_out/t_z2.log
for cfg in 4 3; do timeout 900 python bench.py --config $cfg --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_z2_$cfg.json 2>gpurun_out/b_z2_$cfg.err; done
timeout 900 python bench.py --format i420 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_z2_i420.json 2>gpurun_out/b_z2_i420.err
for f in gpurun_out/b_z2_*.json; do python - "$f" <<'PY'
import json, sys
l = [l for l in open(sys.argv[1]) if l.startswith("{")]
if not l: print(sys.argv[1], "FAILED"); sys.exit()
d = json.loads(l[-1])
print(sys.argv[1], round(d["value"]), round(d["ms_per_step"], 2), "busy", d.get("device_busy_ms_per_step"), d["clocks"]["sm_mhz"])
PY
done
