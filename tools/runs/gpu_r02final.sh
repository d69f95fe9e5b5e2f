#!/bin/bash
# Round-2 evidence run: full GPU suite, smoke, bench lines (c4 default = the driver's command, 4:2:0,
# 8-tap, hybrid encode, c3 latency, c5 on one GPU) and the profile round (launch list + ncu --set full).
T=${TAG:-r02z}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/t_${T}.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_${T}.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_${T}.log 2>&1; echo "SMOKE rc=$?" >> gpurun_out/smoke_${T}.log
timeout 900 python bench.py > gpurun_out/b_${T}_c4.json 2> gpurun_out/b_${T}_c4.err
timeout 900 python bench.py --format i420 > gpurun_out/b_${T}_c4_i420.json 2> gpurun_out/b_${T}_c4_i420.err
timeout 900 python bench.py --interp regular --e2e-steps 0 > gpurun_out/b_${T}_c4_8tap.json 2> gpurun_out/b_${T}_c4_8tap.err
timeout 900 python bench.py --encode --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c4_encode.json 2> gpurun_out/b_${T}_c4_encode.err
timeout 600 python bench.py --config 3 --no-cpu-baseline > gpurun_out/b_${T}_c3.json 2> gpurun_out/b_${T}_c3.err
timeout 900 python bench.py --config 5 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c5.json 2> gpurun_out/b_${T}_c5.err
TAG=$T bash tools/profile_round.sh > gpurun_out/prof_${T}.log 2>&1
tail -2 gpurun_out/t_${T}.log; tail -2 gpurun_out/smoke_${T}.log
for f in gpurun_out/b_${T}_*.json; do python - "$f" <<'PY'
import json, sys
try:
    d = json.loads([l for l in open(sys.argv[1]) if l.startswith("{")][-1])
    print(sys.argv[1], round(d["value"]), round(d["ms_per_step"], 1), d["clocks"], (d.get("e2e") or {}).get("value"),
          (d.get("roofline") or {}).get("frac"), d.get("hybrid_encode"))
except Exception as e:
    print(sys.argv[1], "ERR", e)
PY
done
