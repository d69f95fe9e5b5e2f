#!/bin/bash
# Round-2 closing evidence on the final code: full GPU suite, smoke, every bench line (c4 default = the
# driver's command, global selection, 4:2:0, 8-tap, hybrid encode, c3 latency, c5 on one GPU), the launch
# list + ncu --set full captures of the hot kernels, compute-sanitizer on c1, the host CPU.
T=${TAG:-r02zz}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
lscpu > gpurun_out/lscpu_${T}.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/t_${T}.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_${T}.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_${T}.log 2>&1; echo "SMOKE rc=$?" >> gpurun_out/smoke_${T}.log
timeout 900 python bench.py > gpurun_out/b_${T}_c4.json 2> gpurun_out/b_${T}_c4.err
timeout 900 python bench.py --select global --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c4_global.json 2> gpurun_out/b_${T}_c4_global.err
timeout 900 python bench.py --format i420 > gpurun_out/b_${T}_c4_i420.json 2> gpurun_out/b_${T}_c4_i420.err
timeout 900 python bench.py --interp regular --e2e-steps 0 > gpurun_out/b_${T}_c4_8tap.json 2> gpurun_out/b_${T}_c4_8tap.err
timeout 900 python bench.py --encode --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c4_encode.json 2> gpurun_out/b_${T}_c4_encode.err
timeout 600 python bench.py --config 3 --no-cpu-baseline > gpurun_out/b_${T}_c3.json 2> gpurun_out/b_${T}_c3.err
timeout 900 python bench.py --config 5 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c5.json 2> gpurun_out/b_${T}_c5.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/b_${T}_reference.json 2> gpurun_out/b_${T}_reference.err
TAG=$T bash tools/profile_round.sh > gpurun_out/prof_${T}.log 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_c1.py > gpurun_out/san_${T}_$tool.log 2>&1
  echo "$tool exit $?" >> gpurun_out/san_${T}_summary.txt
  tail -3 gpurun_out/san_${T}_$tool.log >> gpurun_out/san_${T}_summary.txt
done
tail -2 gpurun_out/t_${T}.log; tail -2 gpurun_out/smoke_${T}.log; cat gpurun_out/san_${T}_summary.txt
for f in gpurun_out/b_${T}_*.json; do python - "$f" <<'PY'
import json, sys
try:
    d = json.loads([l for l in open(sys.argv[1]) if l.startswith("{")][-1])
    print(sys.argv[1], round(d["value"]), round(d["ms_per_step"], 1), d.get("clocks"), (d.get("e2e") or {}).get("value"),
          (d.get("roofline") or {}).get("frac"), d.get("hybrid_encode"))
except Exception as e:
    print(sys.argv[1], "ERR", e)
PY
done
