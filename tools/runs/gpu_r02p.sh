#!/bin/bash
# 8-tap MC: c4 bench lines (regular, switchable) + one ncu --set full capture of k_recon8<3>
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python bench.py --interp regular --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_p_regular.json 2> gpurun_out/bench_p_regular.err
timeout 600 python bench.py --interp switchable --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_p_switch.json 2> gpurun_out/bench_p_switch.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_recon8 --launch-skip 20 -c 1 -o gpurun_out/ncu_recon8 -f \
  python bench.py --interp regular --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_p.log 2>&1
python - <<'PY'
import json
for f in ("gpurun_out/bench_p_regular.json", "gpurun_out/bench_p_switch.json"):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, round(d["value"]), d["ms_per_step"], d["rooflines"]["recon"], d["clocks"])
    except Exception as e:
        print(f, "ERR", e)
PY
tail -3 gpurun_out/ncu_p.log
