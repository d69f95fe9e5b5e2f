#!/bin/bash
# Re-entry check: full GPU suite, smoke and the default bench line on the restored tree.
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/t_zj.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_zj.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_zj.log 2>&1; echo "SMOKE rc=$?" >> gpurun_out/smoke_zj.log
timeout 900 python bench.py > gpurun_out/b_zj_c4.json 2> gpurun_out/b_zj_c4.err
tail -2 gpurun_out/t_zj.log; tail -2 gpurun_out/smoke_zj.log
python - <<'PY'
import json
d = json.loads([l for l in open("gpurun_out/b_zj_c4.json") if l.startswith("{")][-1])
print(round(d["value"]), round(d["ms_per_step"], 1), d["clocks"], {k: round(v.get("ms_per_step", 0), 2) for k, v in d["rooflines"].items()})
PY
