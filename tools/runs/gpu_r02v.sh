#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
timeout 600 python bench.py --config 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_v_c3.json 2>gpurun_out/b_v_c3.err
NS_BENCH_NOPROF=1 timeout 600 python bench.py --config 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_v_c3_noprof.json 2>gpurun_out/b_v_c3_noprof.err
timeout 600 python bench.py --config 3 --no-cpu-baseline --e2e-steps 0 --warmup 10 > gpurun_out/b_v_c3_w10.json 2>gpurun_out/b_v_c3_w10.err
for f in gpurun_out/b_v_*.json; do python - "$f" <<'PY'
import json, sys
l = [l for l in open(sys.argv[1]) if l.startswith("{")]
if not l: print(sys.argv[1], "FAILED", open(sys.argv[1].replace(".json", ".err")).read()[-600:]); sys.exit()
d = json.loads(l[-1])
print(sys.argv[1], round(d["ms_per_step"], 2), d.get("step_ms"), d.get("host_enqueue_ms_per_step"))
PY
done
