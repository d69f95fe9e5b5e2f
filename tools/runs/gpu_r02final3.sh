#!/bin/bash
# Round-2 closing evidence, second pass (after the recon edge permutes and the per-shape SR batch):
# smoke, every bench line (c4 default = the driver's command, global selection, 4:2:0, 8-tap, hybrid
# encode, c3 latency, c5 on one GPU, the CPU-oracle reference arm), the launch list and ncu --set full
# captures of the hot kernels.  (The full GPU suite ran on this code in tools/runs/gpu_r02zs.sh: 134 passed.)
T=${TAG:-r02zt}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_${T}.log 2>&1; echo "SMOKE rc=$?" >> gpurun_out/smoke_${T}.log
timeout 900 python bench.py > gpurun_out/b_${T}_c4.json 2> gpurun_out/b_${T}_c4.err
timeout 900 python bench.py --config 5 --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c5.json 2> gpurun_out/b_${T}_c5.err
timeout 900 python bench.py --select global --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c4_global.json 2> gpurun_out/b_${T}_c4_global.err
timeout 900 python bench.py --format i420 > gpurun_out/b_${T}_c4_i420.json 2> gpurun_out/b_${T}_c4_i420.err
timeout 900 python bench.py --interp regular --e2e-steps 0 > gpurun_out/b_${T}_c4_8tap.json 2> gpurun_out/b_${T}_c4_8tap.err
timeout 900 python bench.py --encode --no-cpu-baseline --e2e-steps 0 > gpurun_out/b_${T}_c4_encode.json 2> gpurun_out/b_${T}_c4_encode.err
timeout 600 python bench.py --config 3 --no-cpu-baseline > gpurun_out/b_${T}_c3.json 2> gpurun_out/b_${T}_c3.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/b_${T}_reference.json 2> gpurun_out/b_${T}_reference.err
TAG=$T bash tools/profile_round.sh > gpurun_out/prof_${T}.log 2>&1
tail -2 gpurun_out/smoke_${T}.log
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
