#!/bin/bash
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
for L in default tools/bin/lib_jpeg8.so tools/bin/lib_jpeg16.so; do
  if [ "$L" = default ]; then unset NS_LIB; else export NS_LIB=$PWD/$L; fi
  timeout 900 python bench.py --encode --no-cpu-baseline --e2e-steps 0 --steps 2 > gpurun_out/b_z6.json 2>gpurun_out/b_z6.err
  python - "$L" <<'PY'
import json, sys
l = [x for x in open("gpurun_out/b_z6.json") if x.startswith("{")]
d = json.loads(l[-1]) if l else {}
print(sys.argv[1], d.get("hybrid_encode"))
PY
done
unset NS_LIB
timeout 600 python -m pytest tests/test_gpu_hybrid.py -q -x > gpurun_out/t_z6.log 2>&1; echo "TESTS rc=$?" >> gpurun_out/t_z6.log; tail -2 gpurun_out/t_z6.log
