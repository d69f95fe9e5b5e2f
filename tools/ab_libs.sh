#!/bin/bash
# A/B of library variants on one box: bench (device path only) per NS_LIB; prints value and family ms.
# usage: LIBS="default tools/bin/lib_a.so ..." bash tools/ab_libs.sh
for L in ${LIBS:-default}; do
  unset NS_SR_BATCH NS_OVERLAP_PARTS NS_HOST_GROUPS
  case "$L" in
    default) unset NS_LIB ;;
    env:*) unset NS_LIB; export ${L#env:} ;;
    *) export NS_LIB=$PWD/$L ;;
  esac
  python bench.py --steps ${STEPS:-5} --warmup 3 --no-cpu-baseline --e2e-steps 0 $BENCH_ARGS > gpurun_out/ab.json 2>gpurun_out/ab.err
  python - "$L" <<'PY'
import json, sys
l = [x for x in open("gpurun_out/ab.json") if x.startswith("{")]
if not l:
    print(sys.argv[1], "FAILED", open("gpurun_out/ab.err").read()[-800:]); sys.exit()
d = json.loads(l[-1])
fam = {k: round(v.get("ms_per_step", 0), 2) for k, v in d.get("rooflines", {}).items() if v.get("ms_per_step")}
print(sys.argv[1], round(d["value"]), round(d["ms_per_step"], 1), d["clocks"]["sm_mhz"], fam)
PY
done
