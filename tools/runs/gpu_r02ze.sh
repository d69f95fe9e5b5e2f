#!/bin/bash
# speed-of-light probe: uptail2 without the per-output epilogue math (wrong output, timing only)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || exit 1
LIBS="default tools/bin/lib_up_exp1.so default tools/bin/lib_up_exp1.so" bash tools/ab_libs.sh
