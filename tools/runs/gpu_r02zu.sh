#!/bin/bash
# c4 SR batch size A/B (env NS_SR_BATCH; default = per-shape 16 at 720p)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
LIBS="default env:NS_SR_BATCH=24 env:NS_SR_BATCH=32 default env:NS_SR_BATCH=24 env:NS_SR_BATCH=32" bash tools/ab_libs.sh
