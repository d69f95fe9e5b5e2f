LIBS="default env:NS_SR_BATCH=24 env:NS_SR_BATCH=32 env:NS_SR_BATCH=12 default env:NS_SR_BATCH=24 env:NS_SR_BATCH=32 env:NS_SR_BATCH=12" bash tools/ab_libs.sh > gpurun_out/ab1.txt 2>&1
