#!/bin/bash
# one --set full capture of k_resblock (16 jobs of 1280x720) with source counters
ncu --set full --import-source on --clock-control none -k regex:k_resblock -s 10 -c 1 -o gpurun_out/rb python bench.py --streams 16 --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu_rb.log 2>&1
