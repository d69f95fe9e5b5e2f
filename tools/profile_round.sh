#!/bin/bash
# Round profile evidence on the GPU box (one GPU): the launch list of a c4 bench
# step and one `ncu --set full` capture of each hot kernel.  Output: gpurun_out/prof_<tag>_*
# Summarise here with: python tools/ncu_summary.py gpurun_out/prof_<tag>_launches.csv profiles/<round>_ncu_summary.md gpurun_out/prof_<tag>_*.ncu-rep
set -x
T=${TAG:-r01}
B="python bench.py --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/prof_${T}_launches.csv $B > gpurun_out/prof_${T}_launches.log 2>&1
for k in k_resblock:10 k_recon_step:30 k_uptail2:3 k_conv_rot:5; do
  n=${k%%:*}; s=${k##*:}
  ncu --set full --import-source on --clock-control none -k regex:$n -s $s -c 1 -o gpurun_out/prof_${T}_$n $B > gpurun_out/prof_${T}_$n.log 2>&1
done
ls -la gpurun_out/
