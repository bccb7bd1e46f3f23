#!/bin/bash
# Batch-1 pilot latency: phase stamps + one ncu --set full capture of pilot_kernel (MoE, P512).
mkdir -p gpurun_out
for cfg in moe af tiny; do timeout 120 python tools/prof_pilot.py $cfg 200 1; done > gpurun_out/pilot_stamps.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pilot_kernel" -s 10 -c 2 -o gpurun_out/prof_pilot -f python tools/prof_pilot.py moe 20 1 > gpurun_out/ncu_pilot.log 2>&1; echo "ncu pilot rc=$?"
