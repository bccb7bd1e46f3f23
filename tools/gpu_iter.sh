#!/bin/bash
# Iteration loop: GPU tests (all) + pilot stamps.
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -p no:cacheprovider > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"
tail -3 gpurun_out/gpu_tests.log
for cfg in moe af tiny; do timeout 120 python tools/prof_pilot.py $cfg 200 1; done > gpurun_out/pilot_stamps.txt 2>&1
cat gpurun_out/pilot_stamps.txt
