#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "logits or decode or encode" 2>&1 | tail -3
for c in "moe 200 1" "tiny 200 1" "af 100 1" "moe 100 8" "moe 50 64"; do timeout 60 python tools/prof_pilot.py $c; done 2>&1 | tee gpurun_out/pilot_lat.txt
