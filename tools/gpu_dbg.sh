#!/bin/bash
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,driver_version --format=csv > gpurun_out/dbg.log 2>&1
timeout 600 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest tests/test_gpu_migrate.py -x -q -k "test_tiny_fullsize_default_mechanisms" -p no:cacheprovider >> gpurun_out/dbg.log 2>&1; echo "san rc=$?"
grep -m 30 -A12 "Invalid\|misaligned\|Error" gpurun_out/dbg.log | head -80
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider > gpurun_out/dbg_parity.log 2>&1; echo "parity rc=$?"; tail -5 gpurun_out/dbg_parity.log
