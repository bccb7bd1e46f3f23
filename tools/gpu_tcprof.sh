mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 200 -p no:cacheprovider -k "tensor_cores" -s > gpurun_out/gpu_tc.log 2>&1; echo "tests rc=$?"
grep -E "worst err|passed|failed" gpurun_out/gpu_tc.log | head
python tools/prof_tc.py moe 64
python tools/prof_pilot.py moe 100 64 2>&1 | grep "us/predict"
