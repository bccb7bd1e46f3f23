mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 200 -p no:cacheprovider -k "tensor_cores" -s > gpurun_out/gpu_tc.log 2>&1; echo "rc=$?"
grep -E "worst|passed|failed|Error|assert" gpurun_out/gpu_tc.log | head -30
