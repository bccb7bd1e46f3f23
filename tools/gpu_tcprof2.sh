python tools/prof_tc.py moe 64
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q --timeout 200 -p no:cacheprovider -k "tensor_cores" -s 2>&1 | grep -E "worst err|passed|failed"
