mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider -k "traversal or decode" > gpurun_out/gpu_trav.log 2>&1; echo "rc=$?"
tail -20 gpurun_out/gpu_trav.log
