mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_migrate.py -m gpu -q --timeout 400 -p no:cacheprovider -k "lstm" > gpurun_out/gpu_lstm.log 2>&1; echo "rc=$?"
tail -40 gpurun_out/gpu_lstm.log
