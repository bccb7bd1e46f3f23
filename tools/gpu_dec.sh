mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x --timeout 300 -p no:cacheprovider > gpurun_out/gpu_parity.log 2>&1; echo "parity rc=$?"
tail -3 gpurun_out/gpu_parity.log
for cfg in moe af lstm; do python tools/prof_pilot.py $cfg 50 64 2>&1 | grep "us/predict"; done
python tools/prof_pilot.py moe 200 1 2>&1 | grep "us/predict"
