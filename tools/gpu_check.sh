#!/bin/bash
# One gpurun session: build, GPU tests (optionally filtered), smoke, optional bench lines.
#   tools/gpu_check.sh [pytest -k expr] [bench configs...]
# Writes gpurun_out/{build,tests,smoke,bench_<cfg>}.log
set -u
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
mkdir -p gpurun_out
K="${1:-}"; shift || true
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,pcie.link.gen.current,pcie.link.width.current --format=csv > gpurun_out/gpu.txt 2>&1
if [ "$K" != "none" ]; then
  if [ -n "$K" ]; then timeout 2400 python -m pytest tests -m gpu -q -x -s -k "$K" > gpurun_out/tests.log 2>&1
  else timeout 2400 python -m pytest tests -m gpu -q -s > gpurun_out/tests.log 2>&1; fi
  echo "tests rc=$?"; tail -5 gpurun_out/tests.log
fi
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -3 gpurun_out/smoke.log
for cfg in "$@"; do
  timeout 900 python bench.py --config "$cfg" --steps 10 --warmup 3 > gpurun_out/bench_$cfg.log 2>&1
  echo "bench $cfg rc=$?"; tail -c 600 gpurun_out/bench_$cfg.log; echo
done
