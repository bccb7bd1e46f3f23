#!/bin/bash
# R21 check: build, migrate/plan GPU tests, MoE bench with the per-range order vs strict, plan stamps under SHARE
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
O=gpurun_out/r21; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -20 $O/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -q -x -k "${K:-migrate or share or fault or torch or plan_bitexact}" > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
timeout 900 python bench.py --config moe --steps 10 --warmup 3 --no-cpu-baseline --no-faults > $O/bench_moe.log 2>&1; echo "moe rc=$?"
timeout 900 python bench.py --config moe --steps 10 --warmup 3 --no-cpu-baseline --no-faults --strict-order > $O/bench_moe_strict.log 2>&1; echo "moe strict rc=$?"
PLAN_POLICY=3 timeout 600 python tools/prof_plan.py lstm 64 5 100 300 600 900 > $O/prof_plan_lstm_p3.txt 2>&1; echo "prof rc=$?"
