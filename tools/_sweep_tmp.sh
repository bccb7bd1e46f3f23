cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -x -k "plan or migrate or memo or edges or residency" > gpurun_out/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/tests.log
python tools/prof_plan.py lstm 64 5 100 300 600 900 > gpurun_out/prof_plan.txt 2>&1
head -5 gpurun_out/prof_plan.txt | cut -c1-400
timeout 900 python bench.py --config lstm --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_lstm.log 2>&1; echo "bench rc=$?"
