cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python tools/prof_plan.py lstm 64 5 100 300 600 900 > gpurun_out/prof_plan.txt 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:plan_kernel -c 1 -o gpurun_out/plan_lstm python tools/prof_plan.py lstm 64 5 > gpurun_out/ncu_plan.log 2>&1
nsys_none=1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/plan_launches.csv python tools/prof_plan.py lstm 64 5 > /dev/null 2>&1
cat gpurun_out/prof_plan.txt
