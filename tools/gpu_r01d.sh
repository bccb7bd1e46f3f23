#!/bin/bash
# Round-1 re-measure at HEAD: GPU tests, bench lines (moe headline, lstm, af), ncu launch list,
# TMA-copy DRAM traffic per algorithmic byte, ncu --set full of the copy kernel and the pilot.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1; echo "build rc=$?"
timeout 1200 python -m pytest tests -m gpu -q --timeout 400 -p no:cacheprovider > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?"
tail -2 gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -c 1500 gpurun_out/bench.json; tail -3 gpurun_out/bench.err
for cfg in lstm af; do
  timeout 900 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/bench_$cfg.json 2> gpurun_out/bench_$cfg.err; echo "$cfg rc=$?"
  tail -2 gpurun_out/bench_$cfg.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
DYO_COPY_LOG=gpurun_out/copy_log.txt timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:copy_records -c 400 --csv --log-file gpurun_out/copy_traffic.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_copy.log 2>&1; echo "ncu traffic rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"copy_records" -s 30 -c 4 -o gpurun_out/prof_full -f python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"pilot_kernel" -s 10 -c 2 -o gpurun_out/prof_pilot -f python tools/prof_pilot.py moe 20 1 > gpurun_out/ncu_pilot.log 2>&1; echo "ncu pilot rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"plan_kernel" -s 2 -c 1 -o gpurun_out/prof_plan -f python tools/prof_plan.py moe 1 3 > gpurun_out/ncu_plan.log 2>&1; echo "ncu plan rc=$?"
for cfg in moe af tiny; do timeout 120 python tools/prof_pilot.py $cfg 200 1; done > gpurun_out/pilot_stamps.txt 2>&1
