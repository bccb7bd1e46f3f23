#!/bin/bash
# Round measurement: GPU tests, smoke, bench lines (all configs), reference arm, launch list,
# ncu captures of the top kernels. Outputs under gpurun_out/r02/.
cd "${GRAFT_REPO_ROOT:-$(dirname "$0")/..}"
O=gpurun_out/${OUT:-r02}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1 || { tail -20 $O/build.log; exit 1; }
nvidia-smi > $O/nvidia_smi.txt 2>&1; nvidia-smi topo -m > $O/topo.txt 2>&1
if [ "${SKIP_TESTS:-0}" != 1 ]; then
  timeout 2400 python -m pytest tests -m gpu -q > $O/tests.log 2>&1; echo "tests rc=$?"; tail -2 $O/tests.log
fi
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"
for cfg in ${CFGS:-moe lstm tree af}; do
  timeout 1200 python bench.py --config $cfg --steps 10 --warmup 3 > $O/bench_$cfg.log 2>&1; echo "bench $cfg rc=$?"
done
# B*0 demonstration: the AlphaFold-shaped trace at 16 GiB with SHARE (R20), exposed vs the compute-only harness
timeout 1200 python bench.py --config af --policy 3 --budget-gib 16 --steps 6 --warmup 3 --no-cpu-baseline > $O/bench_af16_share.log 2>&1; echo "bench af16 share rc=$?"
timeout 900 python bench.py --config moe --steps 10 --warmup 3 --no-cpu-baseline --no-faults --strict-order > $O/bench_moe_strict.log 2>&1; echo "bench moe strict rc=$?"
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.log 2>&1; echo "ref rc=$?"
if [ "${SKIP_NCU:-0}" != 1 ]; then
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_moe.csv \
      python bench.py --config moe --steps 2 --warmup 1 --no-cpu-baseline --no-faults > $O/ncu_launch.log 2>&1; echo "ncu launches rc=$?"
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:copy_records_tma -s 40 -c 1 -o $O/copy_full \
      python bench.py --config moe --steps 2 --warmup 1 --no-cpu-baseline --no-faults > $O/ncu_copy.log 2>&1; echo "ncu copy rc=$?"
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:plan_kernel -c 1 -o $O/plan_full \
      python tools/prof_plan.py lstm 64 5 > $O/ncu_plan.log 2>&1; echo "ncu plan rc=$?"
  timeout 900 ncu --set full --import-source on --clock-control none -k regex:pilot_kernel -s 5 -c 1 -o $O/pilot_b64_full \
      python tools/sweep_batch_pilot.py moe 64 > $O/ncu_pilot.log 2>&1; echo "ncu pilot rc=$?"
  cp paper_conf_hpca_renxyzlnwxl24_b200/_build/*.o $O/ 2>/dev/null
fi
python tools/bench_labels.py > $O/labels.json 2> $O/labels.err; echo "labels rc=$?"
python tools/bench_torch.py > $O/torch_rt.json 2> $O/torch_rt.err; echo "torch rc=$?"
