#!/bin/bash
# Live anatomy of copy_records_tma_kernel inside the bench step (DYO_COPY_STAMPS=1).
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for cfg in moe af; do
  DYO_COPY_STAMPS=1 DYO_COPY_STAMPS_OUT=gpurun_out/copy_stamps_$cfg.json timeout 600 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/stamps_bench_$cfg.json 2>gpurun_out/stamps_bench_$cfg.err
  echo "$cfg rc=$?"; python -c "import json;d=json.load(open('gpurun_out/copy_stamps_$cfg.json'));print(json.dumps(d['median']));print(json.dumps(d['median_over_launches_ge_20us']))"
  python -c "import json;d=json.loads(open('gpurun_out/stamps_bench_$cfg.json').read().strip().splitlines()[-1]);r=d['roofline'];print(d['value'],r['achieved'],r['frac'],r['avg_launch_us'])"
done 2>&1 | tee gpurun_out/stamps.txt
