#!/bin/bash
# Live anatomy of copy_records_tma_kernel inside the bench step (DYO_COPY_STAMPS=1), with and
# without the max shared-memory carveout request.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in 0 1; do for cfg in moe af; do
  DYO_TMA_CARVEOUT=$v DYO_COPY_STAMPS=1 DYO_COPY_STAMPS_OUT=gpurun_out/copy_stamps_${cfg}_c$v.json timeout 600 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/stamps_bench_${cfg}_c$v.json 2>gpurun_out/stamps_bench_${cfg}_c$v.err
  echo "$cfg carveout=$v rc=$?"
  python -c "import json;d=json.loads(open('gpurun_out/stamps_bench_${cfg}_c$v.json').read().strip().splitlines()[-1]);r=d['roofline'];print(d['value'],d['ms_per_step'],r['achieved'],r['frac'],r['avg_launch_us'],r.get('in_kernel'))"
done; done 2>&1 | tee gpurun_out/stamps.txt
