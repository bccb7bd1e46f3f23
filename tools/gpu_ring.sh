#!/bin/bash
# TMA copy ring sweep (DYO_TMA_RING x DYO_TMA_CTAS_PER_SM): live roofline of
# copy_records_tma_kernel in the MoE and AF bench steps.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for rc in 4x16:1 4x16:2 4x16:3 8x16:1 8x16:2 4x32:1 6x32:1 3x64:1; do
  r=${rc%:*}; c=${rc#*:}
  echo "isolated $r ctas/SM $c:"; DYO_TMA_RING=$r DYO_TMA_CTAS_PER_SM=$c timeout 120 python tools/prof_copy.py 2>&1 | grep TMA
  for cfg in moe af; do
    DYO_TMA_RING=$r DYO_TMA_CTAS_PER_SM=$c timeout 600 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/ring_${cfg}_${r}_$c.json 2>/dev/null
    python - "$r" "$c" "$cfg" <<'PY'
import json,sys
r_,c_,cfg=sys.argv[1:4]
try:
    d=json.loads(open(f"gpurun_out/ring_{cfg}_{r_}_{c_}.json").read().strip().splitlines()[-1])
    r=d["roofline"]; print(r_, "ctas/SM", c_, cfg, "value", d["value"], "ms/step", d["ms_per_step"], "copy GB/s", r.get("achieved"), "frac", r.get("frac"), "agg", r.get("aggregate_busy_gbs"), "avg_us", round(r.get("avg_launch_us",0),1), "clocks", d.get("clocks"))
except Exception as e: print(r_, c_, cfg, "failed", e)
PY
  done
done 2>&1 | tee gpurun_out/ring_sweep.txt
