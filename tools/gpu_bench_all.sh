mkdir -p gpurun_out
for cfg in lstm af; do
  DYO_BENCH_VERBOSE=1 timeout 900 python bench.py --config $cfg --no-cpu-baseline > gpurun_out/bench_$cfg.json 2> gpurun_out/bench_$cfg.err; echo "$cfg rc=$?"
  tail -c 3000 gpurun_out/bench_$cfg.json; tail -3 gpurun_out/bench_$cfg.err
done
