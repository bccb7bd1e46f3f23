#!/bin/bash
# Per-launch duration + DRAM bytes of the TMA copy kernel inside the MoE bench (ncu serialises
# launches and flushes caches between them; durations are the kernel alone, not its live share).
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:copy_ -c 2000 --csv --log-file gpurun_out/copy_launches.csv \
  python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_copy.log 2>&1; echo "ncu copy rc=$?"
