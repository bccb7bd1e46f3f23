mkdir -p gpurun_out
timeout 300 ncu --set full --clock-control none --import-source on -k regex:"pilot_tc_kernel" -s 3 -c 1 -o gpurun_out/prof_tc -f python tools/prof_pilot.py moe 5 64 > gpurun_out/ncu_tc.log 2>&1; echo "ncu rc=$?"
