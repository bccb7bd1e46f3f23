cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in auto 16 8 4 2; do
  if [ $c = auto ]; then python tools/sweep_batch_pilot.py moe 64; else DYO_PILOT_BATCH_C=$c python tools/sweep_batch_pilot.py moe 64; fi
done > gpurun_out/sweep.txt 2>&1
EXTRA_FLAGS=32 python tools/sweep_batch_pilot.py moe 64 >> gpurun_out/sweep.txt 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:pilot_kernel -c 1 -s 3 -o gpurun_out/pilot_b64 python tools/sweep_batch_pilot.py moe 64 > gpurun_out/ncu_pilot.log 2>&1
cat gpurun_out/sweep.txt
