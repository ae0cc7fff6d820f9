mkdir -p gpurun_out/w
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_jmatch" -s 2 -c 2 -o gpurun_out/w/c5_jmatch -f python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep > gpurun_out/w/ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_join_emit" -s 1 -c 1 -o gpurun_out/w/c3_emit -f python bench.py --config c3 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep > gpurun_out/w/ncu3.log 2>&1
ls -la gpurun_out/w
