mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_scan_chain|k_join_runs" -s 3 -c 3 -o gpurun_out/prof_c3m -f python bench.py --config c3 --steps 1 --warmup 1 --no-e2e --no-unfused --no-cpu > gpurun_out/ncu_c3m.log 2>&1
