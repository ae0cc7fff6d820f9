mkdir -p gpurun_out/k
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_jmatch" -s 2 -c 2 -o gpurun_out/k/c5_jmatch -f python bench.py --config c5 --steps 2 --warmup 1 --no-e2e --no-unfused --no-cpu --no-sweep > gpurun_out/k/ncu.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' -c 40 --csv --log-file gpurun_out/k/launches_c5.csv python bench.py --config c5 --steps 3 --warmup 1 --no-e2e --no-cpu --no-unfused --no-sweep > /dev/null 2>&1
ls -la gpurun_out/k
